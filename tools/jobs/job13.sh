cd $GRAFT_REPO_ROOT
for tool in racecheck synccheck memcheck; do
  for c in reduce_mma_small gather_mma_6_small gather_blocked_6_small; do
    timeout 300 compute-sanitizer --tool $tool python tools/profile_one.py --case $c --iters 2 > gpurun_out/san13_${tool}_$c.txt 2>&1
  done
done
timeout 300 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 2 -c 1 -o gpurun_out/prof13_gather_mma_6 python tools/profile_one.py --case gather_mma_6 > /dev/null 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 2 -c 1 -o gpurun_out/prof13_reduce_mma python tools/profile_one.py --case reduce_mma > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 80 --csv --log-file gpurun_out/launches13_bench.csv python bench.py --steps 5 --warmup 3 --e2e-steps 1 --no-cpu-baseline > /dev/null 2>&1
