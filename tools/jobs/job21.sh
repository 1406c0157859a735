cd $GRAFT_REPO_ROOT
for c in c2 c3 c1b c5T n1 n2 c5peer gather_mma gather_blocked reduce_mma reduce_blocked; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 2 -c 1 -o gpurun_out/prof21_$c python tools/profile_one.py --case $c > gpurun_out/ncu21_$c.log 2>&1
done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 80 --csv --log-file gpurun_out/launches21_bench.csv python bench.py --steps 5 --warmup 3 --e2e-steps 1 --no-cpu-baseline --no-configs > /dev/null 2>&1
ls -la gpurun_out/ | tail -20
