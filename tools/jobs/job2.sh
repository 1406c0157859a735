set -x
cd $GRAFT_REPO_ROOT
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1
timeout 300 python bench.py > gpurun_out/bench1.json 2> gpurun_out/bench1.err
timeout 300 python bench.py --steps 2000 --warmup 20 --no-cpu-baseline > gpurun_out/bench2000.json 2>> gpurun_out/bench1.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/launches_bench.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
for c in c2 c3 c1b c2smem gather_mma gather_blocked reduce_mma; do
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 2 -c 1 -o gpurun_out/prof_$c python tools/profile_one.py --case $c > gpurun_out/ncu_$c.log 2>&1
done
ls -la gpurun_out
