cd $GRAFT_REPO_ROOT
timeout 900 python bench.py > gpurun_out/bench74.json 2> gpurun_out/bench74.err; tail -c 300 gpurun_out/bench74.json
for c in r2_2_0 r2_2_2 r2_4_2; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 1 -c 1 -o gpurun_out/prof74_$c python tools/profile_one.py --case $c --iters 2 > gpurun_out/prof74_$c.log 2>&1
  tail -1 gpurun_out/prof74_$c.log
done
