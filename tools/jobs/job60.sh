cd $GRAFT_REPO_ROOT
# ncu --set full of the slowest linear-tile maps (balanced runs): r2_4_2 (7,5), r2_2_2 (6,7), r2_2_0 (6,6)
for c in r2_4_2 r2_2_2 r2_2_0 r2_2_1; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 1 -c 1 -o gpurun_out/prof60_$c python tools/profile_one.py --case $c --iters 2 > gpurun_out/prof60_$c.log 2>&1
  tail -2 gpurun_out/prof60_$c.log
done
