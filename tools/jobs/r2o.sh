cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2o_build.txt 2>&1
for c in scan_mma_1g gather_blocked_1g reduce_mma; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 2 -c 1 -o gpurun_out/r2o_prof_$c python tools/profile_one.py --case $c --iters 4 > gpurun_out/r2o_prof_$c.log 2>&1
done
ls gpurun_out/r2o*
