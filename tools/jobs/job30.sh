cd $GRAFT_REPO_ROOT
for c in c3b n1; do
timeout 300 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 2 -c 1 -o gpurun_out/prof30_$c python tools/profile_one.py --case $c > /dev/null 2>&1
done
ls gpurun_out | grep prof30
