cd $GRAFT_REPO_ROOT
for c in n2_16x128b n2_16x256b; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 2 -c 1 -o gpurun_out/r2s3r_full_$c python tools/profile_one.py --case $c --iters 4 > gpurun_out/r2s3r_full_$c.log 2>&1
done
