cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2x_build.txt 2>&1
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in racecheck memcheck synccheck initcheck; do
  for c in acc8_small acc8f_small bcastC1 bcastS901; do
    echo "== $tool $c" >> gpurun_out/r2x_sanitizer.txt
    LL_BCAST_CTA=1 timeout 600 $CS --tool $tool --error-exitcode 9 python tools/profile_one.py --case $c --iters 1 >> gpurun_out/r2x_sanitizer.txt 2>&1
    echo "rc=$?" >> gpurun_out/r2x_sanitizer.txt
  done
done
grep -E "^==|rc=|SUMMARY" gpurun_out/r2x_sanitizer.txt
