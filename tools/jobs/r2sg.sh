cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2sg_build.txt 2>&1
CS=/usr/local/cuda/bin/compute-sanitizer
OUT=gpurun_out/r2sg_sanitizer.txt
for tool in racecheck memcheck synccheck initcheck; do
  for c in t4_scan_custom_128_128_0 t4_scan_mma_128_128_1 t4_scan_blocked_128_16_0 t4_reduce_mma_128_128_1 t4_reduce_custom_128_128_0 t4_reduce_blocked_128_16_0 t4_gather_blocked_128_128_1 t4_gather_mma_128_16_1 t4_gather_custom_32_128_1; do
    echo "== $tool $c" >> $OUT
    timeout 600 $CS --tool $tool --error-exitcode 9 python tools/profile_one.py --case $c --iters 1 >> $OUT 2>&1
    echo "rc=$?" >> $OUT
  done
done
grep -E "^==|rc=|ERROR SUMMARY|RACECHECK SUMMARY" $OUT | head -120
