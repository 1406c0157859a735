cd $GRAFT_REPO_ROOT
# ncu --set full of the headline kernel and the configs the register-cap rule changed;
# sanitizers on the new NOOP copy kernel and the capped smem / shuffle kernels
for c in c2 c3 c3b noop; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 2 -c 1 -o gpurun_out/r2s3m_full_$c python tools/profile_one.py --case $c --iters 4 > gpurun_out/r2s3m_full_$c.log 2>&1
  tail -1 gpurun_out/r2s3m_full_$c.log
done
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in racecheck memcheck synccheck initcheck; do
  for c in noop_small c3_small c3b_small c2_small; do
    echo "== $tool $c" >> gpurun_out/r2s3m_sanitizer.txt
    timeout 600 $CS --tool $tool --error-exitcode 9 python tools/profile_one.py --case $c --iters 1 >> gpurun_out/r2s3m_sanitizer.txt 2>&1
    echo "rc=$?" >> gpurun_out/r2s3m_sanitizer.txt
  done
done
grep -E "^==|rc=|ERROR SUMMARY" gpurun_out/r2s3m_sanitizer.txt | head -60
