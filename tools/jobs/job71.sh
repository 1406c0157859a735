cd $GRAFT_REPO_ROOT
for nh in 0 1; do
  LL_NOHOIST=$nh timeout 900 python tools/sweep.py --only lintb > gpurun_out/sweep_nohoist71_$nh.jsonl 2>> gpurun_out/sweep71.err
done
tail -3 gpurun_out/sweep71.err
timeout 600 python -m pytest tests/test_gpu_convert.py -m gpu -q -k "staged or pipeline or register_cap or linear" > gpurun_out/pytest71.txt 2>&1; tail -2 gpurun_out/pytest71.txt
