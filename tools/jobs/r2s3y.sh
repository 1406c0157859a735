cd $GRAFT_REPO_ROOT
LL_FUZZ_SEEDS=41-120 timeout 3000 python -m pytest tests/test_gpu_fuzz.py -q > gpurun_out/r2s3y_fuzz_gpu.txt 2>&1
tail -2 gpurun_out/r2s3y_fuzz_gpu.txt
