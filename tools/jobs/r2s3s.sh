cd $GRAFT_REPO_ROOT
# extended GPU fuzz on the final defaults (40 seeds x 50 cases), then the bench
LL_FUZZ_SEEDS=1-40 timeout 2400 python -m pytest tests/test_gpu_fuzz.py -q > gpurun_out/r2s3s_fuzz_gpu.txt 2>&1
tail -2 gpurun_out/r2s3s_fuzz_gpu.txt
timeout 900 python bench.py > gpurun_out/r2s3s_bench.txt 2>&1
tail -c 300 gpurun_out/r2s3s_bench.txt
