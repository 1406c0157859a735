cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_graphs.py -q > gpurun_out/r2s3x_graphs.txt 2>&1
tail -15 gpurun_out/r2s3x_graphs.txt
