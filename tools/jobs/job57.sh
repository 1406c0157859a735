cd $GRAFT_REPO_ROOT
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu57.txt 2>&1; tail -3 gpurun_out/pytest_gpu57.txt
