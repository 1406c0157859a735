cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x -k "table4 or reduce" > gpurun_out/pytest_gpu14.txt 2>&1
tail -5 gpurun_out/pytest_gpu14.txt
