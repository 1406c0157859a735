cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu9.txt 2>&1
tail -3 gpurun_out/pytest_gpu9.txt
timeout 600 python tools/sweep.py --only lat > gpurun_out/sweep9.txt 2>&1
