cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x -k "gather or reduce" > gpurun_out/pytest_gpu8.txt 2>&1
tail -3 gpurun_out/pytest_gpu8.txt
timeout 600 python tools/sweep.py --only lat > gpurun_out/sweep8.txt 2>&1
timeout 600 python tools/sweep.py --only next > gpurun_out/sweep8b.txt 2>&1
