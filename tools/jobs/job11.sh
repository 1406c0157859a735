cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu11.txt 2>&1
tail -3 gpurun_out/pytest_gpu11.txt
timeout 600 python tools/sweep.py --only lat > gpurun_out/sweep11.txt 2>&1
timeout 600 python tools/sweep.py --only gather,reduce > gpurun_out/sweep11b.txt 2>&1
