cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x -k "scan" > gpurun_out/pytest41.txt 2>&1; tail -8 gpurun_out/pytest41.txt
timeout 300 python tools/sweep.py --only small 2>&1 | grep case
