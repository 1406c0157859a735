cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x -k "scan" > gpurun_out/pytest40.txt 2>&1; tail -2 gpurun_out/pytest40.txt
timeout 300 python tools/sweep.py --only small 2>&1 | grep case
