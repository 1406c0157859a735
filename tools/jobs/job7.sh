cd $GRAFT_REPO_ROOT
timeout 600 python tools/sweep.py --only next > gpurun_out/sweep7.txt 2>&1
