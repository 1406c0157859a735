cd $GRAFT_REPO_ROOT
timeout 900 python tools/sweep.py --only shflocc > gpurun_out/r2s3j_shflocc.jsonl 2>&1
