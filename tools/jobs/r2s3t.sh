cd $GRAFT_REPO_ROOT
timeout 900 python tools/sweep.py --only c5peer > gpurun_out/r2s3t_c5peer.jsonl 2>&1
