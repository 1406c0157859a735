cd $GRAFT_REPO_ROOT
timeout 900 python tools/sweep.py --only smemocc > gpurun_out/r2s3i_smemocc.jsonl 2>&1
