cd $GRAFT_REPO_ROOT
timeout 900 python tools/sweep.py --only asym > gpurun_out/r2s3p_asym.jsonl 2>&1
