cd $GRAFT_REPO_ROOT
timeout 900 python tools/sweep.py --only generic > gpurun_out/sweep51_generic.jsonl 2>&1; cut -c1-200 gpurun_out/sweep51_generic.jsonl
