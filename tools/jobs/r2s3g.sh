cd $GRAFT_REPO_ROOT
timeout 900 python tools/sweep.py --only ctarun > gpurun_out/r2s3g_ctarun.jsonl 2>&1
timeout 900 python tools/sweep.py --only laggards > gpurun_out/r2s3g_laggards.jsonl 2>&1
