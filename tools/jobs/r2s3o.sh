cd $GRAFT_REPO_ROOT
for k in 0 2 0 2; do LL_AUX_MIN_BLOCKS=$k timeout 1200 python tools/sweep.py --only fammb; done > gpurun_out/r2s3o_fammb.jsonl 2>&1
