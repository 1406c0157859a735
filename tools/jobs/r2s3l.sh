cd $GRAFT_REPO_ROOT
for k in 0 1 2 3 0; do LL_AUX_MIN_BLOCKS=$k timeout 600 python tools/sweep.py --only c4rows; done > gpurun_out/r2s3l_c4rows.jsonl 2>&1
