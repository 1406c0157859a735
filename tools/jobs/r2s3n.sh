cd $GRAFT_REPO_ROOT
# config-4 rows: Python launch stream vs CUDA graph of the same calls (host overhead?)
for k in 0 2; do LL_AUX_MIN_BLOCKS=$k timeout 600 python tools/sweep.py --only c4rows; done > gpurun_out/r2s3n_c4rows.jsonl 2>&1
