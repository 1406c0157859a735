cd $GRAFT_REPO_ROOT
timeout 900 python tools/sweep.py --only matrix > gpurun_out/sweep56_matrix.jsonl 2>&1; cut -c1-180 gpurun_out/sweep56_matrix.jsonl | tail -4
