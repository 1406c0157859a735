cd $GRAFT_REPO_ROOT
# default vs pipelined smem exchange vs 128 B per thread on the 1-2 GiB rows (same box)
timeout 600 python tools/sweep.py --only ceiling > gpurun_out/r2s3h_default.jsonl 2>&1
LL_SWEEP_OPTS='{"pipe": "on"}' timeout 600 python tools/sweep.py --only ceiling > gpurun_out/r2s3h_pipe.jsonl 2>&1
LL_SWEEP_OPTS='{"thread_bytes": 128}' timeout 600 python tools/sweep.py --only ceiling > gpurun_out/r2s3h_tb128.jsonl 2>&1
timeout 600 python tools/sweep.py --only ceiling > gpurun_out/r2s3h_default2.jsonl 2>&1
