cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_convert.py -m gpu -q -k "swizzled" > gpurun_out/pytest50.txt 2>&1; tail -3 gpurun_out/pytest50.txt
timeout 900 python tools/sweep.py --only invec > gpurun_out/sweep50_invec.jsonl 2>&1; cut -c1-200 gpurun_out/sweep50_invec.jsonl
