cd $GRAFT_REPO_ROOT
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu52.txt 2>&1; tail -3 gpurun_out/pytest_gpu52.txt
timeout 900 python tools/sweep.py --only generic > gpurun_out/sweep52_linear.jsonl 2>&1; cut -c1-200 gpurun_out/sweep52_linear.jsonl
