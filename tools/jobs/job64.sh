cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests -m gpu -q -k "pipeline or linear or random_memory or autotune or fuzz" > gpurun_out/pytest64.txt 2>&1; tail -3 gpurun_out/pytest64.txt
timeout 900 python tools/sweep.py --only lintb > gpurun_out/sweep_lin64.jsonl 2> gpurun_out/sweep64.err; cat gpurun_out/sweep_lin64.jsonl; tail -3 gpurun_out/sweep64.err
