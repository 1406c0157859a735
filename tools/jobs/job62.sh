cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests -m gpu -q -k "pipeline or linear or random_memory or swizzled or fuzz" > gpurun_out/pytest62.txt 2>&1; tail -3 gpurun_out/pytest62.txt
timeout 900 python tools/sweep.py --only generic > gpurun_out/sweep_generic62.jsonl 2> gpurun_out/sweep62.err; cat gpurun_out/sweep_generic62.jsonl; tail -3 gpurun_out/sweep62.err
