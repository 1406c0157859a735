cd $GRAFT_REPO_ROOT
timeout 900 python tools/sweep.py --only lintb > gpurun_out/sweep_lintb61.jsonl 2> gpurun_out/sweep61.err; cat gpurun_out/sweep_lintb61.jsonl; tail -3 gpurun_out/sweep61.err
