cd $GRAFT_REPO_ROOT
LL_SWEEP_MAXTILE=1 timeout 1200 python tools/sweep.py --only lintb > gpurun_out/sweep_maxtile67.jsonl 2> gpurun_out/sweep67.err; cat gpurun_out/sweep_maxtile67.jsonl | cut -c1-250; tail -3 gpurun_out/sweep67.err
