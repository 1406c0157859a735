cd $GRAFT_REPO_ROOT
timeout 900 python tools/sweep.py --only lintb > gpurun_out/sweep_lin72.jsonl 2> gpurun_out/sweep72.err; tail -3 gpurun_out/sweep72.err
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu72.txt 2>&1; tail -2 gpurun_out/pytest_gpu72.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke72.txt 2>&1; tail -1 gpurun_out/smoke72.txt
