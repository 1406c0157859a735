cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2sa_build.txt 2>&1
timeout 900 python tools/sweep.py --only scanldg > gpurun_out/r2sa_scanldg.jsonl 2> gpurun_out/r2sa_scanldg.err
cat gpurun_out/r2sa_scanldg.jsonl
tail -3 gpurun_out/r2sa_scanldg.err
