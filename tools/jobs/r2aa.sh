cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2aa_build.txt 2>&1
timeout 900 python tools/sweep.py --only n2opts > gpurun_out/r2aa_sweep_n2opts.jsonl 2>&1
cat gpurun_out/r2aa_sweep_n2opts.jsonl
