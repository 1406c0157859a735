cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2sc_build.txt 2>&1
timeout 1200 python tools/sweep.py --only redfam > gpurun_out/r2sc_redfam.jsonl 2> gpurun_out/r2sc_redfam.err
wc -l gpurun_out/r2sc_redfam.jsonl
tail -3 gpurun_out/r2sc_redfam.err
