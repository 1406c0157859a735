cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2se_build.txt 2>&1
timeout 1500 python tools/sweep.py --only gathfam > gpurun_out/r2se_gathfam.jsonl 2> gpurun_out/r2se_gathfam.err
timeout 900 python tools/sweep.py --only redfam > gpurun_out/r2se_redfam.jsonl 2> gpurun_out/r2se_redfam.err
wc -l gpurun_out/r2se_*.jsonl
tail -3 gpurun_out/r2se_gathfam.err
