cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2sd_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "reduce or scan or table4 or fullsize" > gpurun_out/r2sd_pytest.txt 2>&1
tail -2 gpurun_out/r2sd_pytest.txt
timeout 1200 python tools/sweep.py --only redfam > gpurun_out/r2sd_redfam.jsonl 2> gpurun_out/r2sd_redfam.err
timeout 1200 python tools/sweep.py --only gathfam > gpurun_out/r2sd_gathfam.jsonl 2> gpurun_out/r2sd_gathfam.err
wc -l gpurun_out/r2sd_*.jsonl
tail -3 gpurun_out/r2sd_gathfam.err
