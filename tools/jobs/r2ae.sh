cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2ae_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "gather_more_warps" > gpurun_out/r2ae_pytest.txt 2>&1
tail -2 gpurun_out/r2ae_pytest.txt
timeout 900 python tools/sweep.py --only gwarps > gpurun_out/r2ae_sweep_gwarps.jsonl 2>&1
cat gpurun_out/r2ae_sweep_gwarps.jsonl
