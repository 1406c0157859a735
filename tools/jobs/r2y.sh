cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2y_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "reduce or scan" > gpurun_out/r2y_pytest.txt 2>&1
tail -2 gpurun_out/r2y_pytest.txt
timeout 900 python tools/sweep.py --only warps > gpurun_out/r2y_sweep_warps.jsonl 2>&1
cat gpurun_out/r2y_sweep_warps.jsonl
