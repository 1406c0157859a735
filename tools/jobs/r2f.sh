cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2f_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "broadcast" > gpurun_out/r2f_pytest.txt 2>&1
tail -3 gpurun_out/r2f_pytest.txt
timeout 600 python tools/sweep.py --only broadcast > gpurun_out/r2f_sweep_broadcast.jsonl 2>&1
tail -3 gpurun_out/r2f_sweep_broadcast.jsonl
