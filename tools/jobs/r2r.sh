cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2r_build.txt 2>&1
timeout 600 python tools/sweep.py --only scan > gpurun_out/r2r_sweep_scan.jsonl 2>&1
cat gpurun_out/r2r_sweep_scan.jsonl
timeout 900 python -m pytest tests -m gpu -q -x -k "scan" > gpurun_out/r2r_pytest.txt 2>&1
tail -2 gpurun_out/r2r_pytest.txt
