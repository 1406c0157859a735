cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2v_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "broadcast or table3" > gpurun_out/r2v_pytest.txt 2>&1
tail -2 gpurun_out/r2v_pytest.txt
timeout 1200 python tools/sweep.py --only bcastctacmp > gpurun_out/r2v_sweep_bcastctacmp.jsonl 2>&1
tail -2 gpurun_out/r2v_sweep_bcastctacmp.jsonl
