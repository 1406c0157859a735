cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2t_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "permuted or acc_lhs or autotune" > gpurun_out/r2t_pytest.txt 2>&1
tail -2 gpurun_out/r2t_pytest.txt
timeout 900 python tools/sweep.py --only epermfuzz > gpurun_out/r2t_sweep_epermfuzz.jsonl 2>&1
cat gpurun_out/r2t_sweep_epermfuzz.jsonl
