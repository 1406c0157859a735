cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2d_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "broadcast or n2 or next_rows or tmem" > gpurun_out/r2d_pytest.txt 2>&1
tail -3 gpurun_out/r2d_pytest.txt
timeout 900 python tools/sweep.py --only broadcast > gpurun_out/r2d_sweep_broadcast.jsonl 2>&1
tail -4 gpurun_out/r2d_sweep_broadcast.jsonl
timeout 900 python bench.py > gpurun_out/r2d_bench.txt 2>&1
tail -c 600 gpurun_out/r2d_bench.txt
