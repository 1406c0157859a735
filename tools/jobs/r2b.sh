cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x -k "reduce or table4 or lib" > gpurun_out/r2b_pytest_reduce.txt 2>&1
tail -3 gpurun_out/r2b_pytest_reduce.txt
timeout 600 python bench.py > gpurun_out/r2b_bench.txt 2>&1
tail -c 1500 gpurun_out/r2b_bench.txt
