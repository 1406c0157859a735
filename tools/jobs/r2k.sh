cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2k_build.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r2k_pytest_gpu.txt 2>&1
tail -3 gpurun_out/r2k_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2k_smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/r2k_bench.txt 2>&1
tail -c 300 gpurun_out/r2k_bench.txt
