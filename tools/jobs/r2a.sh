cd $GRAFT_REPO_ROOT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r2a_smi.txt
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/r2a_pytest_gpu.txt 2>&1
tail -3 gpurun_out/r2a_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2a_smoke.txt 2>&1
timeout 600 python bench.py > gpurun_out/r2a_bench.txt 2>&1
tail -c 3000 gpurun_out/r2a_bench.txt
