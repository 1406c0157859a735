cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2c_build.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/r2c_pytest_gpu.txt 2>&1
tail -3 gpurun_out/r2c_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2c_smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/r2c_bench.txt 2>&1
tail -c 1200 gpurun_out/r2c_bench.txt
timeout 300 python bench.py --impl reference --steps 20 --warmup 3 > gpurun_out/r2c_ref.txt 2>&1
tail -c 800 gpurun_out/r2c_ref.txt
timeout 120 python bench.py --gpus 2 --steps 3 > gpurun_out/r2c_bench_gpus2.txt 2>&1; echo "gpus2 rc=$?" >> gpurun_out/r2c_bench_gpus2.txt
