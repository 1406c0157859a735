cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2sf_build.txt 2>&1
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r2sf_pytest_gpu.txt 2>&1
tail -3 gpurun_out/r2sf_pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2sf_smoke.txt 2>&1
tail -2 gpurun_out/r2sf_smoke.txt
timeout 900 python bench.py > gpurun_out/r2sf_bench.txt 2>&1
tail -c 300 gpurun_out/r2sf_bench.txt
timeout 1200 python tools/sweep.py --only gathfam > gpurun_out/r2sf_gathfam.jsonl 2> gpurun_out/r2sf_gathfam.err
timeout 900 python tools/sweep.py --only redfam > gpurun_out/r2sf_redfam.jsonl 2> gpurun_out/r2sf_redfam.err
wc -l gpurun_out/r2sf_*.jsonl
