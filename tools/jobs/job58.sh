cd $GRAFT_REPO_ROOT
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu58.txt 2>&1; tail -3 gpurun_out/pytest_gpu58.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke58.txt 2>&1; tail -2 gpurun_out/smoke58.txt
timeout 900 python bench.py > gpurun_out/bench58.json 2> gpurun_out/bench58.err; tail -c 600 gpurun_out/bench58.json
