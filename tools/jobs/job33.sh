cd $GRAFT_REPO_ROOT
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke33.txt 2>&1; tail -2 gpurun_out/smoke33.txt
timeout 1800 python -m pytest tests -m gpu -q --durations=8 > gpurun_out/pytest_gpu33.txt 2>&1; tail -14 gpurun_out/pytest_gpu33.txt
timeout 600 python bench.py > gpurun_out/bench33.json 2>gpurun_out/bench33.err; tail -c 600 gpurun_out/bench33.json
