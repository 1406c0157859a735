cd $GRAFT_REPO_ROOT
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke55.txt 2>&1; tail -1 gpurun_out/smoke55.txt
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu55.txt 2>&1; tail -3 gpurun_out/pytest_gpu55.txt
