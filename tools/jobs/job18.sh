cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_edge_cases.py tests/test_gpu_convert.py::test_e1_exhaustive_generic_gpu -m gpu -q --durations=12 > gpurun_out/pytest_edge18.txt 2>&1
tail -22 gpurun_out/pytest_edge18.txt
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu18.txt 2>&1
tail -4 gpurun_out/pytest_gpu18.txt
