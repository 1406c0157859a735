cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_edge_cases.py tests/test_gpu_convert.py::test_e1_exhaustive_generic_gpu -m gpu -q -x --durations=10 > gpurun_out/pytest_edge17.txt 2>&1
tail -25 gpurun_out/pytest_edge17.txt
