cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests/test_gpu_fuzz.py -m gpu -q --durations=3 > gpurun_out/pytest49_fuzz.txt 2>&1; tail -8 gpurun_out/pytest49_fuzz.txt
