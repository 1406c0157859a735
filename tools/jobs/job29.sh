cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_convert.py -m gpu -q -x -k "autotune" > gpurun_out/pytest29.txt 2>&1; tail -2 gpurun_out/pytest29.txt
timeout 900 python tools/sweep.py --only tune > gpurun_out/sweep29.txt 2>&1; cut -c1-330 gpurun_out/sweep29.txt
