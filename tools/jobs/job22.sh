cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_convert.py tests/test_gpu_edge_cases.py -m gpu -q -x -k "gather" > gpurun_out/pytest_gather23.txt 2>&1
tail -2 gpurun_out/pytest_gather23.txt
timeout 600 python tools/sweep.py --only lat > gpurun_out/sweep23.txt 2>&1; cut -c1-60,200-320 gpurun_out/sweep23.txt
timeout 300 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 2 -c 1 -o gpurun_out/prof23_gather_blocked python tools/profile_one.py --case gather_blocked > /dev/null 2>&1
