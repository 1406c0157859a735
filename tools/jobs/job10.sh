cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x -k "reduce or nccl" > gpurun_out/pytest_gpu10.txt 2>&1
tail -3 gpurun_out/pytest_gpu10.txt
timeout 600 python tools/sweep.py --only gather,reduce > gpurun_out/sweep10.txt 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 2 -c 1 -o gpurun_out/prof10_reduce_mma python tools/profile_one.py --case reduce_mma > gpurun_out/ncu10.log 2>&1
