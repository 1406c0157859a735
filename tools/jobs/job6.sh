cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu6.txt 2>&1
tail -3 gpurun_out/pytest_gpu6.txt
timeout 600 python tools/sweep.py --only next > gpurun_out/sweep6.txt 2>&1
timeout 300 python bench.py > gpurun_out/bench6.json 2>gpurun_out/bench6.err
timeout 300 ncu --set full --clock-control none --import-source on -k regex:ll_ -s 1 -c 1 -o gpurun_out/prof6_c5T python tools/profile_one.py --case c5T > gpurun_out/ncu6_c5T.log 2>&1
