cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests -m gpu -q -x -k "host or gather" > gpurun_out/pytest_gpu12.txt 2>&1
tail -3 gpurun_out/pytest_gpu12.txt
timeout 300 python bench.py > gpurun_out/bench12.json 2> gpurun_out/bench12.err
tail -2 gpurun_out/bench12.err
