cd $GRAFT_REPO_ROOT
timeout 600 python bench.py > gpurun_out/bench19.json 2>gpurun_out/bench19.err; tail -3 gpurun_out/bench19.err; tail -1 gpurun_out/bench19.json
timeout 300 python tools/sweep.py --only next > gpurun_out/sweep19.txt 2>&1; cat gpurun_out/sweep19.txt | cut -c1-200
