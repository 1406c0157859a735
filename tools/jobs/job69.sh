cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_convert.py -m gpu -q -k "staged or pipeline or register_cap" > gpurun_out/pytest69.txt 2>&1; tail -5 gpurun_out/pytest69.txt
timeout 900 python tools/sweep.py --only lintb > gpurun_out/sweep_lin69.jsonl 2> gpurun_out/sweep69.err; cut -c1-260 gpurun_out/sweep_lin69.jsonl; tail -3 gpurun_out/sweep69.err
timeout 900 python tools/sweep.py --only staged > gpurun_out/sweep_staged69.jsonl 2>> gpurun_out/sweep69.err; cat gpurun_out/sweep_staged69.jsonl; tail -3 gpurun_out/sweep69.err
