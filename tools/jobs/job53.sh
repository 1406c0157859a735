cd $GRAFT_REPO_ROOT
timeout 1800 python -m pytest tests/test_gpu_convert.py tests/test_gpu_fuzz.py -m gpu -q -k "linear or fuzz or swizzled or memory" > gpurun_out/pytest53.txt 2>&1; tail -3 gpurun_out/pytest53.txt
timeout 900 python tools/sweep.py --only generic > gpurun_out/sweep53_linear.jsonl 2>&1; cut -c1-200 gpurun_out/sweep53_linear.jsonl
