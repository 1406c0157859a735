cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_peer_exchange.py -m gpu -q -x > gpurun_out/pytest_peer16.txt 2>&1
tail -3 gpurun_out/pytest_peer16.txt
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu16.txt 2>&1
tail -3 gpurun_out/pytest_gpu16.txt
for ex in collective peer; do
  for P in 2 4 8; do
    timeout 300 python tools/bench_device.py --loopback $P --exchange $ex >> gpurun_out/dev16.jsonl 2>&1
  done
done
cat gpurun_out/dev16.jsonl
timeout 300 python bench.py > gpurun_out/bench16.json 2>gpurun_out/bench16.err; tail -1 gpurun_out/bench16.json
