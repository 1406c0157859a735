cd $GRAFT_REPO_ROOT
timeout 600 python bench.py --no-cpu-baseline --steps 20 > gpurun_out/bench36.json 2>gpurun_out/bench36.err; tail -3 gpurun_out/bench36.err
python -c "
import json; d=json.loads(open('gpurun_out/bench36.json').read().strip().splitlines()[-1]); [print(c['workload'][:50], c.get('GBps'), c.get('frac'), c.get('torch_gather_same_bytes_GBps'), c.get('torch_sum_same_bytes_GBps')) for c in d['configs']]"
