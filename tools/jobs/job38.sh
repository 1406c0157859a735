cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x -k "scan" > gpurun_out/pytest38.txt 2>&1; tail -15 gpurun_out/pytest38.txt
timeout 600 python bench.py --no-cpu-baseline --steps 20 > gpurun_out/bench38.json 2>gpurun_out/bench38.err; tail -3 gpurun_out/bench38.err
python -c "
import json; d=json.loads(open('gpurun_out/bench38.json').read().strip().splitlines()[-1]); [print(c['workload'][:60], c.get('GBps'), c.get('frac'), c.get('torch_cumsum_same_bytes_GBps')) for c in d['configs'] if 'scan' in c['workload']]"
