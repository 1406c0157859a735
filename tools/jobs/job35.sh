cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests -m gpu -q -x -k "reduce" > gpurun_out/pytest35.txt 2>&1; tail -2 gpurun_out/pytest35.txt
timeout 600 python bench.py --no-cpu-baseline --steps 20 > gpurun_out/bench35.json 2>gpurun_out/bench35.err
python -c "
import json; d=json.loads(open('gpurun_out/bench35.json').read().strip().splitlines()[-1]); [print(c['workload'][:50], c.get('GBps'), c.get('frac'), c.get('us_per_conversion')) for c in d['configs']]"
