cd $GRAFT_REPO_ROOT
timeout 600 python bench.py > gpurun_out/bench37.json 2>gpurun_out/bench37.err; tail -3 gpurun_out/bench37.err
python -c "
import json; d=json.loads(open('gpurun_out/bench37.json').read().strip().splitlines()[-1]); print(d['value'], d['roofline']['frac'], d.get('torch_baseline')); [print(c['workload'][:50], c.get('GBps'), c.get('frac'), c.get('torch_permute_GBps'), c.get('torch_permute_matches')) for c in d['configs']]"
