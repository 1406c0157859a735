cd $GRAFT_REPO_ROOT
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke43.txt 2>&1; tail -1 gpurun_out/smoke43.txt
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu43.txt 2>&1; tail -2 gpurun_out/pytest_gpu43.txt
timeout 600 python bench.py > gpurun_out/bench43.json 2>gpurun_out/bench43.err; tail -2 gpurun_out/bench43.err
timeout 600 python bench.py --impl reference > gpurun_out/bench43_ref.json 2>&1; tail -c 300 gpurun_out/bench43_ref.json
python -c "
import json; d=json.loads(open('gpurun_out/bench43.json').read().strip().splitlines()[-1]); print(d['value'], d['roofline'], d['e2e']['value'], d['e2e']['frac_of_host_link'], d['clocks'], d['torch_baseline']); [print(c['workload'][:55], c.get('GBps'), c.get('frac'), c.get('us_per_conversion')) for c in d['configs']]"
