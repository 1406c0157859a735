cd $GRAFT_REPO_ROOT
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke46.txt 2>&1; tail -1 gpurun_out/smoke46.txt
timeout 900 python bench.py > gpurun_out/bench46.json 2>gpurun_out/bench46.err; tail -2 gpurun_out/bench46.err
python -c "
import json; d=json.loads(open('gpurun_out/bench46.json').read().strip().splitlines()[-1]); print(d['value'], d['roofline']['frac'], d['e2e']['value'], d['clocks']); [print(c['workload'][:60], c.get('GBps'), c.get('frac'), c.get('size_matched_copy_GBps'), c.get('smem_instructions'), c.get('us_per_conversion')) for c in d['configs']]"
