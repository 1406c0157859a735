cd $GRAFT_REPO_ROOT
LL_SWEEP_TB=1 timeout 900 python tools/sweep.py --only lintb > gpurun_out/sweep_tb76.jsonl 2> gpurun_out/sweep76.err; tail -2 gpurun_out/sweep76.err
python -c "
import json
for l in open('gpurun_out/sweep_tb76.jsonl'):
    d=json.loads(l); print(d['case'][-8:], d['variant'], d['threads'], d['min_blocks'], d['same_bytes'], d['GBps'], d['frac_6539'])"
