cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_convert.py -m gpu -q -x -k "convert_host or gather" > gpurun_out/pytest26.txt 2>&1; tail -2 gpurun_out/pytest26.txt
timeout 800 python tools/e2e_probe.py > gpurun_out/e2e26.txt 2>&1; cat gpurun_out/e2e26.txt | head -20
timeout 600 python bench.py > gpurun_out/bench26.json 2>gpurun_out/bench26.err; tail -2 gpurun_out/bench26.err
python -c "
import json; d=json.loads(open('gpurun_out/bench26.json').read().strip().splitlines()[-1]); print(d['value'], d['roofline']['frac'], d['e2e']); [print(c) for c in d['configs']]"
