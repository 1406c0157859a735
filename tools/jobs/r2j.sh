cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2j_build.txt 2>&1
timeout 600 python tools/sweep.py --only eperm > gpurun_out/r2j_sweep_eperm.jsonl 2>&1
cat gpurun_out/r2j_sweep_eperm.jsonl
timeout 600 python tools/sweep.py --only broadcast > gpurun_out/r2j_sweep_broadcast.jsonl 2>&1
python - <<'PY'
import json, statistics
v=[json.loads(l)["tile"]["GBps"] for l in open("gpurun_out/r2j_sweep_broadcast.jsonl") if l.startswith("{")]
print("bcast min", min(v), "median", statistics.median(v), "max", max(v))
PY
timeout 900 python -m pytest tests -m gpu -q -x -k "n2 or c3b or broadcast or shuffle" > gpurun_out/r2j_pytest.txt 2>&1
tail -3 gpurun_out/r2j_pytest.txt
