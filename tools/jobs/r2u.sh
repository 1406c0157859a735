cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2u_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "broadcast" > gpurun_out/r2u_pytest.txt 2>&1
tail -2 gpurun_out/r2u_pytest.txt
timeout 900 python tools/sweep.py --only bcastcta > gpurun_out/r2u_sweep_bcastcta.jsonl 2>&1
python - <<'PY'
import json, statistics
rows=[json.loads(l) for l in open("gpurun_out/r2u_sweep_bcastcta.jsonl") if l.startswith("{")]
v=[r["tile"]["GBps"] for r in rows]; g=[r["generic"]["GBps"] for r in rows]
print("tile min", min(v), "median", statistics.median(v), "max", max(v), "generic median", statistics.median(g), all(r["tile"]["ok"] for r in rows))
PY
