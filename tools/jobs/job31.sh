cd $GRAFT_REPO_ROOT
for pipe in 0 1; do
  LL_PIPE=$pipe timeout 600 python tools/sweep.py --only tb > gpurun_out/sweep31_pipe$pipe.txt 2>&1
done
python - <<'PY'
import json
for pipe in (0, 1):
    for l in open(f"gpurun_out/sweep31_pipe{pipe}.txt"):
        try: d = json.loads(l)
        except Exception: continue
        if d.get("xchg") == "smem":
            print(pipe, d["case"], d["opts"], d["threads"], d["R"], d["GBps"], d["frac_6539"])
PY
LL_PIPE=1 timeout 900 python -m pytest tests/test_gpu_convert.py -m gpu -q -x > gpurun_out/pytest31.txt 2>&1; tail -2 gpurun_out/pytest31.txt
