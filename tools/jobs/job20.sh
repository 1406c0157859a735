cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu20.txt 2>&1
tail -3 gpurun_out/pytest_gpu20.txt
for pdl in 0 1; do
  LL_PDL=$pdl timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench20_pdl$pdl.json 2>gpurun_out/bench20_pdl$pdl.err
  python - <<PY
import json
d = json.loads(open("gpurun_out/bench20_pdl$pdl.json").read().strip().splitlines()[-1])
print("PDL=$pdl", d["value"], d["roofline"]["frac"])
for c in d["configs"]:
    print("   ", c["workload"][:60], c.get("GBps"), c.get("frac"), c.get("us_per_conversion"))
PY
done
