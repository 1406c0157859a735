cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r2s_build.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "peer or config5 or device" > gpurun_out/r2s_pytest.txt 2>&1
tail -2 gpurun_out/r2s_pytest.txt
timeout 600 python - > gpurun_out/r2s_c5.txt 2>&1 <<'PY'
import json, torch, sys
sys.path.insert(0, ".")
import paper_conf_asplos_0001cgrnls0trm26_b200 as ll
from workloads import configs as W
from tools.sweep import time_fn
for p in (1, 2, 3):
    sa, sb = W.c5(p)
    plan = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), 2, comm=ll.Comm.loopback(1 << p), exchange="peer")
    n = 1 << 30
    src = torch.randint(-2**15, 2**15, (n,), dtype=torch.int16, device="cuda"); dst = torch.empty_like(src)
    ms = time_fn(lambda: ll.ll_convert(src, dst, plan), iters=10)
    print(json.dumps({"P": 1 << p, "ms": round(ms, 4), "GBps": round(4 * n / ms / 1e6, 1)}))
PY
cat gpurun_out/r2s_c5.txt
