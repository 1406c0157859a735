"""Host-link probe for the e2e path: concurrent H2D + D2H of 2 GiB each (torch, pinned
buffers, two streams) vs ll_convert_host with 2-6 streams and several device buffer
sizes on the config-2 plan."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_asplos_0001cgrnls0trm26_b200 as ll  # noqa: E402
from workloads import configs as W  # noqa: E402

n = 1 << 30
h_src = torch.empty(n, dtype=torch.int16, pin_memory=True)
h_dst = torch.empty(n, dtype=torch.int16, pin_memory=True)
d_a = torch.empty(n, dtype=torch.int16, device="cuda")
d_b = torch.empty(n, dtype=torch.int16, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()


def timed(fn, reps=3):
    fn()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    torch.cuda.synchronize()
    e1.record()
    e1.synchronize()
    return e0.elapsed_time(e1) / reps


def h2d():
    with torch.cuda.stream(s1):
        d_a.copy_(h_src, non_blocking=True)


def d2h():
    with torch.cuda.stream(s2):
        h_dst.copy_(d_b, non_blocking=True)


def both():
    h2d()
    d2h()


for name, fn in [("h2d 2GiB", h2d), ("d2h 2GiB", d2h), ("h2d+d2h concurrent 2+2 GiB", both)]:
    ms = timed(fn)
    b = (4 if "concurrent" in name else 2) * 2 ** 30
    print(json.dumps({"case": name, "ms": round(ms, 2), "GBps": round(b / ms / 1e6, 1)}), flush=True)
del d_a, d_b
sa, sb = W.c2(16)
plan = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), 2)
plan.prepare()
for ns in (2, 3, 4, 6):
    for mib in (256, 512, 1024):
        dev_buf = torch.empty(mib << 20, dtype=torch.uint8, device="cuda")
        streams = [torch.cuda.Stream() for _ in range(ns)]
        ms = timed(lambda: ll.ll_convert_host(h_src, h_dst, dev_buf, plan, streams))
        print(json.dumps({"case": f"ll_convert_host streams={ns} dev_buf={mib} MiB", "ms": round(ms, 2),
                          "GBps": round(4 * 2 ** 30 / ms / 1e6, 1)}), flush=True)
        del dev_buf
