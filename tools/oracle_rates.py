"""The CPU oracles timed on each BASELINE config, on bounded samples of the same
workloads, in the GPU side's units: algorithmic GB/s (conversions: read + write of each
element; gather: src + idx + dst; reduce: src + dst).  Context for BASELINE.md §3 only,
like bench.py's cpu_baseline.

    python tools/oracle_rates.py          > profiles/r01_oracle_rates.jsonl  (numpy, 1 thread)
    python tools/oracle_rates.py --cpp    > profiles/r02_oracle_rates_cpp.jsonl
                                            (C++17/OpenMP oracle: all host cores and 1 core)
"""
import json
import os
import sys
import time

os.environ.setdefault("OMP_NUM_THREADS", "1")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

from oracle import ll_oracle as O  # noqa: E402
from workloads import configs as W  # noqa: E402


def timed(fn, budget=4.0):
    n, t0 = 0, time.perf_counter()
    while True:
        fn()
        n += 1
        dt = time.perf_counter() - t0
        if dt >= budget:
            return n, dt


def conv_rate(name, spec, w, chunk_tiles_elems=1 << 17):
    """Pull map over contiguous runs of dst positions (B(h), then A's slack-zero right
    inverse, then the element copy), as bench.py's cpu_baseline."""
    OA, OB = (O.Layout(*W.spec_to_bases(s)) for s in spec)
    rng = np.random.default_rng(0)
    src = rng.integers(0, 1 << 16, size=1 << 22, dtype=np.uint16)
    state = {"h": 0}
    n_dst = 1 << OB.d_in
    step = min(chunk_tiles_elems, n_dst)

    def one():
        hs = (np.arange(state["h"], state["h"] + step, dtype=np.uint64) % np.uint64(n_dst))
        xs = O.apply_all(OB, hs)
        h_src = O.apply_inverse_all(OA, xs).astype(np.int64) & ((1 << 22) - 1)
        _ = src[h_src]
        state["h"] += step
    n, dt = timed(one)
    elems = n * step
    return {"config": name, "GBps": round(2 * w * elems / dt / 1e9, 5), "cores": 1,
            "sample": f"{elems} dst elements in runs of {step}, {dt:.1f}s"}


def c1_single():
    OA, OB = O.Layout(*W.spec_to_bases(W.C1_A)), O.Layout(*W.spec_to_bases(W.C1_B))
    src = np.arange(256, dtype=np.uint32)
    n, dt = timed(lambda: O.convert(OA, OB, src))
    return {"config": "1 single 16x16 fp32 tile", "GBps": round(2 * 4 * 256 * n / dt / 1e9, 6),
            "us_per_conversion": round(dt / n * 1e6, 1), "cores": 1, "sample": f"{n} conversions, {dt:.1f}s"}


def c4_rates(n_i=8):
    out = []
    rng = np.random.default_rng(1)
    for fam in ("mma", "blocked"):
        L = O.Layout(*W.spec_to_bases(W.c4("gather", fam, n_i=n_i)))
        n = 1 << L.d_in
        src = rng.random(n, dtype=np.float32)
        idx = rng.integers(0, 32, n, dtype=np.int32)
        k, dt = timed(lambda: O.gather(L, 1, src, idx))
        out.append({"config": f"4 gather {fam}", "GBps": round(3 * 4 * n * k / dt / 1e9, 5), "cores": 1,
                    "sample": f"[{1 << n_i},4096] rows of the [4096,4096] problem x {k}, {dt:.1f}s"})
        L = O.Layout(*W.spec_to_bases(W.c4("reduce", fam, n_i=n_i)))
        n = 1 << L.d_in
        src = rng.random(n, dtype=np.float32)
        k, dt = timed(lambda: O.reduce_fixed_order_fp32(L, 1, src))
        out.append({"config": f"4 reduce {fam}", "GBps": round(4 * (n + n // 128) * k / dt / 1e9, 5), "cores": 1,
                    "sample": f"[{1 << n_i},4096] rows of the [4096,4096] problem x {k}, {dt:.1f}s"})
    return out


def cpp_rates():
    """oracle/ll_oracle.cpp on every config: all host cores (os.cpu_count() threads) and
    one; each conversion sample is 2^22 dst elements of a smaller batch of the same tiles
    (the block bits only index tiles), gather / reduce on [256, 4096] rows."""
    from oracle import cpp as OC
    ncores = os.cpu_count() or 1
    out = []
    convs = [("1 batch (2^20 tiles)", W.c1_batched(12), 4), ("2 (65536 tiles)", W.c2(8), 2),
             ("3 (16384 tiles)", W.c3(7), 2), ("3b (16384 tiles)", W.c3b(7), 2),
             ("5-T / 5 at P=1 (32768^2 bf16)", W.c5T(0, n=11), 2)]
    for name, (sa, sb), w in convs:
        OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
        src = np.random.default_rng(0).integers(0, 1 << 16, size=((1 << OA.d_in) * w) // 2, dtype=np.uint16)
        dst = np.empty((1 << OB.d_in) * w, dtype=np.uint8)
        row = {"config": name, "impl": "oracle/ll_oracle.cpp", "cpu_model": OC.cpu_model()}
        for th in (ncores, 1):
            k, dt = timed(lambda: OC.convert(OA.cols, OB.cols, OA.d_out, w, src, threads=th, out=dst), budget=3.0)
            row["GBps_%d_cores" % th] = round(2 * w * (1 << OB.d_in) * k / dt / 1e9, 5)
        out.append(row)
    rng = np.random.default_rng(1)
    for fam in ("mma", "blocked"):
        L = O.Layout(*W.spec_to_bases(W.c4("gather", fam, n_i=8)))
        n = 1 << L.d_in
        src = rng.random(n, dtype=np.float32)
        idx = rng.integers(0, 32, n, dtype=np.int32)
        row = {"config": f"4 gather {fam}", "impl": "oracle/ll_oracle.cpp"}
        for th in (ncores, 1):
            k, dt = timed(lambda: OC.gather(L.cols, L.d_out, 0, 5, 4, src, idx, threads=th), budget=3.0)
            row["GBps_%d_cores" % th] = round(12 * n * k / dt / 1e9, 5)
        out.append(row)
        L = O.Layout(*W.spec_to_bases(W.c4("reduce", fam, n_i=8)))
        n = 1 << L.d_in
        src = rng.random(n, dtype=np.float32)
        row = {"config": f"4 reduce {fam}", "impl": "oracle/ll_oracle.cpp"}
        for th in (ncores, 1):
            k, dt = timed(lambda: OC.reduce(L.cols, L.d_out, 0, 12, 7, src, threads=th), budget=3.0)
            row["GBps_%d_cores" % th] = round(4 * (n + n // 128) * k / dt / 1e9, 5)
        out.append(row)
    return out


def main():
    if "--cpp" in sys.argv:
        for r in cpp_rates():
            print(json.dumps(r), flush=True)
        return
    rows = [c1_single(),
            conv_rate("1 batch (2^20 tiles)", W.c1_batched(20), 4),
            conv_rate("2 (65536 tiles)", W.c2(16), 2),
            conv_rate("3 (16384 tiles)", W.c3(14), 2),
            conv_rate("5-T / 5 at P=1 (32768^2 bf16)", W.c5T(0), 2)]
    rows += c4_rates()
    for r in rows:
        print(json.dumps(r), flush=True)


if __name__ == "__main__":
    main()
