"""Developer sweep: time ll_convert / ll_gather / ll_reduce on the BASELINE configs
under several plan options (CUDA events, inputs > L2).  Not the bench contract."""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_asplos_0001cgrnls0trm26_b200 as ll  # noqa: E402
from workloads import configs as W  # noqa: E402


def time_fn(fn, iters=20, warmup=5, batch=None):
    """Median over `iters` samples of the time per call; each sample times `batch`
    back-to-back calls between two events (default: 1, or 20 for calls < 100 us so that
    small kernels are measured as a stream, not one launch latency each)."""
    for _ in range(warmup):
        fn()
    torch.cuda.synchronize()
    if batch is None:
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        b.synchronize()
        batch = 20 if a.elapsed_time(b) < 0.1 else 1
    ts = []
    for _ in range(iters):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(batch):
            fn()
        b.record()
        b.synchronize()
        ts.append(a.elapsed_time(b) / batch)
    ts.sort()
    return ts[len(ts) // 2]


def time_graph(fn, batch, iters=10):
    """Median time per call of `batch` calls captured in one CUDA graph (no host launch
    overhead between the kernels; PDL edges are captured as programmatic dependencies)."""
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for _ in range(batch):
                fn()
        g.replay()
        torch.cuda.synchronize()
        ts = []
        for _ in range(iters):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            g.replay()
            b.record()
            b.synchronize()
            ts.append(a.elapsed_time(b) / batch)
    ts.sort()
    return ts[len(ts) // 2]


def conv_case(name, sa, sb, w, batch=None, **opts):
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    p = ll.ll_plan_convert(A, B, w, **opts)
    n = 1 << A.d_in
    src = torch.randint(-2 ** 15, 2 ** 15, (n * w // 2,), dtype=torch.int16, device="cuda")
    dst = torch.empty_like(src)
    p.prepare()
    ms = time_fn(lambda: ll.ll_convert(src, dst, p), batch=batch)
    gbs = 2 * n * w / ms / 1e6
    d = p.describe()
    t = d.get("tile", {})
    print(json.dumps({"case": name, "opts": opts, "class": d["class"], "xchg": t.get("xchg"), "threads": t.get("threads"),
                      "R": t.get("R"), "ms": round(ms, 4),
                      "GBps": round(gbs, 1), "frac_6539": round(gbs / 6539.5, 3)}), flush=True)
    del src, dst
    torch.cuda.empty_cache()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--only", default="all")
    args = ap.parse_args()
    only = args.only.split(",")
    if "hints" in only:
        return hints()
    if "next" in only:
        return next_rows()
    if "lat" in only:
        return latency_and_ksweep()
    if "n2" in only:
        return n2_options()
    if "tb" in only:
        return thread_bytes_sweep()
    if "tune" in only:
        return autotune_sweep()
    if "big" in only:
        return big_configs()
    if "ceiling" in only:
        return ceiling_cases()
    if "c5peer" in only:
        return c5_peer_tiles()
    if "asym" in only:
        return cta_asym_runs()
    if "fammb" in only:
        return families_min_blocks()
    if "c4rows" in only:
        return c4_rows()
    if "shflocc" in only:
        return shuffle_occupancy()
    if "smemocc" in only:
        return smem_occupancy()
    if "laggards" in only:
        return laggards()
    if "ctarun" in only:
        return cta_run_lengths()
    if "smallcta" in only:
        return small_cta_tiles()
    if "small" in only:
        return small_kernels()
    if "matrix" in only:
        return matrix_tiles()
    if "invec" in only:
        return invec_swizzles()
    if "lintb" in only:
        return linear_thread_bytes()
    if "staged" in only:
        return staged_configs()
    if "generic" in only:
        return generic_maps()
    if "broadcast" in only:
        return broadcast_sweep()
    if "bcastcta" in only:
        return broadcast_sweep(permute_batch=True)
    if "bcastctacmp" in only:
        # CTA-class broadcast: XOR-copy tiles first (default) vs the CTA-tiled broadcast
        for env in ("1", None):
            if env:
                os.environ["LL_BCAST_CTA"] = env
            else:
                os.environ.pop("LL_BCAST_CTA", None)
            print(json.dumps({"LL_BCAST_CTA": env}), flush=True)
            broadcast_sweep(permute_batch=True)
        return
    if "scan" in only:
        # scan output by TMA bulk store (default) vs per-thread STG (LL_SCAN_TMA_STORE=0),
        # config size and 1 GiB; env is read at plan time
        for env in ("1", "0", None):
            if env is None:
                os.environ.pop("LL_SCAN_TMA_STORE", None)
            else:
                os.environ["LL_SCAN_TMA_STORE"] = env
            for fam in ("mma", "blocked"):
                for ni, nj in ((12, 12), (15, 13)):
                    L = ll.Layout.from_spec(W.c4("reduce", fam, n_i=ni, n_j=nj))
                    p = ll.ll_plan_scan(L, 1)
                    n = 1 << L.d_in
                    sets = [(torch.rand(n, device="cuda"), torch.empty(n, device="cuda")) for _ in range(4 if ni == 12 else 1)]
                    it = [0]

                    def f():
                        a = sets[it[0] % len(sets)]
                        it[0] += 1
                        ll.ll_scan(a[0], a[1], p)
                    ms = time_fn(f, batch=20 if ni == 12 else 3)
                    print(json.dumps({"case": f"scan {fam} [{1 << ni},{1 << nj}]", "tma_store": p.describe()["tma_store"],
                                      "ms": round(ms, 4), "GBps": round(8 * n / ms / 1e6, 1)}), flush=True)
                    del sets
        return
    if "scanldg" in only:
        # scans / reduces: TMA stages (one CTA per SM with 3 x 64 KiB stages) vs direct LDG
        # loads (force_class = SHUFFLE: several CTAs per SM), at 512 / 256 / 128 / 64 bytes per
        # thread; config-4 size (4 rotating buffer sets) and 1 GiB
        for kind in ("scan", "reduce"):
            for fam in ("mma", "blocked"):
                for ni, nj in ((12, 12), (15, 13)):
                    L = ll.Layout.from_spec(W.c4("reduce", fam, n_i=ni, n_j=nj))
                    n = 1 << L.d_in
                    nset = 4 if ni == 12 else 1
                    sets = [torch.rand(n, device="cuda") for _ in range(nset)]
                    for opts in ({}, {"thread_bytes": 256}, {"thread_bytes": 128}, {"force_class": "SHUFFLE"},
                                 {"force_class": "SHUFFLE", "thread_bytes": 256},
                                 {"force_class": "SHUFFLE", "thread_bytes": 128},
                                 {"force_class": "SHUFFLE", "thread_bytes": 64}):
                        p = (ll.ll_plan_scan if kind == "scan" else ll.ll_plan_reduce)(L, 1, **opts)
                        m = n if kind == "scan" else p.out_elems()
                        outs = [torch.empty(m, device="cuda") for _ in sets]
                        it = [0]

                        def f():
                            k = it[0] % nset
                            it[0] += 1
                            (ll.ll_scan if kind == "scan" else ll.ll_reduce)(sets[k], outs[k], p)
                        ms = time_fn(f, batch=20 if ni == 12 else 3)
                        d = p.describe()
                        print(json.dumps({"case": f"{kind} {fam} [{1 << ni},{1 << nj}]", "opts": opts, "tma": d["tma"],
                                          "warps": 1 << d["warp_bits"], "R": d["R"], "ms": round(ms, 4),
                                          "GBps": round(4 * (n + m) / ms / 1e6, 1)}), flush=True)
                        del outs
                    del sets
        return
    if "redfam" in only:
        return reduce_scan_families()
    if "gathfam" in only:
        return gather_families()
    if "split" in only:
        # smaller CTA tiles (tile_bytes: independent rows to the grid) for the config-4
        # gather / reduce / scan at the config size (4 rotating sets) and at 1 GiB
        for fam in ("mma", "blocked"):
            for ni, nj in ((12, 12), (15, 13)):
                nset = 4 if ni == 12 else 1
                for kind in ("gather", "reduce", "scan"):
                    L = ll.Layout.from_spec(W.c4("gather" if kind == "gather" else "reduce", fam, n_i=ni, n_j=nj))
                    n = 1 << L.d_in
                    if kind == "gather":
                        sets = [(torch.randint(0, 1 << 30, (n,), dtype=torch.int32, device="cuda"),
                                 torch.randint(0, 32, (n,), dtype=torch.int32, device="cuda"),
                                 torch.empty(n, dtype=torch.int32, device="cuda")) for _ in range(nset)]
                    else:
                        sets = [torch.rand(n, device="cuda") for _ in range(nset)]
                    for tb in (0, 32768, 16384, 8192, 4096, 2048):
                        if kind == "gather":
                            p = ll.ll_plan_gather(L, 1, 4, tile_bytes=tb)
                            outs = None
                            nbytes = 12 * n
                        else:
                            p = (ll.ll_plan_scan if kind == "scan" else ll.ll_plan_reduce)(L, 1, tile_bytes=tb)
                            m = n if kind == "scan" else p.out_elems()
                            outs = [torch.empty(m, device="cuda") for _ in sets]
                            nbytes = 4 * (n + m)
                        it = [0]

                        def f():
                            k = it[0] % nset
                            it[0] += 1
                            if kind == "gather":
                                ll.ll_gather(sets[k][0], sets[k][1], sets[k][2], p)
                            else:
                                (ll.ll_scan if kind == "scan" else ll.ll_reduce)(sets[k], outs[k], p)
                        ms = time_fn(f, batch=20 if ni == 12 else 3)
                        d = p.describe()
                        print(json.dumps({"case": f"{kind} {fam} [{1 << ni},{1 << nj}]", "tile_bytes": tb,
                                          "ctas": d["ctas"], "warps": 1 << d["warp_bits"], "ms": round(ms, 4),
                                          "GBps": round(nbytes / ms / 1e6, 1)}), flush=True)
                        del outs
                    del sets
        return
    if "warps" in only:
        # reduce / scan with non-axis register bits moved to warps (thread_bytes)
        for fam in ("mma", "blocked"):
            for ni, nj in ((12, 12), (15, 13)):
                L = ll.Layout.from_spec(W.c4("reduce", fam, n_i=ni, n_j=nj))
                n = 1 << L.d_in
                sets = [torch.rand(n, device="cuda") for _ in range(4 if ni == 12 else 1)]
                for tb in (512, 256, 128):
                    for kind in ("reduce", "scan"):
                        p = (ll.ll_plan_reduce if kind == "reduce" else ll.ll_plan_scan)(L, 1, thread_bytes=tb)
                        outs = [torch.empty(p.out_elems() if kind == "reduce" else n, device="cuda") for _ in sets]
                        it = [0]

                        def f():
                            k = it[0] % len(sets)
                            it[0] += 1
                            (ll.ll_reduce if kind == "reduce" else ll.ll_scan)(sets[k], outs[k], p)
                        ms = time_fn(f, batch=20 if ni == 12 else 3)
                        nbytes = 4 * n + 4 * (p.out_elems() if kind == "reduce" else n)
                        print(json.dumps({"case": f"{kind} {fam} [{1 << ni},{1 << nj}]", "thread_bytes": tb,
                                          "warps": 1 << p.describe()["warp_bits"], "ms": round(ms, 4),
                                          "GBps": round(nbytes / ms / 1e6, 1)}), flush=True)
        return
    if "n2opts" in only:
        for shape in ("16x256b", "16x128b"):
            sa, sb = W.n2_tmem(shape, 14)
            for opts in ({}, {"thread_bytes": 128}, {"thread_bytes": 64}, {"force_class": "SMEM"},
                         {"sigma": "faithful"}, {"tile_bytes": 65536}):
                conv_case(f"n2 {shape}", sa, sb, 4, **opts)
        for rep in range(3):
            L = ll.Layout.from_spec(W.c4("gather", "mma", n_i=15, n_j=13))
            p = ll.ll_plan_gather(L, 1, 4)
            n = 1 << L.d_in
            a = torch.randint(0, 1 << 30, (n,), dtype=torch.int32, device="cuda")
            i = torch.randint(0, 32, (n,), dtype=torch.int32, device="cuda")
            o = torch.empty_like(a)
            ms = time_fn(lambda: ll.ll_gather(a, i, o, p), batch=3)
            print(json.dumps({"case": "gather mma 1 GiB repeat", "rep": rep, "ms": round(ms, 4), "GBps": round(12 * n / ms / 1e6, 1)}), flush=True)
            del a, i, o
        return
    if "gwarps" in only:
        for fam in ("mma", "blocked"):
            for ni, nj in ((12, 12), (15, 13)):
                L = ll.Layout.from_spec(W.c4("gather", fam, n_i=ni, n_j=nj))
                n = 1 << L.d_in
                sets = [(torch.randint(0, 1 << 30, (n,), dtype=torch.int32, device="cuda"),
                         torch.randint(0, 32, (n,), dtype=torch.int32, device="cuda"),
                         torch.empty(n, dtype=torch.int32, device="cuda")) for _ in range(4 if ni == 12 else 1)]
                for tb in (0, 64, 32):
                    p = ll.ll_plan_gather(L, 1, 4, thread_bytes=tb)
                    it = [0]

                    def f():
                        a = sets[it[0] % len(sets)]
                        it[0] += 1
                        ll.ll_gather(a[0], a[1], a[2], p)
                    ms = time_fn(f, batch=20 if ni == 12 else 3)
                    print(json.dumps({"case": f"gather {fam} [{1 << ni},{1 << nj}]", "thread_bytes": tb,
                                      "warps": 1 << p.describe()["warp_bits"], "ms": round(ms, 4),
                                      "GBps": round(12 * n / ms / 1e6, 1)}), flush=True)
        return
    if "gtma" in only:
        # gather output by TMA bulk store vs per-thread STG, config size and 1 GiB
        for env in ("1", "0", None):
            if env is None:
                os.environ.pop("LL_GATHER_TMA_STORE", None)
            else:
                os.environ["LL_GATHER_TMA_STORE"] = env
            for fam in ("mma", "blocked"):
                for ni, nj in ((12, 12), (15, 13)):
                    L = ll.Layout.from_spec(W.c4("gather", fam, n_i=ni, n_j=nj))
                    p = ll.ll_plan_gather(L, 1, 4)
                    n = 1 << L.d_in
                    sets = [(torch.randint(0, 1 << 30, (n,), dtype=torch.int32, device="cuda"),
                             torch.randint(0, 32, (n,), dtype=torch.int32, device="cuda"),
                             torch.empty(n, dtype=torch.int32, device="cuda")) for _ in range(4 if ni == 12 else 1)]
                    it = [0]

                    def f():
                        a = sets[it[0] % len(sets)]
                        it[0] += 1
                        ll.ll_gather(a[0], a[1], a[2], p)
                    ms = time_fn(f, batch=20 if ni == 12 else 3)
                    print(json.dumps({"case": f"gather {fam} [{1 << ni},{1 << nj}]", "tma_store": p.describe()["tma_store"],
                                      "ms": round(ms, 4), "GBps": round(12 * n / ms / 1e6, 1)}), flush=True)
                    del sets
        return
    if "epermfuzz" in only:
        # random SHUFFLE-class pairs that take the element-permuted shuffle, batched to
        # 2^30 bytes: default (permuted shuffle) vs the smem exchange vs faithful σ
        import numpy as np
        from workloads import gen
        rng = np.random.default_rng(31)
        out = [("i", 5), ("j", 5)]
        done = 0
        for case in range(400):
            r = int(rng.integers(3, 6))
            hw = [("reg", r), ("lane", 5), ("warp", 10 - r - 5)]
            sa = gen.random_distributed(rng, out, hw)
            sb = gen.random_distributed(rng, out, hw)
            for w in (1, 2):
                d = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), w).describe()
                if not d.get("tile", {}).get("element_permutes") or done >= 12:
                    continue
                nb = 20 - (w - 1)
                ba = {"out": [("b", nb)] + list(sa["out"]), "in": list(sa["in"]) + [("block", [f"b{k}" for k in range(nb)])]}
                bb = {"out": [("b", nb)] + list(sb["out"]), "in": list(sb["in"]) + [("block", [f"b{k}" for k in range(nb)])]}
                for opts in ({}, {"force_class": "SMEM"}, {"sigma": "faithful"}):
                    conv_case(f"eperm#{case} w{w}", ba, bb, w, **opts)
                done += 1
        return
    if "eperm" in only:
        # sub-word shuffles with element permutations (plan_shuffle_eperm) vs the smem exchange
        for name, (sa, sb), w in (("c3b", W.c3b(14), 2), ("acc_fp8", W.n2_acc_to_lhs(8, 18), 1)):
            for opts in ({}, {"force_class": "SMEM"}, {"sigma": "faithful"}):
                conv_case(name, sa, sb, w, **opts)
        return
    if "bulk" in only:
        for name, (sa, sb), w in (("c3", W.c3(14), 2), ("c3b", W.c3b(14), 2)):
            for opts in ({}, {"pipe": "bulk"}, {"pipe": "bulkst"}, {"pipe": "staged"}):
                conv_case(name, sa, sb, w, **opts)
        return
    if "all" not in only and "conv" not in only:
        return gather_reduce()
    # raw copy roofline reference
    n = 1 << 30
    a = torch.empty(n, dtype=torch.int16, device="cuda")
    b = torch.empty_like(a)
    ms = time_fn(lambda: b.copy_(a))
    print(json.dumps({"case": "torch_copy_2GiB", "ms": round(ms, 4), "GBps": round(4 * n / ms / 1e6, 1)}), flush=True)
    del a, b
    for grid in ["0", "4", "8", "16"]:
        os.environ["LL_GRID_PER_SM"] = grid
        sa, sb = W.c2(16)
        conv_case(f"c2 grid{grid}", sa, sb, 2)
    os.environ["LL_GRID_PER_SM"] = "0"
    sa, sb = W.c2(16)
    for opts in [dict(force_class="SMEM"), dict(sigma="faithful"), dict(thread_bytes=128), dict(thread_bytes=64)]:
        conv_case("c2", sa, sb, 2, **opts)
    sa, sb = W.c3(14)
    for opts in [dict(), dict(thread_bytes=128), dict(thread_bytes=64), dict(sigma="faithful")]:
        conv_case("c3", sa, sb, 2, **opts)
    sa, sb = W.c3b(14)
    conv_case("c3b", sa, sb, 2)
    sa, sb = W.c1_batched(20)
    for opts in [dict(), dict(force_class="SMEM"), dict(tile_bytes=65536), dict(thread_bytes=16)]:
        conv_case("c1batch", sa, sb, 4, **opts)
    gather_reduce()



def _batched(L, nb):
    """L (reg, lane, warp -> 2 dims) times 2^nb CTAs on a new leading batch dim."""
    ins, outs = L.in_dims, L.out_dims
    vecs = L.bases()
    bases, k = {}, 0
    for n, b in ins:
        bases[n] = [(0,) + tuple(v) for v in vecs[k:k + b]]
        k += b
    bases["block"] = [tuple([1 << q] + [0] * len(outs)) for q in range(nb)]
    return ll.Layout(list(ins) + [("block", nb)], [("b", nb)] + list(outs), bases)


def reduce_scan_families():
    """Reduce and scan over Table 4 families batched to 64 MiB and 1 GiB of
    fp32: TMA stages (one CTA per SM) vs direct LDG loads at 16 warps."""
    import numpy as np
    from workloads import gen
    rng = np.random.default_rng(77)
    fams = {
        "blocked": lambda a, b: ll.ll_layout_blocked([a, b], [1, 4], [8, 4], [4, 1], [1, 0]),
        "mma": lambda a, b: ll.ll_layout_mma_acc(a, b, 4),
        "mma_input": lambda a, b: ll.ll_layout_mma_operand(0, a, b, 16, 4, 1),
        "custom": lambda a, b: ll.Layout.from_spec(gen.random_distributed(
            rng, [("r", a.bit_length() - 1), ("c", b.bit_length() - 1)],
            [("reg", max(1, a.bit_length() + b.bit_length() - 2 - 7)), ("lane", 5), ("warp", 2)],
            zero_ok=["reg", "lane", "warp"])),
    }
    for fam, mk in fams.items():
        for shape in ((128, 128), (128, 16), (32, 128)):
            T = mk(*shape)
            for total in (24, 28):
                L = _batched(T, total - T.d_in)
                n = 1 << L.d_in
                nset = 4 if total == 24 else 1
                sets = [torch.rand(n, device="cuda") for _ in range(nset)]
                for axis in (1, 2):
                    for kind in ("reduce", "scan"):
                        res = {}
                        for tag, opts in (("default", {}), ("tma16w", {"thread_bytes": 128}),
                                          ("ldg", {"force_class": "SHUFFLE"}),
                                          ("ldg16w", {"force_class": "SHUFFLE", "thread_bytes": 128})):
                            try:
                                p = (ll.ll_plan_scan if kind == "scan" else ll.ll_plan_reduce)(L, axis, **opts)
                            except Exception as e:   # noqa: BLE001
                                res[tag] = str(e)[:80]
                                continue
                            m = n if kind == "scan" else p.out_elems()
                            outs = [torch.empty(m, device="cuda") for _ in sets]
                            it = [0]

                            def f():
                                k = it[0] % nset
                                it[0] += 1
                                (ll.ll_scan if kind == "scan" else ll.ll_reduce)(sets[k], outs[k], p)
                            ms = time_fn(f, batch=20 if total == 24 else 3)
                            d = p.describe()
                            res[tag] = {"tma": d["tma"], "warps": 1 << d["warp_bits"],
                                        "GBps": round(4 * (n + m) / ms / 1e6, 1)}
                            del outs
                        print(json.dumps({"kind": kind, "family": fam, "shape": shape, "axis": axis - 1,
                                          "MiB": (4 * n) >> 20, "res": res}), flush=True)
                del sets


def families_min_blocks():
    """Default gather / reduce / scan plans over Table 4 families x 3 tile shapes x 2
    axes at 64 MiB (4 rotated sets, CUDA graph of 20 calls) and 1 GiB (stream of 3),
    under the caller's LL_AUX_MIN_BLOCKS."""
    import numpy as np
    from workloads import gen
    tag = os.environ.get("LL_AUX_MIN_BLOCKS", "0")
    rng = np.random.default_rng(77)
    fams = {
        "blocked": lambda a, b: ll.ll_layout_blocked([a, b], [1, 4], [8, 4], [4, 1], [1, 0]),
        "mma": lambda a, b: ll.ll_layout_mma_acc(a, b, 4),
        "mma_input": lambda a, b: ll.ll_layout_mma_operand(0, a, b, 16, 4, 1),
        "custom": lambda a, b: ll.Layout.from_spec(gen.random_distributed(
            rng, [("r", a.bit_length() - 1), ("c", b.bit_length() - 1)],
            [("reg", max(1, a.bit_length() + b.bit_length() - 2 - 7)), ("lane", 5), ("warp", 2)],
            zero_ok=["reg", "lane", "warp"])),
    }
    for fam, mk in fams.items():
        for shape in ((128, 128), (128, 16), (32, 128)):
            T = mk(*shape)
            for total in (24, 28):
                L = _batched(T, total - T.d_in)
                n = 1 << L.d_in
                nset = 4 if total == 24 else 1
                sets = [torch.rand(n, device="cuda") for _ in range(nset)]
                idx = [torch.randint(0, 1 << 20, (n,), dtype=torch.int32, device="cuda") for _ in range(nset)]
                for axis in (1, 2):
                    for kind in ("reduce", "scan", "gather"):
                        try:
                            if kind == "gather":
                                p = ll.ll_plan_gather(L, axis, 4)
                            else:
                                p = (ll.ll_plan_scan if kind == "scan" else ll.ll_plan_reduce)(L, axis)
                        except Exception as e:   # noqa: BLE001
                            print(json.dumps({"kind": kind, "family": fam, "error": str(e)[:80]}), flush=True)
                            continue
                        m = p.out_elems() if kind == "reduce" else n
                        outs = [torch.empty(m, device="cuda") for _ in sets]
                        it = [0]

                        def f():
                            k = it[0] % nset
                            it[0] += 1
                            if kind == "gather":
                                ll.ll_gather(sets[k], idx[k], outs[k], p)
                            else:
                                (ll.ll_scan if kind == "scan" else ll.ll_reduce)(sets[k], outs[k], p)
                        nbytes = 4 * (n + m) + (4 * n if kind == "gather" else 0)
                        ms = time_graph(f, 20) if total == 24 else time_fn(f, batch=3)
                        print(json.dumps({"kind": kind, "family": fam, "shape": shape, "axis": axis - 1,
                                          "MiB": (4 * n) >> 20, "aux_min_blocks": tag,
                                          "GBps": round(nbytes / ms / 1e6, 1)}), flush=True)
                        del outs
                del sets, idx


def gather_families():
    """Gather (4-byte elements, int32 indices) over Table 4 families batched to 64 MiB and
    1 GiB of src, and the config-4 gather layouts: load path (TMA stages: pipe = bulk;
    direct LDG: pipe = off) x bytes per thread (extra warps) x exchange (auto / smem)."""
    cases = []
    fams = {
        "blocked": lambda a, b: ll.ll_layout_blocked([a, b], [1, 4], [8, 4], [4, 1], [1, 0]),
        "mma": lambda a, b: ll.ll_layout_mma_acc(a, b, 4),
    }
    for fam in ("mma", "blocked"):
        for ni, nj in ((12, 12), (15, 13)):
            cases.append((f"c4_{fam}", (128, 32), ll.Layout.from_spec(W.c4("gather", fam, n_i=ni, n_j=nj)), 1, 32))
    for fam, mk in fams.items():
        for shape in ((128, 128), (128, 16), (32, 128)):
            T = mk(*shape)
            for total in (24, 28):
                for axis in (1, 2):
                    cases.append((fam, shape, _batched(T, total - T.d_in), axis, shape[axis - 1]))
    for fam, shape, L, axis, K in cases:
        n = 1 << L.d_in
        nset = 4 if n <= (1 << 24) else 1
        sets = [(torch.randint(0, 1 << 30, (n,), dtype=torch.int32, device="cuda"),
                 torch.randint(0, K, (n,), dtype=torch.int32, device="cuda"),
                 torch.empty(n, dtype=torch.int32, device="cuda")) for _ in range(nset)]
        res = {}
        for pipe in ("auto", "bulk", "off"):
            for tb in (0, 64, 32, 16):
                for fc in (None, "SMEM"):
                    tag = f"{pipe}/{tb}/{fc or 'auto'}"
                    try:
                        p = ll.ll_plan_gather(L, axis, 4, pipe=pipe, thread_bytes=tb, force_class=fc)
                    except Exception as e:   # noqa: BLE001
                        res[tag] = str(e)[:60]
                        continue
                    it = [0]

                    def f():
                        a = sets[it[0] % nset]
                        it[0] += 1
                        ll.ll_gather(a[0], a[1], a[2], p)
                    ms = time_fn(f, batch=20 if n <= (1 << 24) else 3)
                    d = p.describe()
                    res[tag] = {"tma": d["tma"], "x": d["exchange"], "warps": 1 << d["warp_bits"],
                                "GBps": round(12 * n / ms / 1e6, 1)}
        print(json.dumps({"family": fam, "shape": shape, "axis": axis - 1, "MiB": (4 * n) >> 20, "res": res}), flush=True)
        del sets

def broadcast_sweep(permute_batch=False):
    """Broadcast targets: random bijective A -> B with 5-8 zero columns,
    batched to ~2 GiB of dst, fp32.  GB/s on algorithmic bytes (src read once + every
    dst replica written: (2^dA + 2^dB) * w), the specialised replica-store tile kernel
    vs the generic kernel on the same pair, and the copy roofline."""
    import numpy as np
    from workloads import gen, hashfill
    w = 4
    for nz in (5, 6, 7, 8):
        rng = np.random.default_rng(900 + nz)
        for case in range(6):
            sa, sb = gen.random_broadcast_pair(rng, nz, ki=5, kj=5, batch_bits=19 - nz, permute_batch=permute_batch)
            A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
            src = hashfill.fill(sa, w, case)
            dst = torch.empty(1 << B.d_in, dtype=torch.int32, device="cuda")
            alg = (src.numel() + dst.numel()) * w
            row = {"case": f"bcast{'-cta' if permute_batch else ''} nz={nz} #{case}", "src_MiB": src.numel() * w >> 20, "dst_MiB": dst.numel() * w >> 20}
            for tag, opts in (("tile", {}), ("generic", {"generic": True})):
                p = ll.ll_plan_convert(A, B, w, **opts)
                p.prepare()
                d = p.describe()
                ms = time_fn(lambda: ll.ll_convert(src, dst, p), iters=10, warmup=3)
                ok = hashfill.check(sb, w, case, dst) == 0
                row[tag] = {"exec": d["exec"], "xchg": d.get("tile", {}).get("xchg"), "vst": d.get("tile", {}).get("vst"),
                            "ms": round(ms, 4), "GBps": round(alg / ms / 1e6, 1), "ok": ok}
            print(json.dumps(row), flush=True)
            del src, dst
            torch.cuda.empty_cache()


def matrix_tiles():
    """Thm 5.1 instruction selection: stmatrix / ldmatrix vs vectorised
    ld/st.shared only, same layouts, same bytes."""
    cases = [("c2 faithful smem", W.c2(16), dict(sigma="faithful", force_class="SMEM")),
             ("c2 faithful smem (matrix)", W.c2(16), dict(sigma="faithful", force_class="SMEM", smem_instr="matrix")),
             ("c3 faithful", W.c3(14), dict(sigma="faithful")),
             ("c3 faithful smem", W.c3(14), dict(sigma="faithful", force_class="SMEM")),
             ("c3b", W.c3b(14), dict()),
             ("c3b tb128", W.c3b(14), dict(thread_bytes=128))]
    for name, (sa, sb), opts in cases:
        for mode in ("auto", "vec"):
            conv_case(f"{name} smem_instr={mode}", sa, sb, 2, smem_instr=mode, **opts)
    for mode in ("auto", "matrix"):
        conv_case(f"N1 preshuffle smem_instr={mode}", *W.n1_preshuffle(14, 14), 2, smem_instr=mode)


def invec_swizzles():
    """Def 4.11 swizzles whose XOR reaches below the 16-byte vector: in-vector XOR copy
    (default) vs shrinking the vector (LL_XOR_INVEC=0), 16384^2 elements, both directions."""
    m = n = 14
    R = ll.Layout([("offset", m + n)], [("d0", m), ("d1", n)],
                  {"offset": [((1 << (k - n)) if k >= n else 0, (1 << k) if k < n else 0) for k in range(m + n)]})
    for w in (1, 2, 4):
        for vec, pp, mp in [(1, 1, 8), (2, 1, 8), (4, 2, 4), (8, 1, 8)]:
            S = ll.ll_layout_mma_swizzle(m, n, vec, pp, mp)
            for mode in ("1", "0"):
                os.environ["LL_XOR_INVEC"] = mode
                p = ll.ll_plan_convert(R, S, w)
                p.prepare()
                nbytes = (1 << (m + n)) * w
                src = torch.randint(-2 ** 15, 2 ** 15, (nbytes // 2,), dtype=torch.int16, device="cuda")
                dst = torch.empty_like(src)
                ms = time_fn(lambda: ll.ll_convert(src, dst, p))
                gbs = 2 * nbytes / ms / 1e6
                print(json.dumps({"case": f"row-major -> mma swizzle vec={vec} pp={pp} mp={mp}, 16384^2 x {w} B",
                                  "in_vector_xor": mode == "1", "vld": p.describe()["tile"]["vld"],
                                  "ms": round(ms, 4), "GBps": round(gbs, 1), "frac_6539": round(gbs / 6539.5, 3)}), flush=True)
                del src, dst
    os.environ.pop("LL_XOR_INVEC", None)


def generic_maps():
    """Linear maps outside the specialised decompositions (random Def 4.14 memory
    layouts, R2; a transpose into a swizzled layout): the runtime-generic kernel."""
    import numpy as np
    from workloads import gen
    rng = np.random.default_rng(5)
    d = 28
    for w in (2, 4):
        for case in range(3):
            ca, cb = gen.random_memory_cols(rng, d), gen.random_memory_cols(rng, d)
            A = ll.Layout([("offset", d)], [("x", d)], {"offset": [(c,) for c in ca]})
            B = ll.Layout([("offset", d)], [("x", d)], {"offset": [(c,) for c in cb]})
            nbytes = (1 << d) * w
            src = torch.randint(-2 ** 15, 2 ** 15, (nbytes // 2,), dtype=torch.int16, device="cuda")
            dst = torch.empty_like(src)
            ref = None
            for bal in ("0", "1"):          # linear-tile run choice: widest stores vs balanced runs
                os.environ["LL_LINEAR_BALANCE"] = bal
                p = ll.ll_plan_convert(A, B, w)
                p.prepare()
                ms = time_fn(lambda: ll.ll_convert(src, dst, p))
                out = dst.clone()
                same = ref is None or bool(torch.equal(ref, out))
                ref = out if ref is None else ref
                gbs = 2 * nbytes / ms / 1e6
                t = p.describe().get("tile", {})
                print(json.dumps({"case": f"random R2 memory layouts 2^{d} x {w} B #{case}", "balance": bal,
                                  "exec": p.describe()["exec"], "st_run_bits": t.get("st_run_bits"),
                                  "ld_run_bits": t.get("ld_run_bits"), "smem_bytes": t.get("smem_bytes"),
                                  "same_bytes": same, "ms": round(ms, 4), "GBps": round(gbs, 1),
                                  "frac_6539": round(gbs / 6539.5, 3)}), flush=True)
            os.environ.pop("LL_LINEAR_BALANCE", None)
            del src, dst, ref, out


def linear_thread_bytes():
    """Linear tiles on the random R2 maps of generic_maps(): the automatic plan, the
    pipelined exchange with and without the two-CTAs-per-SM register cap, and the
    plan ll_plan_autotune picks."""
    import numpy as np
    from workloads import gen
    rng = np.random.default_rng(5)
    d = 28
    for w in (2, 4):
        for case in range(3):
            ca, cb = gen.random_memory_cols(rng, d), gen.random_memory_cols(rng, d)
            A = ll.Layout([("offset", d)], [("x", d)], {"offset": [(c,) for c in ca]})
            B = ll.Layout([("offset", d)], [("x", d)], {"offset": [(c,) for c in cb]})
            nbytes = (1 << d) * w
            src = torch.randint(-2 ** 15, 2 ** 15, (nbytes // 2,), dtype=torch.int16, device="cuda")
            dst = torch.empty_like(src)
            ref = None
            variants = [("auto", {}), ("pipe, no cap", {"pipe": "on", "min_blocks": -1}),
                        ("pipe, 2 CTAs/SM", {"pipe": "on", "min_blocks": 2}),
                        ("no pipe, 2 CTAs/SM", {"pipe": "off", "min_blocks": 2}),
                        ("staged (cp.async)", {"pipe": "staged", "min_blocks": -1}), ("autotune", None)]
            if os.environ.get("LL_SWEEP_TB"):
                variants = [(f"thread_bytes {tb}", {"thread_bytes": tb}) for tb in (0, 64, 128, 512)]
            if os.environ.get("LL_SWEEP_MAXTILE"):
                variants = [(f"max tile {mt}, {n}", dict(o, tile_bytes=mt)) for mt in (65536, 32768, 131072)
                            for n, o in (("auto", {}), ("2 CTAs/SM", {"min_blocks": 2}), ("no cap", {"min_blocks": -1}))]
            for name, opts in variants:
                if opts is None:
                    p = ll.ll_plan_autotune(A, B, w, src, dst, iters=5)
                else:
                    p = ll.ll_plan_convert(A, B, w, **opts)
                p.prepare()
                ms = time_fn(lambda: ll.ll_convert(src, dst, p))
                same = ref is None or bool(torch.equal(ref, dst))
                if ref is None:
                    ref = dst.clone()
                gbs = 2 * nbytes / ms / 1e6
                t = p.describe().get("tile", {})
                print(json.dumps({"case": f"random R2 memory layouts 2^{d} x {w} B #{case}", "variant": name,
                                  "exec": p.describe()["exec"], "threads": t.get("threads"),
                                  "pipe": t.get("pipe"), "staged": t.get("staged"), "min_blocks": t.get("min_blocks"),
                                  "st_run_bits": t.get("st_run_bits"), "ld_run_bits": t.get("ld_run_bits"),
                                  "same_bytes": same, "ms": round(ms, 4),
                                  "GBps": round(gbs, 1), "frac_6539": round(gbs / 6539.5, 3)}), flush=True)
            os.environ.pop("LL_PIPE", None)
            os.environ.pop("LL_MIN_BLOCKS", None)
            del src, dst, ref


def staged_configs():
    """The staged (cp.async) smem exchange against the default plan on the smem-class
    BASELINE conversions (config 3, 3b, 5-T, config 1-batch with smem forced)."""
    cases = [("c3", W.c3(14), 2, {}), ("c3b", W.c3b(14), 2, {}), ("c5T", W.c5T(0), 2, {}),
             ("c1b smem", W.c1_batched(20), 4, {"force_class": "SMEM"})]
    for name, (sa, sb), w, o in cases:
        A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
        n = (1 << A.d_in) * w // 2
        src = torch.randint(-2 ** 15, 2 ** 15, (n,), dtype=torch.int16, device="cuda")
        dst = torch.empty_like(src)
        ref = None
        for var, extra in (("default", {}), ("staged", {"pipe": "staged"})):
            p = ll.ll_plan_convert(A, B, w, **o, **extra)
            p.prepare()
            ms = time_fn(lambda: ll.ll_convert(src, dst, p))
            same = ref is None or bool(torch.equal(ref, dst))
            if ref is None:
                ref = dst.clone()
            gbs = 4 * n / ms / 1e6
            print(json.dumps({"case": name, "variant": var, "staged": p.describe()["tile"].get("staged"),
                              "same_bytes": same, "ms": round(ms, 4), "GBps": round(gbs, 1),
                              "frac_6539": round(gbs / 6539.5, 3)}), flush=True)
        del src, dst, ref


def swizzle_case():
    """Row-major -> Def 4.11 mma-swizzled memory layout, 16384 x 16384 bf16 (XOR copy)."""
    m = n = 14
    S = ll.ll_layout_mma_swizzle(m, n, 8, 1, 8)
    R = ll.Layout([("offset", m + n)], [("d0", m), ("d1", n)],
                  {"offset": [((1 << (k - n)) if k >= n else 0, (1 << k) if k < n else 0) for k in range(m + n)]})
    p = ll.ll_plan_convert(R, S, 2)
    p.prepare()
    src = torch.randint(-2 ** 15, 2 ** 15, (1 << (m + n),), dtype=torch.int16, device="cuda")
    dst = torch.empty_like(src)
    ms = time_fn(lambda: ll.ll_convert(src, dst, p))
    gbs = 4 * (1 << (m + n)) / ms / 1e6
    print(json.dumps({"case": "row-major -> mma swizzle (Def 4.11) 16384^2 bf16", "exec": p.describe()["exec"],
                      "ms": round(ms, 4), "GBps": round(gbs, 1), "frac_6539": round(gbs / 6539.5, 3)}), flush=True)


def next_rows():
    """§8(f) N1 pre-shuffle and N2 TMEM-fragment epilogue at scale; CTA-class transpose."""
    swizzle_case()
    conv_case("N1 preshuffle W[16384,16384] bf16 -> mma rhs fragments", *W.n1_preshuffle(14, 14), 2)
    conv_case("N2 tmem 32x32b -> blocked, 8192 tiles 128x128 fp32", *W.n2_tmem_epilogue(13), 4)
    sa, sb = W.c5T(0, n=15)
    for opts in [dict(), dict(tile_bytes=65536), dict(thread_bytes=128), dict(thread_bytes=64),
                 dict(tile_bytes=65536, thread_bytes=128)]:
        conv_case("c5T P=1 transpose", sa, sb, 2, **opts)
    for opts in [dict(), dict(tile_bytes=65536), dict(thread_bytes=128)]:
        conv_case("N1 preshuffle", *W.n1_preshuffle(14, 14), 2, **opts)


def n2_options():
    """N2 (TMEM 32x32b fragment -> blocked) under the plan options."""
    sa, sb = W.n2_tmem_epilogue(13)
    for opts in [dict(), dict(force_class="SMEM"), dict(thread_bytes=32), dict(thread_bytes=128),
                 dict(tile_bytes=32768), dict(tile_bytes=65536), dict(force_class="SMEM", thread_bytes=128),
                 dict(force_class="SMEM", thread_bytes=32)]:
        conv_case("N2 tmem 32x32b -> blocked", sa, sb, 4, **opts)
    sa, sb = W.n1_preshuffle(14, 14)
    for opts in [dict(thread_bytes=32), dict(tile_bytes=32768), dict(force_class="SMEM", thread_bytes=128)]:
        conv_case("N1 preshuffle", sa, sb, 2, **opts)


def thread_bytes_sweep():
    """Every tile-kernel config under thread_bytes 64 / 128 / 256 (default = None)."""
    cases = [("c1b", W.c1_batched(20), 4), ("c2", W.c2(16), 2), ("c3", W.c3(14), 2), ("c3b", W.c3b(14), 2),
             ("n2", W.n2_tmem_epilogue(13), 4), ("c5T", W.c5T(0), 2), ("n1", W.n1_preshuffle(14, 14), 2)]
    for name, (sa, sb), w in cases:
        for tb in (None, 64, 128, 256):
            opts = {} if tb is None else {"thread_bytes": tb}
            try:
                conv_case(name, sa, sb, w, **opts)
            except Exception as e:  # noqa: BLE001
                print(json.dumps({"case": name, "opts": opts, "error": str(e)[:120]}), flush=True)


def autotune_sweep():
    """ll_plan_autotune vs the default plan on every tile-kernel config."""
    cases = [("c1b", W.c1_batched(20), 4), ("c2", W.c2(16), 2), ("c3", W.c3(14), 2), ("c3b", W.c3b(14), 2),
             ("n2", W.n2_tmem_epilogue(13), 4), ("c5T", W.c5T(0), 2), ("n1", W.n1_preshuffle(14, 14), 2)]
    for name, (sa, sb), w in cases:
        A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
        n = 1 << A.d_in
        src = torch.randint(-2 ** 15, 2 ** 15, (n * w // 2,), dtype=torch.int16, device="cuda")
        dst = torch.empty_like(src)
        t0 = time.time()
        p = ll.ll_plan_autotune(A, B, w, src, dst, iters=5)
        tune_s = time.time() - t0
        pd = ll.ll_plan_convert(A, B, w)
        pd.prepare()
        ms_d = time_fn(lambda: ll.ll_convert(src, dst, pd))
        ms_t = time_fn(lambda: ll.ll_convert(src, dst, p))
        d = p.describe()
        print(json.dumps({"case": name, "default_GBps": round(2 * n * w / ms_d / 1e6, 1),
                          "tuned_GBps": round(2 * n * w / ms_t / 1e6, 1),
                          "tuned_frac_6539": round(2 * n * w / ms_t / 1e6 / 6539.5, 3),
                          "tune_seconds": round(tune_s, 1), "chosen": {k: d["tile"][k] for k in ("xchg", "R", "threads")},
                          "candidates": d.get("autotune")}), flush=True)
        del src, dst
        torch.cuda.empty_cache()


def big_configs():
    """The 1-2 GiB conversions only (for A/B tests of code-generation knobs)."""
    for name, (sa, sb), w in [("c2", W.c2(16), 2), ("c3", W.c3(14), 2), ("c1b", W.c1_batched(20), 4),
                              ("c5T", W.c5T(0), 2), ("n1", W.n1_preshuffle(14, 14), 2),
                              ("n2", W.n2_tmem_epilogue(13), 4)]:
        conv_case(name, sa, sb, w)


def ceiling_cases():
    """The 1-2 GiB conversions of the bench's configs list, for A/B against the plain
    streaming ceiling (tools/smem_counter_control.cu, one tile per CTA); extra plan
    options from $LL_SWEEP_OPTS (JSON), env hooks from the caller."""
    extra = json.loads(os.environ.get("LL_SWEEP_OPTS", "{}"))
    for name, (sa, sb), w in [("c2", W.c2(16), 2), ("c3", W.c3(14), 2), ("c3b", W.c3b(14), 2),
                              ("c1b", W.c1_batched(20), 4), ("c5T", W.c5T(0), 2),
                              ("n1", W.n1_preshuffle(15, 15), 2), ("n2_16x256b", W.n2_tmem("16x256b", 14), 4),
                              ("n2_fp8", W.n2_acc_to_lhs(8, 18), 1), ("noop_bf16", W.n2_acc_to_lhs(16, 17), 2)]:
        conv_case(name, sa, sb, w, batch=20, **extra)


def cta_run_lengths():
    """CTA-class transposes (config 5-T, N1): 256-byte runs in 32 / 64 KiB tiles (the
    64 KiB smem cap) vs 512-byte runs in 128 KiB tiles (tile_bytes = 131072, one CTA
    per SM), unpipelined and pipelined; streams of 20 launches."""
    for name, (sa, sb), w in [("c5T", W.c5T(0), 2), ("n1", W.n1_preshuffle(15, 15), 2)]:
        for o in [{}, {"tile_bytes": 65536}, {"tile_bytes": 131072}, {"tile_bytes": 131072, "pipe": "on"},
                  {"tile_bytes": 65536, "pipe": "on"}]:
            conv_case(name, sa, sb, w, batch=20, **o)


def laggards():
    """The in-CTA rows furthest below the streaming ceiling (config 3b, the tcgen05
    16x256b fragment) under the existing plan options; streams of 20 launches."""
    for name, (sa, sb), w, extra in [("c3b", W.c3b(14), 2, [{"smem_instr": "vec"}]),
                                     ("n2_16x256b", W.n2_tmem("16x256b", 14), 4, [{"force_class": "SMEM"}])]:
        for o in [{}, {"pipe": "on"}, {"thread_bytes": 128}, {"tile_bytes": 131072}] + extra:
            conv_case(name, sa, sb, w, batch=20, **o)


def smem_occupancy():
    """64 / 32 KiB smem-exchange tiles: CTAs per SM (registers: min_blocks) x the
    pipelined exchange; streams of 20 launches."""
    for name, (sa, sb), w in [("c3", W.c3(14), 2), ("c3b", W.c3b(14), 2), ("c5T", W.c5T(0), 2),
                              ("n1", W.n1_preshuffle(15, 15), 2)]:
        for o in [{}, {"pipe": "on"}, {"pipe": "on", "min_blocks": 2}, {"pipe": "on", "min_blocks": 3},
                  {"min_blocks": 2}, {}]:
            conv_case(name, sa, sb, w, batch=20, **o)


def shuffle_occupancy():
    """Shuffle-exchange rows under register caps (min_blocks); streams of 20 launches."""
    cases = [("c2", W.c2(16), 2)] + [(f"n2_{sh}", W.n2_tmem(sh, 14), 4) for sh in ("32x32b", "16x64b", "16x128b", "16x256b")]
    for name, (sa, sb), w in cases:
        for o in [{}, {"min_blocks": 1}, {"min_blocks": 2}, {"min_blocks": 3}, {"min_blocks": 4}]:
            conv_case(name, sa, sb, w, batch=20, **o)


def c4_rows():
    """Config-4 gather / reduce / scan at the config size (4 rotated buffer sets,
    streams of 20 calls) and at 1 GiB (streams of 3), as the bench times them; the env
    hooks of the caller apply (e.g. LL_AUX_MIN_BLOCKS)."""
    tag = os.environ.get("LL_AUX_MIN_BLOCKS", "0")
    for fam in ("mma", "blocked"):
        for big in (False, True):
            kw = dict(n_i=15, n_j=13) if big else {}
            Lg = ll.Layout.from_spec(W.c4("gather", fam, **kw))
            Lr = ll.Layout.from_spec(W.c4("reduce", fam, **kw))
            n = 1 << Lg.d_in
            nsets = 1 if big else 4
            src = [torch.rand(n, device="cuda") for _ in range(nsets)]
            idx = [torch.randint(0, 32, (n,), dtype=torch.int32, device="cuda") for _ in range(nsets)]
            out = [torch.empty(n, device="cuda") for _ in range(nsets)]
            pg, pr, ps = ll.ll_plan_gather(Lg, 1, 4), ll.ll_plan_reduce(Lr, 1), ll.ll_plan_scan(Lr, 1)
            ro = [torch.empty(pr.out_elems(), device="cuda") for _ in range(nsets)]
            it = [0]

            def nxt():
                it[0] += 1
                return it[0] % nsets
            rows = [("gather", lambda: (lambda k: ll.ll_gather(src[k], idx[k], out[k], pg))(nxt()), 12 * n),
                    ("reduce", lambda: (lambda k: ll.ll_reduce(src[k], ro[k], pr))(nxt()), 4 * n + 4 * pr.out_elems()),
                    ("scan", lambda: (lambda k: ll.ll_scan(src[k], out[k], ps))(nxt()), 8 * n)]
            for name, fn, nbytes in rows:
                nb = 3 if big else 20
                ms = time_fn(fn, iters=10, warmup=3, batch=nb)
                gms = time_graph(fn, nb)
                print(json.dumps({"case": f"{name} {fam} {'1GiB' if big else 'config'}", "aux_min_blocks": tag,
                                  "ms": round(ms, 4), "GBps": round(nbytes / ms / 1e6, 1),
                                  "graph_ms": round(gms, 4), "graph_GBps": round(nbytes / gms / 1e6, 1)}), flush=True)
            del src, idx, out, ro
            torch.cuda.empty_cache()


def cta_asym_runs():
    """CTA-class transposes with src runs longer / shorter than dst runs (LL_CTA_RUNS=+1
    / -1, 64 KiB tiles) vs the default symmetric 256-byte runs; streams of 20 launches."""
    for e in ("0", "1", "-1", "0"):
        os.environ["LL_CTA_RUNS"] = e
        for name, (sa, sb), w in [("c5T", W.c5T(0), 2), ("n1", W.n1_preshuffle(15, 15), 2)]:
            conv_case(f"{name} runs{e}", sa, sb, w, batch=20)
    os.environ["LL_CTA_RUNS"] = "0"


def c5_peer_tiles():
    """Config 5 at P = 8 on one GPU (loopback windows, peer-store tile kernel): CTA tile
    bytes x bytes per thread of the fused copy tiles; streams of 20 launches."""
    sa, sb = W.c5(3)
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    n = 1 << 30
    src = torch.randint(-2 ** 15, 2 ** 15, (n,), dtype=torch.int16, device="cuda")
    dst = torch.empty_like(src)
    for o in [{}, {"tile_bytes": 32768}, {"tile_bytes": 65536}, {"tile_bytes": 32768, "thread_bytes": 64},
              {"thread_bytes": 128}, {"tile_bytes": 65536, "thread_bytes": 128}, {}]:
        p = ll.ll_plan_convert(A, B, 2, comm=ll.Comm.loopback(8), exchange="peer", **o)
        p.prepare()
        t = p.describe()["fused"]["tile"]
        ms = time_fn(lambda: ll.ll_convert(src, dst, p), batch=20, iters=10)
        print(json.dumps({"case": "c5 P=8 loopback peer", "opts": o, "n": t["n"], "threads": t["threads"],
                          "ms": round(ms, 4), "GBps": round(4 * n / ms / 1e6, 1)}), flush=True)


def small_cta_tiles():
    """Layouts whose own CTA tile is below 16 KiB (grid bits folded up to tile_bytes):
    tile_bytes x thread_bytes, timed as streams of 20 launches like the bench."""
    for name, (sa, sb), w in [("c1b", W.c1_batched(20), 4), ("n2_fp8", W.n2_acc_to_lhs(8, 18), 1),
                              ("n2_bf16_to_fp8_like_c1", W.c1_batched(21), 2)]:
        for tile in (16384, 32768, 65536):
            for tb in (64, 128, 256):
                conv_case(name, sa, sb, w, batch=20, tile_bytes=tile, thread_bytes=tb)


def small_kernels():
    """Config-4 reduce (TMA vs LDG staging) and scan, 4 rotated buffer sets."""
    n = 1 << 24
    for fam in ("mma", "blocked"):
        L = ll.Layout.from_spec(W.c4("reduce", fam))
        for name, mk in [("reduce tma", lambda: ll.ll_plan_reduce(L, 1)),
                         ("reduce ldg", lambda: ll.ll_plan_reduce(L, 1, force_class="SHUFFLE")),
                         ("scan", lambda: ll.ll_plan_scan(L, 1)),
                         ("scan ldg", lambda: ll.ll_plan_scan(L, 1, force_class="SHUFFLE"))]:
            p = mk()
            p.prepare()
            is_scan = name.startswith("scan")
            sets = [(torch.rand(n, device="cuda"),
                     torch.empty(n if is_scan else p.out_elems(), device="cuda")) for _ in range(4)]
            it = [0]

            def f():
                st = sets[it[0] % 4]
                it[0] += 1
                (ll.ll_scan if is_scan else ll.ll_reduce)(st[0], st[1], p)
            ms = time_fn(f)
            b = 8 * n if is_scan else 4 * n + 4 * p.out_elems()
            print(json.dumps({"case": f"{name} {fam}", "ms": round(ms, 4), "GBps": round(b / ms / 1e6, 1)}), flush=True)
            del sets


def latency_and_ksweep():
    """Config 1 single tile (latency-bound: CUDA graph of 1000 ll_convert launches) and
    the config-4 gather K sweep (16 / 32 / 64)."""
    A, B = ll.Layout.from_spec(W.C1_A), ll.Layout.from_spec(W.C1_B)
    for fc in [None, "SMEM"]:
        p = ll.ll_plan_convert(A, B, 4, force_class=fc)
        p.prepare()
        src = torch.randint(0, 1 << 30, (256,), dtype=torch.int32, device="cuda")
        dst = torch.empty_like(src)
        s = torch.cuda.Stream()
        with torch.cuda.stream(s):
            ll.ll_convert(src, dst, p, s)
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=s):
                for _ in range(1000):
                    ll.ll_convert(src, dst, p, torch.cuda.current_stream())
        torch.cuda.synchronize()
        ms = time_fn(lambda: g.replay(), iters=10, warmup=3)
        print(json.dumps({"case": f"c1 single tile (16x16 fp32) {fc or 'auto'}: 1000 launches in a CUDA graph",
                          "us_per_conversion": round(ms, 4), "xchg": p.describe()["tile"]["xchg"]}), flush=True)
    for kb, fam, fc in [(k, f, x) for k in [4, 5, 6] for f in ["mma", "blocked"] for x in ["SHUFFLE", "SMEM", "CTA"]]:
        if True:
            L = ll.Layout.from_spec(W.c4("gather", fam, k_bits=kb))
            p = ll.ll_plan_gather(L, 1, 4, force_class=fc)
            p.prepare()
            n = 1 << 24
            sets = [(torch.randint(-2 ** 31, 2 ** 31 - 1, (n,), dtype=torch.int32, device="cuda"),
                     torch.randint(0, 1 << kb, (n,), dtype=torch.int32, device="cuda"),
                     torch.empty(n, dtype=torch.int32, device="cuda")) for _ in range(4)]
            it = [0]

            def gg():
                st = sets[it[0] % 4]
                it[0] += 1
                ll.ll_gather(st[0], st[1], st[2], p)
            ms = time_fn(gg)
            print(json.dumps({"case": f"gather {fam} K={1 << kb} {fc if fc != 'CTA' else 'auto-exchange, LDG (no TMA)'}", "desc": p.describe(), "ms": round(ms, 4),
                              "GBps": round(12 * n / ms / 1e6, 1)}), flush=True)
            del sets


def hints():
    """Store hint, grid persistence, CTA-class transpose and DEVICE loopback."""
    for hint in ["", "cs"]:
        os.environ["LL_ST_HINT"] = hint
        sa, sb = W.c2(16)
        conv_case(f"c2 st_hint={hint or 'default'}", sa, sb, 2)
        sa, sb = W.c3(14)
        conv_case(f"c3 st_hint={hint or 'default'}", sa, sb, 2)
    os.environ["LL_ST_HINT"] = ""
    sa, sb = W.c5T(0, n=15)          # 2 GiB bf16 transpose (CTA class)
    for opts in [dict(), dict(tile_bytes=32768), dict(tile_bytes=8192)]:
        conv_case("c5T P=1 transpose", sa, sb, 2, **opts)
    # config 5 DEVICE decomposition on one GPU (loopback: memcpy exchange), P = 8
    sa, sb = W.c5(3, n=15)
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    p = ll.ll_plan_convert(A, B, 2, comm=ll.Comm.loopback(8))
    p.prepare()
    n = 1 << 30
    src = torch.randint(-2 ** 15, 2 ** 15, (n,), dtype=torch.int16, device="cuda")
    dst = torch.empty_like(src)
    ws = torch.empty(p.workspace_bytes(), dtype=torch.uint8, device="cuda")
    ms = time_fn(lambda: ll.ll_convert(src, dst, p, workspace=ws), iters=10, warmup=3)
    print(json.dumps({"case": "c5 P=8 loopback (pack + memcpy all-to-all)", "ms": round(ms, 4),
                      "GBps_algorithmic": round(4 * n / ms / 1e6, 1)}), flush=True)
    del src, dst, ws
    torch.cuda.empty_cache()
    for per in ["0", "4", "8", "16"]:
        os.environ["LL_GRID_PER_SM"] = per
        gather_reduce(tag=f" grid{per}", sigmas=["coalesced"])
    os.environ["LL_GRID_PER_SM"] = "0"


def gather_reduce(tag="", sigmas=("coalesced", "faithful")):
    # gather / reduce (4096 x 4096 fp32)
    for fam in ["mma", "blocked"]:
        for sig in sigmas:
            L = ll.Layout.from_spec(W.c4("gather", fam))
            p = ll.ll_plan_gather(L, 1, 4, sigma=sig)
            p.prepare()
            n = 1 << 24
            sets = [(torch.randint(-2 ** 31, 2 ** 31 - 1, (n,), dtype=torch.int32, device="cuda"),
                     torch.randint(0, 32, (n,), dtype=torch.int32, device="cuda"),
                     torch.empty(n, dtype=torch.int32, device="cuda")) for _ in range(4)]
            it = [0]

            def g():
                s = sets[it[0] % 4]
                it[0] += 1
                ll.ll_gather(s[0], s[1], s[2], p)
            ms = time_fn(g)
            print(json.dumps({"case": f"gather {fam} {sig}{tag}", "desc": p.describe(), "ms": round(ms, 4),
                              "GBps": round(12 * n / ms / 1e6, 1)}), flush=True)
        for fc in [None, "SHUFFLE"]:
            L = ll.Layout.from_spec(W.c4("reduce", fam))
            p = ll.ll_plan_reduce(L, 1, force_class=fc)
            p.prepare()
            n = 1 << 24
            sets = [(torch.rand(n, device="cuda"), torch.empty(p.out_elems(), device="cuda")) for _ in range(4)]
            it = [0]

            def r():
                s = sets[it[0] % 4]
                it[0] += 1
                ll.ll_reduce(s[0], s[1], p)
            ms = time_fn(r)
            print(json.dumps({"case": f"reduce {fam}{tag} {'tma' if p.describe()['tma'] else 'ldg'}", "ms": round(ms, 4),
                              "GBps": round((4 * n + 4 * p.out_elems()) / ms / 1e6, 1)}), flush=True)


if __name__ == "__main__":
    main()
