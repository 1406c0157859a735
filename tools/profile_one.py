"""Run one hot-path kernel a few times (for ncu captures): --case c2 | c2smem | c3 |
c3b | c1b | c1bsmem | c5T | n1 | n2 | c5peer | gather_mma | gather_blocked | reduce_mma |
reduce_blocked."""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_asplos_0001cgrnls0trm26_b200 as ll  # noqa: E402
from workloads import configs as W  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--case", default="c2")
ap.add_argument("--iters", type=int, default=3)
ap.add_argument("--opts", default="{}", help="extra ll_plan_convert options as JSON")
a = ap.parse_args()

conv = {"c2": (W.c2(16), 2, {}), "c2smem": (W.c2(16), 2, {"force_class": "SMEM"}),
        "c3": (W.c3(14), 2, {}), "c3b": (W.c3b(14), 2, {}), "c1b": (W.c1_batched(20), 4, {}),
        "c1bsmem": (W.c1_batched(20), 4, {"force_class": "SMEM"}),
        # small variants for compute-sanitizer
        "c1bsmem_small": (W.c1_batched(6), 4, {"force_class": "SMEM"}),
        "c3_small": (W.c3(3), 2, {}), "c3_mid_pipe": (W.c3(9), 2, {"pipe": "on"}), "c2_small": (W.c2(3), 2, {}),
        "c3b_small": (W.c3b(3), 2, {}),
        # NOOP plans (ll_copy_kernel): a partial last CTA tile, and the 2 GiB copy
        "noop_small": (W.n2_acc_to_lhs(16, 3), 2, {}), "noop": (W.n2_acc_to_lhs(16, 17), 2, {}),
        "acc8_small": (W.n2_acc_to_lhs(8, 4), 1, {}), "acc8f_small": (W.n2_acc_to_lhs(8, 4), 1, {"sigma": "faithful"}),
        "c2fsmem_small": (W.c2(3), 2, {"sigma": "faithful", "force_class": "SMEM", "smem_instr": "matrix"}),
        "c3f_small": (W.c3(3), 2, {"sigma": "faithful"}),
        "c5T": (W.c5T(0, n=15), 2, {}), "n1": (W.n1_preshuffle(14, 14), 2, {}),
        "n2": (W.n2_tmem_epilogue(13), 4, {}),
        "n2_16x128b": (W.n2_tmem("16x128b", 14), 4, {}), "n2_16x256b": (W.n2_tmem("16x256b", 14), 4, {}),
        # Thm 5.1: stmatrix / ldmatrix vs vectorised ld/st.shared only
        "c3bvec": (W.c3b(14), 2, {"smem_instr": "vec"}),
        "c2fsmem": (W.c2(16), 2, {"sigma": "faithful", "force_class": "SMEM", "smem_instr": "matrix"}),
        "c2fsmemvec": (W.c2(16), 2, {"sigma": "faithful", "force_class": "SMEM", "smem_instr": "vec"}),
        "c3f": (W.c3(14), 2, {"sigma": "faithful"}),
        "c3fvec": (W.c3(14), 2, {"sigma": "faithful", "smem_instr": "vec"})}
if a.case.startswith("t4_"):
    # t4_<reduce|scan|gather>_<blocked|mma|custom>_<a>_<b>_<axis>: a Table 4 family tile
    # times 8 CTAs, default plan plus --opts (sanitizer runs of the default load paths)
    import json as _json
    import numpy as np
    from workloads import gen
    _, kind, fam, ta, tb, ax = a.case.split("_")
    ta, tb, ax = int(ta), int(tb), int(ax)
    if fam == "blocked":
        T = ll.ll_layout_blocked([ta, tb], [1, 4], [8, 4], [4, 1], [1, 0])
    elif fam == "mma":
        T = ll.ll_layout_mma_acc(ta, tb, 4)
    else:
        T = ll.Layout.from_spec(gen.random_distributed(
            np.random.default_rng(77), [("r", ta.bit_length() - 1), ("c", tb.bit_length() - 1)],
            [("reg", max(1, ta.bit_length() + tb.bit_length() - 2 - 7)), ("lane", 5), ("warp", 2)],
            zero_ok=["reg", "lane", "warp"] if kind != "gather" else []))
    vecs, bases, k = T.bases(), {}, 0
    for nm, nb in T.in_dims:
        bases[nm] = [(0,) + tuple(v) for v in vecs[k:k + nb]]
        k += nb
    bases["block"] = [(1, 0, 0), (2, 0, 0), (4, 0, 0)]
    L = ll.Layout(list(T.in_dims) + [("block", 3)], [("b", 3)] + list(T.out_dims), bases)
    n = 1 << L.d_in
    o = _json.loads(a.opts)
    s = torch.rand(n, device="cuda")
    if kind == "gather":
        p = ll.ll_plan_gather(L, ax + 1, 4, **o)
        K = (ta, tb)[ax]
        i = torch.randint(0, K, (n,), dtype=torch.int32, device="cuda")
        d = torch.empty_like(s)
        run = lambda: ll.ll_gather(s, i, d, p)   # noqa: E731
    elif kind == "scan":
        p = ll.ll_plan_scan(L, ax + 1, **o)
        d = torch.empty_like(s)
        run = lambda: ll.ll_scan(s, d, p)   # noqa: E731
    else:
        p = ll.ll_plan_reduce(L, ax + 1, **o)
        d = torch.empty(p.out_elems(), device="cuda")
        run = lambda: ll.ll_reduce(s, d, p)   # noqa: E731
    print(p.describe())
    for _ in range(a.iters):
        run()
elif a.case.startswith("bcast"):
    # the bench's broadcast row: random bijective A -> B with 8 zero columns (seed 908)
    import numpy as np
    from workloads import gen
    # bcast<seed>: the bench size (8 MiB -> 2 GiB); bcastS<seed>: 2 batch bits (sanitizer size)
    # bcastC<seed>: small, with permuted block bits (CTA class)
    small = a.case.startswith("bcastS") or a.case.startswith("bcastC")
    seed = int(a.case[6:] if small else a.case[5:] or 908)
    sa, sb = gen.random_broadcast_pair(np.random.default_rng(seed), 8 if not small else 5, ki=5, kj=5,
                                       batch_bits=2 if small else 11, permute_batch=a.case.startswith("bcastC"))
    import json
    p = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), 4, **json.loads(a.opts))
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    src = torch.randint(-2 ** 31, 2 ** 31 - 1, (1 << A.d_in,), dtype=torch.int32, device="cuda")
    dst = torch.empty(1 << B.d_in, dtype=torch.int32, device="cuda")
    for _ in range(a.iters):
        ll.ll_convert(src, dst, p)
    torch.cuda.synchronize()
elif a.case == "c5peer":
    # config 5 at P = 8 on one GPU (loopback): one peer-store tile kernel per virtual rank
    sa, sb = W.c5(3)
    p = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), 2, comm=ll.Comm.loopback(8),
                           exchange="peer")
    src = torch.randint(-2 ** 15, 2 ** 15, (1 << 30,), dtype=torch.int16, device="cuda")
    dst = torch.empty_like(src)
    for _ in range(a.iters):
        ll.ll_convert(src, dst, p)
elif a.case in conv:
    (sa, sb), w, opts = conv[a.case]
    import json
    opts = dict(opts, **json.loads(a.opts))
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    p = ll.ll_plan_convert(A, B, w, **opts)
    n = (1 << A.d_in) * w // 2
    src = torch.randint(-2 ** 15, 2 ** 15, (n,), dtype=torch.int16, device="cuda")
    dst = torch.empty_like(src)
    for _ in range(a.iters):
        ll.ll_convert(src, dst, p)
elif a.case.startswith("r2small_") or a.case.startswith("r2mid_"):
    # a 2^16 (2^21) element random R2 map (linear tile, pipelined; compute-sanitizer size)
    import numpy as np
    from workloads import gen
    w = int(a.case.split("_")[1])
    rng = np.random.default_rng(77)
    d = 16 if a.case.startswith("r2small_") else 21
    ca, cb = gen.random_memory_cols(rng, d), gen.random_memory_cols(rng, d)
    A = ll.Layout([("offset", d)], [("x", d)], {"offset": [(c,) for c in ca]})
    B = ll.Layout([("offset", d)], [("x", d)], {"offset": [(c,) for c in cb]})
    import json
    p = ll.ll_plan_convert(A, B, w, **json.loads(a.opts))
    print(json.dumps({k: p.describe()["tile"].get(k) for k in ("linear_tile", "pipe", "min_blocks", "ctas")}))
    src = torch.randint(-2 ** 15, 2 ** 15, ((1 << d) * w // 2,), dtype=torch.int16, device="cuda")
    dst = torch.empty_like(src)
    for _ in range(a.iters):
        ll.ll_convert(src, dst, p)
    torch.cuda.synchronize()
elif a.case.startswith("r2_"):
    # random R2 memory layouts of 2^28 elements, as tools/sweep.py --only generic: r2_<w>_<i>
    import numpy as np
    from workloads import gen
    _, wq, iq = a.case.split("_")
    rng = np.random.default_rng(5)
    d = 28
    for w in (2, 4):
        for i in range(3):
            ca, cb = gen.random_memory_cols(rng, d), gen.random_memory_cols(rng, d)
            if w == int(wq) and i == int(iq):
                A = ll.Layout([("offset", d)], [("x", d)], {"offset": [(c,) for c in ca]})
                B = ll.Layout([("offset", d)], [("x", d)], {"offset": [(c,) for c in cb]})
                p = ll.ll_plan_convert(A, B, w)
                src = torch.randint(-2 ** 15, 2 ** 15, ((1 << d) * w // 2,), dtype=torch.int16, device="cuda")
                dst = torch.empty_like(src)
                for _ in range(a.iters):
                    ll.ll_convert(src, dst, p)
elif a.case.startswith("scan"):
    # scan_<fam>[_1g]: config-4 scan, or at 1 GiB ([32768, 8192])
    parts = a.case.split("_")
    fam = parts[1]
    big = len(parts) > 2 and parts[2] == "1g"
    spec = W.c4("reduce", fam, n_i=15, n_j=13) if big else W.c4("reduce", fam)
    L = ll.Layout.from_spec(spec)
    p = ll.ll_plan_scan(L, 1)
    s = torch.rand(1 << L.d_in, device="cuda")
    d = torch.empty_like(s)
    for _ in range(a.iters):
        ll.ll_scan(s, d, p)
elif a.case.startswith("gather") and a.case.endswith("_1g"):
    fam = a.case.split("_")[1]
    L = ll.Layout.from_spec(W.c4("gather", fam, n_i=15, n_j=13))
    p = ll.ll_plan_gather(L, 1, 4)
    n = 1 << L.d_in
    s = torch.randint(0, 1 << 30, (n,), dtype=torch.int32, device="cuda")
    i = torch.randint(0, 32, (n,), dtype=torch.int32, device="cuda")
    d = torch.empty_like(s)
    for _ in range(a.iters):
        ll.ll_gather(s, i, d, p)
elif a.case.startswith("gather"):
    parts = a.case.split("_")
    fam = parts[1]
    kb = int(parts[2]) if len(parts) > 2 else 5
    small = len(parts) > 3
    spec = W.c4("gather", fam, k_bits=kb) if not small else W.c4("gather", fam, n_i=9, n_j=8, k_bits=kb)
    p = ll.ll_plan_gather(ll.Layout.from_spec(spec), 1, 4)
    n = 1 << (24 if not small else 17)
    s = torch.randint(0, 1 << 30, (n,), dtype=torch.int32, device="cuda")
    i = torch.randint(0, 32, (n,), dtype=torch.int32, device="cuda")
    d = torch.empty_like(s)
    for _ in range(a.iters):
        ll.ll_gather(s, i, d, p)
else:
    parts = a.case.split("_")
    fam = parts[1]
    small = len(parts) > 2
    spec = W.c4("reduce", fam) if not small else W.c4("reduce", fam, n_i=9, n_j=9)
    p = ll.ll_plan_reduce(ll.Layout.from_spec(spec), 1)
    s = torch.rand(1 << (24 if not small else 18), device="cuda")
    d = torch.empty(p.out_elems(), device="cuda")
    for _ in range(a.iters):
        ll.ll_reduce(s, d, p)
torch.cuda.synchronize()
print("done", a.case)
