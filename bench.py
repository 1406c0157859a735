"""Benchmark contract for the linear-layout conversion hot path on B200.

Default workload (BASELINE.json configs[1], the config the metric is quoted on):
config 2 — a batch of 65536 independent 128x128 bf16 tiles converted from the
wgmma m64n128 accumulator layout (x2 m-repetitions) to the blocked
[8,8]/[2,16]/[4,1] layout; the planner executes it with warp shuffles.
One step = one ll_convert over the whole batch (2 GiB in, 2 GiB out).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

Multi-GPU (one rank per GPU): `--gpus N` without a torchrun environment re-launches
itself under torch.distributed.run with N ranks (127.0.0.1); under torchrun the world
size must equal --gpus.  Every rank converts its own 65536-tile batch (weak scaling, no
communication — the block bits are identical in A and B); time = max over ranks of the
CUDA-event time; value = all ranks' bytes / time (the whole-job aggregate the driver's
contract asks for), per_gpu_GBps = value / N (the metric's per-GPU figure).

Correctness: src is hash-filled (src[h] = H(A(h)), workloads/hashfill.py) and after
the timed region every one of the 2^30 dst elements per rank is compared on the device
with the closed form H(B(h)) (O5); a mismatch prints the line with verified = false and
exits 1.
"""
import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

PEAKS_PATH = os.path.join(ROOT, "MEASURED_PEAKS.json")
FALLBACK_HBM = 6650.0   # B200_PROFILING.md fallback (GB/s) if MEASURED_PEAKS.json is absent
C5_TIMEOUT_S = 300.0   # bound on the cross-GPU config-5 leg (N > 1), see main()
METRIC = "layout-conversion GB/s per GPU and % of HBM peak; smem bank conflicts/request"
WORKLOAD = ("config 2: [65536,128,128] bf16, wgmma m64n128 accumulator (x2 m-reps) -> "
            "blocked [8,8]/[2,16]/[4,1], warp-shuffle conversion, 65536 tiles")


def hbm_peak():
    try:
        with open(PEAKS_PATH) as f:
            return float(json.load(f)["hbm_gbs"]), "measured"
    except Exception:
        return FALLBACK_HBM, "fallback"


def smem_conflicts():
    """Bank conflicts per shared request of the SMEM-class kernel (config 3) from the
    committed ncu captures (the metric's second part; config 2 itself uses no smem)."""
    try:
        with open(os.path.join(ROOT, "profiles", "smem_conflicts.json")) as f:
            return json.load(f)
    except Exception:
        return None


def ncu_traffic(key):
    """Per-launch dram bytes (read + write) from the committed ncu --set full capture."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(p) as f:
            return json.load(f).get(key)
    except Exception:
        return None


class ClockSampler:
    """Samples SM clocks and clock-event reasons with NVML during the timed region."""

    REASONS = {
        0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap", 0x8: "hw_slowdown",
        0x10: "sync_boost", 0x20: "sw_thermal_slowdown", 0x40: "hw_thermal_slowdown",
        0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting",
    }

    def __init__(self, device_index):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(device_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None

    def _run(self):
        while not self._stop.is_set():
            try:
                self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
                r = self.nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit and name != "gpu_idle":
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(0.005)

    def __enter__(self):
        if self.nv:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.nv:
            self.t.join()

    def summary(self):
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "samples": len(self.samples), "reasons": sorted(self.reasons)}


def dist_env():
    return int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1)), int(os.environ.get("LOCAL_RANK", 0))


def relaunch_if_needed(args):
    """--gpus N > 1 outside torchrun: re-exec this command under torch.distributed.run
    with N ranks on 127.0.0.1.  Under torchrun: the world size must equal --gpus."""
    if "WORLD_SIZE" in os.environ:
        world = int(os.environ["WORLD_SIZE"])
        if world != args.gpus:
            sys.stderr.write(f"bench.py: WORLD_SIZE={world} but --gpus {args.gpus}\n")
            sys.exit(2)
        return
    if args.gpus <= 1:
        return
    if args.impl == "ours":
        import torch
        have = torch.cuda.device_count()
        if have < args.gpus:
            sys.stderr.write(f"bench.py: --gpus {args.gpus} but only {have} CUDA device(s) visible\n")
            sys.exit(2)
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    sys.stdout.flush()
    os.execv(sys.executable, cmd)


def _oracle_sample(threads, budget_s, tiles=256):
    """The C++17/OpenMP oracle (oracle/ll_oracle.cpp, as it stands) on a bounded sample
    of the config-2 workload: `tiles` 128x128 bf16 tiles of the same A -> B (the block
    bits are a batch index: every tile is the same conversion), repeated until
    `budget_s`.  Per element: B(h) bit by bit, then the slack-zero right inverse of A
    applied linearly, then the 2-byte copy (O5).  Returns (GB/s, elements, seconds)."""
    import numpy as np
    from oracle import cpp as OC
    from oracle import ll_oracle as O
    from workloads import configs as W
    nb = tiles.bit_length() - 1
    sa, sb = W.c2(nb)
    OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
    src = np.random.default_rng(0).integers(0, 1 << 16, size=1 << OA.d_in, dtype=np.uint16)
    out = np.empty(src.size * 2, dtype=np.uint8)
    done, t0 = 0, time.perf_counter()
    while True:
        OC.convert(OA.cols, OB.cols, OA.d_out, 2, src, threads=threads, out=out)
        done += src.size
        dt = time.perf_counter() - t0
        if dt >= budget_s:
            break
    return 2 * 2 * done / dt / 1e9, done, dt


def cpu_baseline_oracle(budget_s=10.0):
    """cpu_baseline: the C++ oracle on all host cores (os.cpu_count() OpenMP threads)
    and on one core, with the CPU model; a baseline only."""
    from oracle import cpp as OC
    ncores = os.cpu_count() or 1
    v_all, n_all, t_all = _oracle_sample(ncores, budget_s * 0.7)
    v_one, n_one, t_one = _oracle_sample(1, budget_s * 0.3)
    return {"value": round(v_all, 4), "unit": "GB/s", "cores": ncores, "kind": "oracle",
            "impl": "oracle/ll_oracle.cpp (C++17, OpenMP, g++ -O2)", "cpu_model": OC.cpu_model(),
            "sample": f"{n_all} elements ({n_all >> 14} tiles) of the config-2 batch in {t_all:.1f}s, "
                      f"pull map B(h) -> A^+ -> copy, {ncores} threads",
            "single_core": {"value": round(v_one, 4), "cores": 1,
                            "sample": f"{n_one} elements in {t_one:.1f}s, 1 thread"}}


def run_reference(args):
    """--impl reference: the oracle (C++17/OpenMP, all host cores) timed on the same
    config / metric; each step is one bounded sample of the workload (256 tiles =
    8 MiB in + 8 MiB out), and ms_per_step is that step's actual duration."""
    rank, world, _ = dist_env()
    if world > 1 and rank != 0:
        return
    from oracle import cpp as OC
    ncores = os.cpu_count() or 1
    for _ in range(args.warmup):
        _oracle_sample(ncores, 0.0)
    per = [_oracle_sample(ncores, 0.0) for _ in range(args.steps)]
    total_bytes = sum(4 * n for _, n, _ in per)
    total_s = sum(t for _, _, t in per)
    value = total_bytes / total_s / 1e9
    ms = total_s / len(per) * 1e3
    sample = f"{per[0][1]} elements (256 tiles) of the config-2 batch per step, {ncores} threads"
    line = {"metric": METRIC, "value": round(value, 4), "unit": "GB/s", "n_gpus": args.gpus, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms, 3),
            "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "bf16", "data": "synthetic", "impl": "reference",
            "config": {"workload": WORKLOAD, "elem_bytes": 2, "step": "one bounded sample: 256 of the 65536 tiles"},
            "cpu_baseline": {"value": round(value, 4), "unit": "GB/s", "cores": ncores, "kind": "oracle",
                             "cpu_model": OC.cpu_model(), "sample": sample},
            "e2e": {"value": round(value, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def _time_stream(fn, torch, samples=10, batch=20, warmup=3):
    """Median over `samples` of the time per call of `batch` back-to-back calls (CUDA
    events on the current stream); small kernels are measured as a stream."""
    for _ in range(warmup):
        fn()
    torch.cuda.synchronize()
    ts = []
    for _ in range(samples):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(batch):
            fn()
        b.record()
        b.synchronize()
        ts.append(a.elapsed_time(b) / batch)
    ts.sort()
    return ts[len(ts) // 2]


def _time_graph(fn, torch, batch=20, samples=10):
    """Median time per call of `batch` calls captured in one CUDA graph: the small
    config-4 kernels (12-31 us) without the Python launch path between them (the
    production form of a launch-bound loop; PDL edges are captured)."""
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        for _ in range(3):
            fn()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            for _ in range(batch):
                fn()
        g.replay()
        torch.cuda.synchronize()
        ts = []
        for _ in range(samples):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            g.replay()
            b.record()
            b.synchronize()
            ts.append(a.elapsed_time(b) / batch)
    ts.sort()
    return ts[len(ts) // 2]


def torch_permute_baseline(torch, A_spec, B_spec, src, w, steps=5):
    """Context for the headline: the same conversion done the way a PyTorch user would —
    the packed buffer viewed as a tensor of 2-sized dims, permuted and made contiguous
    (torch's generic strided copy).  For bijective layouts the dst packed bit k holds the
    logical bit B[k], found at src packed bit A.index(B[k]) (spec bookkeeping only);
    runs of bits that stay adjacent are merged into one dim."""
    a_bits = [b for _, bits in A_spec["in"] for b in bits]
    b_bits = [b for _, bits in B_spec["in"] for b in bits]
    perm = [a_bits.index(x) for x in b_bits]          # dst packed bit -> src packed bit
    n = len(perm)
    runs = []                                           # (src lo bit, length) in dst bit order
    k = 0
    while k < n:
        j = k
        while j + 1 < n and perm[j + 1] == perm[j] + 1:
            j += 1
        runs.append((perm[k], j - k + 1))
        k = j + 1
    src_runs = sorted(runs)                             # src dims, least significant first
    shape = [1 << ln for _, ln in reversed(src_runs)]
    dim_of = {lo: len(src_runs) - 1 - i for i, (lo, _) in enumerate(src_runs)}
    order = [dim_of[lo] for lo, _ in reversed(runs)]   # dst dims, most significant first
    et = {1: torch.uint8, 2: torch.int16, 4: torch.int32, 8: torch.int64}[w]
    x = src.view(et).view(*shape)
    xp = x.permute(*order)
    y = torch.empty(xp.shape, dtype=et, device=src.device)   # preallocated: no allocator churn

    def run():
        y.copy_(xp)                      # the strided copy permute(...).contiguous() runs
    run()
    torch.cuda.synchronize()
    ts = []
    for _ in range(steps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        run()
        b.record()
        b.synchronize()
        ts.append(a.elapsed_time(b))
    ms = sorted(ts)[len(ts) // 2]
    return {"impl": "torch: packed src viewed as %d dims, permute(...) copied into a preallocated "
                    "contiguous tensor (the strided copy of .contiguous()), median of %d" % (len(shape), steps),
            "GBps": round(2 * src.numel() * src.element_size() / (ms / 1e3) / 1e9, 1), "ms": round(ms, 4)}, \
        y.reshape(-1).view(src.dtype)


def size_matched_copy(torch, nbytes, nsets=4):
    """The copy roofline at a small problem size: torch copy_ moving `nbytes` in total
    (nbytes/2 read + nbytes/2 written), rotated over `nsets` buffer sets and timed as a
    stream like the config-4 kernels — launch ramp and tail included, as they are for
    any kernel of that size.  Context for the config-4 fractions, not the roofline."""
    n = nbytes // 8
    bufs = [(torch.empty(n, dtype=torch.int32, device="cuda"), torch.empty(n, dtype=torch.int32, device="cuda"))
            for _ in range(nsets)]
    it = [0]

    def f():
        s = bufs[it[0] % nsets]
        it[0] += 1
        s[1].copy_(s[0])
    ms = _time_stream(f, torch)
    del bufs
    return round(8 * n / ms / 1e6, 1)


def other_configs(ll, W, torch, peak):
    from workloads import hashfill
    """The other BASELINE configs (1, 3, 4, 5) measured live on this GPU, each against
    the same copy roofline: GB/s = algorithmic bytes / median time per call.  Inputs
    larger than L2, or 4 rotated buffer sets for config 4 (192 / 64.5 MiB per set)."""
    out = []

    def conv(name, sa, sb, w, comm=None, batch=5, torch_ref=True, **opts):
        A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
        p = ll.ll_plan_convert(A, B, w, comm=comm, **opts) if comm else ll.ll_plan_convert(A, B, w, **opts)
        p.prepare()
        n = 1 << A.d_in        # all ranks' slices for the loopback communicator (dev bits included)
        nb = 1 << B.d_in       # > n for broadcasting B (replicas written)
        src = hashfill.fill(sa, w, 11)
        dst = torch.empty(nb, dtype=src.dtype, device="cuda")
        ms = _time_stream(lambda: ll.ll_convert(src, dst, p), torch, batch=batch)
        d = p.describe()
        gbs = (n + nb) * w / ms / 1e6   # algorithmic: src read once + every dst element written
        if "tile" in d:
            ex = d["tile"]["xchg"]
        elif d.get("exchange") == "peer":
            ex = "peer stores: %s tile kernel into the receivers' windows" % d["fused"]["tile"]["xchg"]
        else:
            ex = d["exec"]
        entry = {"workload": name, "class": d["class"], "executed": ex, "ms": round(ms, 4),
                 "GBps": round(gbs, 1), "frac": round(gbs / peak, 3),
                 "verified": hashfill.check(sb, w, 11, dst) == 0}
        if "tile" in d and d["tile"]["xchg"] == "smem":     # Thm 5.1 instruction choice
            entry["smem_instructions"] = [d["tile"]["smem_store"], d["tile"]["smem_load"]]
        if comm is None and torch_ref:
            tb, y = torch_permute_baseline(torch, sa, sb, src, w)
            entry["torch_permute_GBps"] = tb["GBps"]
            entry["torch_permute_matches"] = bool(torch.equal(y.view(dst.dtype), dst))
            del y
        out.append(entry)
        del src, dst

    # config 1 single tile: latency of one conversion in a CUDA graph of 1000
    A, B = ll.Layout.from_spec(W.C1_A), ll.Layout.from_spec(W.C1_B)
    p1 = ll.ll_plan_convert(A, B, 4)
    p1.prepare()
    s1 = torch.zeros(256, dtype=torch.int32, device="cuda")
    d1 = torch.empty_like(s1)
    st = torch.cuda.Stream()
    with torch.cuda.stream(st):
        ll.ll_convert(s1, d1, p1, st)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            for _ in range(1000):
                ll.ll_convert(s1, d1, p1, st)
    ms = _time_stream(g.replay, torch, batch=1)
    out.append({"workload": "config 1: one 16x16 fp32 tile (2 warps), 1000 conversions in a CUDA graph",
                "class": p1.cls, "us_per_conversion": round(ms, 4)})
    conv("config 1 batch: 2^20 Fig.-1 tiles (16x16 fp32, A -> B = A^T), 1+1 GiB", *W.c1_batched(20), 4)
    conv("config 3: 16384 tiles 256x128 fp16 blocked -> transposed blocked (optimal swizzle), 1+1 GiB", *W.c3(14), 2)
    conv("config 3b: 16384 tiles 256x128 fp16, [8,8] per thread row- -> column-order (16-byte rows via stmatrix), 1+1 GiB",
         *W.c3b(14), 2)
    conv("config 5-T, P=1: 32768^2 bf16 row-major -> column-major, 2+2 GiB", *W.c5T(0), 2)
    conv("config 5, P=8 loopback on one GPU: row- -> column-sharded, peer-store kernels, 2+2 GiB",
         *W.c5(3), 2, comm=ll.Comm.loopback(8), exchange="peer")
    # §8(f) next rows: N1 (HBM operand pre-shuffle), N2 (Blackwell TMEM fragments ->
    # coalesced epilogue; chained-GEMM accumulator -> register-A operand), broadcast
    conv("N1: [32768,32768] bf16 row-major -> mma m16n8k16 rhs fragment order (HBM pre-shuffle), 2+2 GiB",
         *W.n1_preshuffle(15, 15), 2)
    for shape in ("32x32b", "16x64b", "16x128b", "16x256b"):
        conv(f"N2: 16384 tiles 128x128 fp32 tcgen05.ld.{shape} fragment -> blocked epilogue layout, 1+1 GiB",
             *W.n2_tmem(shape, 14), 4)
    conv("N2: 2^18 tiles 64x64 wgmma accumulator -> fp8 register-A operand of the next wgmma, 1+1 GiB",
         *W.n2_acc_to_lhs(8, 18), 1)
    conv("N2: 2^17 tiles 64x64 wgmma accumulator -> bf16 register-A operand (equal layouts), 1+1 GiB",
         *W.n2_acc_to_lhs(16, 17), 2)
    import numpy as np
    from workloads import gen
    sa_b, sb_b = gen.random_broadcast_pair(np.random.default_rng(908), 8, ki=5, kj=5, batch_bits=11)
    conv("broadcast: bijective A -> B with 8 zero columns (256 replicas), 8 MiB in + 2 GiB out, fp32",
         sa_b, sb_b, 4, torch_ref=False)
    # config 4: gather and reduce, [4096, 4096] fp32 in [128, K=32] / [128, 128] tiles
    for fam in ("mma", "blocked"):
        L = ll.Layout.from_spec(W.c4("gather", fam))
        p = ll.ll_plan_gather(L, 1, 4)
        n = 1 << L.d_in
        sets = [(torch.randint(-2 ** 31, 2 ** 31 - 1, (n,), dtype=torch.int32, device="cuda"),
                 torch.randint(0, 32, (n,), dtype=torch.int32, device="cuda"),
                 torch.empty(n, dtype=torch.int32, device="cuda")) for _ in range(4)]
        it = [0]

        def g1():
            s = sets[it[0] % 4]
            it[0] += 1
            ll.ll_gather(s[0], s[1], s[2], p)
        ms = _time_stream(g1, torch)
        gms = _time_graph(g1, torch)
        d = p.describe()
        gbs = 12 * n / ms / 1e6
        # context: PyTorch's own gather on the logical [4096*128, 32] view, same bytes,
        # same 4-set rotation (a library kernel for the op, not the roofline)
        tsets = [(s[0].view(-1, 32), s[1].view(-1, 32).to(torch.int64) & 31, s[2].view(-1, 32)) for s in sets]

        def tg():
            s = tsets[it[0] % 4]
            it[0] += 1
            torch.gather(s[0], 1, s[1], out=s[2])
        ms_t = _time_stream(tg, torch)
        out.append({"workload": f"config 4 gather: [4096,4096] fp32, {fam} [128,32] tiles", "class": "gather",
                    "executed": d["exchange"] + (" (TMA stages)" if d.get("tma") else ""), "ms": round(ms, 4),
                    "shuffles_per_elem": d.get("shuffles_per_elem"),
                    "GBps": round(gbs, 1), "frac": round(gbs / peak, 3),
                    "graph_GBps": round(12 * n / gms / 1e6, 1), "graph_frac": round(12 * n / gms / 1e6 / peak, 3),
                    "torch_gather_same_bytes_GBps": round(12 * n / ms_t / 1e6, 1),
                    "size_matched_copy_GBps": size_matched_copy(torch, 12 * n)})
        del tsets
        L = ll.Layout.from_spec(W.c4("reduce", fam))
        p = ll.ll_plan_reduce(L, 1)
        rsets = [(torch.rand(n, device="cuda"), torch.empty(p.out_elems(), device="cuda")) for _ in range(4)]

        def r1():
            s = rsets[it[0] % 4]
            it[0] += 1
            ll.ll_reduce(s[0], s[1], p)
        ms = _time_stream(r1, torch)
        gms = _time_graph(r1, torch)
        gbs = (4 * n + 4 * p.out_elems()) / ms / 1e6
        ggbs = (4 * n + 4 * p.out_elems()) / gms / 1e6

        # context: PyTorch's own sum over the logical [4096, 32, 128] view (same bytes)
        def tr():
            s = rsets[it[0] % 4]
            it[0] += 1
            torch.sum(s[0].view(4096, 32, 128), dim=2, out=s[1].view(4096, 32))
        ms_t = _time_stream(tr, torch)
        out.append({"workload": f"config 4 reduce: [4096,4096] fp32 -> [4096,32], {fam} [128,128] tiles",
                    "class": "reduce", "executed": "logical-order steps (register / shfl.bfly / smem)" + (" (TMA stages)" if p.describe().get("tma") else ""),
                    "ms": round(ms, 4), "GBps": round(gbs, 1), "frac": round(gbs / peak, 3),
                    "graph_GBps": round(ggbs, 1), "graph_frac": round(ggbs / peak, 3),
                    "torch_sum_same_bytes_GBps": round((4 * n + 4 * p.out_elems()) / ms_t / 1e6, 1),
                    "size_matched_copy_GBps": size_matched_copy(torch, 4 * n + 4 * p.out_elems())})
        # scan (N3): inclusive prefix sum along the axis inside each [128, 128] tile
        p = ll.ll_plan_scan(L, 1)
        ssets = [(rs[0], torch.empty_like(rs[0])) for rs in rsets]

        def s1():
            s = ssets[it[0] % 4]
            it[0] += 1
            ll.ll_scan(s[0], s[1], p)
        ms = _time_stream(s1, torch)
        gms = _time_graph(s1, torch)
        gbs = 8 * n / ms / 1e6

        def ts():
            s = ssets[it[0] % 4]
            it[0] += 1
            torch.cumsum(s[0].view(4096, 32, 128), dim=2, out=s[1].view(4096, 32, 128))
        ms_t = _time_stream(ts, torch)
        d = p.describe()
        out.append({"workload": f"config 4 scan (N3): [4096,4096] fp32 inclusive prefix sum inside {fam} [128,128] tiles",
                    "class": "scan", "executed": f"{d['steps']} bit-doubling steps, {d['shuffles_per_elem']} shuffles/elem",
                    "ms": round(ms, 4), "GBps": round(gbs, 1), "frac": round(gbs / peak, 3),
                    "graph_GBps": round(8 * n / gms / 1e6, 1), "graph_frac": round(8 * n / gms / 1e6 / peak, 3),
                    "torch_cumsum_same_bytes_GBps": round(8 * n / ms_t / 1e6, 1),
                    "size_matched_copy_GBps": size_matched_copy(torch, 8 * n)})
        del sets, rsets, ssets
    torch.cuda.empty_cache()
    # the same gather / reduce / scan kernels at 1 GiB of input (2^28 fp32, [32768, 8192]
    # in the same tiles): their own ceiling, free of the small problem's launch / ramp
    for fam in ("mma", "blocked"):
        L = ll.Layout.from_spec(W.c4("gather", fam, n_i=15, n_j=13))
        p = ll.ll_plan_gather(L, 1, 4)
        n = 1 << L.d_in
        s0 = torch.randint(-2 ** 31, 2 ** 31 - 1, (n,), dtype=torch.int32, device="cuda")
        i0 = torch.randint(0, 32, (n,), dtype=torch.int32, device="cuda")
        o0 = torch.empty(n, dtype=torch.int32, device="cuda")
        ms = _time_stream(lambda: ll.ll_gather(s0, i0, o0, p), torch, batch=3)
        out.append({"workload": f"config 4 gather at 1 GiB: [32768,8192] fp32, {fam} [128,32] tiles", "class": "gather",
                    "ms": round(ms, 4), "GBps": round(12 * n / ms / 1e6, 1), "frac": round(12 * n / ms / 1e6 / peak, 3)})
        del s0, i0, o0
        L = ll.Layout.from_spec(W.c4("reduce", fam, n_i=15, n_j=13))
        p = ll.ll_plan_reduce(L, 1)
        s0 = torch.rand(n, device="cuda")
        o0 = torch.empty(p.out_elems(), device="cuda")
        ms = _time_stream(lambda: ll.ll_reduce(s0, o0, p), torch, batch=3)
        gbs = (4 * n + 4 * p.out_elems()) / ms / 1e6
        out.append({"workload": f"config 4 reduce at 1 GiB: [32768,8192] fp32 -> [32768,64], {fam} [128,128] tiles",
                    "class": "reduce", "ms": round(ms, 4), "GBps": round(gbs, 1), "frac": round(gbs / peak, 3)})
        p = ll.ll_plan_scan(L, 1)
        o1 = torch.empty_like(s0)
        ms = _time_stream(lambda: ll.ll_scan(s0, o1, p), torch, batch=3)
        out.append({"workload": f"config 4 scan at 1 GiB: [32768,8192] fp32, {fam} [128,128] tiles", "class": "scan",
                    "ms": round(ms, 4), "GBps": round(8 * n / ms / 1e6, 1), "frac": round(8 * n / ms / 1e6 / peak, 3)})
        del s0, o0, o1
        torch.cuda.empty_cache()
    return out


def config5_exchange(ll, W, torch, world, rank, steps=10, warmup=3):
    """Config 5 across the GPUs of this job (N > 1, N a power of two): a [32768, 32768]
    bf16 tensor row-sharded over N ranks, redistributed to column-sharded — the DEVICE
    class over NVLink, with both exchanges: the collective decomposition (pack ->
    grouped ncclSend/ncclRecv -> unpack) and the fused peer-store kernel writing into
    the receivers' windows (CUDA IPC).  Time = max over ranks of CUDA-event time per
    conversion; errors are reported, not raised, so the main line still prints."""
    import torch.distributed as dist
    p = world.bit_length() - 1
    total = 1 << 30
    nloc = total // world
    sa, sb = W.c5(p)
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    src = torch.randint(-2 ** 15, 2 ** 15, (nloc,), dtype=torch.int16, device="cuda")
    dst = torch.empty_like(src)
    flags = torch.zeros(ll.PEER_FLAG_BYTES // 4, dtype=torch.int32, device="cuda")
    out = {"workload": f"config 5: [32768,32768] bf16 row-sharded -> column-sharded over {world} GPUs",
           "bytes_per_gpu_each_way_nvlink": int((world - 1) * nloc * 2 // world)}
    for exchange in ("collective", "peer"):
        try:
            comm = ll.Comm.from_process_group() if exchange == "collective" else ll.Comm.peers(dst, flags)
            plan = ll.ll_plan_convert(A, B, 2, comm=comm, exchange=exchange)
            plan.prepare()
            ws = torch.empty(max(16, plan.workspace_bytes()), dtype=torch.uint8, device="cuda")
            for _ in range(warmup):
                ll.ll_convert(src, dst, plan, workspace=ws)
            torch.cuda.synchronize()
            dist.barrier()
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            for _ in range(steps):
                ll.ll_convert(src, dst, plan, workspace=ws)
            b.record()
            torch.cuda.synchronize()
            t = torch.tensor([a.elapsed_time(b) / steps], device="cuda", dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ms = float(t.item())
            nvl = out["bytes_per_gpu_each_way_nvlink"]
            out[exchange] = {"ms": round(ms, 4), "aggregate_GBps": round(2 * total * 2 / (ms / 1e3) / 1e9, 1),
                             "nvlink_GBps_per_gpu_each_way": round(nvl / (ms / 1e3) / 1e9, 1),
                             # roofline: the measured 770 GB/s peer copy per direction (B200_PROFILING.md);
                             # the nominal 900 is context only
                             "frac_of_measured_770": round(nvl / (ms / 1e3) / 1e9 / 770, 3),
                             "frac_of_nominal_900": round(nvl / (ms / 1e3) / 1e9 / 900, 3),
                             "class": plan.cls, "exchange": plan.describe().get("exchange")}
            del plan, comm, ws
        except Exception as e:  # noqa: BLE001 - reported in the JSON line
            out[exchange] = {"error": f"{type(e).__name__}: {str(e)[:200]}"}
    del src, dst
    torch.cuda.empty_cache()
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=3)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-configs", action="store_true", help="skip the other BASELINE configs (N=1 only)")
    ap.add_argument("--no-config5", action="store_true", help="skip the cross-GPU config-5 exchange (N>1 only)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    relaunch_if_needed(args)
    if args.impl == "reference":
        return run_reference(args)

    import numpy as np
    import torch
    import paper_conf_asplos_0001cgrnls0trm26_b200 as ll
    from workloads import configs as W

    rank, world, local = dist_env()
    torch.cuda.set_device(local)
    if world > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    A_spec, B_spec = W.c2(16)
    A, B = ll.Layout.from_spec(A_spec), ll.Layout.from_spec(B_spec)
    plan = ll.ll_plan_convert(A, B, 2)
    plan.prepare()
    desc = plan.describe()
    w = 2
    n = 1 << A.d_in                       # 2^30 elements per rank
    bytes_per_step = 2 * n * w            # algorithmic: read + write each element once
    from workloads import hashfill
    seed = 1002 + rank
    src = hashfill.fill(A_spec, w, seed)                 # src[h] = H(A(h)): checkable at every element
    dst = torch.empty_like(src)
    stream = torch.cuda.current_stream()

    def barrier():
        if world > 1:
            torch.distributed.barrier()

    for _ in range(args.warmup):
        ll.ll_convert(src, dst, plan, stream)
    torch.cuda.synchronize()
    barrier()
    torch.cuda.synchronize()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    with ClockSampler(local) as clk:
        t_start = torch.cuda.Event(enable_timing=True)
        t_end = torch.cuda.Event(enable_timing=True)
        t_start.record(stream)
        for i in range(args.steps):
            evs[i][0].record(stream)
            ll.ll_convert(src, dst, plan, stream)
            evs[i][1].record(stream)
        t_end.record(stream)
        torch.cuda.synchronize()
    barrier()
    torch.cuda.synchronize()
    total_ms = t_start.elapsed_time(t_end)
    launch_ms = [a.elapsed_time(b) for a, b in evs]
    # every element of the last timed step's output against the closed form H(B(h))
    bad = hashfill.check(B_spec, w, seed, dst)
    tb_ = torch.tensor([bad], device="cuda", dtype=torch.int64)
    if world > 1:
        torch.distributed.all_reduce(tb_)
    bad = int(tb_.item())
    t = torch.tensor([total_ms], device="cuda", dtype=torch.float64)
    if world > 1:
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
    total_ms = float(t.item())
    ms_per_step = total_ms / args.steps
    value = world * bytes_per_step * args.steps / (total_ms / 1e3) / 1e9

    # ---- context for the roofline: the library's own NOOP plan (A -> A) on the same
    # 2+2 GiB runs ll_copy_kernel, a plain streaming copy in the tile kernels' shape —
    # the practical read+write ceiling of a kernel on this GPU (the measured peak in
    # MEASURED_PEAKS.json is a driver copy)
    pc = ll.ll_plan_convert(A, A, 2)
    ceil_ms = _time_stream(lambda: ll.ll_convert(src, dst, pc, stream), torch, samples=5)
    ceil_gbs = bytes_per_step / (ceil_ms / 1e3) / 1e9
    del pc

    # ---- end to end through the C-ABI call with HOST buffers (ll_convert_host): per
    # step the pinned host input is copied in, converted and copied back, chunked over
    # two streams so that H2D, kernels and D2H of different chunks overlap
    h_src = torch.empty(n, dtype=torch.int16, pin_memory=True)
    h_src.copy_(src, non_blocking=False)
    h_dst = torch.empty(n, dtype=torch.int16, pin_memory=True)
    dev_buf = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")   # 2 slots x 512 MiB
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    torch.cuda.synchronize()
    barrier()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(streams[0])
    streams[1].wait_event(e0)
    for _ in range(args.e2e_steps):
        ll.ll_convert_host(h_src, h_dst, dev_buf, plan, streams)
    ev = torch.cuda.Event()
    ev.record(streams[1])
    streams[0].wait_event(ev)
    e1.record(streams[0])
    torch.cuda.synchronize()
    e2e_ms = e0.elapsed_time(e1) / args.e2e_steps
    te = torch.tensor([e2e_ms], device="cuda", dtype=torch.float64)
    if world > 1:
        torch.distributed.all_reduce(te, op=torch.distributed.ReduceOp.MAX)
    e2e_ms = float(te.item())
    # the host-buffer run must produce the device run's bytes
    ll.ll_convert(src, dst, plan, stream)
    torch.cuda.synchronize()
    ok_e2e = hashfill.check(B_spec, w, seed, h_dst.cuda()) == 0      # every element of the host result
    # the host link's own limit for the same traffic: concurrent H2D + D2H of the same
    # bytes with plain pinned copies on two streams (torch), timed the same way
    d_tmp = torch.empty_like(src)
    l0, l1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    l0.record(streams[0])
    streams[1].wait_event(l0)
    for _ in range(args.e2e_steps):
        with torch.cuda.stream(streams[0]):
            d_tmp.copy_(h_src, non_blocking=True)
        with torch.cuda.stream(streams[1]):
            h_dst.copy_(dst, non_blocking=True)
    evl = torch.cuda.Event()
    evl.record(streams[1])
    streams[0].wait_event(evl)
    l1.record(streams[0])
    torch.cuda.synchronize()
    link_ms = l0.elapsed_time(l1) / args.e2e_steps
    del d_tmp
    del dev_buf
    if rank == 0:
        peak, peak_kind = hbm_peak()
        avg_launch_ms = statistics.mean(launch_ms)
        achieved = bytes_per_step / (avg_launch_ms / 1e3) / 1e9
        traffic = ncu_traffic("c2_shuffle")
        line = {
            "metric": METRIC, "value": round(value, 1), "unit": "GB/s", "n_gpus": world, "steps": args.steps,
            "per_gpu_GBps": round(value / world, 1),
            "value_note": "value = whole-job aggregate GB/s over all ranks (driver contract); per_gpu_GBps = value / n_gpus",
            "verified": {"ok": bad == 0, "elements_checked": world * n, "mismatches": bad,
                         "how": "every dst element vs the closed form H(B(h)) of hash-filled src (O5), on the device"},
            "warmup": args.warmup, "ms_per_step": round(ms_per_step, 5), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
            "config": {"workload": WORKLOAD, "tiles_per_gpu": 65536, "elem_bytes": w,
                       "bytes_per_step_per_gpu": bytes_per_step, "class": desc["class"],
                       "executed": desc["tile"]["xchg"], "shuffle_rounds": desc["tile"].get("rounds"),
                       "threads_per_cta": desc["tile"]["threads"], "ctas": desc["tile"]["ctas"],
                       "l2": "inputs 2 GiB/GPU > 126 MB L2 (no flush needed)",
                       "parallelism": f"dp{world} (independent tiles, no communication)"},
            "roofline": {"bound": "hbm", "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                         "frac": round(achieved / peak, 4), "peak_kind": peak_kind,
                         "frac_of_nominal_8TBps": round(achieved / 8000.0, 4),
                         "traffic": traffic, "kernel": "ll_tile_kernel (shuffle)",
                         "traffic_over_algorithmic": round(traffic / bytes_per_step, 4) if traffic else None,
                         "bytes_per_launch": bytes_per_step, "avg_launch_ms": round(avg_launch_ms, 5),
                         "streaming_ceiling": {"GBps": round(ceil_gbs, 1), "frac": round(achieved / ceil_gbs, 4),
                                               "kernel": "ll_copy_kernel (NOOP plan A -> A, same 2+2 GiB, "
                                                         "streams of 20 launches)"}},
            "e2e": {"value": round(world * bytes_per_step / (e2e_ms / 1e3) / 1e9, 2), "unit": "GB/s",
                    "h2d_bytes_per_step": n * w, "d2h_bytes_per_step": n * w, "ms_per_step": round(e2e_ms, 3),
                    "api": "ll_convert_host (chunked H2D -> kernel -> D2H over 2 streams)",
                    "matches_device_run": ok_e2e,
                    "host_link_GBps": round(2 * n * w / (link_ms / 1e3) / 1e9, 2),
                    "frac_of_host_link": round(link_ms / e2e_ms, 3),
                    "host_link": "plain pinned H2D + D2H of the same bytes, concurrent on two streams"},
            "gpu_launches": args.steps,
            "smem_bank_conflicts": smem_conflicts(),
            "clocks": clk.summary(),
        }
        if world == 1 and not args.no_configs:
            # the library baseline must produce the same bytes as our kernel
            tb, y = torch_permute_baseline(torch, A_spec, B_spec, src, w)
            tb["matches"] = bool(torch.equal(y, dst))
            line["torch_baseline"] = tb
            del y
            del src, dst
            torch.cuda.empty_cache()
            line["configs"] = other_configs(ll, W, torch, peak)
        if world == 1 and not args.no_cpu_baseline:   # the oracle baseline: rank 0 at N=1 only
            line["cpu_baseline"] = cpu_baseline_oracle()
    if world > 1 and (world & (world - 1)) == 0 and not args.no_config5:
        # config 5 across the GPUs (NCCL + peer windows).  A watchdog on every rank bounds
        # it: should any rank stall in the exchange, rank 0 still prints the main line
        # (config5_nvlink = the timeout) and every rank exits instead of hanging the job.
        def _stalled():
            if rank == 0:
                line["config5_nvlink"] = {"error": f"timeout after {C5_TIMEOUT_S} s (exchange stalled)"}
                print(json.dumps(line), flush=True)
            os._exit(1 if bad else 0)
        dog = threading.Timer(C5_TIMEOUT_S, _stalled)
        dog.daemon = True
        dog.start()
        c5 = config5_exchange(ll, W, torch, world, rank)
        dog.cancel()
        if rank == 0:
            line["config5_nvlink"] = c5
    if rank == 0:
        print(json.dumps(line), flush=True)
    if world > 1:
        torch.distributed.destroy_process_group()
    if bad:
        sys.exit(1)


if __name__ == "__main__":
    main()
