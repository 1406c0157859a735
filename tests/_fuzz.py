"""Seeded random conversion cases for fuzzing the planner + kernels against the oracle.

No layout arithmetic: random layouts come from workloads.gen (literal specs or
column lists) and are returned as (in_dims, out_dims, bases) triples that both the
product (ll.Layout) and the oracle (O.Layout) ingest with their own constructors.
Each case: (tag, layout_A, layout_B, elem_bytes, opts)."""
from workloads import configs as W
from workloads import gen

OPTION_SETS = [
    {}, {}, {},                                  # the default plan most often
    {"sigma": "faithful"},
    {"force_class": "SMEM"},
    {"force_class": "SMEM", "smem_instr": "matrix"},
    {"force_class": "SMEM", "smem_instr": "vec"},
    {"sigma": "faithful", "force_class": "SMEM", "smem_instr": "matrix"},
    {"thread_bytes": 64},
    {"thread_bytes": 128, "tile_bytes": 32768},
    {"force_class": "SHUFFLE"},
    {"pipe": "bulk"}, {"pipe": "bulkst"}, {"pipe": "staged"},
]
KINDS = ["bijective", "bijective", "broadcast", "memory", "offset_perm", "to_memory",
         "broadcast_many", "subword"]


def _out_dims(rng, d):
    di = int(rng.integers(1, d))
    return [("i", di), ("j", d - di)]


def _with_batch(spec, nb):
    if nb == 0:
        return spec
    return {"out": [("b", nb)] + list(spec["out"]),
            "in": list(spec["in"]) + [("block", [f"b{k}" for k in range(nb)])]}


def _tiling_opts(opts):
    return {k: v for k, v in opts.items() if k in ("thread_bytes", "tile_bytes")}


def fuzz_case(rng):
    kind = KINDS[int(rng.integers(0, len(KINDS)))]
    w = [1, 2, 4, 8][int(rng.integers(0, 4))]
    opts = dict(OPTION_SETS[int(rng.integers(0, len(OPTION_SETS)))])
    if kind in ("bijective", "broadcast"):
        r = int(rng.integers(0, 5))
        wb = int(rng.integers(0, 4))
        zeros = 0 if kind == "bijective" else int(rng.integers(1, 3))
        d = max(2, r + 5 + wb - zeros)
        hw = [("reg", r), ("lane", 5), ("warp", wb)]
        out = _out_dims(rng, d)
        if sum(b for _, b in hw) < d:
            hw = [("reg", r + d - sum(b for _, b in hw)), ("lane", 5), ("warp", wb)]
        if kind == "bijective":
            sa = gen.random_distributed(rng, out, hw)
            sb = gen.random_distributed(rng, out, hw)
        else:
            # zero (broadcast) columns in registers or lanes
            za = "lane" if hw[0][1] < zeros else ["reg", "lane"][int(rng.integers(0, 2))]
            sa = gen.random_distributed(rng, out, hw, zero_ok=[za])
            sb = gen.random_distributed(rng, out, hw, zero_ok=["reg", "lane"])
        nb = int(rng.integers(0, 5))
        return kind, W.spec_to_bases(_with_batch(sa, nb)), W.spec_to_bases(_with_batch(sb, nb)), w, opts
    if kind == "broadcast_many":
        # up to 8 zero columns in B (replica grid bits, dst-order broadcast stores), the
        # batch bits possibly permuted (CTA class)
        nz = int(rng.integers(3, 9))
        sa, sb = gen.random_broadcast_pair(rng, nz, ki=4, kj=4, batch_bits=int(rng.integers(1, 4)),
                                           permute_batch=bool(rng.integers(0, 2)))
        return kind, W.spec_to_bases(sa), W.spec_to_bases(sb), w, _tiling_opts(opts)
    if kind == "subword":
        # 1- / 2-byte elements on random SHUFFLE-class pairs (element-permuted shuffles)
        r = int(rng.integers(3, 6))
        hw = [("reg", r), ("lane", 5), ("warp", 10 - r - 5)]
        out = [("i", 5), ("j", 5)]
        sa, sb = gen.random_distributed(rng, out, hw), gen.random_distributed(rng, out, hw)
        nb = int(rng.integers(0, 3))
        return kind, W.spec_to_bases(_with_batch(sa, nb)), W.spec_to_bases(_with_batch(sb, nb)), \
            [1, 2][int(rng.integers(0, 2))], {}
    if kind == "memory":
        # Def 4.14 memory layouts with 1- and 2-bit columns (swizzles, R2)
        d = int(rng.integers(6, 13))
        out = [("x", d)]
        mk = lambda cols: ([("offset", d)], out, {"offset": [(int(c),) for c in cols]})
        return kind, mk(gen.random_memory_cols(rng, d)), mk(gen.random_memory_cols(rng, d)), w, {}
    if kind == "offset_perm":
        d = int(rng.integers(8, 15))
        out = _out_dims(rng, d)
        names = gen._names(out)
        sa = {"out": out, "in": [("offset", [names[k] for k in rng.permutation(d)])]}
        sb = {"out": out, "in": [("offset", [names[k] for k in rng.permutation(d)])]}
        return kind, W.spec_to_bases(sa), W.spec_to_bases(sb), w, _tiling_opts(opts)
    # to_memory: a distributed tile (plus batch) stored to / loaded from a row-major
    # (identity) memory layout
    r = int(rng.integers(1, 5))
    wb = int(rng.integers(0, 3))
    d = r + 5 + wb
    out = _out_dims(rng, d)
    sa = _with_batch(gen.random_distributed(rng, out, [("reg", r), ("lane", 5), ("warp", wb)]), int(rng.integers(0, 5)))
    sb = {"out": sa["out"], "in": [("offset", gen._names(sa["out"]))]}
    if rng.integers(0, 2):
        sa, sb = sb, sa
    return kind, W.spec_to_bases(sa), W.spec_to_bases(sb), w, _tiling_opts(opts)
