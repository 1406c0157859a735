"""The hot path captured in CUDA graphs (the production form of a launch-bound loop and
how bench.py times the config-4 rows): every specialised kernel is launched with
programmatic dependent launch, so stream capture turns the serialisation into
programmatic graph edges.  Each test captures several calls on rotating buffers —
conversion (config 1 tile, config 2 tiles, NOOP copy), gather, reduce, scan — replays
the graph twice on fresh inputs and compares every output with the oracle."""
import numpy as np
import pytest

from oracle import ll_oracle as O
from workloads import configs as W
from workloads import gen
from tests._util import from_device, to_device

pytestmark = pytest.mark.gpu

ll = pytest.importorskip("paper_conf_asplos_0001cgrnls0trm26_b200")


def _capture(calls):
    """One CUDA graph of `calls` (callables launching on the current stream)."""
    import torch
    st = torch.cuda.Stream()
    st.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(st):
        for c in calls:            # warm-up: kernels loaded before capture
            c()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=st):
            for c in calls:
                c()
    torch.cuda.synchronize()
    return g


def _refill(dev, host):
    dev.copy_(to_device(host))


@pytest.mark.parametrize("case", ["c1", "c2", "noop"])
def test_graph_conversions(case):
    import torch
    rng = np.random.default_rng(1101)
    sa, sb, w = {"c1": (W.C1_A, W.C1_B, 4), "c2": (*W.c2(3), 2),
                 "noop": (W.C1_A, W.C1_A, 4)}[case]
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    OA, OB = (O.Layout(*W.spec_to_bases(x)) for x in (sa, sb))
    plan = ll.ll_plan_convert(A, B, w)
    nsets = 3
    srcs = [to_device(O.pack(OA, gen.random_bits(rng, 1 << OA.d_out, w))) for _ in range(nsets)]
    dsts = [torch.zeros_like(s) for s in srcs]
    g = _capture([(lambda k=k: ll.ll_convert(srcs[k], dsts[k], plan)) for k in range(nsets)])
    for _ in range(2):
        host = [O.pack(OA, gen.random_bits(rng, 1 << OA.d_out, w)) for _ in range(nsets)]
        for k in range(nsets):
            _refill(srcs[k], host[k])
        g.replay()
        torch.cuda.synchronize()
        for k in range(nsets):
            assert np.array_equal(from_device(dsts[k], w), O.convert(OA, OB, host[k])), (case, k)


@pytest.mark.parametrize("family", ["mma", "blocked"])
def test_graph_gather_reduce_scan(family):
    import torch
    rng = np.random.default_rng(1102)
    Lg_spec = W.c4("gather", family, n_i=9, n_j=7)
    Lr_spec = W.c4("reduce", family, n_i=9, n_j=9)
    Lg, Lr = ll.Layout.from_spec(Lg_spec), ll.Layout.from_spec(Lr_spec)
    OLg, OLr = (O.Layout(*W.spec_to_bases(x)) for x in (Lg_spec, Lr_spec))
    pg, pr, ps = ll.ll_plan_gather(Lg, 1, 4), ll.ll_plan_reduce(Lr, 1), ll.ll_plan_scan(Lr, 1)
    ng, nr = 1 << OLg.d_in, 1 << OLr.d_in
    gs, gi, go = (torch.zeros(ng, dtype=torch.int32, device="cuda") for _ in range(3))
    rs = torch.zeros(nr, dtype=torch.float32, device="cuda")
    ro = torch.zeros(pr.out_elems(), dtype=torch.float32, device="cuda")
    so = torch.zeros(nr, dtype=torch.float32, device="cuda")
    g = _capture([lambda: ll.ll_gather(gs, gi, go, pg), lambda: ll.ll_reduce(rs, ro, pr),
                  lambda: ll.ll_scan(rs, so, ps)])
    for _ in range(2):
        src = O.pack(OLg, gen.random_bits(rng, ng, 4))
        idx = O.pack(OLg, rng.integers(0, 1 << 20, size=ng).astype(np.int32))
        rsrc = O.pack(OLr, rng.random(nr, dtype=np.float32))
        gs.copy_(torch.from_numpy(src.view(np.int32)).cuda())
        gi.copy_(torch.from_numpy(idx.view(np.int32)).cuda())
        rs.copy_(torch.from_numpy(rsrc).cuda())
        g.replay()
        torch.cuda.synchronize()
        assert np.array_equal(go.cpu().numpy().view(np.uint32), O.gather(OLg, 1, src, idx).view(np.uint32))
        assert np.array_equal(ro.cpu().numpy().view(np.uint32),
                              O.reduce_fixed_order_fp32(OLr, 1, rsrc).view(np.uint32))
        assert np.array_equal(so.cpu().numpy().view(np.uint32),
                              O.scan_bitdoubling_fp32(OLr, 1, rsrc).view(np.uint32))
