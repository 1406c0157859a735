"""DEVICE plans executed as peer stores (§8(f) N4, LL_EXCHANGE_PEER).

One tile kernel per rank loads that rank's src tiles and stores straight into the
receivers' dst windows; no pack / all-to-all / unpack.  Every rank's slice must equal
the oracle's closed form O12 (dst_r[h] = T[B(h, dev=r)]).

CPU: the fused tile plan's schedule emulated on all ranks' slices back to back
(ll_plan_simulate), for config 5 / 5-T and random distributed layouts with dev bits.
GPU: the loopback communicator (P virtual ranks, one launch per rank through the peer
table), and two processes on the one GPU sharing their windows through CUDA IPC with
the flag barriers between them.
"""
import os
import socket

import numpy as np
import pytest

from oracle import ll_oracle as O
from workloads import configs as W
from workloads import gen

ll = pytest.importorskip("paper_conf_asplos_0001cgrnls0trm26_b200")


def _rank_src(OA, T, r):
    la, off = O.rank_slice(OA, r)
    xs = O.apply_all(la, np.arange(1 << la.d_in, dtype=np.uint64)) ^ np.uint64(off)
    return T[xs.astype(np.int64)]


def _want(OA, OB, T, P):
    return np.concatenate([O.convert_distributed_rank(OA, OB, T, r) for r in range(P)])


@pytest.mark.parametrize("make", ["c5", "c5T"])
@pytest.mark.parametrize("p", [1, 2, 3])
@pytest.mark.parametrize("w", [2, 4, 8])
def test_peer_plan_simulated(make, p, w):
    n = 6
    sa, sb = getattr(W, make)(p, n=n)
    OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
    P = 1 << p
    plan = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), w,
                              comm=ll.Comm.loopback(P), exchange="peer")
    d = plan.describe()
    assert d["class"] == "DEVICE" and d["exchange"] == "peer" and d["workspace_bytes"] == 0
    assert plan.workspace_bytes() == 0
    # the src dev bits are the top CTA-index bits (rank r owns a contiguous tile range)
    nl = 2 * n - p + (1 if w == 8 else 0)
    gsrc = d["fused"]["tile"]["grid_src_bit"]
    assert sorted(gsrc[-p:]) == list(range(nl, nl + p)) and all(b < nl for b in gsrc[:-p])
    assert all(b < nl for b in d["fused"]["tile"]["ld_bit"])
    assert d["rank_tiles"] * P == d["fused"]["tile"]["ctas"]
    T = gen.random_bits(np.random.default_rng(1006 + p), 1 << (2 * n), w)
    src = np.concatenate([_rank_src(OA, T, r) for r in range(P)])
    got = plan.simulate(src, src.size)
    assert np.array_equal(got, _want(OA, OB, T, P))


@pytest.mark.parametrize("seed", range(12))
def test_peer_plan_random_simulated(seed):
    """Random distributed layouts (R1, bijective) with p dev bits on both sides."""
    rng = np.random.default_rng(4000 + seed)
    p = int(rng.integers(1, 4))
    out = [("i", 6), ("j", 6)]
    hw = [("reg", 3), ("lane", 5), ("warp", 4 - p), ("dev", p)]
    sa = gen.random_distributed(rng, out, hw)
    sb = gen.random_distributed(rng, out, hw)
    OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
    P = 1 << p
    w = int(rng.choice([1, 2, 4]))
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    try:
        plan = ll.ll_plan_convert(A, B, w, comm=ll.Comm.loopback(P), exchange="peer")
    except ll.LLError as e:
        # a pair whose dev bits do not cross is not a DEVICE plan at all
        assert O.classify(OA, OB) != "DEVICE", e
        return
    if plan.cls != "DEVICE":
        assert plan.cls == O.classify(OA, OB)
        return
    T = gen.random_bits(rng, 1 << 12, w)
    src = np.concatenate([_rank_src(OA, T, r) for r in range(P)])
    got = plan.simulate(src, src.size)
    assert np.array_equal(got, _want(OA, OB, T, P))


def _peer_comm(nranks, rank, dst, flags, window_bytes=1 << 20):
    import ctypes
    h = ctypes.c_void_p()
    st = ll._lib.ll_comm_create_peers(nranks, rank, (ctypes.c_void_p * max(1, nranks))(*dst),
                                      (ctypes.c_void_p * max(1, nranks))(*flags), window_bytes, ctypes.byref(h))
    return st, (ll.Comm(h, nranks) if st == 0 else None)


def test_peer_comm_and_plan_errors():
    # communicator validation happens before any CUDA call (host pointers suffice here)
    assert _peer_comm(3, 0, [16, 32, 48], [16, 32, 48])[0] == 1          # not a power of two
    assert _peer_comm(2, 2, [16, 32], [16, 32])[0] == 1                  # rank out of range
    assert _peer_comm(2, 0, [16, 0], [16, 32])[0] == 1                   # null window
    assert _peer_comm(2, 0, [16, 40], [16, 32])[0] == 8                  # LL_ERR_MISALIGNED
    st, comm = _peer_comm(2, 0, [1 << 20, 2 << 20], [3 << 20, 4 << 20])
    assert st == 0
    sa, sb = W.c5(1, n=5)
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    # AUTO on a communicator with windows -> peer stores; no workspace
    d = ll.ll_plan_convert(A, B, 2, comm=comm).describe()
    assert d["exchange"] == "peer" and d["workspace_bytes"] == 0
    # the collective exchange needs NCCL (or loopback): refused at plan time
    with pytest.raises(ll.LLError, match="collective exchange"):
        ll.ll_plan_convert(A, B, 2, comm=comm, exchange="collective")
    # AUTO on a loopback communicator keeps the collective decomposition
    assert ll.ll_plan_convert(A, B, 2, comm=ll.Comm.loopback(2)).describe()["exchange"] == "collective"
    # communicator size must match the dev bits
    st, comm4 = _peer_comm(4, 0, [16 * k for k in range(1, 5)], [16 * k for k in range(1, 5)])
    with pytest.raises(ll.LLError, match="communicator size"):
        ll.ll_plan_convert(A, B, 2, comm=comm4)


# ----------------------------------------------------------------------------- GPU
@pytest.mark.gpu
@pytest.mark.parametrize("make", ["c5", "c5T"])
@pytest.mark.parametrize("p", [1, 2, 3])
@pytest.mark.parametrize("w", [2, 8])
def test_peer_loopback_gpu(make, p, w):
    from tests._util import empty_device, from_device, to_device
    n = 9
    sa, sb = getattr(W, make)(p, n=n)
    OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
    P = 1 << p
    plan = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), w,
                              comm=ll.Comm.loopback(P), exchange="peer")
    T = gen.random_bits(np.random.default_rng(1006), 1 << (2 * n), w)
    src = np.concatenate([_rank_src(OA, T, r) for r in range(P)])
    d_src, d_dst = to_device(src), empty_device(src.size, w)
    ll.ll_convert(d_src, d_dst, plan)
    assert np.array_equal(from_device(d_dst, w), _want(OA, OB, T, P))


@pytest.mark.gpu
@pytest.mark.parametrize("seed", range(6))
def test_peer_loopback_random_gpu(seed):
    from tests._util import empty_device, from_device, to_device
    rng = np.random.default_rng(5000 + seed)
    p = int(rng.integers(1, 4))
    out = [("i", 8), ("j", 8)]
    hw = [("reg", 4), ("lane", 5), ("warp", 2), ("block", 5 - p), ("dev", p)]
    sa = gen.random_distributed(rng, out, hw)
    sb = gen.random_distributed(rng, out, hw)
    OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
    P = 1 << p
    w = int(rng.choice([1, 2, 4, 8]))
    plan = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), w,
                              comm=ll.Comm.loopback(P), exchange="peer")
    assert plan.cls == "DEVICE"
    T = gen.random_bits(rng, 1 << 16, w)
    src = np.concatenate([_rank_src(OA, T, r) for r in range(P)])
    d_src, d_dst = to_device(src), empty_device(src.size, w)
    ll.ll_convert(d_src, d_dst, plan)
    assert np.array_equal(from_device(d_dst, w), _want(OA, OB, T, P))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _ipc_worker(rank, world, port, q):
    """One rank: its src slice and dst window on cuda:0, the peers' windows mapped with
    CUDA IPC, three back-to-back conversions (flag-barrier epochs), own slice checked."""
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        from tests._util import from_device, to_device
        n, p = 10, world.bit_length() - 1
        sa, sb = W.c5(p, n=n)
        OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
        nloc = 1 << (2 * n - p)
        window = torch.zeros(nloc, dtype=torch.int16, device="cuda")
        flags = torch.zeros(ll.PEER_FLAG_BYTES // 4, dtype=torch.int32, device="cuda")
        comm = ll.Comm.peers(window, flags)
        plan = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), 2, comm=comm)
        assert plan.describe()["exchange"] == "peer"
        for it in range(3):
            T = gen.random_bits(np.random.default_rng(1006 + it), 1 << (2 * n), 2)
            src = to_device(_rank_src(OA, T, rank))
            ll.ll_convert(src, window, plan)
            torch.cuda.synchronize()
            got = from_device(window, 2)
            assert np.array_equal(got, O.convert_distributed_rank(OA, OB, T, rank)), (rank, it)
            dist.barrier()   # nobody starts the next round while a peer still reads
        del plan, comm
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.timeout(300)
def test_peer_ipc_two_processes_one_gpu():
    """The multi-process peer path for real: two ranks (processes) on the one B200,
    windows shared through CUDA IPC, stores into the peer's window, flag barriers."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ipc_worker, args=(r, 2, port, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    res = dict(q.get(timeout=240) for _ in procs)
    for pr in procs:
        pr.join(timeout=60)
    assert all(v == "ok" for v in res.values()), res
