"""DEVICE class (row a9): pack -> all-to-all -> unpack.

CPU (gloo, world_size 2 and 4): each rank builds the real plan, runs its pack /
unpack stages with the host schedule emulation (ll_plan_simulate) and exchanges the
chunks with torch.distributed.all_to_all_single over gloo; every rank's slice must
equal the oracle's closed form (O12).  GPU (1 B200): the loopback communicator runs
the same decomposition with the CUDA kernels and device memcpys for P = 2, 4, 8."""
import os
import socket

import numpy as np
import pytest

from oracle import ll_oracle as O
from workloads import configs as W
from workloads import gen

ll = pytest.importorskip("paper_conf_asplos_0001cgrnls0trm26_b200")


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank_src(OA, T, r):
    la, off = O.rank_slice(OA, r)
    xs = O.apply_all(la, np.arange(1 << la.d_in, dtype=np.uint64)) ^ np.uint64(off)
    return T[xs.astype(np.int64)]


def src_elems(OA):
    return 1 << (OA.d_in - len(OA.dim_bits("dev")))


def _worker(rank, world, port, n, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        p = world.bit_length() - 1
        cases = [W.c5(p, n=n), W.c5T(p, n=n)]
        if p >= 2:
            cases += [W.c5_partial(p, n=n), W.c5_partial(p, n=n, swap=True)]
        for sa, sb in cases:
            OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
            A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
            # the communicator handle is only consulted for its size at plan time
            plan = ll.ll_plan_convert(A, B, 2, comm=ll.Comm.loopback(world))
            assert plan.cls == "DEVICE"
            pack, unpack, chunk, nr = plan.device_stages()
            assert nr == world
            sp, rp = plan.device_peers(rank)
            assert len(sp) * chunk == len(rp) * chunk == src_elems(OA)
            T = gen.random_bits(np.random.default_rng(1006), 1 << (2 * n), 2)
            src = _rank_src(OA, T, rank)
            send = pack.simulate(src, src.size) if pack else src
            # all_to_all_single takes chunks in rank order: send chunk j to sp[j], file
            # the chunk from rp[i] as recv chunk i (ranks outside the routing get 0);
            # gloo has no 16-bit all_to_all: move the bf16 bits as int32 pairs
            c2 = chunk // 2
            sv = send.view(np.int32).reshape(len(sp), c2)
            order = sorted(range(len(sp)), key=lambda j: sp[j])
            insz = [c2 if q in sp else 0 for q in range(world)]
            outsz = [c2 if q in rp else 0 for q in range(world)]
            recv_t = torch.empty(len(rp) * c2, dtype=torch.int32)
            dist.all_to_all_single(recv_t, torch.from_numpy(np.ascontiguousarray(sv[order]).reshape(-1)),
                                   outsz, insz)
            by_src = dict(zip(sorted(rp), recv_t.numpy().reshape(len(rp), c2)))
            recv = np.concatenate([by_src[rp[i]] for i in range(len(rp))]).view(np.uint16)
            got = unpack.simulate(recv, recv.size) if unpack else recv
            want = O.convert_distributed_rank(OA, OB, T, rank)
            assert np.array_equal(got, want), (sa, rank)
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_device_decomposition_gloo(world):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, 5, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in procs)
    for p in procs:
        p.join(timeout=60)
    assert all(v == "ok" for v in res.values()), res


def test_partial_exchange_routing():
    """Partial exchanges: with the top row bit a dev bit of both A and
    B, each rank sends to and receives from 2^(p-1) ranks — exactly those that agree with
    it on the shared bit (at the same rank position, or moved to rank bit 0 by swap) —
    and every (sender, receiver) pair is routed once."""
    for p in (2, 3):
        for swap in (False, True):
            sa, sb = W.c5_partial(p, n=6, swap=swap)
            plan = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), 2,
                                      comm=ll.Comm.loopback(1 << p))
            assert plan.cls == "DEVICE"
            _, _, chunk, nr = plan.device_stages()
            assert chunk == 1 << (12 - p - (p - 1))
            pairs = set()
            for r in range(nr):
                sp, rp = plan.device_peers(r)
                assert len(sp) == len(rp) == 1 << (p - 1)
                top = (r >> (p - 1)) & 1
                for q in sp:
                    assert ((q >> (0 if swap else p - 1)) & 1) == top
                    pairs.add((r, q))
            for r in range(nr):
                for s in plan.device_peers(r)[1]:
                    assert (s, r) in pairs


def test_device_plan_errors():
    sa, sb = W.c5(1, n=4)
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    with pytest.raises(ll.LLError, match="comm"):
        ll.ll_plan_convert(A, B, 2)
    with pytest.raises(ll.LLError):
        ll.ll_plan_convert(A, B, 2, comm=ll.Comm.loopback(4))   # 2 ranks' worth of dev bits


def test_device_p1_is_noop_and_5T_is_cta():
    sa, sb = W.c5(0, n=5)
    assert ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), 2).cls == "NOOP"
    sa, sb = W.c5T(0, n=5)
    p = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), 2)
    assert p.cls == "CTA" and p.describe()["exec"] == "tile"


@pytest.mark.gpu
@pytest.mark.parametrize("p", [1, 2, 3])
@pytest.mark.parametrize("make", ["c5", "c5T", "c5_partial", "c5_partial_swap"])
def test_device_loopback_gpu(p, make):
    import torch
    from tests._util import empty_device, from_device, to_device
    n = 9
    if make.startswith("c5_partial"):
        if p < 2:
            pytest.skip("partial exchanges need >= 2 dev bits")
        sa, sb = W.c5_partial(p, n=n, swap=make.endswith("swap"))
    else:
        sa, sb = getattr(W, make)(p, n=n)
    OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    P = 1 << p
    plan = ll.ll_plan_convert(A, B, 2, comm=ll.Comm.loopback(P))
    T = gen.random_bits(np.random.default_rng(1006), 1 << (2 * n), 2)
    src = np.concatenate([_rank_src(OA, T, r) for r in range(P)])
    d_src, d_dst = to_device(src), empty_device(src.size, 2)
    ws = torch.empty(max(1, plan.workspace_bytes()), dtype=torch.uint8, device="cuda")
    ll.ll_convert(d_src, d_dst, plan, workspace=ws)
    got = from_device(d_dst, 2).reshape(P, -1)
    for r in range(P):
        assert np.array_equal(got[r], O.convert_distributed_rank(OA, OB, T, r)), r


@pytest.mark.gpu
def test_device_loopback_config5_large():
    """Config 5 shape at P = 8 with a 2^13 x 2^13 bf16 tensor (128 MiB): every rank's
    slice checked on sampled outputs against the oracle's closed form."""
    import torch
    n, p = 13, 3
    sa, sb = W.c5(p, n=n)
    OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    P = 1 << p
    plan = ll.ll_plan_convert(A, B, 2, comm=ll.Comm.loopback(P))
    total = 1 << (2 * n)
    g = torch.Generator(device="cuda").manual_seed(1006)
    T = torch.randint(-2 ** 15, 2 ** 15, (total,), dtype=torch.int16, device="cuda", generator=g)
    # rank slices of A: src_r[h] = T[A(h, dev=r)], built from the oracle's index map
    nloc = total // P
    rng = np.random.default_rng(0)
    src = torch.empty(total, dtype=torch.int16, device="cuda")
    for r in range(P):
        la, off = O.rank_slice(OA, r)
        xs = O.apply_all(la, np.arange(nloc, dtype=np.uint64)) ^ np.uint64(off)
        src[r * nloc:(r + 1) * nloc] = T[torch.from_numpy(xs.astype(np.int64)).cuda()]
    dst = torch.empty_like(src)
    ws = torch.empty(max(1, plan.workspace_bytes()), dtype=torch.uint8, device="cuda")
    ll.ll_convert(src, dst, plan, workspace=ws)
    torch.cuda.synchronize()
    for r in range(P):
        hs = rng.integers(0, nloc, size=1 << 16).astype(np.uint64)
        lb, offb = O.rank_slice(OB, r)
        xs = (O.apply_all(lb, hs) ^ np.uint64(offb)).astype(np.int64)
        got = dst[r * nloc + torch.from_numpy(hs.astype(np.int64)).cuda()]
        assert torch.equal(got, T[torch.from_numpy(xs).cuda()]), r


@pytest.mark.gpu
def test_nccl_comm_bootstrap_single_rank():
    """NCCL through dlopen: ncclGetUniqueId + ncclCommInitRank (one rank on this GPU)
    and destroy — the bootstrap every DEVICE plan uses (the multi-GPU exchange itself
    needs >1 GPU, unavailable in this run)."""
    import ctypes
    uid = (ctypes.c_char * 128)()
    ll._check(ll._lib.ll_comm_get_unique_id(uid))
    assert any(b != 0 for b in bytes(uid))
    h = ctypes.c_void_p()
    ll._check(ll._lib.ll_comm_create(uid, 1, 0, ctypes.byref(h)))
    assert h.value
    ll._lib.ll_comm_destroy(h)


def _with_dev(spec, p):
    """The top p block bits of a batched spec become `dev` bits."""
    ins, dev = [], []
    for n, bits in spec["in"]:
        if n == "block":
            ins.append(("block", bits[:-p]))
            dev = bits[-p:]
        else:
            ins.append((n, bits))
    ins.append(("dev", dev))
    return {"out": spec["out"], "in": ins}


def _weak_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        p = world.bit_length() - 1
        for make, w in ((lambda: W.c2(4), 2), (lambda: W.c3(3), 2), (lambda: W.c1_batched(4), 4)):
            sa, sb = (_with_dev(s, p) for s in make())
            OA, OB = O.Layout(*W.spec_to_bases(sa)), O.Layout(*W.spec_to_bases(sb))
            plan = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), w)
            # Q is the identity on the dev bits: a local class, no communicator needed
            assert plan.cls == O.classify(OA, OB) and plan.cls != "DEVICE"
            T = gen.random_bits(np.random.default_rng(1002), 1 << OA.d_out, w)
            src = _rank_src(OA, T, rank)
            got = plan.simulate(src, src.size)
            ok = np.array_equal(got, O.convert_distributed_rank(OA, OB, T, rank))
            # the bench's max-over-ranks reduction, on a per-rank figure
            t = torch.tensor([float(rank + 1)], dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            assert ok and t.item() == world
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_weak_sharding_independent_tiles_gloo(world):
    """Row e(1): configs 1-batch, 2 and 3 sharded over ranks by declaring the top block
    bits `dev` in both layouts — each rank plans and converts its own slice with no
    communication (host schedule emulation), equal to the oracle's rank slice (O12)."""
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_weak_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = dict(q.get(timeout=300) for _ in procs)
    for pr in procs:
        pr.join(timeout=60)
    assert all(v == "ok" for v in res.values()), res


def test_device_peers_errors():
    """ll_plan_device_peers: only collective DEVICE plans, rank in range."""
    A, B = ll.Layout.from_spec(W.C1_A), ll.Layout.from_spec(W.C1_B)
    with pytest.raises(ll.LLError, match="INVALID_ARG"):
        ll.ll_plan_convert(A, B, 4).device_peers(0)
    sa, sb = W.c5(1, n=4)
    plan = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), 2, comm=ll.Comm.loopback(2))
    assert plan.device_peers(0) == ([0, 1], [0, 1])
    with pytest.raises(ll.LLError, match="INVALID_ARG"):
        plan.device_peers(2)


def _gpu_stage_worker(rank, world, port, q):
    """One process per virtual rank on the one GPU: the collective DEVICE plan's real
    pack and unpack kernels (ll_convert of the stage plans) around an exchange carried
    by gloo (NCCL refuses two ranks on one device), routed by ll_plan_device_peers;
    every element of this rank's slice against the closed form H(B(h, dev = r))."""
    import torch
    import torch.distributed as dist
    from workloads import hashfill as HF
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        p = world.bit_length() - 1
        n = 10
        res = []
        for sa, sb in ([W.c5(p, n=n), W.c5T(p, n=n)] + ([W.c5_partial(p, n=n), W.c5_partial(p, n=n, swap=True)]
                                                        if p >= 2 else [])):
            plan = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), 2, comm=ll.Comm.loopback(world))
            pack, unpack, chunk, nr = plan.device_stages()
            sp, rp = plan.device_peers(rank)
            nloc = 1 << (2 * n - p)
            src = HF.fill(sa, 2, 5, h0=rank * nloc, n=nloc)
            send = torch.empty_like(src)
            if pack:
                ll.ll_convert(src, send, pack)
            else:
                send.copy_(src)
            c2 = chunk // 2
            sv = send.view(torch.int32).view(len(sp), c2).cpu()
            order = sorted(range(len(sp)), key=lambda j: sp[j])
            insz = [c2 if qq in sp else 0 for qq in range(world)]
            outsz = [c2 if qq in rp else 0 for qq in range(world)]
            recv_t = torch.empty(len(rp) * c2, dtype=torch.int32)
            dist.all_to_all_single(recv_t, sv[order].contiguous().view(-1), outsz, insz)
            by_src = dict(zip(sorted(rp), recv_t.view(len(rp), c2)))
            recv = torch.cat([by_src[rp[i]] for i in range(len(rp))]).cuda().view(torch.int16)
            dst = torch.empty_like(src)
            if unpack:
                ll.ll_convert(recv, dst, unpack)
            else:
                dst.copy_(recv)
            torch.cuda.synchronize()
            res.append(HF.check(sb, 2, 5, dst, h0=rank * nloc))
        q.put((rank, res))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.timeout(600)
@pytest.mark.parametrize("world", [2, 4])
def test_collective_stages_multiprocess_one_gpu(world):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_gpu_stage_worker, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = dict(q.get(timeout=540) for _ in procs)
    for pr in procs:
        pr.join(timeout=60)
    for r, v in res.items():
        assert isinstance(v, list) and all(x == 0 for x in v), (r, v)
