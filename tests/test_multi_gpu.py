"""Multi-GPU paths on real GPUs (§8(e)): one process per GPU over NCCL, world size
min(2, device_count).  Skipped cleanly on a one-GPU box (the driver's GPU tier and
gpurun are one GPU); the host logic of the same paths runs on CPU with gloo
(test_device_dist.py, test_peer_exchange.py).

* config 5 (DEVICE class) with the collective exchange (pack -> grouped
  ncclSend/ncclRecv -> unpack) and with peer stores into the other rank's window
  (CUDA IPC over NVLink): every element of every rank's slice against the closed form
  dst_r[h] = H(B(h, dev = r)) of hash-filled src (O5 / O12);
* independent tiles (config 2 with the top block bit as a dev bit in both A and B):
  no communicator needed, every element checked the same way.
Also (CPU): bench.py --gpus N fails loudly when N GPUs are not there.
"""
import os
import socket
import subprocess
import sys

import pytest

from workloads import configs as W
from workloads import hashfill as H

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(rank)
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", rank))
    try:
        import paper_conf_asplos_0001cgrnls0trm26_b200 as ll
        p = world.bit_length() - 1
        n = 12
        sa, sb = W.c5(p, n=n)
        nloc = 1 << (2 * n - p)
        res = {}
        for exchange in ("collective", "peer"):
            seed = 1006 + len(res)
            src = H.fill(sa, 2, seed, h0=rank * nloc, n=nloc)
            dst = torch.zeros(nloc, dtype=torch.int16, device="cuda")
            flags = torch.zeros(ll.PEER_FLAG_BYTES // 4, dtype=torch.int32, device="cuda")
            comm = ll.Comm.from_process_group() if exchange == "collective" else ll.Comm.peers(dst, flags)
            plan = ll.ll_plan_convert(ll.Layout.from_spec(sa), ll.Layout.from_spec(sb), 2, comm=comm,
                                      exchange=exchange)
            assert plan.cls == "DEVICE"
            ws = torch.empty(max(16, plan.workspace_bytes()), dtype=torch.uint8, device="cuda")
            for _ in range(3):
                ll.ll_convert(src, dst, plan, workspace=ws)
            torch.cuda.synchronize()
            res[exchange] = H.check(sb, 2, seed, dst, h0=rank * nloc)
            dist.barrier()
            del plan, comm
        # independent tiles: config 2 with dev = the top batch bit in A and B
        sa2, sb2 = W.c2(3)
        for spec in (sa2, sb2):
            blk = dict(spec["in"])["block"]
            spec["in"] = [(nm, bits) for nm, bits in spec["in"] if nm != "block"] + \
                [("block", blk[:-1]), ("dev", blk[-1:])]
        plan = ll.ll_plan_convert(ll.Layout.from_spec(sa2), ll.Layout.from_spec(sb2), 2)
        n2 = 1 << (ll.Layout.from_spec(sa2).d_in - 1)
        src = H.fill(sa2, 2, 7, h0=rank * n2, n=n2)
        dst = torch.empty_like(src)
        ll.ll_convert(src, dst, plan)
        torch.cuda.synchronize()
        res["independent"] = H.check(sb2, 2, 7, dst, h0=rank * n2)
        q.put((rank, res))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.gpu
@pytest.mark.timeout(600)
def test_two_gpus_nccl_config5_and_independent_tiles():
    import torch
    if torch.cuda.device_count() < 2:
        pytest.skip("needs 2 GPUs (one process per GPU over NCCL); this box has %d" % torch.cuda.device_count())
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for pr in procs:
        pr.start()
    res = dict(q.get(timeout=540) for _ in procs)
    for pr in procs:
        pr.join(timeout=60)
    for r, v in res.items():
        assert isinstance(v, dict), (r, v)
        assert v == {"collective": 0, "peer": 0, "independent": 0}, (r, v)


def test_bench_gpus_mismatch_fails_loudly():
    """bench.py --gpus 2 must not silently benchmark one GPU: with fewer visible devices
    it exits non-zero; under a torchrun environment whose WORLD_SIZE differs from --gpus
    it exits non-zero too."""
    import torch
    env = dict(os.environ)
    if torch.cuda.device_count() < 2:
        r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "3"],
                           capture_output=True, text=True, env=env, timeout=300)
        assert r.returncode == 2, r.stdout + r.stderr
        assert "n_gpus" not in r.stdout
        assert "CUDA device" in r.stderr
    env.update(WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "4", "--steps", "3"],
                       capture_output=True, text=True, env=env, timeout=300)
    assert r.returncode == 2 and "WORLD_SIZE=1" in r.stderr, r.stdout + r.stderr
