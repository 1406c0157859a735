"""Config 5: a 32K x 32K bf16 tensor row-sharded over P GPUs,
redistributed to column-sharded — the DEVICE class: pack (CTA-class tile kernel) ->
grouped ncclSend/ncclRecv all-to-all over NVLink -> unpack (identity here).

    torchrun --nproc-per-node P --master-addr 127.0.0.1 tools/bench_device.py [--n 15]
    python tools/bench_device.py --loopback 8      # one GPU, P virtual ranks (memcpy exchange)
    python tools/bench_device.py --loopback 8 --exchange peer   # one GPU, fused peer-store kernel

Prints one JSON line: aggregate GB/s (2 x tensor bytes / time, max over ranks), the
per-GPU NVLink bytes and their fraction of 900 GB/s per direction (nominal) and of the
measured 770 GB/s peer copy (B200_PROFILING.md), and the pack kernel's HBM GB/s."""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_asplos_0001cgrnls0trm26_b200 as ll  # noqa: E402
from workloads import configs as W  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=15, help="log2 of the square tensor side")
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--loopback", type=int, default=0)
    ap.add_argument("--exchange", default="collective", choices=["collective", "peer"],
                    help="collective: pack -> all-to-all -> unpack; peer: one tile kernel storing into "
                         "the receivers' windows (CUDA IPC over NVLink), §8(f) N4")
    args = ap.parse_args()
    rank, world = int(os.environ.get("RANK", 0)), int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    torch.cuda.set_device(local)
    if args.loopback:
        P = args.loopback
        comm = ll.Comm.loopback(P)
    else:
        P = world
        if world > 1:
            import torch.distributed as dist
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
            comm = None if args.exchange == "peer" else ll.Comm.from_process_group()
        else:
            comm = None
    p = P.bit_length() - 1
    total = 1 << (2 * args.n)
    local_elems = total // P
    slices = P if args.loopback else 1
    src = torch.randint(-2 ** 15, 2 ** 15, (local_elems * slices,), dtype=torch.int16, device="cuda")
    dst = torch.empty_like(src)
    if args.exchange == "peer" and not args.loopback and world > 1:
        flags = torch.zeros(ll.PEER_FLAG_BYTES // 4, dtype=torch.int32, device="cuda")
        comm = ll.Comm.peers(dst, flags)
    sa, sb = W.c5(p, n=args.n)
    A, B = ll.Layout.from_spec(sa), ll.Layout.from_spec(sb)
    plan = ll.ll_plan_convert(A, B, 2, comm=comm, exchange=args.exchange) if p else ll.ll_plan_convert(A, B, 2)
    plan.prepare()
    ws = torch.empty(max(16, plan.workspace_bytes()), dtype=torch.uint8, device="cuda")
    for _ in range(args.warmup):
        ll.ll_convert(src, dst, plan, workspace=ws)
    torch.cuda.synchronize()
    if world > 1 and not args.loopback:
        torch.distributed.barrier()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(args.steps):
        ll.ll_convert(src, dst, plan, workspace=ws)
    b.record()
    torch.cuda.synchronize()
    ms = a.elapsed_time(b) / args.steps
    t = torch.tensor([ms], device="cuda", dtype=torch.float64)
    if world > 1 and not args.loopback:
        torch.distributed.all_reduce(t, op=torch.distributed.ReduceOp.MAX)
    ms = float(t.item())
    nvl = (P - 1) / P * local_elems * 2          # bytes each GPU sends (and receives)
    if rank == 0:
        d = plan.describe()
        print(json.dumps({
            "workload": f"config 5: [{1 << args.n},{1 << args.n}] bf16 row-sharded -> column-sharded, P={P}"
                        + (" (loopback)" if args.loopback else ""),
            "class": d["class"], "exec": d["exec"], "exchange": d.get("exchange"), "ms_per_step": round(ms, 4),
            "value_GBps": round(2 * total * 2 / (ms / 1e3) / 1e9, 1),
            "nvlink_bytes_per_gpu_each_way": int(nvl),
            "nvlink_GBps_per_gpu": round(nvl / (ms / 1e3) / 1e9, 1) if P > 1 else None,
            "frac_of_900": round(nvl / (ms / 1e3) / 1e9 / 900, 3) if P > 1 else None,
            "frac_of_770_measured_peer": round(nvl / (ms / 1e3) / 1e9 / 770, 3) if P > 1 else None,
        }), flush=True)
    if world > 1 and not args.loopback:
        torch.distributed.destroy_process_group()


if __name__ == "__main__":
    main()
