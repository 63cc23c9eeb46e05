#!/usr/bin/env python
"""C5 (BASELINE configs[4]) at G GPUs: TMV 65536^2 fp32 sharded by column
blocks and a 64M-item x 64 loop-reduce sharded by item blocks (contiguous
outer ranges), outputs gathered to rank 0 -- NCCL send/recv, or
fused into the kernels' master stores through CUDA IPC (--gather fused), or
the library's own NCCL group (--gather native, cudanp_group_gather).

    torchrun --nproc-per-node G --master-addr 127.0.0.1 tools/c5_scale.py [--gather nccl|fused|native]

Strong scaling: the problem is fixed, each rank owns 1/G of it, generated on
its device from global indices.  Per op, rank 0 prints one JSON record with
the max-over-ranks kernel time, the gather time, the end-to-end time
(kernel + gather, device events, max over ranks), aggregate GB/s of
algorithmic bytes over the max kernel time and over e2e, and whether the
gathered result equals the unsharded single-GPU result bit for bit.
CUDANP_BENCH_BACKEND=gloo lets several ranks share one GPU (logic test only;
use --gather fused and --scale to shrink the problem).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

from paper_conf_ppopp_yangz14_b200 import cudanp as C  # noqa: E402
from paper_conf_ppopp_yangz14_b200 import parallel as P  # noqa: E402


def ev():
    return torch.cuda.Event(enable_timing=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gather", choices=["nccl", "fused", "native"], default="nccl")
    ap.add_argument("--scale", type=int, default=1, help="divide n (TMV) and N (reduce) by this")
    ap.add_argument("--reps", type=int, default=10)
    ap.add_argument("--tmv-cfg", default="16,cyclic,inter")
    ap.add_argument("--reduce-cfg", default="8,block,intra")
    a = ap.parse_args()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    backend = os.environ.get("CUDANP_BENCH_BACKEND", "nccl")
    dev = local % max(torch.cuda.device_count(), 1)
    torch.cuda.set_device(dev)
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev))
        else:
            dist.init_process_group(backend)
    C.load()
    fused = world > 1 and a.gather == "fused"
    native = P.NativeGroup(rank, world) if world > 1 and a.gather == "native" else None
    maps = {"intra": C.INTRA_WARP, "inter": C.INTER_WARP, "inter_tma": C.INTER_WARP_TMA}
    dists = {"cyclic": C.CYCLIC, "block": C.BLOCK}

    def cfg(s):
        S, d, m = s.split(",")
        return int(S), dists[d], maps[m]

    def max_ranks(v):
        if world == 1:
            return v
        t = torch.tensor([v], dtype=torch.float64, device="cuda" if backend == "nccl" else "cpu")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    n = 65536 // a.scale
    N, L = (1 << 26) // a.scale, 64
    for op in ("tmv", "reduce"):
        total = n if op == "tmv" else N
        b, e = P.shard(total, world, rank)
        if op == "tmv":
            S, d, m = cfg(a.tmv_cfg)
            A = torch.empty(n, e - b, device="cuda")
            C.cudanp_generate(A, "f32_unit", stream_id=1, col0=b, w_global=n)
            x = torch.empty(n, device="cuda")
            C.cudanp_generate(x, "f32_unit", stream_id=2)
            nbytes = 4 * n * n + 4 * n + 4 * n
        else:
            S, d, m = cfg(a.reduce_cfg)
            A = torch.empty(e - b, L, device="cuda")
            C.cudanp_generate(A, "f32_unit", stream_id=1, row0=b, w_global=L)
            nbytes = 4 * N * L + 4 * N
        y = torch.empty(e - b, device="cuda")
        root = torch.empty(total, device="cuda") if rank == 0 else None
        fg = P.FusedGather(root, total, rank, world) if fused else None
        out = fg.out_ptr() if fused else y

        def kernel():
            if op == "tmv":
                C.cudanp_tmv(A, x, out, S=S, dist=d, map=m, n_outer=e - b)
            else:
                C.cudanp_batched_loop_reduce(A, None, out, S=S, dist=d, map=m)

        def gather():
            if native is not None:
                native.gather(y, root, total)
            elif world > 1 and not fused:
                P.gather_to_root(y, root, total, rank, world)
            elif world == 1:
                root.copy_(y)

        for _ in range(2):
            kernel()
            gather()
        if fused:
            fg.finish()
        tk, tg = [], []
        for _ in range(a.reps):
            if world > 1:
                dist.barrier()
            torch.cuda.synchronize()
            e0, e1, e2 = ev(), ev(), ev()
            e0.record()
            kernel()
            e1.record()
            gather()
            e2.record()
            torch.cuda.synchronize()
            if fused:
                fg.finish()  # the peer stores are complete and visible to rank 0
            tk.append(e0.elapsed_time(e1))
            tg.append(e1.elapsed_time(e2))
        k_ms = max_ranks(statistics.median(tk))
        g_ms = max_ranks(statistics.median(tg))
        e_ms = max_ranks(statistics.median([p + q for p, q in zip(tk, tg)]))
        rec = {"config": "C5", "op": op, "G": world, "gather": a.gather if world > 1 else "none",
               "n_or_N": total, "L": n if op == "tmv" else L, "S": S, "dist": d, "map": m,
               "kernel_max_us": round(k_ms * 1e3, 1), "gather_us": round(g_ms * 1e3, 1),
               "e2e_us": round(e_ms * 1e3, 1), "alg_bytes": nbytes,
               "agg_gbs_kernel": round(nbytes / (k_ms * 1e-3) / 1e9, 1),
               "agg_gbs_e2e": round(nbytes / (e_ms * 1e-3) / 1e9, 1)}
        if rank == 0:
            # pin P4 (the result does not depend on the rank count): recompute the
            # whole problem unsharded on rank 0 with the same kernel and compare
            # bit for bit (the kernels' parity with the CPU oracle at C5 size is
            # tests/test_gpu_parity.py::test_full_size_C5_single_gpu_sampled)
            del A
            torch.cuda.empty_cache()
            if op == "tmv":
                Af = torch.empty(n, n, device="cuda")
                C.cudanp_generate(Af, "f32_unit", stream_id=1)
                full = C.cudanp_tmv(Af, x, S=S, dist=d, map=m)
            else:
                Af = torch.empty(N, L, device="cuda")
                C.cudanp_generate(Af, "f32_unit", stream_id=1)
                full = C.cudanp_batched_loop_reduce(Af, None, S=S, dist=d, map=m)
            torch.cuda.synchronize()
            rec["sharded_equals_unsharded"] = bool(torch.equal(full, root))
            del Af, full
            print(json.dumps(rec), flush=True)
        else:
            del A
        if fg:
            fg.close()
        del y, root
        torch.cuda.empty_cache()
    if native is not None:
        native.close()
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
