#!/usr/bin/env python
"""Benchmark of the CUDA-NP hot path on B200 (the driver's contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl cudanp|reference]
    torchrun --nproc-per-node N --master-addr 127.0.0.1 bench.py --gpus N ...

Workload (BASELINE.json configs[1], "C2"): TMV y=A^T x and MV y=A x on a
16384 x 16384 fp32 matrix, one item per output (master), inner loop 16384.
One *step* = one cudanp_tmv + one cudanp_mv over the resident matrix (+ the
NCCL gather of every rank's outputs to rank 0 when N > 1).  Before timing,
every (S, dist, map) is measured once -- the paper's exhaustive autotune over
slave counts and NP types -- and the best of each op is
timed; the per-S sweep (GB/s and speedup vs the S=1 no-NP kernel) is part of
the JSON line because the metric is quoted "per slave count".

Multi-GPU (weak scaling): rank g owns column block g of a 16384 x 16384*N
TMV matrix and row block g of a 16384*N x 16384 MV matrix (contiguous outer
ranges); its outputs are gathered to rank 0 with NCCL.

Metric value = algorithmic HBM bytes of all ranks / max-over-ranks step time
(GB/s).  Inputs (1 GiB per matrix) exceed the 126 MB L2, so no flush is
needed between steps.

The same line carries a `c5` block: BASELINE configs[4] (TMV 65536^2 by column
shards + the 64M x 64 loop-reduce by item shards, strong scaling over the N
ranks, outputs gathered to rank 0), with max-over-ranks kernel and gather
times, aggregate GB/s, the fraction of N x peak and a bit-exact check of the
sharded result against the unsharded one (pin P4).  `--no-c5` skips it.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "HBM GB/s and speedup vs S=1 no-NP kernel per slave count, at 1/2/4/8 B200"
H = W = 16384
SEED = 20140215
MAPN = {1: "intra", 2: "inter", 3: "inter_tma", 4: "intra_tma"}   # cudanp_map


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=400)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", choices=["cudanp", "reference"], default="cudanp")
    ap.add_argument("--n", type=int, default=H, help="matrix size (default 16384 = C2)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=5)
    ap.add_argument("--no-sweep", action="store_true",
                    help="skip the autotune sweep and comparisons (for ncu launch lists); "
                         "use --tmv-cfg / --mv-cfg")
    ap.add_argument("--gather", choices=["auto", "nccl", "fused", "native"], default="auto",
                    help="N > 1: gather outputs to rank 0 with NCCL send/recv through "
                         "torch.distributed, fused into the kernels' master stores through CUDA IPC "
                         "over NVLink (SURVEY f4), or with the library's own NCCL group "
                         "(cudanp_group_gather); auto = fused when every rank can map rank 0's "
                         "buffers, else nccl")
    ap.add_argument("--tmv-cfg", default="8,cyclic,inter_tma")
    ap.add_argument("--mv-cfg", default="256,cyclic,intra")
    ap.add_argument("--no-c5", action="store_true", help="skip the C5 strong-scaling block")
    ap.add_argument("--c5-steps", type=int, default=10)
    ap.add_argument("--oracle-timing", default=None, metavar="JSONL",
                    help="time the CPU oracle on C1-C5 (1 core / all cores / generation only; "
                         "SURVEY §8(d)) into JSONL and exit (no GPU work)")
    ap.add_argument("--oracle-cap-s", type=float, default=12.0,
                    help="--oracle-timing: seconds per (config, op, cores) before extrapolating")
    ap.add_argument("--cpu-sample-json", action="store_true", help=argparse.SUPPRESS)
    ap.add_argument("--cpu-rows", type=int, default=4096,
                    help="rows of the C2 matrix in the oracle's CPU sample (both arms)")
    return ap.parse_args()


def peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


def hbm_peak():
    p = peaks()
    if "hbm_gbs" in p:
        return float(p["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy read+write)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled during the timed region."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.rows = []
        self.proc = None
        self.thread = None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "100"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except Exception:
            self.proc = None
            return
        self.thread = threading.Thread(target=self._read, daemon=True)
        self.thread.start()

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([c.strip() for c in line.split(",")])

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        if self.thread:
            self.thread.join(timeout=2)
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in self.rows:
            try:
                sm.append(float(r[1]))
                mx.append(float(r[2]))
                for name, v in zip(names, r[5:9]):
                    if v.lower().startswith("active"):
                        reasons.add(name)
            except Exception:
                continue
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------ distributed plumbing
def dist_init(ngpus):
    import torch
    import torch.distributed as dist
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != ngpus:
        raise SystemExit(f"--gpus {ngpus} but WORLD_SIZE={world}")
    # CUDANP_BENCH_BACKEND=gloo (testing only): lets several ranks share one GPU
    # to exercise the multi-rank logic where NCCL refuses duplicate devices.
    backend = os.environ.get("CUDANP_BENCH_BACKEND", "nccl")
    dev = local % max(torch.cuda.device_count(), 1)
    torch.cuda.set_device(dev)
    if world > 1 and backend == "nccl":
        # NCCL's communicator log (the init lines name nranks and the transport)
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", dev))
        else:
            dist.init_process_group(backend)
    return rank, world, dev


def barrier(world):
    if world > 1:
        import torch.distributed as dist
        dist.barrier()


def max_over_ranks(v: float, world: int) -> float:
    if world == 1:
        return v
    import torch
    import torch.distributed as dist
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor([v], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def max_over_ranks_list(vals, world: int):
    if world == 1:
        return list(vals)
    import torch
    import torch.distributed as dist
    dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
    t = torch.tensor(vals, dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return t.tolist()


# ------------------------------------------------------------------ cudanp arm
def alg_bytes_matvec(h, w):
    # A once, x once, y once
    return 4 * h * w + 4 * h + 4 * w


def time_op(fn, reps=5, warm=2):
    import torch
    st = torch.cuda.current_stream()
    for _ in range(warm):
        fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for _ in range(reps):
        fn()
    e1.record(st)
    e1.synchronize()
    return e0.elapsed_time(e1) / reps


def run_cudanp(args):
    import torch
    from paper_conf_ppopp_yangz14_b200 import cudanp as C
    from paper_conf_ppopp_yangz14_b200 import parallel as P

    rank, world, local = dist_init(args.gpus)
    C.load()
    n = args.n
    # ---- inputs, resident in HBM (generated on the device: global indices)
    c0, c1 = C.cudanp_shard_range(n * world, world, rank)   # TMV column block
    r0, r1 = c0, c1                                         # MV row block
    wt, hm = c1 - c0, r1 - r0
    A_t = torch.empty(n, wt, dtype=torch.float32, device="cuda")
    C.cudanp_generate(A_t, "f32_unit", stream_id=1, col0=c0, w_global=n * world)
    x_t = torch.empty(n, dtype=torch.float32, device="cuda")
    C.cudanp_generate(x_t, "f32_unit", stream_id=2)
    if world == 1:
        A_m = A_t  # C2: the same 16384^2 matrix for TMV and MV
    else:
        A_m = torch.empty(hm, n, dtype=torch.float32, device="cuda")
        C.cudanp_generate(A_m, "f32_unit", stream_id=1, row0=r0, w_global=n)
    x_m = x_t
    y_t = torch.empty(wt, dtype=torch.float32, device="cuda")
    y_m = torch.empty(hm, dtype=torch.float32, device="cuda")
    torch.cuda.synchronize()

    bytes_t = alg_bytes_matvec(n, wt)
    bytes_m = alg_bytes_matvec(hm, n)

    # ---- autotune: every (S, dist, map) version timed on the resident operands --
    # the paper's exhaustive version selection, run by the
    # library's native cudanp_autotune; max over ranks so every rank picks the same.
    sweep = {"tmv": {}, "mv": {}}
    if args.no_sweep:
        def parse_cfg(s):
            S, d, m = s.split(",")
            return (int(S), {"cyclic": C.CYCLIC, "block": C.BLOCK}[d],
                    {"intra": C.INTRA_WARP, "inter": C.INTER_WARP, "inter_tma": C.INTER_WARP_TMA,
                     "auto": C.AUTO}[m])
        sweep["tmv"][parse_cfg(args.tmv_cfg)] = 1.0
        sweep["mv"][parse_cfg(args.mv_cfg)] = 1.0
    else:
        for op, A_, x_, y_, h_, w_ in (("tmv", A_t, x_t, y_t, wt, n), ("mv", A_m, x_m, y_m, hm, n)):
            _, table = C.cudanp_autotune(op, A_, x_, y_, lda=A_.shape[1], n_outer=h_, n_inner=w_,
                                         reps=5)
            cands = list(table)
            vals = max_over_ranks_list([min(table[c], 1e30) for c in cands], world)
            for cand, ms in zip(cands, vals):
                if ms < 1e29:  # not supported for this shape
                    sweep[op][cand] = ms
    best = {op: min(sweep[op], key=sweep[op].get) for op in sweep}
    best_ms = {op: sweep[op][best[op]] for op in sweep}
    if not args.no_sweep:
        # refine: the three fastest versions of each op re-timed with 30 launches
        # each (the 5-launch sweep is noisy at the 1-2 % level), max over ranks
        for op, A_, x_, y_, w_ in (("tmv", A_t, x_t, y_t, wt), ("mv", A_m, x_m, y_m, None)):
            top = sorted(sweep[op], key=sweep[op].get)[:3]
            fn = C.cudanp_tmv if op == "tmv" else C.cudanp_mv
            kw = {"n_outer": w_} if op == "tmv" else {}
            ref = [max_over_ranks(time_op(lambda c=c: fn(A_, x_, y_, S=c[0], dist=c[1], map=c[2], **kw),
                                          reps=30, warm=3), world) for c in top]
            best[op] = top[min(range(len(top)), key=ref.__getitem__)]
            best_ms[op] = min(ref)
    # literal S=1 (Fig 2) and DP (per-CTA / per-thread) comparison, once each
    comp = {}
    C.cudanp_dp_set_pending_launch_limit(1 << 16)
    for op, fn in () if args.no_sweep else (("tmv_s1_literal", lambda: C.cudanp_tmv_variant(C.S1_LITERAL, A_t, x_t, y_t)),
                   ("mv_s1_literal", lambda: C.cudanp_mv_variant(C.S1_LITERAL, A_m, x_m, y_m)),
                   ("tmv_s1_tiled", lambda: C.cudanp_tmv_variant(C.S1_TILED, A_t, x_t, y_t)),
                   ("mv_s1_tiled", lambda: C.cudanp_mv_variant(C.S1_TILED, A_m, x_m, y_m)),
                   ("tmv_dp_block", lambda: C.cudanp_tmv_variant(C.DP_BLOCK, A_t, x_t, y_t)),
                   ("mv_dp_block", lambda: C.cudanp_mv_variant(C.DP_BLOCK, A_m, x_m, y_m)),
                   ("tmv_dp_thread", lambda: C.cudanp_tmv_variant(C.DP_THREAD, A_t, x_t, y_t)),
                   ("mv_dp_thread", lambda: C.cudanp_mv_variant(C.DP_THREAD, A_m, x_m, y_m))):
        comp[op] = max_over_ranks(time_op(fn, reps=2 if "dp_" in op or "literal" in op else 10,
                                          warm=1), world)
    dp_err = C.cudanp_dp_error_count(reset=True)
    # the library's own version choice (S = CUDANP_S_AUTO, MAP_AUTO): what a
    # caller gets with default arguments, against the autotuned best
    auto = {}
    if not args.no_sweep:
        for op, fn, A_, x_, y_, kw in (("tmv", C.cudanp_tmv, A_t, x_t, y_t, {"n_outer": wt}),
                                       ("mv", C.cudanp_mv, A_m, x_m, y_m, {})):
            auto[op] = max_over_ranks(time_op(lambda: fn(A_, x_, y_, **kw), reps=30, warm=3), world)

    (St, dt, mt), (Sm, dm, mm) = best["tmv"], best["mv"]
    st = torch.cuda.current_stream()
    y_root = torch.empty(n * world, dtype=torch.float32, device="cuda") if rank == 0 else None
    ym_root = torch.empty(n * world, dtype=torch.float32, device="cuda") if rank == 0 else None

    fused = world > 1 and args.gather in ("fused", "auto")
    native = P.NativeGroup(rank, world) if world > 1 and args.gather == "native" else None
    if fused:
        fg_t = P.FusedGather(y_root, n * world, rank, world)
        fg_m = P.FusedGather(ym_root, n * world, rank, world)
        if not P.FusedGather.all_ok([fg_t, fg_m], world):
            if args.gather == "fused":
                raise SystemExit(f"--gather fused: CUDA IPC unavailable ({fg_t.error or fg_m.error})")
            fg_t.close()
            fg_m.close()
            fused = False   # auto: fall back to the NCCL send/recv gather
    if fused:
        out_t, out_m = fg_t.out_ptr(), fg_m.out_ptr()
    else:
        out_t, out_m = y_t, y_m
    gather_used = ("fused" if fused else ("native" if native else "nccl")) if world > 1 else "none"

    def step(evs=None):
        if evs:
            evs[0].record(st)
        C.cudanp_tmv(A_t, x_t, out_t, S=St, dist=dt, map=mt, n_outer=wt)
        if evs:
            evs[1].record(st)
        C.cudanp_mv(A_m, x_m, out_m, S=Sm, dist=dm, map=mm)
        if evs:
            evs[2].record(st)
        if native is not None:
            native.gather(y_t, y_root, n * world)
            native.gather(y_m, ym_root, n * world)
        elif world > 1 and not fused:
            # both gathers back to back on NCCL's stream, then one stream wait.
            # They are not overlapped with the MV kernel on purpose: its
            # persistent grid is sized to fill every SM, and an NCCL kernel
            # holding part of one SM would push a CTA of it into a second wave.
            works = P.gather_to_root(y_t, y_root, n * world, rank, world, async_op=True)
            works += P.gather_to_root(y_m, ym_root, n * world, rank, world, async_op=True)
            for wk in works:
                wk.wait()

    for _ in range(args.warmup):
        step()
    if fused:
        fg_t.finish()
    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.3)
    per_step = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(args.steps)]
    barrier(world)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(st)
    for k in range(args.steps):
        step()
    e1.record(st)
    torch.cuda.synchronize()
    barrier(world)   # with --gather fused this is also the stores' completion point
    ms = max_over_ranks(e0.elapsed_time(e1) / args.steps, world)
    # Per-kernel durations (roofline.achieved): the same K steps again with an
    # event pair around each kernel.  Kept out of the headline pass: an event
    # recorded between two kernels ends the programmatic-dependent-launch
    # overlap and cost the step ~3 % (tools/exp_step_events.py).
    barrier(world)
    torch.cuda.synchronize()
    for k in range(args.steps):
        step(per_step[k])
    torch.cuda.synchronize()
    barrier(world)
    clk = clocks.stop()
    t_tmv = statistics.mean(ev[0].elapsed_time(ev[1]) for ev in per_step)
    t_mv = statistics.mean(ev[1].elapsed_time(ev[2]) for ev in per_step)
    t_tmv = max_over_ranks(t_tmv, world)
    t_mv = max_over_ranks(t_mv, world)
    total_bytes = (bytes_t + bytes_m) * world   # per step, all ranks
    value = total_bytes / (ms * 1e-3) / 1e9

    # ---- end to end through the public API with HOST buffers (pinned)
    e2e = None
    if args.e2e_steps > 0:
        A_h = torch.empty(A_t.shape, dtype=torch.float32, pin_memory=True)
        A_h.copy_(A_t)
        if A_m is A_t:
            Am_h = A_h
        else:
            Am_h = torch.empty(A_m.shape, dtype=torch.float32, pin_memory=True)
            Am_h.copy_(A_m)
        x_h = torch.empty(n, dtype=torch.float32, pin_memory=True)
        x_h.copy_(x_t)
        yt_h = torch.empty(wt, dtype=torch.float32, pin_memory=True)
        ym_h = torch.empty(hm, dtype=torch.float32, pin_memory=True)
        torch.cuda.synchronize()

        def e2e_step():
            A_t.copy_(A_h, non_blocking=True)
            if Am_h is not A_h:
                A_m.copy_(Am_h, non_blocking=True)
            x_t.copy_(x_h, non_blocking=True)
            C.cudanp_tmv(A_t, x_t, y_t, S=St, dist=dt, map=mt)
            C.cudanp_mv(A_m, x_m, y_m, S=Sm, dist=dm, map=mm)
            yt_h.copy_(y_t, non_blocking=True)
            ym_h.copy_(y_m, non_blocking=True)
        e2e_step()
        barrier(world)
        torch.cuda.synchronize()
        f0, f1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        f0.record(st)
        for _ in range(args.e2e_steps):
            e2e_step()
        f1.record(st)
        torch.cuda.synchronize()
        e2e_ms = max_over_ranks(f0.elapsed_time(f1) / args.e2e_steps, world)
        h2d = A_h.numel() * 4 + (0 if Am_h is A_h else Am_h.numel() * 4) + x_h.numel() * 4
        d2h = (yt_h.numel() + ym_h.numel()) * 4
        # the PCIe bound of this path: the same pinned H2D copies alone
        f0.record(st)
        for _ in range(args.e2e_steps):
            A_t.copy_(A_h, non_blocking=True)
            if Am_h is not A_h:
                A_m.copy_(Am_h, non_blocking=True)
            x_t.copy_(x_h, non_blocking=True)
        f1.record(st)
        torch.cuda.synchronize()
        copy_ms = max_over_ranks(f0.elapsed_time(f1) / args.e2e_steps, world)
        e2e = {"value": round(total_bytes / (e2e_ms * 1e-3) / 1e9, 3), "unit": "GB/s",
               "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
               "ms_per_step": round(e2e_ms, 4),
               "h2d_alone_ms": round(copy_ms, 4),
               "h2d_gbs": round(h2d / (copy_ms * 1e-3) / 1e9, 1),
               "bound": "PCIe host->device: the step's H2D copies alone take "
                        f"{100 * copy_ms / e2e_ms:.1f} % of the e2e step",
               "path": "pinned host A,x -> H2D -> cudanp_tmv + cudanp_mv -> D2H y (per rank)"}
        del A_h, Am_h

    # ---- C5 (BASELINE configs[4]): strong scaling over the N ranks
    c5 = None
    if not args.no_c5:
        del A_t, A_m, x_t, x_m, y_t, y_m
        torch.cuda.empty_cache()
        # C5's outputs are bulk (64M floats for the reduce): "auto" gathers them
        # with NCCL's bulk send/recv rather than as 16-byte remote stores from
        # the kernel's masters; --gather fused / native force those paths.
        c5_gather = "nccl" if args.gather == "auto" else gather_used
        c5 = run_c5(C, P, rank, world, args.c5_steps, c5_gather if world > 1 else "none")

    if rank != 0:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()
        return

    peak, peak_src = hbm_peak()
    if c5 is not None:
        for rec in (c5["tmv"], c5["reduce"]):
            rec["frac_of_n_peak"] = round(rec["agg_gbs_kernel"] / (world * peak), 4)
    dom = "tmv" if t_tmv >= t_mv else "mv"
    dom_bytes = bytes_t if dom == "tmv" else bytes_m
    dom_ms = t_tmv if dom == "tmv" else t_mv
    achieved = dom_bytes / (dom_ms * 1e-3) / 1e9
    traffic = None
    try:
        tr = json.load(open(os.path.join(ROOT, "profiles", "ncu_traffic.json")))
        traffic = tr.get(dom, {}).get("dram_bytes_per_launch")
    except Exception:
        pass

    def gbs(nb, t):
        return round(nb / (t * 1e-3) / 1e9, 1)

    # "tuned S=1" = the best no-NP kernel: the S=1 instantiations, the literal and
    # the TMA-tiled S=1 kernel (rows staged through shared memory: the paper's
    # "already optimized" SMM-style baseline)
    def best_s1(op):
        c = [v for (S, d, m), v in sweep[op].items() if S == 1]
        for extra in (f"{op}_s1_literal", f"{op}_s1_tiled"):  # every no-NP kernel we have
            if extra in comp:
                c.append(comp[extra])
        return min(c or [float("nan")])

    per_S = {}
    for op, nb in (("tmv", bytes_t), ("mv", bytes_m)):
        s1 = best_s1(op)
        for S in sorted(set(C.SLAVE_SIZES + C.INTER_ONLY_SIZES + C.MULTI_WARP_SIZES
                            + C.TMV_CLUSTER_SIZES + C.CLUSTER_SIZES)):
            cand = {k: v for k, v in sweep[op].items() if k[0] == S}
            if not cand:
                continue
            k = min(cand, key=cand.get)
            per_S.setdefault(str(S), {})[op] = {
                "gbs": gbs(nb, cand[k]), "ms": round(cand[k], 4),
                "speedup_vs_s1": round(s1 / cand[k], 3),
                "dist": "cyclic" if k[1] == C.CYCLIC else "block",
                "map": MAPN[k[2]],
                "all": {f"{'cyc' if d == C.CYCLIC else 'blk'}/{MAPN[m]}":
                        gbs(nb, v) for (SS, d, m), v in cand.items()}}
    s1_tmv, s1_mv = best_s1("tmv"), best_s1("mv")

    line = {
        "metric": METRIC, "value": round(value, 2), "unit": "GB/s", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms, 5),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic (device counter-based generator, f32_unit in (0,1); SURVEY C-4)",
        "config": {
            "workload": f"C2: TMV y=A^T x + MV y=A x, {n}x{n} fp32 per rank (BASELINE configs[1])",
            "h": n, "w": n, "outer_items_per_rank": {"tmv": wt, "mv": hm}, "inner_count": n,
            "tmv": {"S": St, "dist": "cyclic" if dt == 0 else "block", "map": MAPN[mt]},
            "mv": {"S": Sm, "dist": "cyclic" if dm == 0 else "block", "map": MAPN[mm]},
            "parallelism": (f"dp{world}: contiguous outer-item shards + "
                            + ("gather fused into the master stores (CUDA IPC over NVLink; no "
                               "collective kernel)" if fused else "NCCL send/recv gather to rank 0"
                               + (" (library group, cudanp_group_gather)" if native else "")))
                           if world > 1 else "single GPU",
            "gather": gather_used,
            "l2": "no flush: each matrix is 1 GiB > 126 MB L2",
            "step": "cudanp_tmv + cudanp_mv (+ gather when n_gpus > 1)",
        },
        "roofline": {"bound": "hbm", "kernel": f"cudanp_{dom}", "achieved": round(achieved, 1),
                     "peak": peak, "unit": "GB/s", "frac": round(achieved / peak, 4),
                     "traffic": traffic, "peak_source": peak_src,
                     "alg_bytes_per_launch": dom_bytes, "avg_launch_ms": round(dom_ms, 5),
                     "launch_timing": "event pair around each kernel over a second pass of the "
                                      "same K steps right after the headline pass"},
        "kernels": {"tmv": {"avg_ms": round(t_tmv, 5), "gbs": gbs(bytes_t, t_tmv),
                            "speedup_vs_s1": round(s1_tmv / t_tmv, 3),
                            "s1_tuned_ms": round(s1_tmv, 5)},
                    "mv": {"avg_ms": round(t_mv, 5), "gbs": gbs(bytes_m, t_mv),
                           "speedup_vs_s1": round(s1_mv / t_mv, 3),
                           "s1_tuned_ms": round(s1_mv, 5)}},
        "auto": {op: {"gbs": gbs(bytes_t if op == "tmv" else bytes_m, v),
                      "vs_autotuned_best": round(best_ms[op] / v, 4),
                      "choice": dict(zip(("S", "dist", "map"),
                                         C.cudanp_choose_version(op, wt if op == "tmv" else hm, n)))}
                 for op, v in auto.items()},
        "per_S": per_S,
        "comparison_ms": {k: round(v, 4) for k, v in comp.items()} | {"dp_launch_errors": dp_err},
        "gpu_launches": 2 * args.steps,
        "clocks": clk,
        "e2e": e2e,
        # the paper's own speedups (other hardware): context, not a target
        "paper_context": {"speedup_over_optimized_baseline": {"max": 6.69, "geomean": 2.18,
                                                              "range_min": 1.36},
                          "tmv_vs_cublas": 4.9, "tmv_dp_slowdown": 7.61,
                          "hardware": "GTX 680 (DP: Tesla K20c)",
                          "source": "PAPER.md P:23, P:41, P:417, P:451, P:482"},
    }
    if c5 is not None:
        line["c5"] = c5
    if not args.no_cpu_baseline:
        line["cpu_baseline"] = cpu_baseline_subprocess(n, args.cpu_rows)
    print(json.dumps(line), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()


# ------------------------------------------------------------------ C5 strong scaling
C5_N_TMV = 65536
C5_N_RED, C5_L_RED = 1 << 26, 64


def run_c5(C, P, rank, world, steps, gather_mode):
    """BASELINE configs[4]: TMV 65536 x 65536 fp32 sharded by column blocks and
    a 64M-item x 64 fp32 loop-reduce sharded by item blocks (contiguous outer
    ranges), outputs gathered to rank 0.  Strong scaling: the
    problem is fixed, each rank generates its 1/N from global indices.  Per op:
    version = the library's autotune on the shard (max over ranks), timed
    `steps` times as kernel + gather with device events, max over ranks; the
    library's own choice (S_AUTO) timed beside it; then pin P4 on exact data:
    the gathered result must equal, bit for bit, the unsharded result that
    rank 0 computes alone (at N = 1 the run is the unsharded one)."""
    import torch
    import torch.distributed as dist
    fused = world > 1 and gather_mode == "fused"
    native = P.NativeGroup(rank, world) if world > 1 and gather_mode == "native" else None
    st = torch.cuda.current_stream()
    out = {"workload": "C5: TMV 65536x65536 fp32 by column shards + 64M x 64 fp32 loop-reduce by "
                       "item shards (BASELINE configs[4])",
           "scaling": "strong", "n_gpus": world,
           "gather": (gather_mode if world > 1 else "none (single GPU: outputs written in place)"),
           "l2": "no flush: 16 GiB operands per op"}
    for op in ("tmv", "reduce"):
        total = C5_N_TMV if op == "tmv" else C5_N_RED
        b, e = P.shard(total, world, rank)
        if op == "tmv":
            n = C5_N_TMV
            A = torch.empty(n, e - b, dtype=torch.float32, device="cuda")
            x = torch.empty(n, dtype=torch.float32, device="cuda")
            nbytes = 4 * n * n + 8 * n
        else:
            A = torch.empty(e - b, C5_L_RED, dtype=torch.float32, device="cuda")
            x = None
            nbytes = 4 * C5_N_RED * C5_L_RED + 4 * C5_N_RED

        def fill(kind):
            if op == "tmv":
                C.cudanp_generate(A, kind, stream_id=1, col0=b, w_global=C5_N_TMV)
                C.cudanp_generate(x, kind, stream_id=2)
            else:
                C.cudanp_generate(A, kind, stream_id=1, row0=b, w_global=C5_L_RED)
        fill("f32_unit")
        root = torch.empty(total, dtype=torch.float32, device="cuda") if rank == 0 else None
        y = root if world == 1 else torch.empty(e - b, dtype=torch.float32, device="cuda")
        fg = P.FusedGather(root, total, rank, world) if fused else None
        if fg is not None and not P.FusedGather.all_ok([fg], world):
            fg.close()
            fg, fused = None, False  # fall back to the NCCL send/recv gather
            out["gather"] = "nccl (CUDA IPC unavailable)"
        dst = fg.out_ptr() if fused else y

        def kernel(S, d, m, o=None):
            o = dst if o is None else o
            if op == "tmv":
                C.cudanp_tmv(A, x, o, S=S, dist=d, map=m, n_outer=e - b)
            else:
                C.cudanp_batched_loop_reduce(A, None, o, S=S, dist=d, map=m)

        def gather():
            if native is not None:
                native.gather(y, root, total)
            elif world > 1 and not fused:
                P.gather_to_root(y, root, total, rank, world)

        # version selection on this rank's shard, max over ranks so all agree
        _, table = C.cudanp_autotune(op, A, x, y, lda=A.shape[1], n_outer=e - b,
                                     n_inner=C5_N_TMV if op == "tmv" else C5_L_RED, reps=3)
        cands = list(table)
        vals = max_over_ranks_list([min(table[c], 1e30) for c in cands], world)
        S, d, m = cands[min(range(len(cands)), key=vals.__getitem__)]
        for _ in range(2):
            kernel(S, d, m)
            gather()
        if fused:
            fg.finish()
        tk, tg = [], []
        for _ in range(steps):
            barrier(world)
            torch.cuda.synchronize()
            e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
            e0.record(st)
            kernel(S, d, m)
            e1.record(st)
            gather()
            e2.record(st)
            torch.cuda.synchronize()
            if fused:
                fg.finish()
            tk.append(e0.elapsed_time(e1))
            tg.append(e1.elapsed_time(e2))
        k_ms = max_over_ranks(statistics.median(tk), world)
        g_ms = max_over_ranks(statistics.median(tg), world)
        e_ms = max_over_ranks(statistics.median([p + q for p, q in zip(tk, tg)]), world)
        # the library's own choice (S_AUTO), kernel only
        ta = max_over_ranks(time_op(lambda: kernel(C.S_AUTO, C.CYCLIC, C.AUTO, y), reps=steps, warm=2), world)
        rec = {"S": S, "dist": "cyclic" if d == C.CYCLIC else "block", "map": MAPN.get(m, str(m)),
               "outer_total": total, "inner": C5_N_TMV if op == "tmv" else C5_L_RED,
               "alg_bytes": nbytes, "kernel_max_ms": round(k_ms, 4), "gather_ms": round(g_ms, 4),
               "e2e_ms": round(e_ms, 4),
               "agg_gbs_kernel": round(nbytes / (k_ms * 1e-3) / 1e9, 1),
               "agg_gbs_e2e": round(nbytes / (e_ms * 1e-3) / 1e9, 1),
               "auto": {"choice": dict(zip(("S", "dist", "map"),
                                           C.cudanp_choose_version(op, e - b, C5_N_TMV if op == "tmv" else C5_L_RED))),
                        "kernel_ms": round(ta, 4), "vs_autotuned_best": round(k_ms / ta, 4)}}
        # pin P4 on exact data (every summation order gives the same bits)
        fill("f32_int4")
        kernel(S, d, m)
        gather()
        torch.cuda.synchronize()
        if fused:
            fg.finish()
        if rank == 0 and world > 1:
            A = None
            torch.cuda.empty_cache()
            if op == "tmv":
                Af = torch.empty(C5_N_TMV, C5_N_TMV, dtype=torch.float32, device="cuda")
                C.cudanp_generate(Af, "f32_int4", stream_id=1)
                full = C.cudanp_tmv(Af, x, S=S, dist=d, map=m)
            else:
                Af = torch.empty(C5_N_RED, C5_L_RED, dtype=torch.float32, device="cuda")
                C.cudanp_generate(Af, "f32_int4", stream_id=1)
                full = C.cudanp_batched_loop_reduce(Af, None, S=S, dist=d, map=m)
            torch.cuda.synchronize()
            rec["p4_sharded_equals_unsharded"] = bool(torch.equal(full, root))
            del Af, full
        elif rank == 0:
            rec["p4_sharded_equals_unsharded"] = "n/a at N = 1 (the run is unsharded)"
        barrier(world)
        if fg:
            fg.close()
        out[op] = rec
        A = x = y = root = dst = None
        torch.cuda.empty_cache()
    if native is not None:
        native.close()
    return out


# ------------------------------------------------------------------ oracle (CPU) legs
def _cpu_sample(n, rows):
    """The CPU sample both arms time: the first `rows` rows of the C2 matrix
    (generated on the host by synth, the same values the device generator
    makes) and x."""
    import synth
    rows = min(rows, n)
    return synth.matrix(rows, n, "f32_unit"), synth.vector(n, "f32_unit"), rows


def _oracle_pass(A, x, rows, threads):
    """One oracle pass over the sample: TMV over its rows (all columns) and MV
    over its rows; threads > 1 runs the same oracle functions over contiguous
    outer-item ranges."""
    import oracle as O
    t0 = time.perf_counter()
    if threads > 1:
        O.tmv_parallel(A, x[:rows], threads)
        O.mv_parallel(A, x, threads)
    else:
        O.tmv(A, x[:rows])
        O.mv(A, x)
    dt = time.perf_counter() - t0
    return dt, 2 * alg_bytes_matvec(rows, A.shape[1])


def _timed_oracle(A, x, rows, threads, budget_s=None, passes=None):
    tot_t, tot_b, reps = 0.0, 0, 0
    while (passes is not None and reps < passes) or (passes is None and tot_t < budget_s and reps < 5000):
        dt, nb = _oracle_pass(A, x, rows, threads)
        tot_t += dt
        tot_b += nb
        reps += 1
        if passes is not None and tot_t > 150:
            break
    return tot_b / tot_t / 1e9, reps, tot_t


def _cpu_warm(A, x, rows, threads, passes=1, min_s=2.0):
    """Untimed passes (page-in, thread start-up, core clocks ramping): at least
    `passes` and at least `min_s` seconds, in both arms alike."""
    t0 = time.perf_counter()
    k = 0
    while k < passes or time.perf_counter() - t0 < min_s:
        _oracle_pass(A, x, rows, threads)
        k += 1


def _sample_text(n, rows, cores):
    return (f"TMV + MV over the first {rows} of {n} rows of the C2 matrix (1/{n // rows} of one "
            f"step; the oracle's plain fp64-accumulating loops), {cores} threads over contiguous "
            f"outer-item ranges")


def cpu_baseline(n, rows):
    """The oracle as it stands on the bounded sample (_cpu_sample) -- the same
    sample and thread count the `--impl reference` arm times -- about 10 s on
    all host cores, plus about 10 s on one core."""
    A, x, rows = _cpu_sample(n, rows)
    cores = os.cpu_count() or 1
    _cpu_warm(A, x, rows, cores)
    v_all, reps_all, t_all = _timed_oracle(A, x, rows, cores, budget_s=10.0)
    v_one, reps_one, t_one = _timed_oracle(A, x, rows, 1, budget_s=10.0)
    return {"value": round(v_all, 4), "unit": "GB/s", "cores": cores, "kind": "oracle",
            "sample": _sample_text(n, rows, cores) + f": {reps_all} passes in {t_all:.1f} s; "
                      f"1 core: {reps_one} passes in {t_one:.1f} s",
            "value_1core": round(v_one, 4), "cpu": _cpu_model()}


def cpu_baseline_subprocess(n, rows):
    """cpu_baseline in a fresh process with no CUDA context (the same
    function the --impl reference arm runs): this process's GPU state --
    pinned host buffers, driver threads -- slowed the oracle by up to 40 %
    when it ran in-process (bench r02t: 3.8 vs 5.3 GB/s)."""
    r = subprocess.run([sys.executable, os.path.abspath(__file__), "--cpu-sample-json", "--n", str(n),
                        "--cpu-rows", str(rows)], capture_output=True, text=True, timeout=600)
    try:
        return json.loads(r.stdout.strip().splitlines()[-1])
    except Exception:
        return {"value": None, "unit": "GB/s", "kind": "oracle", "error": (r.stderr or r.stdout)[-300:]}


def _cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip() + f" x{os.cpu_count()}"
    except Exception:
        pass
    return None


def run_reference(args):
    """--impl reference: the oracle on the host cores, same metric/config; each
    step = one oracle pass over the same sample the cudanp arm's cpu_baseline
    times (so the run states one CPU rate)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    n = args.n
    A, x, rows = _cpu_sample(n, args.cpu_rows)
    cores = os.cpu_count() or 1
    _cpu_warm(A, x, rows, cores, passes=max(args.warmup, 1))
    value, steps, tot_t = _timed_oracle(A, x, rows, cores, passes=max(args.steps, 1))
    ms = tot_t / steps * 1e3
    sample = "each step: " + _sample_text(n, rows, cores)
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": round(value, 4), "unit": "GB/s",
        "n_gpus": args.gpus, "steps": steps, "warmup": args.warmup, "ms_per_step": round(ms, 3),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64-accum",
        "data": "synthetic (counter-based generator, f32_unit)",
        "config": {"workload": f"C2: TMV y=A^T x + MV y=A x, {n}x{n} fp32 per rank (BASELINE configs[1]); "
                               f"sampled rows", "h": n, "w": n, "sample_rows": rows},
        "cpu_baseline": {"value": round(value, 4), "unit": "GB/s", "cores": cores, "kind": "oracle",
                         "sample": sample, "cpu": _cpu_model()},
        "e2e": {"value": round(value, 4), "unit": "GB/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }), flush=True)


def oracle_timing(path, cap_s):
    """SURVEY §8(d) "Oracle timing": the oracle's on-the-fly-generating forms
    (orc_*_gen: inputs recomputed from the counter-based generator, no
    multi-GiB host copies) timed on C1-C5 on 1 core and on all host cores
    (contiguous outer-item ranges, one thread each), plus a generation-only
    pass over the same input elements.  A run that would exceed `cap_s` is
    stopped after whole chunks and extrapolated (the record says the fraction
    done).  The oracle as it stands -- never tuned for this."""
    import ctypes
    from concurrent.futures import ThreadPoolExecutor

    import oracle as O
    L = O.lib()
    cores = os.cpu_count() or 1
    seed = O.SEED
    K = O.KIND

    def tmv_chunk(h, w):
        def f(lo, hi):
            cols = np.arange(lo, hi, dtype=np.int64)
            y = np.empty(hi - lo, np.float32)
            L.orc_tmv_gen(seed, K["f32_unit"], K["f32_unit"], h, w, cols.ctypes.data, hi - lo, y.ctypes.data)
        return f

    def mv_chunk(h, w):
        def f(lo, hi):
            rows = np.arange(lo, hi, dtype=np.int64)
            y = np.empty(hi - lo, np.float32)
            L.orc_mv_gen(seed, K["f32_unit"], K["f32_unit"], h, w, rows.ctypes.data, hi - lo, y.ctypes.data)
        return f

    def reduce_chunk(Lc):
        def f(lo, hi):
            it = np.arange(lo, hi, dtype=np.int64)
            o = np.empty(hi - lo, np.float32)
            L.orc_reduce_gen(seed, O.F32, K["f32_unit"], 1 << 20, -1, Lc, O.SUM, it.ctypes.data, hi - lo,
                             o.ctypes.data)
        return f

    def scan_chunk(Lc):
        def f(lo, hi):
            it = np.arange(lo, hi, dtype=np.int64)
            o = np.empty((hi - lo) * Lc, np.int32)
            L.orc_scan_gen(seed, O.I32, K["i32_small"], 1 << 15, -1, Lc, it.ctypes.data, hi - lo, o.ctypes.data)
        return f

    def gen_chunk():
        buf = {}

        def f(lo, hi):  # generation only: the same input elements, materialized in a scratch buffer
            b = buf.setdefault(threading.get_ident(), np.empty(1 << 22, np.float32))
            i = lo
            while i < hi:
                n = min(hi - i, b.size)
                L.orc_gen_f32(seed, 1, K["f32_unit"], i, n, b.ctypes.data)
                i += n
        return f

    def timed(fn, n_outer, chunk, threads):
        """Run fn over [0, n_outer) in chunks of `chunk`, on `threads` threads,
        until done or cap_s; return (seconds extrapolated to all, fraction done)."""
        bounds = [(lo, min(lo + chunk, n_outer)) for lo in range(0, n_outer, chunk)]
        done, t0 = 0, time.perf_counter()
        with ThreadPoolExecutor(threads) as ex:
            for k in range(0, len(bounds), threads):
                list(ex.map(lambda b: fn(*b), bounds[k:k + threads]))
                done += sum(b[1] - b[0] for b in bounds[k:k + threads])
                if time.perf_counter() - t0 > cap_s:
                    break
        dt = time.perf_counter() - t0
        return dt * n_outer / done, done / n_outer

    cases = [("C1", "tmv", 1024, 1024, tmv_chunk(1024, 1024), 4 * 1024 * 1024 + 8 * 1024, 1024 * 1024),
             ("C2", "tmv", 16384, 16384, tmv_chunk(16384, 16384), 4 * 16384 ** 2 + 8 * 16384, 16384 ** 2),
             ("C2", "mv", 16384, 16384, mv_chunk(16384, 16384), 4 * 16384 ** 2 + 8 * 16384, 16384 ** 2)]
    cases += [("C3", "reduce", 1 << 22, Lc, reduce_chunk(Lc), 4 * (1 << 22) * Lc + 4 * (1 << 22), (1 << 22) * Lc)
              for Lc in (32, 64, 128, 256)]
    cases += [("C4", "scan", 1 << 21, Lc, scan_chunk(Lc), 8 * (1 << 21) * Lc, (1 << 21) * Lc)
              for Lc in (64, 128, 256, 512, 1024)]
    cases += [("C5", "tmv", 65536, 65536, tmv_chunk(65536, 65536), 4 * 65536 ** 2 + 8 * 65536, 65536 ** 2),
              ("C5", "reduce", 1 << 26, 64, reduce_chunk(64), 4 * (1 << 26) * 64 + 4 * (1 << 26), (1 << 26) * 64)]
    with open(path, "w") as f:
        for cfg, op, N, Lc, fn, nbytes, elems in cases:
            chunk = max(1, N // (64 * cores))
            rec = {"config": cfg, "op": op, "N": N, "L": Lc, "alg_bytes": nbytes, "elements": elems,
                   "cpu": _cpu_model(), "cores": cores, "kind": "oracle (on-the-fly generation)"}
            for name, threads in (("1core", 1), ("allcore", cores)):
                t, frac = timed(fn, N, chunk, threads)
                rec[f"s_{name}"] = round(t, 3)
                rec[f"gbs_{name}"] = round(nbytes / t / 1e9, 4)
                rec[f"frac_done_{name}"] = round(frac, 4)
            tg, fg = timed(gen_chunk(), elems, max(1, elems // (64 * cores)), cores)
            rec["s_gen_only_allcore"] = round(tg, 3)
            rec["frac_done_gen_only"] = round(fg, 4)
            rec["s_compute_allcore"] = round(max(rec["s_allcore"] - tg, 0.0), 3)
            f.write(json.dumps(rec) + "\n")
            f.flush()
            print(json.dumps(rec), flush=True)
    del ctypes


def main():
    args = parse()
    if args.oracle_timing:
        oracle_timing(args.oracle_timing, args.oracle_cap_s)
        return
    if args.cpu_sample_json:
        print(json.dumps(cpu_baseline(args.n, args.cpu_rows)), flush=True)
        return
    if args.impl == "reference":
        run_reference(args)
    else:
        run_cudanp(args)


if __name__ == "__main__":
    main()
