#!/usr/bin/env python
"""Sweep every config of BASELINE.json (C1-C5 at G=1) over S x dist x map,
plus the S=1 literal (Fig 2) and dynamic-parallelism comparison kernels --
the analog of the paper's Figs 11, 13, 14 and its DP comparison.

    python tools/sweep.py [--configs C1,C2,C3,C4,C5] [--out gpurun_out/sweep.jsonl]

One JSON record per (config, op, dtype, L, S, dist, map, impl): median time,
algorithmic bytes, GB/s, fraction of the measured HBM peak, speedup vs the
best no-NP kernel ("tuned S=1": the faster of the S=1 instantiations and the
literal) and vs the literal Fig 2 kernel.
Timing: CUDA events on the launching stream, 2 warm-ups, median of reps.
Inputs >= 512 MB exceed the 126 MB L2; C1 (4 MiB) is timed as a CUDA graph
of 64 launches over 64 distinct copies (256 MiB) so every launch reads cold.
"""
from __future__ import annotations

import argparse
import itertools
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_ppopp_yangz14_b200 import cudanp as C  # noqa: E402

PEAK = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))).get("hbm_gbs", 6537.0) \
    if os.path.exists(os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6537.0
DN = {C.CYCLIC: "cyclic", C.BLOCK: "block"}
MN = {C.INTRA_WARP: "intra", C.INTER_WARP: "inter", C.INTER_WARP_TMA: "inter_tma", C.INTRA_WARP_TMA: "intra_tma"}
OUT = None


def emit(rec):
    rec["frac_hbm"] = round(rec["gbs"] / PEAK, 4) if rec.get("gbs") else None
    line = json.dumps(rec)
    print(line, flush=True)
    if OUT:
        OUT.write(line + "\n")
        OUT.flush()


_FLUSH = None


def flush_l2():
    """Read a buffer twice the 126 MB L2 so the next launch reads cold HBM.
    (Reading, not writing: a write-flush leaves ~126 MB of dirty lines whose
    write-back then competes with the timed kernel.)"""
    global _FLUSH
    if _FLUSH is None:
        _FLUSH = torch.ones(64 << 20, dtype=torch.int32, device="cuda")
    _FLUSH.max()


def time_ms(fn, reps=5, warm=2, flush=False):
    st = torch.cuda.current_stream()
    for _ in range(warm):
        fn()
    ts = []
    for _ in range(reps):
        if flush:
            flush_l2()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        fn()
        b.record(st)
        b.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts), min(ts)


def steady_ms(fn, R=20, reps=5):
    """Per-launch time of R back-to-back launches between one event pair: the
    rate a pipeline of repeated calls sees (launch latency and the grid's
    ramp/tail overlap the neighbouring launches through PDL)."""
    for _ in range(3):
        fn()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(R):
            fn()
        b.record()
        b.synchronize()
        ts.append(a.elapsed_time(b) / R)
    return statistics.median(ts)


def graph_time_ms(fns, reps=5):
    """Capture a CUDA graph calling every fn once; return per-launch time."""
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for f in fns:
            f()
    torch.cuda.current_stream().wait_stream(s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        for f in fns:
            f()
    g.replay()
    torch.cuda.synchronize()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        g.replay()
        b.record()
        b.synchronize()
        ts.append(a.elapsed_time(b) / len(fns))
    return statistics.median(ts), min(ts)


def sweep_np(cfg, op, nbytes, run, extra, s1_ref=None, literal=None, comps=(), maps=None, call=None,
             big=(), auto=None):
    """run(S, dist, map) -> (median_ms, min_ms).  s1_ref: extra no-NP kernel
    times (e.g. the TMA-staged S=1 TMV) that count toward "tuned S=1".
    call(S, dist, map) -> a one-launch callable: the best NP and the best S=1
    version are then also timed back to back (steady state)."""
    res = {}
    if maps is None:  # TMV and reduce also have TMA-staged kernels
        maps = (C.INTRA_WARP, C.INTER_WARP) + {"tmv": (C.INTER_WARP_TMA,),
                                               "reduce": (C.INTRA_WARP_TMA,)}.get(op, ())
    cands = list(itertools.product(C.SLAVE_SIZES, (C.CYCLIC, C.BLOCK), maps)) + \
        [(S, d, m) for S, m in big for d in (C.CYCLIC, C.BLOCK)]
    if C.INTER_WARP in maps and op in ("tmv", "mv", "reduce", "scan"):
        # non-power-of-two inter-warp teams (Fig 12)
        cands += list(itertools.product(C.INTER_ONLY_SIZES, (C.CYCLIC, C.BLOCK), (C.INTER_WARP,)))
    for S, d, m in cands:
        try:
            res[(S, d, m)] = run(S, d, m)
        except C.CudanpError:
            if m in (C.INTER_WARP_TMA, C.INTRA_WARP_TMA):
                continue  # e.g. the TMA reduce needs L % 4 == 0
            raise
    # "tuned S=1" = the best no-NP kernel: the S=1 NP-path instantiations and the
    # Fig 2 literal, whichever is faster.
    s1 = min([v[0] for k, v in res.items() if k[0] == 1] + ([literal] if literal else [])
             + list(s1_ref or []))
    for (S, d, m), (med, mn) in res.items():
        rec = {"config": cfg, "op": op, **extra, "S": S, "dist": DN[d], "map": MN[m], "impl": "np",
               "t_median_us": round(med * 1e3, 2), "t_min_us": round(mn * 1e3, 2),
               "alg_bytes": nbytes, "gbs": round(nbytes / (med * 1e-3) / 1e9, 1),
               "speedup_vs_s1_tuned": round(s1 / med, 3)}
        if literal:
            rec["speedup_vs_s1_literal"] = round(literal / med, 3)
        emit(rec)
    best = min(res, key=lambda k: res[k][0])
    for name, t in comps:
        emit({"config": cfg, "op": op, **extra, "impl": name, "t_median_us": round(t * 1e3, 2),
              "alg_bytes": nbytes, "gbs": round(nbytes / (t * 1e-3) / 1e9, 1),
              "speedup_of_best_np": round(t / res[best][0], 3)})
    bS, bd, bm = best
    # Fig 12 analog: each non-power-of-two inter-warp S against the power of two
    # it would be padded to under intra-warp NP's limit
    for S in C.INTER_ONLY_SIZES:
        P2 = 1 << (S - 1).bit_length()
        for d in (C.CYCLIC, C.BLOCK):
            k, kp = (S, d, C.INTER_WARP), (P2, d, C.INTER_WARP)
            if k in res and kp in res:
                emit({"config": cfg, "op": op, **extra, "impl": "fig12", "S": S, "S_padded": P2,
                      "dist": DN[d], "map": "inter", "t_median_us": round(res[k][0] * 1e3, 2),
                      "t_padded_us": round(res[kp][0] * 1e3, 2), "alg_bytes": nbytes,
                      "gbs": round(nbytes / (res[k][0] * 1e-3) / 1e9, 1),
                      "gbs_padded": round(nbytes / (res[kp][0] * 1e-3) / 1e9, 1),
                      "speedup_vs_padded": round(res[kp][0] / res[k][0], 3)})
    if auto is not None:  # the library's own choice (S = S_AUTO, MAP_AUTO)
        ta = auto()[0]
        emit({"config": cfg, "op": op, **extra, "impl": "auto", "t_median_us": round(ta * 1e3, 2),
              "alg_bytes": nbytes, "gbs": round(nbytes / (ta * 1e-3) / 1e9, 1),
              "vs_best_np": round(res[best][0] / ta, 3), "vs_s1_tuned": round(s1 / ta, 3)})
    steady = {}
    if call is not None:
        best1 = min((k for k in res if k[0] == 1), key=lambda k: res[k][0])
        tb, t1 = steady_ms(call(*best)), steady_ms(call(*best1))
        steady = {"t_steady_us": round(tb * 1e3, 2), "gbs_steady": round(nbytes / (tb * 1e-3) / 1e9, 1),
                  "s1_steady": f"{best1[0]},{DN[best1[1]]},{MN[best1[2]]}",
                  "gbs_s1_steady": round(nbytes / (t1 * 1e-3) / 1e9, 1),
                  "speedup_vs_s1_steady": round(t1 / tb, 3)}
    emit({"config": cfg, "op": op, **extra, "impl": "best_np", "S": bS, "dist": DN[bd], "map": MN[bm],
          "t_median_us": round(res[best][0] * 1e3, 2), "alg_bytes": nbytes,
          "gbs": round(nbytes / (res[best][0] * 1e-3) / 1e9, 1),
          "speedup_vs_s1_tuned": round(s1 / res[best][0], 3),
          **({"speedup_vs_s1_literal": round(literal / res[best][0], 3)} if literal else {}), **steady})
    return res, best


def gen(shape, kind, dtype=torch.float32, stream_id=1, B=1 << 20):
    t = torch.empty(*shape, dtype=dtype, device="cuda")
    C.cudanp_generate(t, kind, stream_id=stream_id, B=B)
    return t


def c1():
    n, copies = 1024, 64
    As = [gen((n, n), "f32_unit") for _ in range(copies)]
    x = gen((n,), "f32_unit", stream_id=2)
    ys = [torch.empty(n, device="cuda") for _ in range(copies)]
    nb = 4 * n * n + 8 * n

    def run(S, d, m):
        return graph_time_ms([lambda i=i: C.cudanp_tmv(As[i], x, ys[i], S=S, dist=d, map=m)
                              for i in range(copies)])
    lit = graph_time_ms([lambda i=i: C.cudanp_tmv_variant(C.S1_LITERAL, As[i], x, ys[i]) for i in range(copies)])[0]
    tiled = graph_time_ms([lambda i=i: C.cudanp_tmv_variant(C.S1_TILED, As[i], x, ys[i]) for i in range(copies)])[0]
    comps = [("s1_literal", lit), ("s1_tiled", tiled)]
    for impl, name in ((C.DP_BLOCK, "dp_block"), (C.DP_THREAD, "dp_thread")):
        comps.append((name, time_ms(lambda: C.cudanp_tmv_variant(impl, As[0], x, ys[0]), reps=5)[0]))
    sweep_np("C1", "tmv", nb, run, {"dtype": "f32", "N": n, "L": n}, literal=lit, comps=comps, s1_ref=[tiled],
             auto=lambda: graph_time_ms([lambda i=i: C.cudanp_tmv(As[i], x, ys[i]) for i in range(copies)]))
    for S in (64, 128):  # teams larger than a warp (inter-warp, 8 masters per CTA)
        for d in (C.CYCLIC, C.BLOCK):
            med, mn = run(S, d, C.INTER_WARP)
            emit({"config": "C1", "op": "tmv_bigS", "dtype": "f32", "N": n, "L": n, "S": S, "dist": DN[d],
                  "map": "inter", "impl": "np", "t_median_us": round(med * 1e3, 2), "alg_bytes": nb,
                  "gbs": round(nb / (med * 1e-3) / 1e9, 1)})


def c2():
    n = 16384
    A = gen((n, n), "f32_unit")
    x = gen((n,), "f32_unit", stream_id=2)
    y = torch.empty(n, device="cuda")
    nb = 4 * n * n + 8 * n
    for op, fnp, fv in (("tmv", C.cudanp_tmv, C.cudanp_tmv_variant), ("mv", C.cudanp_mv, C.cudanp_mv_variant)):
        lit = time_ms(lambda: fv(C.S1_LITERAL, A, x, y), reps=3)[0]
        # the no-NP kernel with rows staged through shared memory by TMA (the
        # paper's SMM-style "already optimized" baseline) is part of the
        # tuned S=1 baseline
        t_tiled = time_ms(lambda: fv(C.S1_TILED, A, x, y))[0]
        comps = [("s1_literal", lit), ("s1_tiled", t_tiled)]
        s1_ref = [t_tiled]
        for impl, name in ((C.DP_BLOCK, "dp_block"), (C.DP_THREAD, "dp_thread")):
            comps.append((name, time_ms(lambda: fv(impl, A, x, y), reps=3, warm=1)[0]))
        # vendor-library context (the paper's CUBLAS comparison, Figs 13/14; not
        # part of the product path): torch.mv on the same operands = cuBLAS sgemv
        At = A.t() if op == "tmv" else A
        comps.append(("cublas_sgemv", time_ms(lambda: torch.mv(At, x, out=y))[0]))
        # teams larger than a warp (MV: S/32 warps of a CTA; TMV: 8-master inter-warp CTAs
        # and clusters)
        big = ([(S, C.INTRA_WARP) for S in C.MULTI_WARP_SIZES] if op == "mv" else
               [(S, C.INTER_WARP) for S in (64, 128) + C.TMV_CLUSTER_SIZES])
        sweep_np("C2", op, nb, lambda S, d, m: time_ms(lambda: fnp(A, x, y, S=S, dist=d, map=m)),
                 {"dtype": "f32", "N": n, "L": n}, s1_ref=s1_ref, literal=lit, comps=comps, big=big,
                 call=lambda S, d, m: (lambda: fnp(A, x, y, S=S, dist=d, map=m)),
                 auto=lambda: time_ms(lambda: fnp(A, x, y)))
    tma_sweep("C2", A, x, y, n)
    del A


def tma_sweep(cfg, A, x, y, n):
    """TMA-staged TMV (cudanp_tmv_tma), every S x dist."""
    nb = 4 * n * n + 8 * n
    for S in C.SLAVE_SIZES:
        for d in (C.CYCLIC, C.BLOCK):
            med, mn = time_ms(lambda: C.cudanp_tmv_tma(A, x, y, S=S, dist=d))
            emit({"config": cfg, "op": "tmv_tma", "dtype": "f32", "N": n, "L": n, "S": S, "dist": DN[d],
                  "map": "inter", "impl": "np_tma", "t_median_us": round(med * 1e3, 2),
                  "alg_bytes": nb, "gbs": round(nb / (med * 1e-3) / 1e9, 1)})


def dp_thread_time(full, prefix, N, Np=65536):
    """DP with one child launch per item, timed on a 65,536-item prefix and
    scaled (SURVEY §8(d) DP budget rule).  A full-size attempt (2M-4M device
    launches) did not finish within 20 minutes on B200, so it is not tried."""
    C.cudanp_dp_error_count(reset=True)
    tp = time_ms(prefix, reps=3, warm=1)[0]
    return f"dp_thread_prefix{Np}_scaled", tp * N / Np


def c3(Ls=(32, 64, 128, 256, 80, 150)):
    N = 1 << 22
    for L in Ls:
        for dtype, op, kind, tdt in ((C.F32, C.SUM, "f32_unit", torch.float32),
                                     (C.F32, C.MAX, "f32_signed", torch.float32),
                                     (C.I32, C.SUM, "i32_small", torch.int32),
                                     (C.I32, C.MAX, "i32_full", torch.int32)):
            x = gen((N, L), kind, tdt)
            out = torch.empty(N, dtype=tdt, device="cuda")
            nb = 4 * N * L + 4 * N
            lit = time_ms(lambda: C.cudanp_batched_loop_reduce_variant(C.S1_LITERAL, x, None, out, op=op))[0]
            comps = [("s1_literal", lit),
                     ("dp_block", time_ms(lambda: C.cudanp_batched_loop_reduce_variant(C.DP_BLOCK, x, None, out, op=op), reps=3, warm=1)[0])]
            s1_ref = []
            if L % 4 == 0:  # one thread per item, rows staged by TMA (S1_TILED)
                s1_ref.append(time_ms(lambda: C.cudanp_batched_loop_reduce_variant(C.S1_TILED, x, None, out, op=op))[0])
                comps.append(("s1_tiled", s1_ref[-1]))
            # DP per thread: one device launch per item (full size if the runtime takes it)
            Np = 65536
            xp, op_ = x[:Np], out[:Np]
            comps.append(dp_thread_time(
                lambda: C.cudanp_batched_loop_reduce_variant(C.DP_THREAD, x, None, out, op=op),
                lambda: C.cudanp_batched_loop_reduce_variant(C.DP_THREAD, xp, None, op_, op=op), N, Np))
            sweep_np("C3", "reduce", nb,
                     lambda S, d, m: time_ms(lambda: C.cudanp_batched_loop_reduce(x, None, out, op=op, S=S, dist=d, map=m)),
                     {"dtype": "f32" if dtype == C.F32 else "i32", "opname": "sum" if op == C.SUM else "max",
                      "N": N, "L": L}, literal=lit, comps=comps, s1_ref=s1_ref,
                     call=lambda S, d, m: (lambda: C.cudanp_batched_loop_reduce(x, None, out, op=op, S=S, dist=d, map=m)),
                     auto=lambda: time_ms(lambda: C.cudanp_batched_loop_reduce(x, None, out, op=op)))
            del x, out
            torch.cuda.empty_cache()


def c4(Ls=(64, 128, 256, 512, 1024)):
    N = 1 << 21
    for L in Ls:
        for dtype, kind, tdt in ((C.I32, "i32_small", torch.int32), (C.F32, "f32_unit", torch.float32)):
            x = gen((N, L), kind, tdt, B=1 << 15)
            out = torch.empty_like(x)
            nb = 8 * N * L
            lit = time_ms(lambda: C.cudanp_batched_loop_scan_variant(C.S1_LITERAL, x, None, out), reps=3)[0]
            t_tiled = time_ms(lambda: C.cudanp_batched_loop_scan_variant(C.S1_TILED, x, None, out), reps=3)[0]
            comps = [("s1_literal", lit), ("s1_tiled", t_tiled),
                     ("dp_block", time_ms(lambda: C.cudanp_batched_loop_scan_variant(C.DP_BLOCK, x, None, out), reps=3, warm=1)[0])]
            Np = 65536
            xp, op_ = x[:Np], out[:Np]
            comps.append(dp_thread_time(
                lambda: C.cudanp_batched_loop_scan_variant(C.DP_THREAD, x, None, out),
                lambda: C.cudanp_batched_loop_scan_variant(C.DP_THREAD, xp, None, op_), N, Np))
            sweep_np("C4", "scan", nb,
                     lambda S, d, m: time_ms(lambda: C.cudanp_batched_loop_scan(x, None, out, S=S, dist=d, map=m), reps=3),
                     {"dtype": "f32" if dtype == C.F32 else "i32", "N": N, "L": L}, literal=lit, comps=comps,
                     s1_ref=[t_tiled],
                     call=lambda S, d, m: (lambda: C.cudanp_batched_loop_scan(x, None, out, S=S, dist=d, map=m)),
                     auto=lambda: time_ms(lambda: C.cudanp_batched_loop_scan(x, None, out), reps=3))
            del x, out
            torch.cuda.empty_cache()


def c5():
    n = 65536
    A = gen((n, n), "f32_unit")
    x = gen((n,), "f32_unit", stream_id=2)
    y = torch.empty(n, device="cuda")
    nb = 4 * n * n + 8 * n
    tma_sweep("C5", A, x, y, n)
    for S, d in itertools.product((8, 16, 32), (C.CYCLIC, C.BLOCK)):
        med, mn = time_ms(lambda: C.cudanp_tmv(A, x, y, S=S, dist=d, map=C.INTER_WARP), reps=3)
        emit({"config": "C5", "op": "tmv", "dtype": "f32", "N": n, "L": n, "G": 1, "S": S, "dist": DN[d],
              "map": "inter", "impl": "np", "t_median_us": round(med * 1e3, 1), "alg_bytes": nb,
              "gbs": round(nb / (med * 1e-3) / 1e9, 1)})
    med, _ = time_ms(lambda: C.cudanp_tmv(A, x, y), reps=3)
    emit({"config": "C5", "op": "tmv", "dtype": "f32", "N": n, "L": n, "G": 1, "impl": "auto",
          "choice": C.cudanp_choose_version("tmv", n, n), "t_median_us": round(med * 1e3, 1),
          "alg_bytes": nb, "gbs": round(nb / (med * 1e-3) / 1e9, 1)})
    del A
    torch.cuda.empty_cache()
    N, L = 1 << 26, 64
    xr = gen((N, L), "f32_unit")
    out = torch.empty(N, device="cuda")
    nb = 4 * N * L + 4 * N
    for S, d in itertools.product((4, 8, 16), (C.CYCLIC, C.BLOCK)):
        med, mn = time_ms(lambda: C.cudanp_batched_loop_reduce(xr, None, out, S=S, dist=d, map=C.INTRA_WARP), reps=3)
        emit({"config": "C5", "op": "reduce", "dtype": "f32", "N": N, "L": L, "G": 1, "S": S, "dist": DN[d],
              "map": "intra", "impl": "np", "t_median_us": round(med * 1e3, 1), "alg_bytes": nb,
              "gbs": round(nb / (med * 1e-3) / 1e9, 1)})
    med, _ = time_ms(lambda: C.cudanp_batched_loop_reduce(xr, None, out), reps=3)
    emit({"config": "C5", "op": "reduce", "dtype": "f32", "N": N, "L": L, "G": 1, "impl": "auto",
          "choice": C.cudanp_choose_version("reduce", N, L), "t_median_us": round(med * 1e3, 1),
          "alg_bytes": nb, "gbs": round(nb / (med * 1e-3) / 1e9, 1)})
    del xr, out
    torch.cuda.empty_cache()


def r1(means=(16, 64, 256, 1024)):
    """f1: ragged CSR segments, N = 4M items, uniform and exponential lengths."""
    import synth
    N = 1 << 22
    cases = [(N, m, d) for m in means for d in ("uniform", "exp")] + [(1 << 15, 8192, "exp")]
    for N, mean, dist in cases:
        if True:
            off = torch.from_numpy(synth.offsets_from_lengths(synth.lengths(N, mean, dist))).cuda()
            total = int(off[-1].item())
            x = gen((total,), "f32_unit")
            out = torch.empty(N, device="cuda")
            nb = 4 * total + 8 * (N + 1) + 4 * N
            lit = time_ms(lambda: C.cudanp_ragged_loop_reduce_literal(x, off, None, out))[0]
            if N < (1 << 20):  # few, long segments: multi-warp teams too
                for S in (64, 128, 256, 512, 1024):
                    for d in (C.CYCLIC, C.BLOCK):
                        med, _ = time_ms(lambda: C.cudanp_ragged_loop_reduce(x, off, None, out, S=S, dist=d))
                        emit({"config": "R1", "op": "ragged_reduce_bigS", "dtype": "f32", "N": N,
                              "L": f"{dist}{mean}", "S": S, "dist": DN[d], "map": "intra", "impl": "np",
                              "t_median_us": round(med * 1e3, 2), "alg_bytes": nb,
                              "gbs": round(nb / (med * 1e-3) / 1e9, 1)})
            comps = [("s1_literal", lit)]
            for th in (64, 128, 256, 512):  # adaptive team size per segment
                comps.append((f"adaptive_t{th}", time_ms(
                    lambda: C.cudanp_ragged_loop_reduce_adaptive(x, off, None, out, threshold=th))[0]))
            sweep_np("R1", "ragged_reduce", nb,
                     lambda S, d, m: time_ms(lambda: C.cudanp_ragged_loop_reduce(x, off, None, out, S=S, dist=d, map=m)),
                     {"dtype": "f32", "N": N, "L": f"{dist}{mean}"}, literal=lit, comps=comps,
                     call=lambda S, d, m: (lambda: C.cudanp_ragged_loop_reduce(x, off, None, out, S=S, dist=d, map=m)))
            del x, out, off
            torch.cuda.empty_cache()


def f2(L=150):
    """f2: LE multi-section items (Figs 5-6), N = 2M items x 150 points, both
    layouts, every map x dist x S including the non-power-of-two inter-warp S
    of Fig 12 (3, 5, 10, 15)."""
    N = 1 << 21
    for layout in (0, 1):
        x = gen((N, L) if layout == 0 else (L, N), "f32_unit")
        g = torch.empty(N, device="cuda")
        st = [torch.empty(N, device="cuda") for _ in range(3)]
        nb = 4 * N * L + 4 * N * 4
        def run(S, d, m):
            return time_ms(lambda: C.load().cudanp_le_gicov(x.data_ptr(), g.data_ptr(), *(t.data_ptr() for t in st),
                                                           N, L, 0.02, layout, S, d, m, None))
        lit = time_ms(lambda: C.load().cudanp_le_gicov_literal(x.data_ptr(), g.data_ptr(), *(t.data_ptr() for t in st),
                                                               N, L, 0.02, layout, None))[0]
        res = {}
        for S in (1, 2, 3, 4, 5, 8, 10, 15, 16, 32):
            for d in (C.CYCLIC, C.BLOCK):
                for m in (C.INTRA_WARP, C.INTER_WARP):
                    if m == C.INTRA_WARP and S & (S - 1):
                        continue
                    res[(S, d, m)] = run(S, d, m)
        s1 = min([v[0] for k, v in res.items() if k[0] == 1] + [lit])  # best no-NP kernel
        for (S, d, m), (med, mn) in res.items():
            emit({"config": "F2", "op": "le_gicov", "dtype": "f32", "N": N, "L": L,
                  "layout": "point-major" if layout else "item-major", "S": S, "dist": DN[d], "map": MN[m],
                  "impl": "np", "t_median_us": round(med * 1e3, 2), "alg_bytes": nb,
                  "gbs": round(nb / (med * 1e-3) / 1e9, 1), "speedup_vs_s1_tuned": round(s1 / med, 3),
                  "speedup_vs_s1_literal": round(lit / med, 3)})
        best = min(res, key=lambda k: res[k][0])
        emit({"config": "F2", "op": "le_gicov", "dtype": "f32", "N": N, "L": L,
              "layout": "point-major" if layout else "item-major", "impl": "s1_literal", "t_median_us": round(lit * 1e3, 2), "alg_bytes": nb,
              "gbs": round(nb / (lit * 1e-3) / 1e9, 1)})
        emit({"config": "F2", "op": "le_gicov", "dtype": "f32", "N": N, "L": L,
              "layout": "point-major" if layout else "item-major", "impl": "best_np", "S": best[0], "dist": DN[best[1]], "map": MN[best[2]],
              "t_median_us": round(res[best][0] * 1e3, 2), "alg_bytes": nb,
              "gbs": round(nb / (res[best][0] * 1e-3) / 1e9, 1),
              "speedup_vs_s1_tuned": round(s1 / res[best][0], 3),
              "speedup_vs_s1_literal": round(lit / res[best][0], 3)})
        # Fig 15 analog: the home of Grad (6c registers = above, 6b shared memory
        # staged by TMA, 6a global = loop 3 re-reads the input), intra-warp teams
        for pl, name in ((C.GRAD_SHARED, "grad_shared"), (C.GRAD_GLOBAL, "grad_global")):
            # item-major: intra-warp teams; point-major: the shared placement is
            # built for inter-warp teams (S <= 16, any of the Fig 12 sizes)
            pm_shared = pl == C.GRAD_SHARED and layout == 1
            mp = C.INTER_WARP if pm_shared else C.INTRA_WARP
            for S in ((1, 2, 3, 4, 5, 8, 10, 15, 16) if pm_shared else C.SLAVE_SIZES):
                for d in (C.CYCLIC, C.BLOCK):
                    med, _ = time_ms(lambda: C.load().cudanp_le_gicov_placement(
                        x.data_ptr(), g.data_ptr(), *(t.data_ptr() for t in st), N, L, 0.02, layout, S,
                        d, mp, pl, None))
                    emit({"config": "F2", "op": "le_gicov", "dtype": "f32", "N": N, "L": L,
                          "layout": "point-major" if layout else "item-major", "placement": name,
                          "S": S, "dist": DN[d], "map": MN[mp], "impl": "np_" + name,
                          "t_median_us": round(med * 1e3, 2), "alg_bytes": nb,
                          "gbs": round(nb / (med * 1e-3) / 1e9, 1),
                          "speedup_vs_s1_literal": round(lit / med, 3)})
        del x, g, st
        torch.cuda.empty_cache()


def f3(total=1 << 26):
    """f3: Fig 1 on B200 -- copy 64M floats; plain kernel without and
    with -rdc, and DP with m parent threads x n = total/m child threads."""
    x = gen((total,), "f32_unit")
    out = torch.empty_like(x)
    nb = 8 * total
    for variant, name in ((0, "plain"), (1, "plain_rdc")):
        med, mn = time_ms(lambda: C.cudanp_dp_memcopy(x, out, variant=variant))
        emit({"config": "F3", "op": "memcopy", "impl": name, "m": 1, "n": total,
              "t_median_us": round(med * 1e3, 2), "alg_bytes": nb, "gbs": round(nb / (med * 1e-3) / 1e9, 1)})
    for m in (1, 4, 16, 64, 256, 1024, 4096, 16384, 65536):
        med, mn = time_ms(lambda: C.cudanp_dp_memcopy(x, out, m=m, variant=2), reps=3, warm=1)
        emit({"config": "F3", "op": "memcopy", "impl": "dp", "m": m, "n": total // m,
              "t_median_us": round(med * 1e3, 2), "alg_bytes": nb, "gbs": round(nb / (med * 1e-3) / 1e9, 1)})
    del x, out
    torch.cuda.empty_cache()


def e9(Ls=(32, 64, 128)):
    """Fig 16 analog: team reduction by shfl vs shared memory vs
    redux.sync under intra-warp NP (cyclic), C3 shapes."""
    N = 1 << 22
    for L in Ls:
        for dtype, op, kind, tdt in ((C.I32, C.SUM, "i32_small", torch.int32),
                                     (C.F32, C.MAX, "f32_signed", torch.float32)):
            x = gen((N, L), kind, tdt)
            out = torch.empty(N, dtype=tdt, device="cuda")
            nb = 4 * N * L + 4 * N
            for S in C.SLAVE_SIZES:
                for be, name in ((C.SHFL, "shfl"), (C.SMEM, "smem"), (C.REDUX, "redux")):
                    med, mn = time_ms(lambda: C.cudanp_batched_loop_reduce_backend(x, None, out, op=op, S=S, backend=be))
                    emit({"config": "E9", "op": "reduce", "dtype": "f32" if dtype == C.F32 else "i32",
                          "opname": "sum" if op == C.SUM else "max", "N": N, "L": L, "S": S,
                          "backend": name, "impl": "np", "t_median_us": round(med * 1e3, 2),
                          "alg_bytes": nb, "gbs": round(nb / (med * 1e-3) / 1e9, 1)})
            del x, out
            torch.cuda.empty_cache()


def big():
    """Teams larger than a warp (S = 64..1024) and than a CTA (S = 2048..8192,
    cluster teams) on the shapes that need them: MV with few long
    rows (the Fig 14 axis: fixed width, growing height) and a batched reduce
    over few long items.  L2 is flushed before every timed launch (several of
    these working sets fit the 126 MB L2)."""
    cases = [("mv", h, 65536) for h in (16, 64, 256, 1024, 4096)] + \
            [("reduce", N, L) for N, L in ((16, 1 << 22), (64, 1 << 20), (256, 262144), (2048, 16384), (16384, 4096))] + \
            [("scan", N, L) for N, L in ((16, 1 << 22), (256, 262144))] + \
            [("tmv", w, h) for w, h in ((256, 262144), (1024, 65536), (4096, 16384))]
    only = os.environ.get("CUDANP_BIG_OPS")  # e.g. "scan": restrict an A/B run to one op
    if only:
        cases = [c for c in cases if c[0] in only.split(",")]
    for op, N, L in cases:
        if op == "tmv":  # N = columns (masters), L = rows (the loop)
            A = gen((L, N), "f32_unit")
            x = gen((L,), "f32_unit", stream_id=2)
            y = torch.empty(N, device="cuda")
            nb = 4 * N * L + 4 * N + 4 * L
            fn = lambda S, d: C.cudanp_tmv(A, x, y, S=S, dist=d, map=C.INTER_WARP if S > 32 else C.AUTO)  # noqa: E731
        elif op == "mv":
            A = gen((N, L), "f32_unit")
            x = gen((L,), "f32_unit", stream_id=2)
            y = torch.empty(N, device="cuda")
            nb = 4 * N * L + 4 * N + 4 * L
            fn = lambda S, d: C.cudanp_mv(A, x, y, S=S, dist=d, map=C.INTRA_WARP)  # noqa: E731
        elif op == "reduce":
            A = gen((N, L), "f32_unit")
            y = torch.empty(N, device="cuda")
            nb = 4 * N * L + 4 * N
            fn = lambda S, d: C.cudanp_batched_loop_reduce(A, None, y, S=S, dist=d, map=C.INTRA_WARP)  # noqa: E731
        else:
            A = gen((N, L), "i32_small", torch.int32, B=1 << 15)
            y = torch.empty_like(A)
            nb = 8 * N * L
            fn = lambda S, d: C.cudanp_batched_loop_scan(A, None, y, S=S, dist=d, map=C.INTRA_WARP)  # noqa: E731
        sizes = (C.SLAVE_SIZES + (64, 128, 256, 1024)) if op == "tmv" else \
            (C.SLAVE_SIZES + (64, 128, 256, 512, 1024, 2048, 4096, 8192))
        for S in sizes:
            for d in (C.CYCLIC, C.BLOCK):
                try:
                    med, mn = time_ms(lambda: fn(S, d), flush=True)
                except C.CudanpError:
                    continue  # e.g. the cluster-team scan is block-only
                emit({"config": "BIG", "op": op, "dtype": "f32" if op != "scan" else "i32", "N": N, "L": L, "S": S, "dist": DN[d],
                      "map": "intra", "impl": "np", "t_median_us": round(med * 1e3, 2), "alg_bytes": nb,
                      "gbs": round(nb / (med * 1e-3) / 1e9, 1)})
        del A, y
        torch.cuda.empty_cache()


def main():
    global OUT
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C1,C2,C3,C4,C5,R1,F2,F3,E9,BIG")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "sweep.jsonl"))
    ap.add_argument("--lib", default=None, help="alternative libcudanp.so (build experiments)")
    a = ap.parse_args()
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    OUT = open(a.out, "w")
    C.load(a.lib) if a.lib else C.load()
    C.cudanp_dp_set_pending_launch_limit(1 << 17)
    t0 = time.time()
    for c in a.configs.split(","):
        {"C1": c1, "C2": c2, "C3": c3, "C4": c4, "C5": c5, "R1": r1, "F2": f2, "F3": f3, "E9": e9, "BIG": big}[c.strip()]()
        print(f"# {c} done at {time.time() - t0:.0f}s", file=sys.stderr, flush=True)
    print(f"# dp launch errors: {C.cudanp_dp_error_count(reset=True)}", file=sys.stderr)


if __name__ == "__main__":
    main()
