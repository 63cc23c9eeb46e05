#!/usr/bin/env python
"""Small launches of every kernel family for compute-sanitizer
(memcheck / racecheck / synccheck):

    compute-sanitizer --tool racecheck python tools/sanitize_cases.py

Shapes are tiny but ragged (several teams, partial warps/CTAs, tails), and
cover both maps, both distributions, every S, the smem broadcast / reduce /
scan barriers of the inter-warp teams and every masked shuffle.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ppopp_yangz14_b200 import cudanp as C  # noqa: E402


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def main():
    C.load()
    quick = "--quick" in sys.argv
    no_dp = "--no-dp" in sys.argv  # racecheck/synccheck do not support dynamic parallelism
    Ss = (1, 8, 32) if quick else C.SLAVE_SIZES
    A = dev(synth.matrix(37, 70, "f32_unit"))
    A4 = dev(synth.matrix(37, 68, "f32_unit"))
    xt, xm, xm4 = dev(synth.vector(37)), dev(synth.vector(70)), dev(synth.vector(68))
    Xf = dev(synth.items(70, 36, "f32_unit"))
    Xi = dev(synth.items(70, 37, "i32_small"))
    Xi4 = dev(synth.items(70, 36, "i32_small"))
    inif, inii = dev(synth.init(70, "f32_unit")), dev(synth.init(70, "i32_small"))
    lens = synth.lengths(50, 9)
    off = dev(synth.offsets_from_lengths(lens))
    xr = dev(synth.gen(1, "f32_unit", 0, int(lens.sum()) + 3))
    le = dev(synth.items(40, 30, "f32_unit"))
    for S in Ss:
        for d in (C.CYCLIC, C.BLOCK):
            for m in (C.INTRA_WARP, C.INTER_WARP):
                C.cudanp_tmv(A, xt, S=S, dist=d, map=m, n_outer=70)
                C.cudanp_tmv(A4, xt, S=S, dist=d, map=m)
                C.cudanp_mv(A, xm, S=S, dist=d, map=m)
                C.cudanp_mv(A4, xm4, S=S, dist=d, map=m)
                for X, ini in ((Xf, inif), (Xi, inii)):
                    C.cudanp_batched_loop_reduce(X, ini, op=C.SUM, S=S, dist=d, map=m)
                    C.cudanp_batched_loop_reduce(X, None, op=C.MAX, S=S, dist=d, map=m)
                    C.cudanp_batched_loop_scan(X, ini, S=S, dist=d, map=m)
                C.cudanp_ragged_loop_reduce(xr, off, S=S, dist=d, map=m)
                C.cudanp_le_gicov(le, 0.01, S=S, dist=d, map=m)
        for be in (C.SHFL, C.SMEM, C.REDUX):
            C.cudanp_batched_loop_reduce_backend(Xi4, inii, S=S, backend=be)
    for th in (1, 4, 16):  # ragged reduce with the team size chosen per segment
        C.cudanp_ragged_loop_reduce_adaptive(xr, off, threshold=th)
    for S in (64, 256, 1024):  # multi-warp teams
        for d in (C.CYCLIC, C.BLOCK):
            for X, ini in ((Xf, inif), (Xi, inii)):
                C.cudanp_batched_loop_reduce(X, ini, S=S, dist=d)
                C.cudanp_batched_loop_scan(X, ini, S=S, dist=d)
            C.cudanp_mv(A, xm, S=S, dist=d)
            C.cudanp_ragged_loop_reduce(xr, off, S=S, dist=d)
            if S == 64:
                C.cudanp_tmv(A, xt, S=S, dist=d, map=C.INTER_WARP, n_outer=70)
    Xc = dev(synth.items(300, 97, "i32_small"))      # cluster teams: more items than clusters
    Xcf = dev(synth.items(7, 5003, "f32_unit"))       # (grid stride, both slot buffers), L % 4 != 0
    for S in (2048, 4096, 8192):
        for d in (C.CYCLIC, C.BLOCK):
            C.cudanp_batched_loop_reduce(Xc, None, S=S, dist=d)
            C.cudanp_batched_loop_reduce(Xcf, None, op=C.MAX, S=S, dist=d)
        for d in (C.CYCLIC, C.BLOCK):
            C.cudanp_batched_loop_scan(Xc, None, S=S, dist=d)
            C.cudanp_batched_loop_scan(Xcf, None, S=S, dist=d)
        C.cudanp_mv(A, xm, S=S, dist=C.CYCLIC)
    # narrow TMV S = 64 / 128 in each CTA layout (V = 4 with 4 / 8 masters, V = 1), ragged
    # last CTA, with the L2 bulk prefetch before the dependency wait
    for h, w in ((1024, 1028), (300, 4800), (3000, 1024), (64, 1022)):
        An, xn = dev(synth.matrix(h, w, "f32_unit")), dev(synth.vector(h))
        for S in (64, 128):
            for d in (C.CYCLIC, C.BLOCK):
                C.cudanp_tmv(An, xn, S=S, dist=d, map=C.INTER_WARP)
    for S in (256, 1024):  # TMV cluster teams
        for d in (C.CYCLIC, C.BLOCK):
            C.cudanp_tmv(A, xt, S=S, dist=d, map=C.INTER_WARP, n_outer=70)
            C.cudanp_tmv(A4, xt, S=S, dist=d, map=C.INTER_WARP)
    Xp = dev(synth.items(70, 37, "i32_small").reshape(-1))  # peeled rows, every misalignment
    for sh in range(4):
        v = Xp[sh:sh + 69 * 37].view(69, 37)
        for S in Ss:
            C.cudanp_batched_loop_reduce(v, None, S=S, map=C.INTRA_WARP)
    At = dev(synth.matrix(600, 132, "f32_unit"))   # tall: the rings wrap several times
    xtt = dev(synth.vector(600))
    for S in (1, 2, 4, 8, 16, 32):  # TMA-staged TMV, auto and pinned shapes
        for d in (C.CYCLIC, C.BLOCK):
            C.cudanp_tmv_tma(A4, xt, S=S, dist=d)
            C.cudanp_tmv(At, xtt, S=S, dist=d, map=C.INTER_WARP_TMA)
            for cols, rs in ((32, 0), (64, 1), (128, 2)):
                try:
                    C.cudanp_tmv_tma(At, xtt, S=S, dist=d, cols=cols, rows_sel=rs, stages=2)
                except C.CudanpError:
                    pass  # ring larger than shared memory for this S
    Xt4 = dev(synth.items(300, 36, "i32_small"))   # TMA-staged reduce: rings that wrap
    for S in (1, 4, 8, 32):
        for d in (C.CYCLIC, C.BLOCK):
            C.cudanp_batched_loop_reduce(Xi4, inii, S=S, dist=d, map=C.INTRA_WARP_TMA)
            C.cudanp_batched_loop_reduce_tma(Xt4, None, op=C.MAX, S=S, dist=d, stage_bytes=1024, stages=2)
    if not quick:  # native group, world 1
        g = C.cudanp_group_create(C.cudanp_group_unique_id(), 1, 0)
        yr = torch.empty(68, device="cuda")
        C.cudanp_sharded_tmv(g, A4, xt, torch.empty(68, device="cuda"), yr, 68, S=8)
        torch.cuda.synchronize()
        C.cudanp_group_destroy(g)
    for S in (3, 5, 10, 15):
        C.cudanp_le_gicov(le, 0.01, S=S, map=C.INTER_WARP, layout=0)
        for d in (C.CYCLIC, C.BLOCK):  # non-power-of-two inter-warp teams
            C.cudanp_tmv(A, xt, S=S, dist=d, map=C.INTER_WARP, n_outer=70)
            C.cudanp_mv(A4, xm4, S=S, dist=d, map=C.INTER_WARP)
            for X, ini in ((Xf, inif), (Xi, inii)):
                C.cudanp_batched_loop_reduce(X, ini, S=S, dist=d, map=C.INTER_WARP)
                C.cudanp_batched_loop_scan(X, ini, S=S, dist=d, map=C.INTER_WARP)
    # more items than one persistent wave of the multi-warp kernels (their
    # grid-stride loops), S = 64 reduce/scan and S = 256 MV
    Xw = dev(synth.items(5003, 16, "i32_small"))
    Xwf = dev(synth.items(5003, 16, "f32_unit"))
    Aw = dev(synth.matrix(2500, 64, "f32_unit"))
    xw = dev(synth.vector(64))
    for d in (C.CYCLIC, C.BLOCK):
        C.cudanp_batched_loop_reduce(Xw, None, S=64, dist=d)
        C.cudanp_batched_loop_scan(Xwf, None, S=64, dist=d)
        C.cudanp_mv(Aw, xw, S=256, dist=d)
    # point-major LE, inter-warp: several groups per CTA through the
    # double-buffered loop 1 (np_le.cu DB), and the S = 32 single-buffer path
    lpm = dev(synth.items(30, 40003, "f32_unit"))  # (L, N) point-major
    for S in (5, 8, 16, 32):
        for d in (C.CYCLIC, C.BLOCK):
            C.cudanp_le_gicov(lpm, 0.01, S=S, dist=d, map=C.INTER_WARP, layout=1)
    # the library's own version choice (S = S_AUTO) and the TMA fallbacks
    C.cudanp_tmv(A4, xt)
    C.cudanp_mv(A4, xm4)
    C.cudanp_batched_loop_reduce(Xi4)
    C.cudanp_batched_loop_scan(Xf)
    yb = torch.empty(69, device="cuda")
    C.cudanp_tmv(A4, xt, yb[1:], S=8, map=C.INTER_WARP_TMA)  # y off 16-byte alignment
    # tiled S = 1 baselines (TMA rings that wrap; TMA stores for the scan)
    Am = dev(synth.matrix(300, 1000, "f32_unit"))
    xmm = dev(synth.vector(1000))
    C.cudanp_mv_variant(C.S1_TILED, Am, xmm)
    C.cudanp_mv_variant(C.S1_TILED, A4, xm4)
    Xs = dev(synth.items(300, 1000, "i32_small"))
    C.cudanp_batched_loop_scan_variant(C.S1_TILED, Xs, dev(synth.init(300, "i32_small")))
    C.cudanp_batched_loop_scan_variant(C.S1_TILED, Xf)
    if not quick:
        C.cudanp_dp_set_pending_launch_limit(1 << 12)
        for impl in (C.S1_LITERAL,) if no_dp else (C.S1_LITERAL, C.DP_THREAD, C.DP_BLOCK):
            C.cudanp_tmv_variant(impl, A, xt, n_outer=70)
            C.cudanp_mv_variant(impl, A, xm)
            C.cudanp_batched_loop_reduce_variant(impl, Xi, inii)
            C.cudanp_batched_loop_scan_variant(impl, Xf, inif)
    torch.cuda.synchronize()
    print("sanitize cases done")


if __name__ == "__main__":
    main()
