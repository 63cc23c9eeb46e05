#!/usr/bin/env python
"""Launch one hot-path kernel a few times for ncu (`-k regex:... -s 1 -c 1`).

    python tools/ncu_target.py --op tmv --S 32 --dist block --map inter [--n 16384]
    python tools/ncu_target.py --op reduce --S 8 --L 64 --N 4194304
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_ppopp_yangz14_b200 import cudanp as C  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--op", required=True, choices=["tmv", "mv", "reduce", "scan", "tmv_literal",
                                                    "mv_literal", "reduce_literal", "scan_literal",
                                                    "ragged", "le", "le_literal", "tmv_tma",
                                                    "mv_tiled", "tmv_tiled", "scan_tiled", "reduce_tiled"])
    ap.add_argument("--lens", default="uniform", help="ragged: length distribution")
    ap.add_argument("--layout", type=int, default=0, help="le: 0 item-major, 1 point-major")
    ap.add_argument("--S", type=int, default=8)
    ap.add_argument("--dist", default="cyclic")
    ap.add_argument("--map", default="auto")
    ap.add_argument("--n", type=int, default=16384)
    ap.add_argument("--N", type=int, default=1 << 22)
    ap.add_argument("--L", type=int, default=64)
    ap.add_argument("--dtype", default="f32")
    ap.add_argument("--reps", type=int, default=3)
    a = ap.parse_args()
    d = {"cyclic": C.CYCLIC, "block": C.BLOCK}[a.dist]
    m = {"auto": C.AUTO, "intra": C.INTRA_WARP, "inter": C.INTER_WARP, "inter_tma": C.INTER_WARP_TMA,
         "intra_tma": C.INTRA_WARP_TMA}[a.map]
    C.load()
    if a.op == "ragged":
        import synth
        off = torch.from_numpy(synth.offsets_from_lengths(synth.lengths(a.N, a.L, a.lens))).cuda()
        X = torch.empty(int(off[-1].item()), device="cuda")
        C.cudanp_generate(X, "f32_unit")
        o1 = torch.empty(a.N, device="cuda")
        fns = {"ragged": lambda: C.cudanp_ragged_loop_reduce(X, off, None, o1, S=a.S, dist=d, map=m)}
    elif a.op in ("le", "le_literal"):
        X = torch.empty(*((a.N, a.L) if a.layout == 0 else (a.L, a.N)), device="cuda")
        C.cudanp_generate(X, "f32_unit")
        fns = {"le": lambda: C.cudanp_le_gicov(X, 0.02, layout=a.layout, S=a.S, dist=d, map=m),
               "le_literal": lambda: C.cudanp_le_gicov(X, 0.02, layout=a.layout, literal=True)}
    elif a.op.startswith(("tmv", "mv")):
        A = torch.empty(a.n, a.n, device="cuda")
        C.cudanp_generate(A, "f32_unit")
        x = torch.empty(a.n, device="cuda")
        C.cudanp_generate(x, "f32_unit", stream_id=2)
        y = torch.empty(a.n, device="cuda")
        fns = {"tmv": lambda: C.cudanp_tmv(A, x, y, S=a.S, dist=d, map=m),
               "tmv_tma": lambda: C.cudanp_tmv_tma(A, x, y, S=a.S, dist=d),
               "mv": lambda: C.cudanp_mv(A, x, y, S=a.S, dist=d, map=m),
               "tmv_literal": lambda: C.cudanp_tmv_variant(C.S1_LITERAL, A, x, y),
               "mv_literal": lambda: C.cudanp_mv_variant(C.S1_LITERAL, A, x, y),
               "mv_tiled": lambda: C.cudanp_mv_variant(C.S1_TILED, A, x, y),
               "tmv_tiled": lambda: C.cudanp_tmv_variant(C.S1_TILED, A, x, y)}
    else:
        dt = torch.float32 if a.dtype == "f32" else torch.int32
        X = torch.empty(a.N, a.L, dtype=dt, device="cuda")
        C.cudanp_generate(X, "f32_unit" if a.dtype == "f32" else "i32_small", B=1 << 15)
        o1 = torch.empty(a.N, dtype=dt, device="cuda")
        o2 = torch.empty_like(X) if "scan" in a.op else None
        fns = {"reduce": lambda: C.cudanp_batched_loop_reduce(X, None, o1, S=a.S, dist=d, map=m),
               "scan": lambda: C.cudanp_batched_loop_scan(X, None, o2, S=a.S, dist=d, map=m),
               "reduce_literal": lambda: C.cudanp_batched_loop_reduce_variant(C.S1_LITERAL, X, None, o1),
               "scan_literal": lambda: C.cudanp_batched_loop_scan_variant(C.S1_LITERAL, X, None, o2),
               "reduce_tiled": lambda: C.cudanp_batched_loop_reduce_variant(C.S1_TILED, X, None, o1),
               "scan_tiled": lambda: C.cudanp_batched_loop_scan_variant(C.S1_TILED, X, None, o2)}
    for _ in range(a.reps):
        fns[a.op]()
    torch.cuda.synchronize()


if __name__ == "__main__":
    main()
