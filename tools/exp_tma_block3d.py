#!/usr/bin/env python
"""TMA TMV, block distribution: S boxes per stage (2-D map) vs one 3-D box
(A viewed as [S][h/S][w]) when S divides h.  C2 shape, 20 launches back to
back per event pair; h = 16383 forces the 2-D path for comparison."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_ppopp_yangz14_b200 import cudanp as C  # noqa: E402


def t_ms(fn, reps=20):
    for _ in range(3):
        fn()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    b.synchronize()
    return a.elapsed_time(b) / reps


C.load()
n = 16384
A = torch.empty(n, n, device="cuda")
C.cudanp_generate(A, "f32_unit")
x = torch.empty(n, device="cuda")
C.cudanp_generate(x, "f32_unit", stream_id=2)
y = torch.empty(n, device="cuda")
for h in (n, n - 1):  # S | h: 3-D box; h = 16383: S boxes
    for S in (2, 4, 8, 16, 32):
        for d in (C.BLOCK, C.CYCLIC):
            ms = t_ms(lambda: C.cudanp_tmv(A[:h], x[:h], y, S=S, dist=d, map=C.INTER_WARP_TMA))
            print(json.dumps({"h": h, "w": n, "S": S, "dist": "block" if d == C.BLOCK else "cyclic",
                              "box3d": d == C.BLOCK and h % S == 0,
                              "gbs": round((4 * h * n + 4 * h + 4 * n) / ms / 1e6, 1)}), flush=True)
