#!/usr/bin/env python
"""Launch-shape exploration for the TMA-staged TMV (cudanp_tmv_tma_ex):
every S x dist x strip width x rows-per-slave x ring depth on a resident
h x w fp32 matrix, GB/s of algorithmic bytes (4hw + 4h + 4w), CUDA events.
Each shape is first checked bit-exact against cudanp_tmv on exact data.

    python tools/tma_explore.py [--n 16384] [--w 16384] [--out gpurun_out/tma_explore.jsonl]
"""
from __future__ import annotations

import argparse
import itertools
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_ppopp_yangz14_b200 import cudanp as C  # noqa: E402


def time_ms(fn, reps=7, warm=2):
    st = torch.cuda.current_stream()
    for _ in range(warm):
        fn()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(st)
        fn()
        b.record(st)
        b.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=16384)
    ap.add_argument("--w", type=int, default=16384)
    ap.add_argument("--out", default=None)
    ap.add_argument("--S", default="1,2,4,8,16,32")
    ap.add_argument("--full", action="store_true", help="also every pinned shape")
    a = ap.parse_args()
    C.load()
    h, w = a.n, a.w
    out = open(a.out, "a") if a.out else None
    A = torch.empty(h, w, dtype=torch.float32, device="cuda")
    x = torch.empty(h, dtype=torch.float32, device="cuda")
    y = torch.empty(w, dtype=torch.float32, device="cuda")
    ref = torch.empty(w, dtype=torch.float32, device="cuda")
    nb = 4 * h * w + 4 * h + 4 * w
    Ss = [int(s) for s in a.S.split(",")]

    def emit(rec):
        line = json.dumps(rec)
        print(line, flush=True)
        if out:
            out.write(line + "\n")
            out.flush()

    # parity pass on exact data (f32_int4: every order gives the same sum)
    C.cudanp_generate(A, "f32_int4", stream_id=1)
    C.cudanp_generate(x, "f32_int4", stream_id=2)
    C.cudanp_tmv(A, x, ref, S=8, map=C.INTER_WARP)
    shapes = [(0, -1, 0)]
    if a.full:
        shapes += list(itertools.product((32, 64, 128), (0, 1, 2), (0, 2, 3, 4, 6)))
    ok = {}
    for S, d, (cols, rs, st) in itertools.product(Ss, (C.CYCLIC, C.BLOCK), shapes):
        try:
            C.cudanp_tmv_tma(A, x, y, S=S, dist=d, cols=cols, rows_sel=rs, stages=st)
            torch.cuda.synchronize()
            ok[(S, d, cols, rs, st)] = bool(torch.equal(y, ref))
        except C.CudanpError as e:
            ok[(S, d, cols, rs, st)] = None
    bad = [k for k, v in ok.items() if v is False]
    print("parity failures:", bad, flush=True)
    C.cudanp_generate(A, "f32_unit", stream_id=1)
    C.cudanp_generate(x, "f32_unit", stream_id=2)
    t = time_ms(lambda: C.cudanp_tmv(A, x, y, S=32, dist=C.BLOCK, map=C.INTER_WARP))
    emit({"h": h, "w": w, "impl": "ldg", "S": 32, "dist": "block", "gbs": round(nb / t / 1e6, 1)})
    for (S, d, cols, rs, st), good in ok.items():
        if good is None:
            continue
        t = time_ms(lambda: C.cudanp_tmv_tma(A, x, y, S=S, dist=d, cols=cols, rows_sel=rs, stages=st))
        info = C.cudanp_launch_info("tmv_tma", w, h, S=S, dist=d) if cols == 0 else {}
        emit({"h": h, "w": w, "impl": "tma", "S": S, "dist": "cyclic" if d == 0 else "block",
              "cols": cols, "rows_sel": rs, "stages": st, "parity": good,
              "gbs": round(nb / t / 1e6, 1), "ms": round(t, 4), "auto_info": info})


if __name__ == "__main__":
    main()
