#!/usr/bin/env python
"""A/B for the inter-warp LE kernel's double-buffered loop 1 (np_le.cu, DB):
F2 shapes (2M items x 150 points), every inter-warp S x dist, both layouts.
Run twice: CUDANP_LE_DB=0 and CUDANP_LE_DB=1 (the switch is read once per process).

    CUDANP_LE_DB=1 python tools/exp_le_db.py --out gpurun_out/exp_le_db1_<tag>.jsonl
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import torch  # noqa: E402

from paper_conf_ppopp_yangz14_b200 import cudanp as C  # noqa: E402
from sweep import time_ms  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", required=True)
    ap.add_argument("--L", type=int, default=150)
    a = ap.parse_args()
    C.load()
    N, L = 1 << 21, a.L
    db = os.environ.get("CUDANP_LE_DB", "1")
    with open(a.out, "w") as f:
        for layout in (1, 0):
            x = torch.empty((L, N) if layout else (N, L), device="cuda")
            C.cudanp_generate(x, "f32_unit")
            nb = 4 * N * L + 4 * N * 4
            g = torch.empty(N, device="cuda")
            st = [torch.empty(N, device="cuda") for _ in range(3)]
            lib = C.load()
            for S in (2, 3, 4, 5, 8, 10, 15, 16, 32):
                for d in (C.CYCLIC, C.BLOCK):
                    med, mn = time_ms(lambda: lib.cudanp_le_gicov(
                        x.data_ptr(), g.data_ptr(), *(t.data_ptr() for t in st), N, L, 0.02, layout, S, d,
                        C.INTER_WARP, None), reps=7)
                    rec = {"db": db, "layout": "pm" if layout else "im", "L": L, "S": S,
                           "dist": "cyc" if d == C.CYCLIC else "blk", "us": round(med * 1e3, 1),
                           "gbs": round(nb / (med * 1e-3) / 1e9, 1)}
                    f.write(json.dumps(rec) + "\n")
                    print(json.dumps(rec), flush=True)
            del x
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
