#!/usr/bin/env python
"""TMV width sweep: where does the TMA-staged inter-warp kernel beat the LDG
inter-warp kernel?  (The rule behind MAP_AUTO / S_AUTO for TMV, abi.cu
tmv_wide.)  For each (h, w): the best TMA version (S x dist) and the best LDG
inter-warp version (S x dist), 20 launches back to back per event pair.

    python tools/tmv_width_sweep.py --out gpurun_out/tmv_width_<tag>.jsonl

--narrow: narrow matrices (w <= 8192, the latency-bound band around C1) --
every LDG inter-warp (S, dist) incl. S = 64 / 128 and the library's S_AUTO
choice, each timed as a CUDA graph over enough distinct copies of A that
every launch reads cold HBM (tools/c1_latency.py's method).
"""
from __future__ import annotations

import argparse
import itertools
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_ppopp_yangz14_b200 import cudanp as C  # noqa: E402


def t_ms(fn, reps=20, warm=3):
    for _ in range(warm):
        fn()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(reps):
        fn()
    e1.record()
    e1.synchronize()
    return e0.elapsed_time(e1) / reps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default="gpurun_out/tmv_width.jsonl")
    ap.add_argument("--narrow", action="store_true")
    a = ap.parse_args()
    C.load()
    if a.narrow:
        return narrow(a.out)
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    shapes = [(16384, w) for w in (4096, 8192, 12288, 16384, 18944, 20480, 24576, 32768, 49152, 65536)]
    shapes += [(65536, w) for w in (8192, 16384, 32768, 65536)]
    with open(a.out, "w") as f:
        for h, w in shapes:
            A = torch.empty(h, w, device="cuda")
            C.cudanp_generate(A, "f32_unit", stream_id=1)
            x = torch.empty(h, device="cuda")
            C.cudanp_generate(x, "f32_unit", stream_id=2)
            y = torch.empty(w, device="cuda")
            nb = 4 * h * w + 4 * h + 4 * w
            res = {}
            for S, d in itertools.product((4, 8, 16, 32), (C.CYCLIC, C.BLOCK)):
                res[("tma", S, d)] = t_ms(lambda: C.cudanp_tmv(A, x, y, S=S, dist=d, map=C.INTER_WARP_TMA))
            for S, d in itertools.product((8, 16, 32, 64, 128), (C.CYCLIC, C.BLOCK)):
                res[("ldg", S, d)] = t_ms(lambda: C.cudanp_tmv(A, x, y, S=S, dist=d, map=C.INTER_WARP))
            res[("auto", 0, 0)] = t_ms(lambda: C.cudanp_tmv(A, x, y))
            bt = min((k for k in res if k[0] == "tma"), key=res.get)
            bl = min((k for k in res if k[0] == "ldg"), key=res.get)
            rec = {"h": h, "w": w, "strips128_per_sm": round(((w + 127) // 128) / sms, 3),
                   "tma_best": {"S": bt[1], "dist": bt[2], "gbs": round(nb / res[bt] / 1e6, 1)},
                   "ldg_best": {"S": bl[1], "dist": bl[2], "gbs": round(nb / res[bl] / 1e6, 1)},
                   "auto_gbs": round(nb / res[("auto", 0, 0)] / 1e6, 1),
                   "auto_choice": C.cudanp_choose_version("tmv", w, h),
                   "all": {f"{k[0]}/{k[1]}/{'cyc' if k[2] == C.CYCLIC else 'blk'}": round(nb / v / 1e6, 1)
                           for k, v in res.items()}}
            f.write(json.dumps(rec) + "\n")
            f.flush()
            print(json.dumps({k: rec[k] for k in ("h", "w", "strips128_per_sm", "tma_best", "ldg_best",
                                                  "auto_gbs")}), flush=True)
            del A
            torch.cuda.empty_cache()


def narrow(out):
    sys.path.insert(0, os.path.join(ROOT, "tools"))
    from c1_latency import graph_us
    shapes = [(1024, 512), (1024, 1024), (1024, 2048), (1024, 4096), (4096, 1024), (4096, 2048),
              (16384, 1024), (16384, 2048), (16384, 4096), (16384, 8192), (65536, 1024)]
    with open(out, "w") as f:
        for h, w in shapes:
            copies = max(2, min(64, (512 << 20) // (4 * h * w)))
            As = []
            for k in range(copies):
                t = torch.empty(h, w, device="cuda")
                C.cudanp_generate(t, "f32_unit", stream_id=1, seed=k)
                As.append(t)
            x = torch.empty(h, device="cuda")
            C.cudanp_generate(x, "f32_unit", stream_id=2)
            ys = [torch.empty(w, device="cuda") for _ in range(copies)]
            nb = 4 * h * w + 4 * h + 4 * w
            res = {}
            for S, d in itertools.product((8, 16, 32, 64, 128), (C.CYCLIC, C.BLOCK)):
                res[(S, d)] = graph_us([lambda i=i: C.cudanp_tmv(As[i], x, ys[i], S=S, dist=d,
                                                                 map=C.INTER_WARP)
                                        for i in range(copies)])
            auto = graph_us([lambda i=i: C.cudanp_tmv(As[i], x, ys[i]) for i in range(copies)])
            best = min(res, key=res.get)
            rec = {"h": h, "w": w, "copies": copies,
                   "best": {"S": best[0], "dist": "cyclic" if best[1] == C.CYCLIC else "block",
                            "us": round(res[best], 3), "gbs": round(nb / res[best] / 1e3, 1)},
                   "auto": {"choice": C.cudanp_choose_version("tmv", w, h), "us": round(auto, 3),
                            "gbs": round(nb / auto / 1e3, 1), "vs_best": round(res[best] / auto, 3)},
                   "all_us": {f"{S}/{'cyc' if d == C.CYCLIC else 'blk'}": round(v, 3)
                              for (S, d), v in res.items()}}
            f.write(json.dumps(rec) + "\n")
            f.flush()
            print(json.dumps({k: rec[k] for k in ("h", "w", "best", "auto")}), flush=True)
            del As
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
