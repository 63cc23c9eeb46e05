#!/usr/bin/env python
"""C1 (TMV 1024^2, 4 MiB) is launch/latency-bound: per-launch time of a CUDA
graph of 64 launches over 64 distinct input copies (256 MiB > L2, every
launch cold), for the best NP shapes, plus the graph floor of a trivial
kernel (torch's fill of 4 bytes).  Run twice -- CUDANP_PDL=1 (default) and
CUDANP_PDL=0 -- to measure programmatic dependent launch.

    CUDANP_PDL=0 python tools/c1_latency.py --out gpurun_out/c1_latency.jsonl
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from paper_conf_ppopp_yangz14_b200 import cudanp as C  # noqa: E402


def graph_us(fns, reps=9):
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
        ts.append(a.elapsed_time(b) * 1e3 / len(fns))
    return statistics.median(ts)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=None)
    ap.add_argument("--n", type=int, default=1024)
    a = ap.parse_args()
    C.load()
    n, copies = a.n, 64
    As = []
    for _ in range(copies):
        t = torch.empty(n, n, device="cuda")
        C.cudanp_generate(t, "f32_unit")
        As.append(t)
    x = torch.empty(n, device="cuda")
    C.cudanp_generate(x, "f32_unit", stream_id=2)
    ys = [torch.empty(n, device="cuda") for _ in range(copies)]
    nb = 4 * n * n + 8 * n
    pdl = os.environ.get("CUDANP_PDL", "1")
    out = open(a.out, "a") if a.out else None

    def emit(rec):
        rec.update({"pdl": pdl, "n": n})
        line = json.dumps(rec)
        print(line, flush=True)
        if out:
            out.write(line + "\n")

    tiny = torch.empty(1, device="cuda")
    emit({"impl": "graph_floor_torch_fill", "us": round(graph_us([lambda: tiny.fill_(1.0)] * copies), 3)})
    emit({"impl": "graph_floor_cudanp_tmv_empty",
          "us": round(graph_us([lambda i=i: C.cudanp_tmv(As[i][:0], x[:0], ys[i], S=32, dist=C.CYCLIC,
                                                         map=C.INTER_WARP, n_outer=n)
                                for i in range(copies)]), 3)})
    for S in (8, 16, 32, 64, 128, 256, 1024):  # 256 / 1024: cluster teams
        for d in (C.CYCLIC, C.BLOCK):
            us = graph_us([lambda i=i: C.cudanp_tmv(As[i], x, ys[i], S=S, dist=d, map=C.INTER_WARP)
                           for i in range(copies)])
            emit({"impl": "np", "S": S, "dist": "cyclic" if d == 0 else "block", "map": "inter",
                  "us": round(us, 3), "gbs": round(nb / us / 1e3, 1)})
    for S in (8, 16, 32):
        us = graph_us([lambda i=i: C.cudanp_tmv(As[i], x, ys[i], S=S, dist=C.CYCLIC, map=C.INTRA_WARP)
                       for i in range(copies)])
        emit({"impl": "np", "S": S, "dist": "cyclic", "map": "intra", "us": round(us, 3),
              "gbs": round(nb / us / 1e3, 1)})
    # tuned S = 1 (no nesting): the LDG kernel of each map and the TMA-staged one
    for m, name in ((C.INTER_WARP, "inter"), (C.INTRA_WARP, "intra"), (C.INTER_WARP_TMA, "inter_tma")):
        us = graph_us([lambda i=i: C.cudanp_tmv(As[i], x, ys[i], S=1, dist=C.CYCLIC, map=m)
                       for i in range(copies)])
        emit({"impl": "s1_tuned", "S": 1, "map": name, "us": round(us, 3), "gbs": round(nb / us / 1e3, 1)})
    us = graph_us([lambda i=i: C.cudanp_tmv(As[i], x, ys[i]) for i in range(copies)])
    emit({"impl": "auto", "us": round(us, 3), "gbs": round(nb / us / 1e3, 1)})
    us = graph_us([lambda i=i: C.cudanp_tmv_variant(C.S1_LITERAL, As[i], x, ys[i]) for i in range(copies)])
    emit({"impl": "s1_literal", "us": round(us, 3), "gbs": round(nb / us / 1e3, 1)})


if __name__ == "__main__":
    main()
