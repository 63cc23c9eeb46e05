#!/usr/bin/env python
"""C1 per-launch time from cold HBM (64 copies) vs from L2 (one copy reused):
how much of the 2.6 us is DRAM latency + transfer, how much the kernel."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import torch  # noqa: E402

from c1_latency import graph_us  # noqa: E402
from paper_conf_ppopp_yangz14_b200 import cudanp as C  # noqa: E402

C.load()
n, copies = 1024, 64
As = []
for _ in range(copies):
    t = torch.empty(n, n, device="cuda")
    C.cudanp_generate(t, "f32_unit")
    As.append(t)
x = torch.empty(n, device="cuda")
C.cudanp_generate(x, "f32_unit", stream_id=2)
ys = [torch.empty(n, device="cuda") for _ in range(copies)]
out = {}
for S, d in ((64, C.BLOCK), (32, C.CYCLIC), (128, C.BLOCK)):
    out[f"cold_S{S}"] = round(graph_us([lambda i=i: C.cudanp_tmv(As[i], x, ys[i], S=S, dist=d, map=C.INTER_WARP)
                                        for i in range(copies)]), 3)
    out[f"warm_S{S}"] = round(graph_us([lambda i=i: C.cudanp_tmv(As[0], x, ys[i], S=S, dist=d, map=C.INTER_WARP)
                                        for i in range(copies)]), 3)
tiny = torch.empty(1, device="cuda")
out["floor"] = round(graph_us([lambda: tiny.fill_(1.0)] * copies), 3)
print(json.dumps(out))
