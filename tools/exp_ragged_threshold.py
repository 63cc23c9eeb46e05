#!/usr/bin/env python
"""Adaptive ragged reduce: small team-size thresholds on the short-segment
mixes (R1 mean 16 / 64, N = 4M), beside the best fixed-S kernel."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_ppopp_yangz14_b200 import cudanp as C  # noqa: E402
from sweep import time_ms  # noqa: E402

C.load()
N = 1 << 22
for mean in (16, 64, 256):
    for dist in ("uniform", "exp"):
        off = torch.from_numpy(synth.offsets_from_lengths(synth.lengths(N, mean, dist))).cuda()
        total = int(off[-1].item())
        x = torch.empty(total, device="cuda")
        C.cudanp_generate(x, "f32_unit")
        out = torch.empty(N, device="cuda")
        nb = 4 * total + 8 * (N + 1) + 4 * N
        res = {}
        for th in (64, 128):
            res[f"adaptive_t{th}"] = time_ms(lambda: C.cudanp_ragged_loop_reduce_adaptive(x, off, None, out, threshold=th))[0]
        for S, d, m in ((1, C.CYCLIC, C.INTRA_WARP), (1, C.BLOCK, C.INTER_WARP), (4, C.BLOCK, C.INTRA_WARP)):
            res[f"np_S{S}_{'cyc' if d == C.CYCLIC else 'blk'}_{'intra' if m == C.INTRA_WARP else 'inter'}"] = \
                time_ms(lambda: C.cudanp_ragged_loop_reduce(x, off, None, out, S=S, dist=d, map=m))[0]
        print(json.dumps({"L": f"{dist}{mean}", "gbs": {k: round(nb / (v * 1e-3) / 1e9, 1) for k, v in res.items()}}),
              flush=True)
        del x, out, off
        torch.cuda.empty_cache()
