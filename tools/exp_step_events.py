#!/usr/bin/env python
"""Does recording CUDA events between the step's two kernels cost anything
(programmatic dependent launch across an event record)?  C2 step (TMV TMA
S=8 cyclic + MV S=256 cyclic), 20 steps per event pair, with and without
per-kernel events, and each kernel alone back to back."""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_ppopp_yangz14_b200 import cudanp as C  # noqa: E402


def main():
    C.load()
    n = 16384
    A = torch.empty(n, n, device="cuda")
    C.cudanp_generate(A, "f32_unit")
    x = torch.empty(n, device="cuda")
    C.cudanp_generate(x, "f32_unit", stream_id=2)
    yt, ym = torch.empty(n, device="cuda"), torch.empty(n, device="cuda")
    tmv = lambda: C.cudanp_tmv(A, x, yt, S=8, dist=C.CYCLIC, map=C.INTER_WARP_TMA)  # noqa: E731
    mv = lambda: C.cudanp_mv(A, x, ym, S=256, dist=C.CYCLIC, map=C.INTRA_WARP)  # noqa: E731
    st = torch.cuda.current_stream()
    K = 20

    def run(body, reps=7):
        for _ in range(3):
            body(None)
        ts = []
        for _ in range(reps):
            evs = [[torch.cuda.Event(enable_timing=True) for _ in range(3)] for _ in range(K)]
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record(st)
            for k in range(K):
                body(evs[k])
            e1.record(st)
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1) / K)
        return statistics.median(ts)

    def step_ev(ev):
        if ev:
            ev[0].record(st)
        tmv()
        if ev:
            ev[1].record(st)
        mv()
        if ev:
            ev[2].record(st)

    res = {
        "step_tmv_mv_events": run(step_ev),
        "step_tmv_mv_no_events": run(lambda ev: (tmv(), mv())),
        "step_mv_tmv_no_events": run(lambda ev: (mv(), tmv())),
        "tmv_only": run(lambda ev: tmv()),
        "mv_only": run(lambda ev: mv()),
    }
    nb = 4 * n * n + 8 * n
    out = {k: {"ms": round(v, 5), "gbs": round((2 if "step" in k else 1) * nb / v / 1e6, 1)} for k, v in res.items()}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
