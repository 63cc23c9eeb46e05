#!/usr/bin/env python
"""PDL A/B (run twice: CUDANP_PDL=1 / 0): back-to-back launches of C2 TMV+MV
steps, C3 reduce L=32/256, C4 scan L=64, 20 per event pair; prints GB/s."""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from paper_conf_ppopp_yangz14_b200 import cudanp as C  # noqa: E402


def run(body, K=20, reps=7):
    for _ in range(3):
        body()
    ts = []
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        for _ in range(K):
            body()
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1) / K)
    return statistics.median(ts)


def main():
    C.load()
    out = {"pdl": os.environ.get("CUDANP_PDL", "1")}
    n = 16384
    A = torch.empty(n, n, device="cuda")
    C.cudanp_generate(A, "f32_unit")
    x = torch.empty(n, device="cuda")
    C.cudanp_generate(x, "f32_unit", stream_id=2)
    yt, ym = torch.empty(n, device="cuda"), torch.empty(n, device="cuda")
    nb = 4 * n * n + 8 * n
    t = run(lambda: (C.cudanp_tmv(A, x, yt), C.cudanp_mv(A, x, ym)))
    out["C2_step"] = round(2 * nb / t / 1e6, 1)
    out["C2_tmv"] = round(nb / run(lambda: C.cudanp_tmv(A, x, yt)) / 1e6, 1)
    out["C2_mv"] = round(nb / run(lambda: C.cudanp_mv(A, x, ym)) / 1e6, 1)
    del A
    N = 1 << 22
    for L in (32, 256):
        X = torch.empty(N, L, device="cuda")
        C.cudanp_generate(X, "f32_unit")
        o = torch.empty(N, device="cuda")
        out[f"C3_L{L}"] = round((4 * N * L + 4 * N) / run(lambda: C.cudanp_batched_loop_reduce(X, None, o)) / 1e6, 1)
        del X
    N = 1 << 21
    X = torch.empty(N, 64, dtype=torch.int32, device="cuda")
    C.cudanp_generate(X, "i32_small", B=1 << 15)
    O = torch.empty_like(X)
    out["C4_L64"] = round(8 * N * 64 / run(lambda: C.cudanp_batched_loop_scan(X, None, O)) / 1e6, 1)
    print(json.dumps(out))


if __name__ == "__main__":
    main()
