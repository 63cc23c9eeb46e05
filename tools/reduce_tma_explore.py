#!/usr/bin/env python
"""Ring-shape exploration for the TMA-staged batched reduce
(cudanp_batched_loop_reduce_tma) on C3 (4M items x L), against the best LDG
intra-warp kernel on the same operands.  GB/s of algorithmic bytes 4NL + 4N.

    python tools/reduce_tma_explore.py [--out gpurun_out/reduce_tma_explore.jsonl]
"""
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
    ap.add_argument("--out", default=None)
    ap.add_argument("--N", type=int, default=1 << 22)
    ap.add_argument("--Ls", default="32,64,128,256")
    a = ap.parse_args()
    C.load()
    out_f = open(a.out, "a") if a.out else None
    N = a.N
    for L in [int(v) for v in a.Ls.split(",")]:
        x = torch.empty(N, L, device="cuda")
        C.cudanp_generate(x, "f32_unit", stream_id=1)
        out = torch.empty(N, device="cuda")
        ref = torch.empty(N, device="cuda")
        nb = 4 * N * L + 4 * N

        def emit(rec):
            rec.update({"N": N, "L": L})
            line = json.dumps(rec)
            print(line, flush=True)
            if out_f:
                out_f.write(line + "\n")
                out_f.flush()

        best_ldg = min((time_ms(lambda: C.cudanp_batched_loop_reduce(x, None, out, S=S, dist=d, map=C.INTRA_WARP)), S, d)
                       for S, d in itertools.product(C.SLAVE_SIZES, (C.CYCLIC, C.BLOCK)))
        emit({"impl": "ldg_best", "S": best_ldg[1], "dist": best_ldg[2], "gbs": round(nb / best_ldg[0] / 1e6, 1)})
        for S, d in itertools.product(C.SLAVE_SIZES, (C.CYCLIC, C.BLOCK)):
            C.cudanp_batched_loop_reduce(x, None, ref, S=S, dist=d, map=C.INTRA_WARP)
            for sb, st in ((0, 0), (16384, 0), (65536, 0), (32768, 3), (32768, 4)):
                try:
                    t = time_ms(lambda: C.cudanp_batched_loop_reduce_tma(x, None, out, S=S, dist=d,
                                                                        stage_bytes=sb, stages=st))
                except C.CudanpError:
                    continue
                same = bool(torch.equal(out, ref))
                emit({"impl": "tma", "S": S, "dist": "cyclic" if d == 0 else "block", "stage_bytes": sb,
                      "stages": st, "gbs": round(nb / t / 1e6, 1), "same_as_ldg": same})
        del x
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
