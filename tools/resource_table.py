#!/usr/bin/env python
"""Table 1 analog (per-thread REG/SM bytes, baseline vs NP): the
launch shape each NP instantiation uses on this B200 -- block size, grid,
registers per thread, static shared memory -- for the bench/sweep configs,
via cudanp_launch_info.  Writes gpurun_out/resources_<tag>.md."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_ppopp_yangz14_b200 import cudanp as C  # noqa: E402


def main(tag="r01"):
    C.load()
    rows = ["| op | N × L | S | dist | map | block | grid | regs/thread | smem/CTA (B) | REG B/thread | SM B/thread |",
            "|---|---|---|---|---|---|---|---|---|---|---|"]
    cases = [("tmv", 16384, 16384, C.F32, C.SUM), ("tmv", 1024, 1024, C.F32, C.SUM),
             ("mv", 16384, 16384, C.F32, C.SUM), ("reduce", 1 << 22, 64, C.F32, C.SUM),
             ("scan", 1 << 21, 256, C.I32, C.SUM)]
    for op, N, L, dt, o in cases:
        for S in C.SLAVE_SIZES:
            for d in (C.CYCLIC, C.BLOCK):
                for m in (C.INTRA_WARP, C.INTER_WARP):
                    vec = not (op == "tmv" and N < 8192)
                    i = C.cudanp_launch_info(op, N, L, dtype=dt, op=o, S=S, dist=d, map=m, vec4=vec)
                    rows.append(f"| {op} | {N}×{L} | {S} | {'cyc' if d == 0 else 'blk'} | {i['map']} | "
                                f"{i['block_threads']} | {i['grid_ctas']} | {i['regs_per_thread']} | "
                                f"{i['smem_bytes']} | {4 * i['regs_per_thread']} | "
                                f"{i['smem_bytes'] / max(i['block_threads'], 1):.1f} |")
    txt = "# Resource use per NP instantiation (Table 1 analog, P:94-115)\n\n" \
          "REG/SM bytes per thread as in the paper's Table 1 (registers x 4 B; static smem / block).\n\n" \
          + "\n".join(rows) + "\n"
    out = os.path.join(ROOT, "gpurun_out")  # merged back by gpurun; copied to profiles/ by hand
    os.makedirs(out, exist_ok=True)
    open(os.path.join(out, f"resources_{tag}.md"), "w").write(txt)
    print(txt)


if __name__ == "__main__":
    main(*(sys.argv[1:2]))
