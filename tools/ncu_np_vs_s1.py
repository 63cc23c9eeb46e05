#!/usr/bin/env python
"""ncu counters of the best NP kernel beside its no-NP (S=1) and literal
comparison kernels, per config: the evidence for *why* nesting wins on B200
(occupancy, coalescing = sectors per request, DRAM throughput, issue rate).

    python tools/ncu_np_vs_s1.py run  --out gpurun_out/npvs1     # on the GPU box
    python tools/ncu_np_vs_s1.py summarize --out gpurun_out/npvs1 --md profiles/ncu_np_vs_s1_<tag>.md

`run` launches `ncu --metrics <list> --clock-control none` on tools/ncu_target.py
once per case (one kernel captured after a warm-up launch).  ncu durations
are serialised and cold-cache: they rank kernels, they are not bench numbers.
"""
import argparse
import csv
import io
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

METRICS = [
    ("gpu__time_duration.sum", "duration us", 1e-3),
    ("dram__bytes_read.sum", "DRAM read MB", 1e-6),
    ("dram__bytes_write.sum", "DRAM write MB", 1e-6),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM % of peak", 1),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %", 1),
    ("sm__maximum_warps_per_active_cycle_pct", "theoretical occupancy %", 1),
    ("launch__registers_per_thread", "registers/thread", 1),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %", 1),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "threads/instruction", 1),
    ("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "L1 ld sectors (M)", 1e-6),
    ("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "L1 ld requests (M)", 1e-6),
    ("launch__grid_size", "grid", 1),
    ("launch__block_size", "block", 1),
]

# (config, label, ncu_target args, kernel regex)
CASES = [
    ("C1 TMV 1024²", "S=1 inter (no NP)", "--op tmv --n 1024 --S 1 --dist cyclic --map inter", "tmv_"),
    ("C1 TMV 1024²", "literal Fig 2", "--op tmv_literal --n 1024", "tmv_"),
    ("C1 TMV 1024²", "S=1 TMA (no NP)", "--op tmv --n 1024 --S 1 --dist cyclic --map inter_tma", "tmv_"),
    ("C1 TMV 1024²", "NP S=32 cyclic inter", "--op tmv --n 1024 --S 32 --dist cyclic --map inter", "tmv_"),
    ("C1 TMV 1024²", "NP S=64 block inter", "--op tmv --n 1024 --S 64 --dist block --map inter", "tmv_"),
    ("C1 TMV 1024²", "NP S=128 cyclic inter (V=4, 4 masters)", "--op tmv --n 1024 --S 128 --dist cyclic --map inter", "tmv_"),
    ("C2 MV 16384²", "S=1 inter (no NP)", "--op mv --S 1 --dist cyclic --map inter", "mv_"),
    ("C2 MV 16384²", "literal", "--op mv_literal", "mv_"),
    ("C2 MV 16384²", "S=1 TMA-tiled (no NP; SMM-style)", "--op mv_tiled", "mv_"),
    ("C2 MV 16384²", "NP S=32 cyclic intra", "--op mv --S 32 --dist cyclic --map intra", "mv_"),
    ("C2 MV 16384²", "NP S=256 cyclic (multi-warp)", "--op mv --S 256 --dist cyclic --map intra", "mv_"),
    ("C2 TMV 16384²", "S=1 inter LDG (no NP)", "--op tmv --S 1 --dist cyclic --map inter", "tmv_"),
    ("C2 TMV 16384²", "S=1 TMA (no NP)", "--op tmv --S 1 --dist cyclic --map inter_tma", "tmv_"),
    ("C2 TMV 16384²", "NP S=8 block TMA", "--op tmv --S 8 --dist block --map inter_tma", "tmv_"),
    ("C3 reduce 4M×256", "S=1 inter (no NP)", "--op reduce --L 256 --S 1 --dist block --map inter", "reduce_"),
    ("C3 reduce 4M×256", "literal", "--op reduce_literal --L 256", "reduce_"),
    ("C3 reduce 4M×256", "S=1 TMA-tiled (no NP)", "--op reduce_tiled --L 256", "reduce_"),
    ("C3 reduce 4M×256", "NP S=32 block intra", "--op reduce --L 256 --S 32 --dist block --map intra", "reduce_"),
    ("C4 scan 2M×256 i32", "S=1 inter (no NP)", "--op scan --N 2097152 --L 256 --dtype i32 --S 1 --dist block --map inter", "scan_"),
    ("C4 scan 2M×256 i32", "literal", "--op scan_literal --N 2097152 --L 256 --dtype i32", "scan_"),
    ("C4 scan 2M×256 i32", "S=1 TMA-tiled (no NP)", "--op scan_tiled --N 2097152 --L 256 --dtype i32", "scan_"),
    ("C4 scan 2M×256 i32", "NP S=16 cyclic intra", "--op scan --N 2097152 --L 256 --dtype i32 --S 16 --dist cyclic --map intra", "scan_"),
    ("F2 LE 2M×150 item-major", "literal Fig 5", "--op le_literal --N 2097152 --L 150 --layout 0", "le_"),
    ("F2 LE 2M×150 item-major", "S=1 intra (no NP)", "--op le --N 2097152 --L 150 --layout 0 --S 1 --dist cyclic --map intra", "le_"),
    ("F2 LE 2M×150 item-major", "NP S=8 cyclic intra", "--op le --N 2097152 --L 150 --layout 0 --S 8 --dist cyclic --map intra", "le_"),
    ("F2 LE 2M×150 point-major", "NP S=5 block inter", "--op le --N 2097152 --L 150 --layout 1 --S 5 --dist block --map inter", "le_"),
    ("reduce 16×4M (few items)", "NP S=1024 (one CTA per item)", "--op reduce --N 16 --L 4194304 --S 1024", "reduce_"),
    ("reduce 16×4M (few items)", "NP S=4096 (cluster per item)", "--op reduce --N 16 --L 4194304 --S 4096", "reduce_"),
]


def run(out, only=None):
    os.makedirs(out, exist_ok=True)
    mlist = ",".join(m for m, _, _ in METRICS)
    for i, (cfg, label, args, rx) in enumerate(CASES):
        if only and only not in cfg:
            continue
        log = os.path.join(out, f"case{i:02d}.csv")
        cmd = (f"ncu --metrics {mlist} --clock-control none --csv --log-file {log} -k regex:{rx} -s 1 -c 1 "
               f"{sys.executable} {os.path.join(ROOT, 'tools', 'ncu_target.py')} {args} --reps 2")
        r = subprocess.run(cmd, shell=True, capture_output=True, text=True, timeout=600)
        print(f"case {i} ({cfg} / {label}): rc={r.returncode}", flush=True)


def parse(path):
    txt = open(path).read()
    lines = txt.splitlines()
    try:
        start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    except StopIteration:
        return None, {}
    rows = list(csv.reader(io.StringIO("\n".join(lines[start:]))))
    hdr = rows[0]
    ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    ui = hdr.index("Metric Unit")
    name, vals = None, {}
    for r in rows[1:]:
        name = r[ki]
        try:
            v = float(r[vi].replace(",", ""))
        except ValueError:
            continue
        unit = r[ui]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1, "usecond": 1e3,
                 "msecond": 1e6}.get(unit, 1)
        vals[r[mi]] = v * scale
    return name, vals


def summarize(out, md):
    lines = ["# ncu: best NP kernel vs no-NP (S=1) and literal kernels", "",
             "`tools/ncu_np_vs_s1.py` (`ncu --metrics … --clock-control none`, one launch after a warm-up). "
             "Durations are ncu's (serialised, cold caches): they rank kernels, they are not bench numbers. "
             "Sectors/request = L1 global-load sectors ÷ requests (4 = one 128-byte line per warp request of "
             "32 lanes × 4 B; 16 = 32 lanes × 16 B fully coalesced; 32 = every lane on its own sector).", ""]
    hdr = "| config | kernel | " + " | ".join(h for _, h, _ in METRICS) + " | sectors/request |"
    lines += [hdr, "|" + "---|" * (len(METRICS) + 3)]
    for i, (cfg, label, _, _) in enumerate(CASES):
        p = os.path.join(out, f"case{i:02d}.csv")
        if not os.path.exists(p):
            continue
        name, v = parse(p)
        if not v:
            lines.append(f"| {cfg} | {label} | (no capture) |")
            continue
        cells = []
        for m, _, sc in METRICS:
            x = v.get(m)
            cells.append("—" if x is None else (f"{x * sc:.1f}" if x * sc < 1e5 else f"{x * sc:.3g}"))
        sec, req = v.get("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum"), v.get("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum")
        spr = f"{sec / req:.1f}" if sec and req else "—"
        kname = (name or "").split("(")[0].replace("void ", "")
        lines.append(f"| {cfg} | {label}<br>`{kname}` | " + " | ".join(cells) + f" | {spr} |")
    txt = "\n".join(lines) + "\n"
    open(md, "w").write(txt)
    print(txt)


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("mode", choices=["run", "summarize"])
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "npvs1"))
    ap.add_argument("--md", default=os.path.join(ROOT, "profiles", "ncu_np_vs_s1.md"))
    ap.add_argument("--only", default=None, help="run: configs containing this substring")
    a = ap.parse_args()
    run(a.out, a.only) if a.mode == "run" else summarize(a.out, a.md)
