#!/usr/bin/env python
"""Summarise ncu reports (.ncu-rep, `--set full`) and a launch list (CSV of
gpu__time_duration.sum) into profiles/.

    python tools/ncu_summary.py --tag r01 [--dir gpurun_out]

Writes profiles/ncu_<tag>.md (key counters per captured kernel and the
launch-list shares), and profiles/ncu_traffic.json (DRAM bytes per launch of
the bench's TMV and MV kernels, read by bench.py for roofline.traffic).
"""
import argparse
import csv
import glob
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("sm__maximum_warps_per_active_cycle_pct", "theoretical occupancy %"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "threads per instruction"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__shared_mem_per_block_static", "static smem/CTA"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("launch__waves_per_multiprocessor", "waves/SM"),
    ("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "L1 global load sectors"),
    ("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "L1 global load requests"),
    ("lts__t_sectors_srcunit_tex_op_read.sum", "L2 read sectors (from L1)"),
    ("sm__cycles_elapsed.avg.per_second", "SM clock"),
    ("smsp__average_warp_latency_issue_stalled_long_scoreboard", "stall long_scoreboard"),
    ("smsp__pcsamp_warps_issue_stalled_long_scoreboard", "pc samples long_scoreboard"),
]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return []
    hdr, units = rows[0], rows[1]
    res = []
    for vals in rows[2:]:
        d = {}
        for i, h in enumerate(hdr):
            d[h] = (vals[i], units[i] if i < len(units) else "")
        res.append(d)
    return res


def num(v):
    try:
        return float(v.replace(",", ""))
    except Exception:
        return None


def to_bytes(val, unit):
    x = num(val)
    if x is None:
        return None
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(unit, 1)
    return x * scale


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr_i = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[hdr_i]
    ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    ui = hdr.index("Metric Unit")
    out = []
    for r in rows[hdr_i + 1:]:
        if len(r) > vi and r[mi] == "gpu__time_duration.sum":
            t = num(r[vi])
            if r[ui] == "usecond":
                t *= 1e3
            elif r[ui] == "msecond":
                t *= 1e6
            out.append((r[ki], t))  # ns
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tag", default="r01")
    ap.add_argument("--dir", default=os.path.join(ROOT, "gpurun_out"))
    a = ap.parse_args()
    md = [f"# ncu summary — {a.tag}", "",
          "Captured with `ncu --set full --clock-control none --import-source on` on one B200 "
          "(`tools/gpu_round.sh`); kernels isolated by `tools/ncu_target.py`. Durations here are "
          "ncu's (cold caches, serialised) and are NOT bench numbers.", ""]
    traffic = {}
    for rep in sorted(glob.glob(os.path.join(a.dir, f"prof_*_{a.tag}.ncu-rep"))):
        op = os.path.basename(rep).split("_")[1]
        for d in raw(rep):
            name = d.get("Kernel Name", ("?", ""))[0]
            md.append(f"## {op}: `{name}`")
            md.append("")
            md.append("| counter | value |")
            md.append("|---|---|")
            for m, label in METRICS:
                if m in d:
                    md.append(f"| {label} (`{m}`) | {d[m][0]} {d[m][1]} |")
            rb = to_bytes(*d.get("dram__bytes_read.sum", ("", "")))
            wb = to_bytes(*d.get("dram__bytes_write.sum", ("", "")))
            if rb is not None and wb is not None:
                traffic[op] = {"kernel": name, "dram_bytes_per_launch": rb + wb,
                               "dram_read": rb, "dram_write": wb, "source": os.path.basename(rep)}
                md.append(f"| DRAM read+write per launch | {rb + wb:.4g} B |")
            md.append("")
    fpath = os.path.join(a.dir, f"launches_full_{a.tag}.csv")
    if os.path.exists(fpath):
        ls = launches(fpath)
        tot = sum(t for _, t in ls) or 1
        agg = {}
        for k, t in ls:
            short = k.split("(")[0]
            c, s_ = agg.get(short, (0, 0.0))
            agg[short] = (c + 1, s_ + t)
        md += ["## Launch list of the driver's command `python bench.py` (ncu gpu__time_duration, "
               "--clock-control none; includes the autotune sweep, comparison kernels and e2e steps)", "",
               "| kernel | launches | total µs | share |", "|---|---|---|---|"]
        for k, (c, s_) in sorted(agg.items(), key=lambda kv: -kv[1][1])[:25]:
            md.append(f"| `{k}` | {c} | {s_ / 1e3:.1f} | {100 * s_ / tot:.1f} % |")
        md.append("")
    lpath = os.path.join(a.dir, f"launches_{a.tag}.csv")
    if os.path.exists(lpath):
        ls = launches(lpath)
        tot = sum(t for _, t in ls) or 1
        agg = {}
        for k, t in ls:
            short = k.split("(")[0]
            c, s = agg.get(short, (0, 0.0))
            agg[short] = (c + 1, s + t)
        md += ["## Launch list of `bench.py --no-sweep` (ncu gpu__time_duration, --clock-control none)", "",
               "| kernel | launches | total µs | share |", "|---|---|---|---|"]
        for k, (c, s) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
            md.append(f"| `{k}` | {c} | {s / 1e3:.1f} | {100 * s / tot:.1f} % |")
        md.append("")
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    open(os.path.join(ROOT, "profiles", f"ncu_{a.tag}.md"), "w").write("\n".join(md) + "\n")
    if traffic:
        json.dump(traffic, open(os.path.join(ROOT, "profiles", "ncu_traffic.json"), "w"), indent=1)
    print("\n".join(md))


if __name__ == "__main__":
    sys.exit(main())
