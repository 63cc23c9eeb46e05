#!/usr/bin/env python
"""Summarise tools/sweep.py JSONL into a Markdown table (per config/op/dtype/L:
best GB/s per S, best overall, speedups vs tuned S=1, literal S=1 and DP)."""
import collections
import json
import sys


def peak_gbs():
    """The measured copy peak of this pod (MEASURED_PEAKS.json), else the survey's 6537."""
    import os
    p = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")
    try:
        return float(json.load(open(p))["hbm_gbs"])
    except (OSError, KeyError, ValueError):
        return 6537.0


def main(path, out=None):
    recs = [json.loads(l) for l in open(path) if l.strip()]
    PEAK = peak_gbs()
    special = [r for r in recs if r["config"] in ("F3", "E9")]
    recs = [r for r in recs if r["config"] not in ("F3", "E9")]
    groups = collections.OrderedDict()
    for r in recs:
        key = (r["config"], r["op"], r.get("dtype"), r.get("opname", "") or r.get("layout", ""), r.get("L"))
        groups.setdefault(key, []).append(r)
    lines = ["| config | op | dtype | L | S=1 | S=2 | S=4 | S=8 | S=16 | S=32 | best (S,dist,map) | best GB/s | % HBM | vs tuned S=1 | vs literal S=1 | vs DP-CTA | vs DP-thread |",
             "|---|---|---|---|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
    for (cfg, op, dt, opn, L), rs in groups.items():
        np_ = [r for r in rs if r["impl"] == "np"]
        perS = {}
        for r in np_:
            perS[r["S"]] = max(perS.get(r["S"], 0), r["gbs"])
        best = [r for r in rs if r["impl"] == "best_np"]
        if best:
            b = best[0]
        elif np_:
            b = max(np_, key=lambda r: r["gbs"])
        else:
            continue
        comp = {r["impl"]: r for r in rs if r["impl"] not in ("np", "best_np", "fig12", "auto")}

        def vs(name):
            c = comp.get(name)
            return f"{c['t_median_us'] / b['t_median_us']:.2f}x" if c else "—"
        dp_thr = next((k for k in comp if k.startswith("dp_thread")), None)
        lines.append(
            f"| {cfg} | {op}{(' ' + opn) if opn else ''} | {dt} | {L} | "
            + " | ".join(f"{perS.get(S, float('nan')):.0f}" for S in (1, 2, 4, 8, 16, 32))
            + f" | {b['S']},{b['dist']},{b['map']} | {b['gbs']:.0f} | {100 * b['gbs'] / PEAK:.1f} | "
            + f"{b.get('speedup_vs_s1_tuned', float('nan')):.2f}x | {vs('s1_literal')} | {vs('dp_block')} | "
            + (vs(dp_thr) if dp_thr else "—") + " |")
    st = [r for r in recs if r["impl"] == "best_np" and "gbs_steady" in r]
    if st:
        lines += ["", f"Steady state (20 back-to-back launches per event pair; % of the {PEAK:.0f} GB/s copy peak)", "",
                  "| config | op | dtype | L | best NP | single GB/s | steady GB/s | steady % | best S=1 | S=1 steady GB/s | NP/S=1 steady |",
                  "|---|---|---|---|---|---|---|---|---|---|---|"]
        for r in st:
            lines.append(f"| {r['config']} | {r['op']}{(' ' + r['opname']) if r.get('opname') else ''} | {r['dtype']} | "
                         f"{r['L']} | {r['S']},{r['dist']},{r['map']} | {r['gbs']:.0f} | {r['gbs_steady']:.0f} | "
                         f"{100 * r['gbs_steady'] / PEAK:.1f} | {r['s1_steady']} | {r['gbs_s1_steady']:.0f} | "
                         f"{r['speedup_vs_s1_steady']:.2f}x |")
    au = [r for r in recs if r["impl"] == "auto" and "vs_best_np" in r]
    if au:
        lines += ["", "Library's own choice (S = S_AUTO, MAP_AUTO) against the swept best NP version", "",
                  "| config | op | dtype | L | auto GB/s | auto / best NP | auto / tuned S=1 |", "|---|---|---|---|---|---|---|"]
        lines += [f"| {r['config']} | {r['op']}{(' ' + r['opname']) if r.get('opname') else ''} | {r['dtype']} | "
                  f"{r['L']} | {r['gbs']:.0f} | {r['vs_best_np']:.3f} | {r['vs_s1_tuned']:.2f}x |" for r in au]
    f12 = [r for r in recs if r["impl"] == "fig12"]
    if f12:
        lines += ["", "Fig 12 analog: non-power-of-two inter-warp S vs the power of two it pads to (GB/s)", "",
                  "| config | op | dtype | L | S | dist | GB/s | padded S | padded GB/s | S / padded |",
                  "|---|---|---|---|---|---|---|---|---|---|"]
        lines += [f"| {r['config']} | {r['op']}{(' ' + r['opname']) if r.get('opname') else ''} | {r['dtype']} | "
                  f"{r['L']} | {r['S']} | {r['dist']} | {r['gbs']:.0f} | {r['S_padded']} | {r['gbs_padded']:.0f} | "
                  f"{r['speedup_vs_padded']:.2f}x |" for r in f12]
    rv = [r for r in recs if r["config"] == "R1" and str(r["impl"]).startswith("adaptive")]
    if rv:
        lines += ["", "R1 — ragged versions beside the swept NP kernels (GB/s; x = time of the best NP / its time)", "",
                  "| L | impl | GB/s | % HBM | vs best NP |", "|---|---|---|---|---|"]
        lines += [f"| {r['L']} | {r['impl']} | {r['gbs']:.0f} | {100 * r['gbs'] / PEAK:.1f} | "
                  f"{1 / r['speedup_of_best_np']:.2f}x |" for r in rv]
    f3 = [r for r in special if r["config"] == "F3"]
    if f3:
        lines += ["", "F3 — Fig 1 memcopy (64M floats): impl, m parents x n children, GB/s", "",
                  "| impl | m | n | GB/s |", "|---|---|---|---|"]
        lines += [f"| {r['impl']} | {r['m']} | {r['n']} | {r['gbs']:.0f} |" for r in f3]
    e9 = [r for r in special if r["config"] == "E9"]
    if e9:
        t = collections.OrderedDict()
        for r in e9:
            t.setdefault((r["dtype"], r["opname"], r["L"], r["S"]), {})[r["backend"]] = r["gbs"]
        lines += ["", "E9 — Fig 16 analog: team reduction backend (GB/s)", "",
                  "| dtype | op | L | S | shfl | smem | redux |", "|---|---|---|---|---|---|---|"]
        lines += [f"| {k[0]} | {k[1]} | {k[2]} | {k[3]} | {v.get('shfl', 0):.0f} | {v.get('smem', 0):.0f} | "
                  f"{v.get('redux', 0):.0f} |" for k, v in t.items()]
    txt = "\n".join(lines)
    print(txt)
    if out:
        open(out, "w").write(txt + "\n")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else None)
