#!/usr/bin/env python
"""Summarise tools/sweep.py JSONL into a Markdown table (per config/op/dtype/L:
best GB/s per S, best overall, speedups vs tuned S=1, literal S=1 and DP)."""
import collections
import json
import sys


def main(path, out=None):
    recs = [json.loads(l) for l in open(path) if l.strip()]
    groups = collections.OrderedDict()
    for r in recs:
        key = (r["config"], r["op"], r.get("dtype"), r.get("opname", ""), r.get("L"))
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
        comp = {r["impl"]: r for r in rs if r["impl"] not in ("np", "best_np")}

        def vs(name):
            c = comp.get(name)
            return f"{c['t_median_us'] / b['t_median_us']:.2f}x" if c else "—"
        dp_thr = next((k for k in comp if k.startswith("dp_thread")), None)
        lines.append(
            f"| {cfg} | {op}{(' ' + opn) if opn else ''} | {dt} | {L} | "
            + " | ".join(f"{perS.get(S, float('nan')):.0f}" for S in (1, 2, 4, 8, 16, 32))
            + f" | {b['S']},{b['dist']},{b['map']} | {b['gbs']:.0f} | {100 * b['gbs'] / 6537:.1f} | "
            + f"{b.get('speedup_vs_s1_tuned', float('nan')):.2f}x | {vs('s1_literal')} | {vs('dp_block')} | "
            + (vs(dp_thr) if dp_thr else "—") + " |")
    txt = "\n".join(lines)
    print(txt)
    if out:
        open(out, "w").write(txt + "\n")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else None)
