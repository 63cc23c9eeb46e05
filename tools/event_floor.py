#!/usr/bin/env python
"""The floor of a single launch timed by its own pair of CUDA events on this
pod: an empty torch fill and batched reduces of growing size (C3 shape,
L = 32, S = 4 block).  Sub-100 us single-launch numbers in the sweeps carry
this floor; the steady-state columns (20 launches per event pair) do not.

    python tools/event_floor.py
"""
import sys, torch, statistics
sys.path.insert(0, __import__('os').path.dirname(__import__('os').path.dirname(__import__('os').path.abspath(__file__))))
from paper_conf_ppopp_yangz14_b200 import cudanp as C
C.load()
x = torch.rand(4 << 20, 32, device='cuda'); y = torch.empty(4 << 20, device='cuda')
def single(fn, reps=20):
    for _ in range(3): fn()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); b.synchronize(); ts.append(a.elapsed_time(b) * 1e3)
    return statistics.median(ts)
for n in (32, 4096, 1 << 16, 1 << 20, 4 << 20):
    xs, ys = x[:n], y[:n]
    print(n, "single us", round(single(lambda: C.cudanp_batched_loop_reduce(xs, None, ys, S=4, dist=1)), 2), flush=True)
print("empty torch fill single us", round(single(lambda: y[:1].fill_(1.0)), 2))
