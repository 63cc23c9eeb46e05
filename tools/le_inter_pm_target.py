#!/usr/bin/env python
"""Launch the point-major LE inter-warp kernel (Grad in registers) a few times
for ncu: python tools/le_inter_pm_target.py <S> [block|cyclic]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ppopp_yangz14_b200 import cudanp as C  # noqa: E402

C.load()
N, L = 1 << 21, 150
x = torch.empty(L, N, device="cuda")
C.cudanp_generate(x, "f32_unit")
S = int(sys.argv[1]) if len(sys.argv) > 1 else 4
d = C.CYCLIC if len(sys.argv) > 2 and sys.argv[2] == "cyclic" else C.BLOCK
for _ in range(3):
    C.cudanp_le_gicov(x, 0.02, layout=1, S=S, dist=d, map=C.INTER_WARP)
torch.cuda.synchronize()
