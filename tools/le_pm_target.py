import sys, torch
sys.path.insert(0, ".")
from paper_conf_ppopp_yangz14_b200 import cudanp as C
C.load()
N, L = 1 << 21, 150
x = torch.empty(L, N, device="cuda")
C.cudanp_generate(x, "f32_unit")
S = int(sys.argv[1]) if len(sys.argv) > 1 else 8
for _ in range(3):
    C.cudanp_le_gicov(x, 0.02, layout=1, S=S, dist=C.BLOCK, map=C.INTER_WARP, placement=C.GRAD_SHARED)
torch.cuda.synchronize()
