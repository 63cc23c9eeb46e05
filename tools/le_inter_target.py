# ncu target: LE point-major inter-warp (F2 shape), S from argv, block distribution.
import sys, torch
sys.path.insert(0, ".")
from paper_conf_ppopp_yangz14_b200 import cudanp as C
lib = C.load()
N, L = 1 << 21, 150
x = torch.empty(L, N, device="cuda"); C.cudanp_generate(x, "f32_unit")
g = torch.empty(N, device="cuda"); st = [torch.empty(N, device="cuda") for _ in range(3)]
S = int(sys.argv[1]); d = C.BLOCK
for _ in range(3):
    lib.cudanp_le_gicov(x.data_ptr(), g.data_ptr(), *(t.data_ptr() for t in st), N, L, 0.02, 1, S, d, C.INTER_WARP, None)
torch.cuda.synchronize()
