import json, os, sys
sys.path.insert(0, "."); sys.path.insert(0, "tools")
import torch
from c1_latency import graph_us
from paper_conf_ppopp_yangz14_b200 import cudanp as C
C.load()
n, copies = 1024, 64
As = []
for _ in range(copies):
    t = torch.empty(n, n, device="cuda"); C.cudanp_generate(t, "f32_unit"); As.append(t)
x = torch.empty(n, device="cuda"); C.cudanp_generate(x, "f32_unit", stream_id=2)
ys = [torch.empty(n, device="cuda") for _ in range(copies)]
out = {"lib": os.environ.get("CUDANP_LIB", "default")}
for S in (64, 128, 256):
    for d in (C.CYCLIC, C.BLOCK):
        out[f"S{S}{'c' if d == 0 else 'b'}"] = round(graph_us([lambda i=i: C.cudanp_tmv(As[i], x, ys[i], S=S, dist=d, map=C.INTER_WARP) for i in range(copies)]), 3)
# correctness vs S=32 cyclic (exact data)
C.cudanp_generate(As[0], "f32_int4"); C.cudanp_generate(x, "f32_int4", stream_id=2)
ref = C.cudanp_tmv(As[0], x, S=32, dist=C.CYCLIC, map=C.INTER_WARP).clone()
for S in (64, 128, 256):
    for d in (0, 1):
        assert torch.equal(C.cudanp_tmv(As[0], x, S=S, dist=d, map=C.INTER_WARP), ref), (S, d)
print(json.dumps(out))
