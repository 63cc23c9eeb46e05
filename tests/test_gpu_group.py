"""Native multi-GPU group (cudanp_group_*, cudanp_sharded_*) on the one GPU
this box has: a world-1 NCCL communicator runs the whole path (shard = all
items, gather = the root's own copy) against the oracle.  World > 1 needs one
GPU per rank (NCCL rejects duplicate devices); the gather's multi-rank logic
is covered by tests/test_parallel_gloo.py and the same-GPU IPC tests."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import oracle as O
import synth
from paper_conf_ppopp_yangz14_b200 import build as B
from paper_conf_ppopp_yangz14_b200 import cudanp as C

pytestmark = pytest.mark.gpu


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def test_world1_group_sharded_calls_match_oracle():
    B.build()
    C.load()
    g = C.cudanp_group_create(C.cudanp_group_unique_id(), 1, 0)
    try:
        A = synth.matrix(300, 516, "f32_int4")
        x = synth.vector(300, "f32_int4")
        Ad, xd = dev(A), dev(x)
        y_shard = torch.empty(516, device="cuda")
        y_root = torch.full((516,), -1.0, device="cuda")
        for S, m in ((8, C.INTER_WARP), (16, C.INTER_WARP_TMA), (4, C.INTRA_WARP)):
            C.cudanp_sharded_tmv(g, Ad, xd, y_shard, y_root, 516, S=S, map=m)
            torch.cuda.synchronize()
            assert np.array_equal(y_root.cpu().numpy(), O.tmv(A, x)), (S, m)
        X = synth.items(1001, 64, "i32_full")
        ini = synth.init(1001, "i32_small")
        out_s = torch.empty(1001, dtype=torch.int32, device="cuda")
        out_r = torch.zeros(1001, dtype=torch.int32, device="cuda")
        C.cudanp_sharded_batched_loop_reduce(g, dev(X), dev(ini), out_s, out_r, 1001, op=C.MAX, S=8)
        torch.cuda.synchronize()
        assert np.array_equal(out_r.cpu().numpy(), O.reduce(X, op=O.MAX, init=ini))
        # gather into the root buffer in place (local is the root's own slice)
        buf = torch.arange(10, dtype=torch.float32, device="cuda")
        C.cudanp_group_gather(g, buf, buf, 10)
        torch.cuda.synchronize()
        assert np.array_equal(buf.cpu().numpy(), np.arange(10, dtype=np.float32))
    finally:
        C.cudanp_group_destroy(g)
