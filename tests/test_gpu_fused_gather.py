"""f4: fused gather -- every rank's kernel stores its shard straight into
rank 0's buffer through CUDA IPC.  Two processes share the
one GPU of this test box (same-device IPC is the same mechanism as peer
NVLink mapping); the gathered result must equal the unsharded oracle."""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu

H, W = 300, 1001
N, L = 5000, 64


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch.distributed as dist

    from paper_conf_ppopp_yangz14_b200 import cudanp as C
    from paper_conf_ppopp_yangz14_b200 import parallel as P
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    try:
        # TMV column shards (outer items = columns)
        root = torch.full((W,), float("nan"), device="cuda") if rank == 0 else None
        fg = P.FusedGather(root, W, rank, world)
        b, e = fg.begin, fg.end
        A = torch.empty(H, e - b, device="cuda")
        C.cudanp_generate(A, "f32_int4", stream_id=1, col0=b, w_global=W)
        x = torch.empty(H, device="cuda")
        C.cudanp_generate(x, "f32_int4", stream_id=2)
        C.cudanp_tmv(A, x, fg.out_ptr(), S=8)
        fg.finish()
        # batched reduce item shards, int32
        rroot = torch.full((N,), -1, dtype=torch.int32, device="cuda") if rank == 0 else None
        fr = P.FusedGather(rroot, N, rank, world)
        X = torch.empty(fr.end - fr.begin, L, dtype=torch.int32, device="cuda")
        C.cudanp_generate(X, "i32_full", stream_id=1, row0=fr.begin, w_global=L)
        C.cudanp_batched_loop_reduce(X, None, fr.out_ptr(), S=8)
        fr.finish()
        if rank == 0:
            q.put((root.cpu().numpy(), rroot.cpu().numpy()))
        dist.barrier()
        fg.close()
        fr.close()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_fused_gather_equals_unsharded(world):
    import oracle as O
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    y, r = q.get(timeout=300)
    for p in ps:
        p.join(timeout=120)
        assert p.exitcode == 0
    A = O.gen_f32(1, "f32_int4", 0, H * W).reshape(H, W)
    x = O.gen_f32(2, "f32_int4", 0, H)
    assert np.array_equal(y, O.tmv(A, x))
    X = O.gen_i32(1, "i32_full", 0, N * L).reshape(N, L)
    assert np.array_equal(r, O.reduce(X))


def _nccl_g1(q, port):
    import torch.distributed as dist

    import oracle as O
    from paper_conf_ppopp_yangz14_b200 import cudanp as C
    from paper_conf_ppopp_yangz14_b200 import parallel as P
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        A = torch.empty(H, W, device="cuda")
        C.cudanp_generate(A, "f32_int4", stream_id=1)
        x = torch.empty(H, device="cuda")
        C.cudanp_generate(x, "f32_int4", stream_id=2)
        y = C.cudanp_tmv(A, x, S=8)
        root = torch.empty(W, device="cuda")
        P.gather_to_root(y, root, W, 0, 1)
        ref = O.tmv(O.gen_f32(1, "f32_int4", 0, H * W).reshape(H, W), O.gen_f32(2, "f32_int4", 0, H))
        q.put(bool(np.array_equal(root.cpu().numpy(), ref)))
    finally:
        dist.destroy_process_group()


def test_nccl_world1_degenerate_gather():
    # NCCL with G = 1 is a degenerate but real path
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    p = ctx.Process(target=_nccl_g1, args=(q, _port()))
    p.start()
    ok = q.get(timeout=300)
    p.join(timeout=60)
    assert ok and p.exitcode == 0
