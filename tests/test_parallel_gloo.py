"""Multi-process (world_size 2 and 3, gloo, CPU) checks of the sharding and
gather plumbing used for N > 1 GPUs.  Each rank computes its
contiguous shard of the outer items with the ORACLE (the CUDA kernels need a
GPU; here only the host logic is under test) and the shards are gathered to
rank 0, which must reproduce the unsharded result bit for bit (pin P4: the
result does not depend on the rank count)."""
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch

    import oracle as O
    import synth
    from paper_conf_ppopp_yangz14_b200 import parallel as P

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        h, n_total = 64, 1001          # TMV: outer items = columns of a 64 x 1001 matrix
        b, e = P.shard(n_total, world, rank)
        A_shard = synth.matrix(h, e - b, "f32_unit", col0=b, w_global=n_total)
        x = synth.vector(h, "f32_unit")
        y_local = torch.from_numpy(O.tmv(A_shard, x))
        root = torch.empty(n_total, dtype=torch.float32) if rank == 0 else None
        P.gather_to_root(y_local, root, n_total, rank, world)
        # batched reduce: items sharded, int32
        N, L = 777, 33
        b, e = P.shard(N, world, rank)
        items = synth.items(e - b, L, "i32_full", n0=b)
        r_local = torch.from_numpy(O.reduce(items))
        r_root = torch.empty(N, dtype=torch.int32) if rank == 0 else None
        # asynchronous form (bench.py overlaps the TMV gather with the MV kernel):
        # two gathers in flight, then wait on every pending work
        works = P.gather_to_root(r_local, r_root, N, rank, world, async_op=True)
        r2_root = torch.empty(N, dtype=torch.int32) if rank == 0 else None
        works += P.gather_to_root(r_local, r2_root, N, rank, world, async_op=True)
        for wk in works:
            wk.wait()
        if rank == 0:
            assert torch.equal(r_root, r2_root)
        if rank == 0:
            q.put((root.numpy().copy(), r_root.numpy().copy()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_sharded_gather_matches_unsharded(world):
    import oracle as O
    import synth
    from paper_conf_ppopp_yangz14_b200 import build as B
    B.build()  # the shard ranges come from the library (host logic, no GPU needed)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    y, r = q.get(timeout=120)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    A = synth.matrix(64, 1001, "f32_unit")
    x = synth.vector(64, "f32_unit")
    assert np.array_equal(y, O.tmv(A, x))
    assert np.array_equal(r, O.reduce(synth.items(777, 33, "i32_full")))
