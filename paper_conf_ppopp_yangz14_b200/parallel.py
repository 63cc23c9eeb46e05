"""Multi-GPU plumbing: one process per GPU, outer items sharded by contiguous
ranges (outer items are independent),
results gathered to rank 0 with torch.distributed (NCCL on GPUs, gloo in the
CPU tests).  The ranges come from the library's cudanp_shard_range, so the
kernels and the gather agree on ownership.

Row-wise split-K for TMV is deliberately not offered: it would change the
summation order with the rank count.
"""
from __future__ import annotations

from . import cudanp as C


def shard(n_outer: int, world: int, rank: int) -> tuple[int, int]:
    return C.cudanp_shard_range(n_outer, world, rank)


def gather_to_root(local, root_buf, n_total: int, rank: int, world: int, root: int = 0):
    """Grouped point-to-point gather (NCCL has no gather primitive): every rank
    sends its shard, the root receives shard g into root_buf[begin_g:end_g].
    Shards may be uneven.  Returns root_buf on the root, None elsewhere."""
    import torch.distributed as dist
    b_me, e_me = shard(n_total, world, rank)
    if local.shape[0] != e_me - b_me:
        raise ValueError(f"rank {rank}: local shard has {local.shape[0]} items, expected {e_me - b_me}")
    if world == 1:
        root_buf[b_me:e_me].copy_(local)
        return root_buf
    ops = []
    if rank == root:
        for g in range(world):
            b, e = shard(n_total, world, g)
            if g == root:
                root_buf[b:e].copy_(local)
            elif e > b:
                ops.append(dist.P2POp(dist.irecv, root_buf[b:e], g))
    elif e_me > b_me:
        ops.append(dist.P2POp(dist.isend, local.contiguous(), root))
    if ops:
        for r in dist.batch_isend_irecv(ops):
            r.wait()
    return root_buf if rank == root else None
