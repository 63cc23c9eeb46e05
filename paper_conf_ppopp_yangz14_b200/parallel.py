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


def gather_to_root(local, root_buf, n_total: int, rank: int, world: int, root: int = 0,
                   async_op: bool = False):
    """Grouped point-to-point gather (NCCL has no gather primitive): every rank
    sends its shard, the root receives shard g into root_buf[begin_g:end_g].
    Shards may be uneven.  Returns root_buf on the root, None elsewhere; with
    async_op=True returns the list of pending works instead (the caller waits
    on them -- on NCCL that only orders its current stream after the
    transfers -- before it reuses `local` or reads root_buf), so the gather of
    one op's outputs can overlap the next op's kernel."""
    import torch.distributed as dist
    b_me, e_me = shard(n_total, world, rank)
    if world > 1 and local.is_cuda and dist.get_backend() == "gloo":
        # test mode only (several ranks sharing one GPU, where NCCL refuses
        # duplicate devices): gloo moves host memory, so stage through the host
        cpu_root = root_buf.cpu() if rank == root else None
        gather_to_root(local.cpu(), cpu_root, n_total, rank, world, root)
        if rank == root:
            root_buf.copy_(cpu_root)
        return [] if async_op else (root_buf if rank == root else None)
    if local.shape[0] != e_me - b_me:
        raise ValueError(f"rank {rank}: local shard has {local.shape[0]} items, expected {e_me - b_me}")
    if world == 1:
        root_buf[b_me:e_me].copy_(local)
        return [] if async_op else root_buf
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
    works = dist.batch_isend_irecv(ops) if ops else []
    if async_op:
        return works
    for r in works:
        r.wait()
    return root_buf if rank == root else None


class FusedGather:
    """Gather fused into the kernels' master stores.

    Rank 0 exports its result buffer through CUDA IPC; every other rank maps
    it once, and then passes ``out_ptr()`` -- rank 0's buffer at the start of
    its own shard -- as the output pointer of a cudanp call, so each master
    thread's store lands in rank 0's HBM over NVLink with no separate
    collective.  ``finish()`` orders the stores before rank 0 reads:
    stream synchronize + a process-group barrier.
    """

    def __init__(self, root_buf, n_total: int, rank: int, world: int, elem_bytes: int = 4,
                 root: int = 0):
        import torch.distributed as dist
        self.rank, self.world, self.root = rank, world, root
        self.begin, self.end = shard(n_total, world, rank)
        self.mapped, self.error = None, None
        obj = [None]
        if rank == root:
            self.base = root_buf.data_ptr()
            try:
                obj = [C.cudanp_ipc_get_handle(root_buf)]
            except C.CudanpError as e:  # every rank still joins the broadcast
                self.error = str(e)
        dist.broadcast_object_list(obj, src=root)
        if obj[0] is None:
            self.error = self.error or "rank 0 could not export its buffer"
            self.handle, self.offset = None, 0
        else:
            self.handle, self.offset = obj[0]
        if rank != root and self.handle is not None:
            try:
                self.mapped = C.cudanp_ipc_open(self.handle, self.offset)
                self.base = self.mapped
            except C.CudanpError as e:
                self.error = str(e)
        self.elem_bytes = elem_bytes

    @property
    def ok(self) -> bool:
        """This rank can store into rank 0's buffer (collective agreement is
        the caller's: see all_ok)."""
        return self.error is None

    @staticmethod
    def all_ok(gathers, world: int) -> bool:
        """True when every rank opened every buffer (an all-reduce MIN)."""
        import torch
        import torch.distributed as dist
        flag = 1.0 if all(g.ok for g in gathers) else 0.0
        dev = "cuda" if dist.get_backend() == "nccl" else "cpu"
        t = torch.tensor([flag], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MIN)
        return bool(t.item() > 0)

    def out_ptr(self) -> int:
        return self.base + self.begin * self.elem_bytes

    def finish(self):
        import torch
        import torch.distributed as dist
        torch.cuda.current_stream().synchronize()
        dist.barrier()

    def close(self):
        if self.mapped is not None:
            C.cudanp_ipc_close(self.mapped, self.offset)
            self.mapped = None


class NativeGroup:
    """The library's own multi-GPU group (cudanp_group_*, include/cudanp.h):
    an NCCL communicator rank created natively from a unique id that rank 0
    makes and torch.distributed broadcasts once.  ``gather`` enqueues the
    shard gather to rank 0 on the current stream (NCCL send/recv in the
    library); ``sharded_tmv`` / ``sharded_reduce`` run this rank's shard and
    the gather in one C call."""

    def __init__(self, rank: int, world: int):
        import torch.distributed as dist
        self.rank, self.world = rank, world
        obj = [C.cudanp_group_unique_id() if rank == 0 else None]
        if world > 1:
            dist.broadcast_object_list(obj, src=0)
        self.handle = C.cudanp_group_create(obj[0], world, rank)

    def gather(self, local, root_buf, n_total: int):
        C.cudanp_group_gather(self.handle, local, root_buf, n_total)
        return root_buf if self.rank == 0 else None

    def sharded_tmv(self, A_shard, x, y_shard, y_root, n_total: int, **kw):
        C.cudanp_sharded_tmv(self.handle, A_shard, x, y_shard, y_root, n_total, **kw)

    def sharded_reduce(self, in_shard, init_shard, out_shard, out_root, n_total: int, **kw):
        C.cudanp_sharded_batched_loop_reduce(self.handle, in_shard, init_shard, out_shard, out_root,
                                             n_total, **kw)

    def close(self):
        if self.handle:
            C.cudanp_group_destroy(self.handle)
            self.handle = None
