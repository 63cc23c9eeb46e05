"""B200-native CUDA-NP hot path (Yang & Zhou, PPoPP'14).

``libcudanp.so`` (C ABI in ``include/cudanp.h``) holds hand-written sm_100a
master/slave kernels for TMV, MV, batched loop-reduce and batched loop-scan,
plus the S=1 and dynamic-parallelism comparison kernels.  ``cudanp`` is the
ctypes binding (argument marshalling only); ``parallel`` shards outer items
over ranks (one process per GPU) and gathers results.
"""
from . import cudanp  # noqa: F401
from .cudanp import (  # noqa: F401
    AUTO, BLOCK, CYCLIC, F32, I32, INTER_WARP, INTRA_WARP, MAX, SUM, SLAVE_SIZES,
    S1_LITERAL, DP_THREAD, DP_BLOCK, CudanpError,
    cudanp_tmv, cudanp_mv, cudanp_batched_loop_reduce, cudanp_batched_loop_scan,
    cudanp_tmv_variant, cudanp_mv_variant, cudanp_batched_loop_reduce_variant,
    cudanp_batched_loop_scan_variant, cudanp_generate, cudanp_shard_range,
    cudanp_launch_info, cudanp_dp_set_pending_launch_limit, cudanp_dp_error_count,
)

__version__ = "0.1.0"
