"""Thin Python binding of libcudanp.so (include/cudanp.h).

Argument marshalling only: every step of the hot path runs in the library's
sm_100a kernels.  torch supplies device memory and the current CUDA stream.
There is no CPU fallback: if the shared library is missing this module raises
on first use, and a non-OK status from the library raises CudanpError.

Function names follow the C ABI (``cudanp_tmv``, ``cudanp_mv``,
``cudanp_batched_loop_reduce``, ``cudanp_batched_loop_scan`` and the
``*_variant`` comparison calls).
"""
from __future__ import annotations

import ctypes
import os
import threading

import numpy as np

_PKG = os.path.dirname(os.path.abspath(__file__))
# CUDANP_LIB selects a build-variant library (experiments, e.g. -DCUDANP_LDG256)
LIB_PATH = os.environ.get("CUDANP_LIB") or os.path.join(_PKG, "libcudanp.so")

OK, ERR_INVALID, ERR_UNSUPPORTED, ERR_CUDA, ERR_NCCL = 0, 1, 2, 3, 4
CYCLIC, BLOCK = 0, 1
AUTO, INTRA_WARP, INTER_WARP, INTER_WARP_TMA, INTRA_WARP_TMA = 0, 1, 2, 3, 4
F32, I32 = 0, 1
SUM, MAX = 0, 1
S1_LITERAL, DP_THREAD, DP_BLOCK, S1_TILED = 1, 2, 3, 4
GRAD_REGISTERS, GRAD_SHARED, GRAD_GLOBAL = 0, 1, 2   # LE: home of Grad (Fig 6c / 6b / 6a)
S_AUTO = 0                                            # S argument: the library picks (S, dist, map)
SLAVE_SIZES = (1, 2, 4, 8, 16, 32)                    # one warp (intra) or S warps (inter)
INTER_ONLY_SIZES = (3, 5, 10, 15)                     # non-power-of-two: inter-warp map only
MULTI_WARP_SIZES = (64, 128, 256, 512, 1024)          # S/32 warps of one CTA (reduce, scan, MV;
                                                      # TMV: 64, 128 inter-warp)
CLUSTER_SIZES = (2048, 4096, 8192)                    # a cluster of 8 CTAs (reduce, scan, MV);
TMV_CLUSTER_SIZES = (256, 1024)                       # TMV: 8 CTAs x 8 masters x 32/128 warps
KIND = {"f32_unit": 0, "f32_signed": 1, "f32_int4": 2, "i32_small": 3, "i32_full": 4,
        "ones_f32": 5, "ones_i32": 6}
SEED = 20140215

_i64, _u64, _int, _vp, _sz = ctypes.c_int64, ctypes.c_uint64, ctypes.c_int, ctypes.c_void_p, ctypes.c_size_t
_P32 = ctypes.POINTER(ctypes.c_int32)
_SIGS = {
    "cudanp_tmv": [_vp, _i64, _vp, _vp, _i64, _i64, _int, _int, _int, _vp],
    "cudanp_mv": [_vp, _i64, _vp, _vp, _i64, _i64, _int, _int, _int, _vp],
    "cudanp_tmv_tma": [_vp, _i64, _vp, _vp, _i64, _i64, _int, _int, _vp],
    "cudanp_tmv_tma_ex": [_vp, _i64, _vp, _vp, _i64, _i64, _int, _int, _int, _int, _int, _vp],
    "cudanp_batched_loop_reduce": [_vp, _vp, _vp, _i64, _i64, _int, _int, _int, _int, _int, _vp],
    "cudanp_batched_loop_reduce_tma": [_vp, _vp, _vp, _i64, _i64, _int, _int, _int, _int, _int, _int,
                                       _vp],
    "cudanp_batched_loop_scan": [_vp, _vp, _vp, _i64, _i64, _int, _int, _int, _int, _vp],
    "cudanp_batched_loop_reduce_backend": [_vp, _vp, _vp, _i64, _i64, _int, _int, _int, _int, _vp],
    "cudanp_ragged_loop_reduce": [_vp, _vp, _vp, _vp, _i64, _int, _int, _int, _int, _int, _vp],
    "cudanp_ragged_loop_reduce_literal": [_vp, _vp, _vp, _vp, _i64, _int, _int, _vp],
    "cudanp_ragged_loop_reduce_adaptive": [_vp, _vp, _vp, _vp, _i64, _int, _int, _i64, _vp],
    "cudanp_le_gicov": [_vp, _vp, _vp, _vp, _vp, _i64, _i64, ctypes.c_float, _int, _int, _int,
                        _int, _vp],
    "cudanp_le_gicov_placement": [_vp, _vp, _vp, _vp, _vp, _i64, _i64, ctypes.c_float, _int, _int,
                                  _int, _int, _int, _vp],
    "cudanp_le_gicov_literal": [_vp, _vp, _vp, _vp, _vp, _i64, _i64, ctypes.c_float, _int, _vp],
    "cudanp_tmv_variant": [_int, _vp, _i64, _vp, _vp, _i64, _i64, _vp],
    "cudanp_mv_variant": [_int, _vp, _i64, _vp, _vp, _i64, _i64, _vp],
    "cudanp_batched_loop_reduce_variant": [_int, _vp, _vp, _vp, _i64, _i64, _int, _int, _vp],
    "cudanp_batched_loop_scan_variant": [_int, _vp, _vp, _vp, _i64, _i64, _int, _vp],
    "cudanp_dp_set_pending_launch_limit": [_sz],
    "cudanp_dp_error_count": [_int, ctypes.POINTER(_i64)],
    "cudanp_dp_memcopy": [_vp, _vp, _i64, _i64, _int, _vp],
    "cudanp_autotune_count": [_int],
    "cudanp_autotune_candidate": [_int, _int, ctypes.POINTER(_int), ctypes.POINTER(_int),
                                  ctypes.POINTER(_int)],
    "cudanp_autotune": [_int, _vp, _vp, _vp, _i64, _i64, _i64, _int, _int, _int,
                        ctypes.POINTER(ctypes.c_float), ctypes.POINTER(_int), _vp],
    "cudanp_launch_info": [_int, _i64, _i64, _int, _int, _int, _int, _int, _int,
                           ctypes.POINTER(_int), ctypes.POINTER(_i64), ctypes.POINTER(_int),
                           ctypes.POINTER(_int), ctypes.POINTER(_int), ctypes.POINTER(_int),
                           ctypes.POINTER(_int)],
    "cudanp_choose_version": [_int, _i64, _i64, _int, _int, ctypes.POINTER(_int), ctypes.POINTER(_int),
                              ctypes.POINTER(_int)],
    "cudanp_group_unique_id": [_vp],
    "cudanp_group_create": [_vp, _int, _int, ctypes.POINTER(_vp)],
    "cudanp_group_destroy": [_vp],
    "cudanp_group_rank": [_vp, ctypes.POINTER(_int), ctypes.POINTER(_int)],
    "cudanp_group_gather": [_vp, _vp, _vp, _i64, _int, _vp],
    "cudanp_sharded_tmv": [_vp, _vp, _i64, _vp, _vp, _vp, _i64, _i64, _int, _int, _int, _vp],
    "cudanp_sharded_batched_loop_reduce": [_vp, _vp, _vp, _vp, _vp, _i64, _i64, _int, _int, _int, _int,
                                           _int, _vp],
    "cudanp_shard_range": [_i64, _int, _int, ctypes.POINTER(_i64), ctypes.POINTER(_i64)],
    "cudanp_ipc_get_handle": [_vp, _vp, ctypes.POINTER(_i64)],
    "cudanp_ipc_open": [_vp, _i64, ctypes.POINTER(_vp)],
    "cudanp_ipc_close": [_vp, _i64],
    "cudanp_generate": [_vp, _i64, _i64, _i64, _i64, _i64, _i64, _int, _int, _i64, _u64, _vp],
    "cudanp_debug_owner_map": [_i64, _int, _int, _int, _P32],
    "cudanp_debug_team_ids": [_int, _int, _P32, _P32, ctypes.POINTER(_int)],
    "cudanp_debug_broadcast": [_int, _int, _P32, ctypes.POINTER(_int)],
    "cudanp_status_string": [_int],
    "cudanp_last_error": [],
    "cudanp_version": [],
}
EXPORTS = tuple(_SIGS)

_lock = threading.Lock()
_lib = None


class CudanpError(RuntimeError):
    def __init__(self, status: int, where: str, detail: str):
        super().__init__(f"{where}: status {status} ({_status_name(status)}): {detail}")
        self.status = status


def _status_name(s: int) -> str:
    return {0: "OK", 1: "ERR_INVALID", 2: "ERR_UNSUPPORTED", 3: "ERR_CUDA", 4: "ERR_NCCL"}.get(s, "?")


def load(path: str = LIB_PATH) -> ctypes.CDLL:
    """Load libcudanp.so.  Raises if it has not been built (no fallback)."""
    global _lib
    with _lock:
        if _lib is None:
            if not os.path.exists(path):
                raise ImportError(f"{path} not found: build it with "
                                  "`python -m paper_conf_ppopp_yangz14_b200.build`")
            L = ctypes.CDLL(path)
            for name, args in _SIGS.items():
                f = getattr(L, name)
                f.argtypes = args
                f.restype = ctypes.c_char_p if name in ("cudanp_status_string", "cudanp_last_error") else _int
            _lib = L
    return _lib


def _check(rc: int, where: str) -> None:
    if rc != OK:
        raise CudanpError(rc, where, load().cudanp_last_error().decode())


def _stream(stream) -> int | None:
    import torch
    if stream is None:
        return torch.cuda.current_stream().cuda_stream or None
    if isinstance(stream, int):
        return stream or None
    return stream.cuda_stream or None


def _ptr(t) -> int | None:
    """Device pointer of a CUDA tensor, or a raw device address passed as int
    (e.g. an IPC-mapped peer buffer, cudanp_ipc_open)."""
    if t is None:
        return None
    if isinstance(t, int):
        return t or None
    if not t.is_cuda:
        raise ValueError("tensor must be on a CUDA device (the library takes device pointers)")
    return t.data_ptr() or None


def _dtype_code(t) -> int:
    import torch
    if t.dtype == torch.float32:
        return F32
    if t.dtype == torch.int32:
        return I32
    raise TypeError(f"unsupported dtype {t.dtype}: float32 or int32")


# ---------------------------------------------------------------- argument checks
# The C ABI takes raw pointers plus sizes and a leading dimension; these checks
# make sure the tensors handed over really have that layout, dtype and length,
# so a strided view or a short buffer raises here instead of being misread.
def _mat(A, what: str):
    """(rows, cols, lda) of a row-major fp32 CUDA matrix; lda = A.stride(0)."""
    import torch
    if not isinstance(A, torch.Tensor) or A.dim() != 2:
        raise ValueError(f"{what}: A must be a 2-D tensor")
    if A.dtype != torch.float32:
        raise TypeError(f"{what}: A must be float32 (got {A.dtype})")
    rows, cols = A.shape
    if rows > 0 and cols > 1 and A.stride(1) != 1:
        raise ValueError(f"{what}: A must have unit column stride (row-major; use A.contiguous())")
    lda = A.stride(0) if rows > 1 else cols
    if rows > 1 and cols > 0 and lda < cols:
        raise ValueError(f"{what}: A rows overlap (stride(0) = {lda} < {cols} columns)")
    return rows, cols, lda


def _buf(t, n: int, dtype, what: str) -> None:
    """t holds at least n contiguous elements of dtype (raw int pointers pass)."""
    import torch
    if t is None or isinstance(t, int):
        return
    if not isinstance(t, torch.Tensor):
        raise TypeError(f"{what} must be a CUDA tensor")
    if t.dtype != dtype:
        raise TypeError(f"{what} must be {dtype} (got {t.dtype})")
    if not t.is_contiguous():
        raise ValueError(f"{what} must be contiguous")
    if t.numel() < n:
        raise ValueError(f"{what} holds {t.numel()} elements, needs {n}")


def _items(x, what: str):
    """(N, L) of an item-major [N][L] batch (contiguous, fp32 or int32)."""
    import torch
    if not isinstance(x, torch.Tensor) or x.dim() != 2:
        raise ValueError(f"{what}: input must be a 2-D (N, L) tensor")
    _dtype_code(x)
    if not x.is_contiguous():
        raise ValueError(f"{what}: input must be contiguous item-major (N, L) (use .contiguous())")
    return x.shape


# ---------------------------------------------------------------- hot-path calls
def _tmv_args(A, x, y, n_outer, what):
    import torch
    h, cols, lda = _mat(A, what)
    w = cols if n_outer is None else n_outer
    if w > cols:
        raise ValueError(f"{what}: n_outer {w} > A's {cols} columns")
    _buf(x, h, torch.float32, f"{what}: x")
    _buf(y, w, torch.float32, f"{what}: y")
    return h, w, lda


def _mv_args(A, x, y, n_inner, what):
    import torch
    h, cols, lda = _mat(A, what)
    w = cols if n_inner is None else n_inner
    if w > cols:
        raise ValueError(f"{what}: n_inner {w} > A's {cols} columns")
    _buf(x, w, torch.float32, f"{what}: x")
    _buf(y, h, torch.float32, f"{what}: y")
    return h, w, lda


def _batched_args(x, init, out, per_item: bool, what):
    N, L = _items(x, what)
    _buf(init, N, x.dtype, f"{what}: init")
    _buf(out, N if per_item else N * L, x.dtype, f"{what}: out")
    return N, L


def cudanp_tmv(A, x, y=None, *, S=S_AUTO, dist=CYCLIC, map=AUTO, n_outer=None, stream=None):
    """y[j] = sum_i A[i, j] * x[i] (Fig 2).  A: (h, >= w) fp32, unit column
    stride, lda = A.stride(0)."""
    import torch
    h, w, lda = _tmv_args(A, x, y, n_outer, "cudanp_tmv")
    if y is None:
        y = torch.empty(w, dtype=torch.float32, device=A.device)
    _check(load().cudanp_tmv(_ptr(A), lda, _ptr(x), _ptr(y), w, h, S, dist, map, _stream(stream)),
           "cudanp_tmv")
    return y


def cudanp_tmv_tma(A, x, y=None, *, S=8, dist=CYCLIC, n_outer=None, stream=None,
                   cols=0, rows_sel=-1, stages=0):
    """TMV with TMA-staged tiles (inter-warp map); same result contract as cudanp_tmv.
    cols / rows_sel / stages pin the launch shape (cudanp_tmv_tma_ex); defaults = auto."""
    import torch
    h, w, lda = _tmv_args(A, x, y, n_outer, "cudanp_tmv_tma")
    if y is None:
        y = torch.empty(w, dtype=torch.float32, device=A.device)
    if cols == 0 and rows_sel == -1 and stages == 0:
        rc = load().cudanp_tmv_tma(_ptr(A), lda, _ptr(x), _ptr(y), w, h, S, dist, _stream(stream))
    else:
        rc = load().cudanp_tmv_tma_ex(_ptr(A), lda, _ptr(x), _ptr(y), w, h, S, dist, cols,
                                      rows_sel, stages, _stream(stream))
    _check(rc, "cudanp_tmv_tma")
    return y


def cudanp_mv(A, x, y=None, *, S=S_AUTO, dist=CYCLIC, map=AUTO, n_inner=None, stream=None):
    """y[i] = sum_j A[i, j] * x[j].  A: (h, >= w) fp32, unit column stride,
    lda = A.stride(0)."""
    import torch
    h, w, lda = _mv_args(A, x, y, n_inner, "cudanp_mv")
    if y is None:
        y = torch.empty(h, dtype=torch.float32, device=A.device)
    _check(load().cudanp_mv(_ptr(A), lda, _ptr(x), _ptr(y), h, w, S, dist, map, _stream(stream)),
           "cudanp_mv")
    return y


def cudanp_batched_loop_reduce(x, init=None, out=None, *, op=SUM, S=S_AUTO, dist=CYCLIC, map=AUTO,
                               stream=None):
    """out[n] = init[n] (op) fold_i x[n, i].  x: (N, L) fp32/int32."""
    import torch
    N, L = _batched_args(x, init, out, True, "cudanp_batched_loop_reduce")
    if out is None:
        out = torch.empty(N, dtype=x.dtype, device=x.device)
    _check(load().cudanp_batched_loop_reduce(_ptr(x), _ptr(init), _ptr(out), N, L, _dtype_code(x),
                                             op, S, dist, map, _stream(stream)),
           "cudanp_batched_loop_reduce")
    return out


SHFL, SMEM, REDUX = 0, 1, 2


def cudanp_batched_loop_reduce_backend(x, init=None, out=None, *, op=SUM, S=8, backend=SHFL,
                                       stream=None):
    """Fig 16 ablation: intra-warp cyclic reduce with the team reduction done by
    shfl (0), shared memory (1) or redux.sync (2)."""
    import torch
    N, L = _batched_args(x, init, out, True, "cudanp_batched_loop_reduce_backend")
    if out is None:
        out = torch.empty(N, dtype=x.dtype, device=x.device)
    _check(load().cudanp_batched_loop_reduce_backend(_ptr(x), _ptr(init), _ptr(out), N, L,
                                                     _dtype_code(x), op, S, backend,
                                                     _stream(stream)),
           "cudanp_batched_loop_reduce_backend")
    return out


def cudanp_batched_loop_reduce_tma(x, init=None, out=None, *, op=SUM, S=8, dist=CYCLIC,
                                   stage_bytes=0, stages=0, stream=None):
    """cudanp_batched_loop_reduce with the rows staged by TMA bulk copies (same result)."""
    import torch
    N, L = _batched_args(x, init, out, True, "cudanp_batched_loop_reduce_tma")
    if out is None:
        out = torch.empty(N, dtype=x.dtype, device=x.device)
    _check(load().cudanp_batched_loop_reduce_tma(_ptr(x), _ptr(init), _ptr(out), N, L, _dtype_code(x),
                                                 op, S, dist, stage_bytes, stages, _stream(stream)),
           "cudanp_batched_loop_reduce_tma")
    return out


def cudanp_batched_loop_scan(x, init=None, out=None, *, S=S_AUTO, dist=CYCLIC, map=AUTO, stream=None):
    """Inclusive scan out[n, k] = init[n] + sum_{i<=k} x[n, i]."""
    import torch
    N, L = _batched_args(x, init, out, False, "cudanp_batched_loop_scan")
    if out is None:
        out = torch.empty_like(x)
    _check(load().cudanp_batched_loop_scan(_ptr(x), _ptr(init), _ptr(out), N, L, _dtype_code(x),
                                           S, dist, map, _stream(stream)),
           "cudanp_batched_loop_scan")
    return out


def _ragged_args(x, offsets, init, out, what):
    """N of a CSR batch.  The offsets' values (0 <= off[n] <= off[n+1] <=
    x.numel()) live on the device and are the caller's contract."""
    import torch
    if not isinstance(x, torch.Tensor) or x.dim() != 1 or not x.is_contiguous():
        raise ValueError(f"{what}: values must be a contiguous 1-D tensor")
    _dtype_code(x)
    if not isinstance(offsets, torch.Tensor) or offsets.dim() != 1 or offsets.shape[0] < 1:
        raise ValueError(f"{what}: offsets must be a 1-D tensor of N+1 entries")
    if offsets.dtype != torch.int64:
        raise TypeError("offsets must be int64")
    _buf(offsets, offsets.shape[0], torch.int64, f"{what}: offsets")
    N = offsets.shape[0] - 1
    _buf(init, N, x.dtype, f"{what}: init")
    _buf(out, N, x.dtype, f"{what}: out")
    return N


def cudanp_ragged_loop_reduce(x, offsets, init=None, out=None, *, op=SUM, S=8, dist=CYCLIC,
                              map=AUTO, stream=None):
    """out[n] = init[n] (op) fold_{offsets[n] <= i < offsets[n+1]} x[i].
    x: 1-D fp32/int32; offsets: 1-D int64 of N+1 entries."""
    import torch
    N = _ragged_args(x, offsets, init, out, "cudanp_ragged_loop_reduce")
    if out is None:
        out = torch.empty(N, dtype=x.dtype, device=x.device)
    _check(load().cudanp_ragged_loop_reduce(_ptr(x), _ptr(offsets), _ptr(init), _ptr(out), N,
                                            _dtype_code(x), op, S, dist, map, _stream(stream)),
           "cudanp_ragged_loop_reduce")
    return out


def cudanp_ragged_loop_reduce_adaptive(x, offsets, init=None, out=None, *, op=SUM, threshold=128,
                                       stream=None):
    """Ragged reduce with the team size chosen per segment (S = 1 below
    `threshold` elements, a warp-wide team of 32 above)."""
    import torch
    N = _ragged_args(x, offsets, init, out, "cudanp_ragged_loop_reduce_adaptive")
    if out is None:
        out = torch.empty(N, dtype=x.dtype, device=x.device)
    _check(load().cudanp_ragged_loop_reduce_adaptive(_ptr(x), _ptr(offsets), _ptr(init), _ptr(out), N,
                                                     _dtype_code(x), op, threshold, _stream(stream)),
           "cudanp_ragged_loop_reduce_adaptive")
    return out


def cudanp_ragged_loop_reduce_literal(x, offsets, init=None, out=None, *, op=SUM, stream=None):
    import torch
    N = _ragged_args(x, offsets, init, out, "cudanp_ragged_loop_reduce_literal")
    if out is None:
        out = torch.empty(N, dtype=x.dtype, device=x.device)
    _check(load().cudanp_ragged_loop_reduce_literal(_ptr(x), _ptr(offsets), _ptr(init), _ptr(out),
                                                    N, _dtype_code(x), op, _stream(stream)),
           "cudanp_ragged_loop_reduce_literal")
    return out


def cudanp_le_gicov(x, threshold, gicov=None, *, layout=0, S=8, dist=CYCLIC, map=AUTO,
                    want_stats=True, literal=False, placement=GRAD_REGISTERS, stream=None):
    """LE multi-section item (Figs 5-6): returns (gicov, ave, var, ep).
    x: (N, L) when layout == 0, (L, N) when layout == 1.  gicov entries whose
    test fails are left as given (default: filled with -1)."""
    import torch
    if not isinstance(x, torch.Tensor) or x.dim() != 2 or x.dtype != torch.float32 or not x.is_contiguous():
        raise ValueError("cudanp_le_gicov: x must be a contiguous 2-D float32 tensor")
    N, L = (x.shape if layout == 0 else x.shape[::-1])
    _buf(gicov, N, torch.float32, "cudanp_le_gicov: gicov")
    if gicov is None:
        gicov = torch.full((N,), -1.0, dtype=torch.float32, device=x.device)
    stats = [torch.empty(N, dtype=torch.float32, device=x.device) for _ in range(3)] \
        if want_stats else [None, None, None]
    if literal:
        rc = load().cudanp_le_gicov_literal(_ptr(x), _ptr(gicov), *(_ptr(t) for t in stats), N, L,
                                            threshold, layout, _stream(stream))
    elif placement != GRAD_REGISTERS:
        rc = load().cudanp_le_gicov_placement(_ptr(x), _ptr(gicov), *(_ptr(t) for t in stats), N, L,
                                              threshold, layout, S, dist, map, placement,
                                              _stream(stream))
    else:
        rc = load().cudanp_le_gicov(_ptr(x), _ptr(gicov), *(_ptr(t) for t in stats), N, L,
                                    threshold, layout, S, dist, map, _stream(stream))
    _check(rc, "cudanp_le_gicov")
    return (gicov, *stats)


# ---------------------------------------------------------------- comparison kernels
def cudanp_tmv_variant(impl, A, x, y=None, *, n_outer=None, stream=None):
    import torch
    h, w, lda = _tmv_args(A, x, y, n_outer, "cudanp_tmv_variant")
    if y is None:
        y = torch.empty(w, dtype=torch.float32, device=A.device)
    _check(load().cudanp_tmv_variant(impl, _ptr(A), lda, _ptr(x), _ptr(y), w, h, _stream(stream)),
           "cudanp_tmv_variant")
    return y


def cudanp_mv_variant(impl, A, x, y=None, *, n_inner=None, stream=None):
    import torch
    h, w, lda = _mv_args(A, x, y, n_inner, "cudanp_mv_variant")
    if y is None:
        y = torch.empty(h, dtype=torch.float32, device=A.device)
    _check(load().cudanp_mv_variant(impl, _ptr(A), lda, _ptr(x), _ptr(y), h, w, _stream(stream)),
           "cudanp_mv_variant")
    return y


def cudanp_batched_loop_reduce_variant(impl, x, init=None, out=None, *, op=SUM, stream=None):
    import torch
    N, L = _batched_args(x, init, out, True, "cudanp_batched_loop_reduce_variant")
    if out is None:
        out = torch.empty(N, dtype=x.dtype, device=x.device)
    _check(load().cudanp_batched_loop_reduce_variant(impl, _ptr(x), _ptr(init), _ptr(out), N, L,
                                                     _dtype_code(x), op, _stream(stream)),
           "cudanp_batched_loop_reduce_variant")
    return out


def cudanp_batched_loop_scan_variant(impl, x, init=None, out=None, *, stream=None):
    N, L = _batched_args(x, init, out, False, "cudanp_batched_loop_scan_variant")
    if out is None:
        import torch
        out = torch.empty_like(x)
    _check(load().cudanp_batched_loop_scan_variant(impl, _ptr(x), _ptr(init), _ptr(out), N, L,
                                                   _dtype_code(x), _stream(stream)),
           "cudanp_batched_loop_scan_variant")
    return out


def cudanp_dp_set_pending_launch_limit(n: int) -> None:
    _check(load().cudanp_dp_set_pending_launch_limit(n), "cudanp_dp_set_pending_launch_limit")


def cudanp_dp_error_count(reset: bool = True) -> int:
    c = _i64(0)
    _check(load().cudanp_dp_error_count(int(reset), ctypes.byref(c)), "cudanp_dp_error_count")
    return c.value


def cudanp_dp_memcopy(x, out=None, *, m=1, variant=2, stream=None):
    """Fig 1 memcopy: variant 0 plain, 1 plain built with -rdc, 2 DP
    with m parent threads each launching a child of numel/m threads."""
    import torch
    if out is None:
        out = torch.empty_like(x)
    _check(load().cudanp_dp_memcopy(_ptr(x), _ptr(out), x.numel(), m, variant, _stream(stream)),
           "cudanp_dp_memcopy")
    return out


OP_KINDS = {"tmv": 0, "mv": 1, "reduce": 2, "scan": 3}


def cudanp_autotune_candidates(op_kind: str) -> list[tuple[int, int, int]]:
    L = load()
    k = OP_KINDS[op_kind]
    out = []
    for i in range(L.cudanp_autotune_count(k)):
        S, d, m = _int(), _int(), _int()
        _check(L.cudanp_autotune_candidate(k, i, ctypes.byref(S), ctypes.byref(d), ctypes.byref(m)),
               "cudanp_autotune_candidate")
        out.append((S.value, d.value, m.value))
    return out


def cudanp_autotune(op_kind: str, a, b, out, *, lda=0, n_outer, n_inner, dtype=F32, op=SUM,
                    reps=5, stream=None):
    """Time every (S, dist, map) candidate on these operands.
    Returns (best (S, dist, map), {candidate: ms})."""
    k = OP_KINDS[op_kind]
    cands = cudanp_autotune_candidates(op_kind)
    table = (ctypes.c_float * len(cands))()
    best = _int()
    _check(load().cudanp_autotune(k, _ptr(a), _ptr(b), _ptr(out), lda, n_outer, n_inner, dtype, op,
                                  reps, table, ctypes.byref(best), _stream(stream)), "cudanp_autotune")
    return cands[best.value], {c: table[i] for i, c in enumerate(cands)}


# ---------------------------------------------------------------- support
def cudanp_launch_info(op_kind: str, n_outer: int, n_inner: int, *, dtype=F32, op=SUM, S=8,
                       dist=CYCLIC, map=AUTO, vec4=True) -> dict:
    kinds = {"tmv": 0, "mv": 1, "reduce": 2, "scan": 3, "tmv_tma": 4, "reduce_tma": 5}
    b, g, r, s, m, su, du = _int(), _i64(), _int(), _int(), _int(), _int(), _int()
    _check(load().cudanp_launch_info(kinds[op_kind], n_outer, n_inner, dtype, op, S, dist, map,
                                     int(vec4), ctypes.byref(b), ctypes.byref(g), ctypes.byref(r),
                                     ctypes.byref(s), ctypes.byref(m), ctypes.byref(su),
                                     ctypes.byref(du)), "cudanp_launch_info")
    return {"block_threads": b.value, "grid_ctas": g.value, "regs_per_thread": r.value,
            "smem_bytes": s.value, "map": MAP_NAMES.get(m.value, "?"), "S": su.value,
            "dist": "cyclic" if du.value == CYCLIC else "block"}


MAP_NAMES = {1: "intra_warp", 2: "inter_warp", 3: "inter_warp_tma", 4: "intra_warp_tma"}


def cudanp_choose_version(op_kind: str, n_outer: int, n_inner: int, *, vec4=True,
                          map=AUTO) -> tuple[int, int, int]:
    """(S, dist, map) the library runs for S = S_AUTO on this shape (host-only rule)."""
    S, d, m = _int(), _int(), _int()
    _check(load().cudanp_choose_version(OP_KINDS[op_kind], n_outer, n_inner, int(vec4), map,
                                        ctypes.byref(S), ctypes.byref(d), ctypes.byref(m)),
           "cudanp_choose_version")
    return S.value, d.value, m.value


def cudanp_ipc_get_handle(t) -> tuple[bytes, int]:
    """(64-byte IPC handle of t's allocation, byte offset of t in it)."""
    buf = ctypes.create_string_buffer(64)
    off = _i64()
    _check(load().cudanp_ipc_get_handle(_ptr(t), buf, ctypes.byref(off)), "cudanp_ipc_get_handle")
    return buf.raw, off.value


def cudanp_ipc_open(handle: bytes, offset: int) -> int:
    p = _vp()
    _check(load().cudanp_ipc_open(handle, offset, ctypes.byref(p)), "cudanp_ipc_open")
    return p.value


def cudanp_ipc_close(ptr: int, offset: int) -> None:
    _check(load().cudanp_ipc_close(ptr, offset), "cudanp_ipc_close")


# ---------------------------------------------------------------- native multi-GPU group
def cudanp_group_unique_id() -> bytes:
    """128-byte NCCL unique id (rank 0 creates it; every rank needs the same bytes)."""
    buf = ctypes.create_string_buffer(128)
    _check(load().cudanp_group_unique_id(buf), "cudanp_group_unique_id")
    return buf.raw


def cudanp_group_create(uid: bytes, nranks: int, rank: int) -> int:
    """This process's rank of the group, on the current CUDA device (collective)."""
    h = _vp()
    _check(load().cudanp_group_create(ctypes.create_string_buffer(uid, 128), nranks, rank,
                                      ctypes.byref(h)), "cudanp_group_create")
    return h.value


def cudanp_group_destroy(group: int) -> None:
    _check(load().cudanp_group_destroy(group), "cudanp_group_destroy")


def cudanp_group_gather(group: int, local, root_buf, n_total: int, stream=None) -> None:
    _check(load().cudanp_group_gather(group, _ptr(local), _ptr(root_buf), n_total, _dtype_code(local),
                                      _stream(stream)), "cudanp_group_gather")


def cudanp_sharded_tmv(group: int, A_shard, x, y_shard, y_root, n_outer_total: int, *, S=32,
                       dist=CYCLIC, map=AUTO, stream=None) -> None:
    import torch
    h, w, lda = _mat(A_shard, "cudanp_sharded_tmv")
    _buf(x, h, torch.float32, "cudanp_sharded_tmv: x")
    _buf(y_shard, w, torch.float32, "cudanp_sharded_tmv: y_shard")
    _buf(y_root, n_outer_total if y_root is not None and not isinstance(y_root, int) else 0,
         torch.float32, "cudanp_sharded_tmv: y_root")
    _check(load().cudanp_sharded_tmv(group, _ptr(A_shard), lda, _ptr(x), _ptr(y_shard), _ptr(y_root),
                                     n_outer_total, h, S, dist, map, _stream(stream)),
           "cudanp_sharded_tmv")


def cudanp_sharded_batched_loop_reduce(group: int, in_shard, init_shard, out_shard, out_root,
                                       n_outer_total: int, *, op=SUM, S=8, dist=CYCLIC, map=AUTO,
                                       stream=None) -> None:
    N, L = _items(in_shard, "cudanp_sharded_batched_loop_reduce")
    _buf(init_shard, N, in_shard.dtype, "cudanp_sharded_batched_loop_reduce: init")
    _buf(out_shard, N, in_shard.dtype, "cudanp_sharded_batched_loop_reduce: out_shard")
    _check(load().cudanp_sharded_batched_loop_reduce(group, _ptr(in_shard), _ptr(init_shard),
                                                     _ptr(out_shard), _ptr(out_root), n_outer_total, L,
                                                     _dtype_code(in_shard), op, S, dist, map,
                                                     _stream(stream)),
           "cudanp_sharded_batched_loop_reduce")


def cudanp_shard_range(n_outer: int, nranks: int, rank: int) -> tuple[int, int]:
    b, e = _i64(), _i64()
    _check(load().cudanp_shard_range(n_outer, nranks, rank, ctypes.byref(b), ctypes.byref(e)),
           "cudanp_shard_range")
    return b.value, e.value


def cudanp_generate(out, kind: str, *, stream_id=1, row0=0, col0=0, w_global=None, B=1 << 20,
                    seed=SEED, stream=None):
    """Fill a 1-D or 2-D CUDA tensor with the counter-based generator (test/bench support)."""
    if out.dim() == 1:
        rows, cols, ld = 1, out.shape[0], out.shape[0]
    else:
        rows, cols = out.shape
        ld = out.stride(0)
    wg = cols if w_global is None else w_global
    if out.dim() == 1 and w_global is None:
        wg = 0  # 1-D: idx = col0 + c
    _check(load().cudanp_generate(_ptr(out), rows, cols, ld, row0, col0, wg, stream_id, KIND[kind],
                                  B, seed, _stream(stream)), "cudanp_generate")
    return out


def cudanp_debug_owner_map(n_inner: int, S: int, dist: int, V: int = 1) -> np.ndarray:
    out = np.empty(max(n_inner, 0), np.int32)
    _check(load().cudanp_debug_owner_map(n_inner, S, dist, V, out.ctypes.data_as(_P32)),
           "cudanp_debug_owner_map")
    return out


def cudanp_debug_team_ids(S: int, map_: int):
    n_max = 1024
    m = np.empty(n_max, np.int32)
    s = np.empty(n_max, np.int32)
    n = _int()
    _check(load().cudanp_debug_team_ids(S, map_, m.ctypes.data_as(_P32), s.ctypes.data_as(_P32),
                                        ctypes.byref(n)), "cudanp_debug_team_ids")
    return m[: n.value].copy(), s[: n.value].copy()


def cudanp_debug_broadcast(S: int, map_: int) -> np.ndarray:
    out = np.empty(1024, np.int32)
    n = _int()
    _check(load().cudanp_debug_broadcast(S, map_, out.ctypes.data_as(_P32), ctypes.byref(n)),
           "cudanp_debug_broadcast")
    return out[: n.value].copy()


def cudanp_status_string(status: int) -> str:
    return load().cudanp_status_string(status).decode()


def cudanp_version() -> int:
    return load().cudanp_version()
