"""CPU oracle for the CUDA-NP hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The
product path (``paper_conf_ppopp_yangz14_b200``) never imports it; it shares no
code with it.  The arithmetic lives in ``cudanp_oracle.c`` (plain C, fp64
accumulation, one rounding; int32 modulo 2^32); this module only compiles it
with gcc and marshals numpy arrays through ctypes.

Every function is the plain definition of what a CUDA-NP master thread ends up
computing (NP only redistributes a parallel loop's
iterations): TMV per Fig 2, MV, reduction and scan
(P:209), the iteration mapping and the thread remap
(P:189-191).  See DESIGN.md "Readings" for every choice the paper leaves open.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "cudanp_oracle.c")
_SO = os.path.join(_HERE, "libcudanp_oracle.so")
_lock = threading.Lock()
_lib = None

F32, I32 = 0, 1
SUM, MAX = 0, 1
CYCLIC, BLOCK = 0, 1
INTRA_WARP, INTER_WARP = 1, 2
KIND = {"f32_unit": 0, "f32_signed": 1, "f32_int4": 2, "i32_small": 3, "i32_full": 4,
        "ones": 5, "iota": 6}
SEED = 20140215

_i64 = ctypes.c_int64
_u64 = ctypes.c_uint64
_int = ctypes.c_int
_vp = ctypes.c_void_p


def build(force: bool = False) -> str:
    """Compile cudanp_oracle.c -> libcudanp_oracle.so (gcc, -O2, no fast-math)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-ffp-contract=off", "-fno-fast-math",
                               "-fPIC", "-shared", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _SO)
    return _SO


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_SO)
            sig = {
                "orc_splitmix64": (_u64, [_u64]),
                "orc_hash": (_u64, [_u64, _u64, _u64]),
                "orc_gen_f32": (None, [_u64, _u64, _int, _u64, _i64, _vp]),
                "orc_gen_i32": (None, [_u64, _u64, _int, _i64, _u64, _i64, _vp]),
                "orc_tmv": (None, [_vp, _i64, _vp, _vp, _i64, _i64]),
                "orc_tmv_serial_f32": (None, [_vp, _i64, _vp, _vp, _i64, _i64]),
                "orc_mv": (None, [_vp, _i64, _vp, _vp, _i64, _i64]),
                "orc_reduce_f32": (None, [_vp, _vp, _vp, _i64, _i64, _int]),
                "orc_reduce_i32": (None, [_vp, _vp, _vp, _i64, _i64, _int]),
                "orc_scan_f32": (None, [_vp, _vp, _vp, _i64, _i64]),
                "orc_scan_i32": (None, [_vp, _vp, _vp, _i64, _i64]),
                "orc_ragged_reduce_f32": (None, [_vp, _vp, _vp, _vp, _i64, _int]),
                "orc_ragged_reduce_i32": (None, [_vp, _vp, _vp, _vp, _i64, _int]),
                "orc_le_gicov": (None, [_vp, _vp, _vp, _vp, _vp, _i64, _i64, ctypes.c_float, _int]),
                "orc_tmv_gen": (None, [_u64, _int, _int, _i64, _i64, _vp, _i64, _vp]),
                "orc_mv_gen": (None, [_u64, _int, _int, _i64, _i64, _vp, _i64, _vp]),
                "orc_reduce_gen": (None, [_u64, _int, _int, _i64, _int, _i64, _int, _vp, _i64, _vp]),
                "orc_scan_gen": (None, [_u64, _int, _int, _i64, _int, _i64, _vp, _i64, _vp]),
                "orc_owner_map": (_int, [_i64, _int, _int, _int, _vp]),
                "orc_team_ids": (_int, [_int, _int, _i64, _vp, _vp]),
            }
            for name, (res, args) in sig.items():
                f = getattr(L, name)
                f.restype = res
                f.argtypes = args
            _lib = L
    return _lib


def _p(a: np.ndarray | None):
    if a is None:
        return None
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data


# ---------------------------------------------------------------- generator
def hash64(stream: int, idx: int, seed: int = SEED) -> int:
    return lib().orc_hash(seed, stream, idx)


def gen_f32(stream: int, kind: str, idx0: int, n: int, seed: int = SEED) -> np.ndarray:
    out = np.empty(n, np.float32)
    lib().orc_gen_f32(seed, stream, KIND[kind], idx0, n, _p(out))
    return out


def gen_i32(stream: int, kind: str, idx0: int, n: int, B: int = 1 << 20, seed: int = SEED) -> np.ndarray:
    out = np.empty(n, np.int32)
    lib().orc_gen_i32(seed, stream, KIND[kind], B, idx0, n, _p(out))
    return out


# ---------------------------------------------------------------- definitions
def tmv(A: np.ndarray, x: np.ndarray, w: int | None = None) -> np.ndarray:
    """y[j] = sum_i A[i, j] * x[i] (Fig 2); A is (h, lda) row-major."""
    A = np.ascontiguousarray(A, np.float32)
    x = np.ascontiguousarray(x, np.float32)
    h, lda = A.shape
    w = lda if w is None else w
    y = np.empty(w, np.float32)
    lib().orc_tmv(_p(A), lda, _p(x), _p(y), w, h)
    return y


def tmv_serial_f32(A: np.ndarray, x: np.ndarray) -> np.ndarray:
    A = np.ascontiguousarray(A, np.float32)
    x = np.ascontiguousarray(x, np.float32)
    h, w = A.shape
    y = np.empty(w, np.float32)
    lib().orc_tmv_serial_f32(_p(A), w, _p(x), _p(y), w, h)
    return y


def tmv_parallel(A: np.ndarray, x: np.ndarray, threads: int) -> np.ndarray:
    """orc_tmv over `threads` contiguous column ranges in parallel (outer items
    are independent; the arithmetic per output is unchanged).  For the
    all-core CPU baseline only."""
    from concurrent.futures import ThreadPoolExecutor
    A = np.ascontiguousarray(A, np.float32)
    x = np.ascontiguousarray(x, np.float32)
    h, lda = A.shape
    y = np.empty(lda, np.float32)
    bounds = [(g * lda // threads, (g + 1) * lda // threads) for g in range(threads)]
    L = lib()

    def run(b):
        j0, j1 = b
        if j1 > j0:
            L.orc_tmv(A.ctypes.data + 4 * j0, lda, _p(x), y.ctypes.data + 4 * j0, j1 - j0, h)
    with ThreadPoolExecutor(threads) as ex:
        list(ex.map(run, bounds))
    return y


def mv_parallel(A: np.ndarray, x: np.ndarray, threads: int) -> np.ndarray:
    """orc_mv over `threads` contiguous row ranges in parallel."""
    from concurrent.futures import ThreadPoolExecutor
    A = np.ascontiguousarray(A, np.float32)
    x = np.ascontiguousarray(x, np.float32)
    h, lda = A.shape
    y = np.empty(h, np.float32)
    bounds = [(g * h // threads, (g + 1) * h // threads) for g in range(threads)]
    L = lib()

    def run(b):
        i0, i1 = b
        if i1 > i0:
            L.orc_mv(A.ctypes.data + 4 * i0 * lda, lda, _p(x), y.ctypes.data + 4 * i0, i1 - i0, lda)
    with ThreadPoolExecutor(threads) as ex:
        list(ex.map(run, bounds))
    return y


def mv(A: np.ndarray, x: np.ndarray, w: int | None = None) -> np.ndarray:
    """y[i] = sum_j A[i, j] * x[j]; A is (h, lda) row-major."""
    A = np.ascontiguousarray(A, np.float32)
    x = np.ascontiguousarray(x, np.float32)
    h, lda = A.shape
    w = lda if w is None else w
    y = np.empty(h, np.float32)
    lib().orc_mv(_p(A), lda, _p(x), _p(y), h, w)
    return y


def reduce(x: np.ndarray, op: int = SUM, init: np.ndarray | None = None) -> np.ndarray:
    """out[n] = init[n] (+|max) fold_i x[n, i]. x is (N, L)."""
    x = np.ascontiguousarray(x)
    N, L = x.shape
    out = np.empty(N, x.dtype)
    if init is not None:
        init = np.ascontiguousarray(init, x.dtype)
    if x.dtype == np.float32:
        lib().orc_reduce_f32(_p(x), _p(init), _p(out), N, L, op)
    elif x.dtype == np.int32:
        lib().orc_reduce_i32(_p(x), _p(init), _p(out), N, L, op)
    else:
        raise TypeError(x.dtype)
    return out


def scan(x: np.ndarray, init: np.ndarray | None = None) -> np.ndarray:
    """Inclusive scan out[n, k] = init[n] + sum_{i<=k} x[n, i] (reading R1)."""
    x = np.ascontiguousarray(x)
    N, L = x.shape
    out = np.empty_like(x)
    if init is not None:
        init = np.ascontiguousarray(init, x.dtype)
    if x.dtype == np.float32:
        lib().orc_scan_f32(_p(x), _p(init), _p(out), N, L)
    elif x.dtype == np.int32:
        lib().orc_scan_i32(_p(x), _p(init), _p(out), N, L)
    else:
        raise TypeError(x.dtype)
    return out


def ragged_reduce(x: np.ndarray, offsets: np.ndarray, op: int = SUM,
                  init: np.ndarray | None = None) -> np.ndarray:
    """out[n] = init[n] (op) fold_{offsets[n] <= i < offsets[n+1]} x[i]."""
    x = np.ascontiguousarray(x)
    offsets = np.ascontiguousarray(offsets, np.int64)
    N = len(offsets) - 1
    out = np.empty(N, x.dtype)
    if init is not None:
        init = np.ascontiguousarray(init, x.dtype)
    f = {np.dtype(np.float32): lib().orc_ragged_reduce_f32,
         np.dtype(np.int32): lib().orc_ragged_reduce_i32}[x.dtype]
    f(_p(x), _p(offsets), _p(init), _p(out), N, op)
    return out


def le_gicov(x: np.ndarray, thr: float, layout: int = 0, gicov_fill: float = -1.0):
    """Fig 5: per item, ave, var, ep and the conditional gicov.
    x is (N, L) for layout 0 (item-major) or (L, N) for layout 1 (point-major).
    Items whose test fails keep gicov_fill."""
    x = np.ascontiguousarray(x, np.float32)
    N, L = (x.shape if layout == 0 else x.shape[::-1])
    g = np.full(N, gicov_fill, np.float32)
    a, v, e = (np.empty(N, np.float32) for _ in range(3))
    lib().orc_le_gicov(_p(x), _p(g), _p(a), _p(v), _p(e), N, L, thr, layout)
    return g, a, v, e


def tmv_gen(h: int, w: int, cols, kindA="f32_unit", kindx="f32_unit", seed: int = SEED) -> np.ndarray:
    cols = np.ascontiguousarray(cols, np.int64)
    y = np.empty(len(cols), np.float32)
    lib().orc_tmv_gen(seed, KIND[kindA], KIND[kindx], h, w, _p(cols), len(cols), _p(y))
    return y


def mv_gen(h: int, w: int, rows, kindA="f32_unit", kindx="f32_unit", seed: int = SEED) -> np.ndarray:
    rows = np.ascontiguousarray(rows, np.int64)
    y = np.empty(len(rows), np.float32)
    lib().orc_mv_gen(seed, KIND[kindA], KIND[kindx], h, w, _p(rows), len(rows), _p(y))
    return y


def reduce_gen(L: int, items, dtype: int, kind: str, op: int = SUM, B: int = 1 << 20,
               init_kind: str | None = None, seed: int = SEED) -> np.ndarray:
    items = np.ascontiguousarray(items, np.int64)
    out = np.empty(len(items), np.float32 if dtype == F32 else np.int32)
    ik = -1 if init_kind is None else KIND[init_kind]
    lib().orc_reduce_gen(seed, dtype, KIND[kind], B, ik, L, op, _p(items), len(items), _p(out))
    return out


def scan_gen(L: int, items, dtype: int, kind: str, B: int = 1 << 20,
             init_kind: str | None = None, seed: int = SEED) -> np.ndarray:
    items = np.ascontiguousarray(items, np.int64)
    out = np.empty((len(items), L), np.float32 if dtype == F32 else np.int32)
    ik = -1 if init_kind is None else KIND[init_kind]
    lib().orc_scan_gen(seed, dtype, KIND[kind], B, ik, L, _p(items), len(items), _p(out))
    return out


# ---------------------------------------------------------------- structure
def owner_map(L: int, S: int, dist: int, V: int = 1) -> np.ndarray:
    out = np.empty(max(L, 0), np.int32)
    rc = lib().orc_owner_map(L, S, dist, V, _p(out))
    if rc != 0:
        raise ValueError("bad owner_map arguments")
    return out


def team_ids(S: int, map_: int, nthreads: int):
    m = np.empty(nthreads, np.int32)
    s = np.empty(nthreads, np.int32)
    rc = lib().orc_team_ids(S, map_, nthreads, _p(m), _p(s))
    if rc != 0:
        raise ValueError("bad team_ids arguments")
    return m, s
