"""Seeded synthetic inputs -- no method arithmetic here.

A counter-based generator: element ``idx`` of stream ``s`` is
``h = splitmix64(splitmix64(SEED ^ (s << 56)) ^ idx)`` mapped to a value.
It serves both sides of the parity tests for small inputs (numpy arrays that
the tests pass to the oracle and upload to the GPU).  The oracle
(``oracle/cudanp_oracle.c``) and the CUDA library (``cudanp_generate``) each
carry their own independent implementation for full-size inputs; the tests
check all three agree bit for bit (pin P8).

Streams: 1 = A or ``in``, 2 = x, 3 = init.  Index conventions: ``A[i][j]`` has
idx ``i*w + j`` with the global width ``w``; ``in[n][i]`` has idx ``n*L + i``.
"""
from __future__ import annotations

import numpy as np

SEED = 20140215
STREAM_A, STREAM_X, STREAM_INIT = 1, 2, 3

_M1 = np.uint64(0x9E3779B97F4A7C15)
_M2 = np.uint64(0xBF58476D1CE4E5B9)
_M3 = np.uint64(0x94D049BB133111EB)


def splitmix64(z):
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = z + _M1
        z = (z ^ (z >> np.uint64(30))) * _M2
        z = (z ^ (z >> np.uint64(27))) * _M3
    return z ^ (z >> np.uint64(31))


def hash64(stream: int, idx, seed: int = SEED):
    key = splitmix64(np.uint64(seed) ^ (np.uint64(stream) << np.uint64(56)))
    return splitmix64(key ^ np.asarray(idx, dtype=np.uint64))


def values(h, kind: str, B: int = 1 << 20, idx=None):
    """Map 64-bit hashes to values of the named distribution."""
    h = np.asarray(h, dtype=np.uint64)
    if kind == "f32_unit":          # in (0,1), exact, never 0
        k = (h >> np.uint64(40)) | np.uint64(1)
        return (k.astype(np.float64) * 2.0 ** -24).astype(np.float32)
    if kind == "f32_signed":        # in (-1,1), exact
        k = ((h >> np.uint64(40)) | np.uint64(1)).astype(np.int64)
        return ((k * 2 - (1 << 24)).astype(np.float64) * 2.0 ** -24).astype(np.float32)
    if kind == "f32_int4":          # {0,1,2,3}: keeps fp32 sums exact (pin P3)
        return (h >> np.uint64(62)).astype(np.float32)
    if kind == "i32_small":         # [-B, B)
        hi = (h >> np.uint64(32)).astype(np.int64)
        return ((hi & (2 * B - 1)) - B).astype(np.int32)
    if kind == "i32_full":
        return (h >> np.uint64(32)).astype(np.uint32).view(np.int32)
    if kind == "ones_f32":
        return np.ones(h.shape, np.float32)
    if kind == "ones_i32":
        return np.ones(h.shape, np.int32)
    raise ValueError(kind)


def gen(stream: int, kind: str, idx0: int, n: int, B: int = 1 << 20, seed: int = SEED):
    idx = np.arange(idx0, idx0 + n, dtype=np.uint64)
    return values(hash64(stream, idx, seed), kind, B)


def matrix(h: int, w: int, kind: str = "f32_unit", seed: int = SEED, row0: int = 0,
           col0: int = 0, w_global: int | None = None):
    """A[i][j] for rows [row0,row0+h) and columns [col0,col0+w) of a matrix of
    global width ``w_global`` (default w): idx = i*w_global + j."""
    wg = w if w_global is None else w_global
    i = np.arange(row0, row0 + h, dtype=np.uint64)[:, None]
    j = np.arange(col0, col0 + w, dtype=np.uint64)[None, :]
    return values(hash64(STREAM_A, i * np.uint64(wg) + j, seed), kind)


def vector(n: int, kind: str = "f32_unit", seed: int = SEED, stream: int = STREAM_X):
    return gen(stream, kind, 0, n, seed=seed)


def items(N: int, L: int, kind: str, B: int = 1 << 20, seed: int = SEED, n0: int = 0):
    """in[n][i] for items [n0, n0+N): idx = n*L + i."""
    return gen(STREAM_A, kind, n0 * L, N * L, B, seed).reshape(N, L)


def init(N: int, kind: str, B: int = 1 << 20, seed: int = SEED, n0: int = 0):
    return gen(STREAM_INIT, kind, n0, N, B, seed)


STREAM_LEN = 4


def lengths(N: int, mean: int, dist: str = "uniform", seed: int = SEED, cap: int | None = None):
    """Per-item loop trip counts (structure of a ragged workload):
    'uniform' -> integers in [0, 2*mean]; 'exp' -> floor(-mean*ln(u)), an
    exponential (skewed) mix capped at `cap` (default 16*mean)."""
    h = hash64(STREAM_LEN, np.arange(N, dtype=np.uint64), seed)
    if dist == "uniform":
        return ((h >> np.uint64(32)) % np.uint64(2 * mean + 1)).astype(np.int64)
    if dist == "exp":
        u = ((h >> np.uint64(11)).astype(np.float64) + 1.0) * 2.0 ** -53
        L = np.floor(-mean * np.log(u)).astype(np.int64)
        return np.minimum(L, cap if cap is not None else 16 * mean)
    raise ValueError(dist)


def offsets_from_lengths(lens):
    off = np.zeros(len(lens) + 1, np.int64)
    np.cumsum(lens, out=off[1:])
    return off
