"""Pins for the CPU oracle (CPU only).  Each test checks the oracle against
something other than itself: the paper's worked examples, closed forms,
exact rational arithmetic (brute force), or a second formulation.

See DESIGN.md section "Oracle pins" for which plausible mistake each catches.
"""
import json
import os
from fractions import Fraction

import numpy as np
import pytest

import synth

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "paper_examples.json")))


# ------------------------------------------------------------------ generator
def test_splitmix64_public_vectors(orc):
    g = GOLD["splitmix64_public"]
    for z, want in zip(g["mix_of"], g["out"]):
        assert orc.lib().orc_splitmix64(int(z, 16)) == int(want, 16)
        assert int(synth.splitmix64(np.uint64(int(z, 16)))) == int(want, 16)


@pytest.mark.parametrize("stream", [1, 2, 3])
def test_generator_oracle_vs_synth(orc, stream):
    # two independent implementations of SURVEY C-4 agree bit for bit (pin P8)
    idx0 = (1 << 32) - 100  # straddles 2^32: 64-bit index handling
    for kind in ["f32_unit", "f32_signed", "f32_int4"]:
        a = orc.gen_f32(stream, kind, idx0, 1000)
        b = synth.gen(stream, kind, idx0, 1000)
        assert a.tobytes() == b.tobytes(), kind
    for kind, B in [("i32_small", 1 << 20), ("i32_small", 1 << 15), ("i32_full", 0)]:
        a = orc.gen_i32(stream, kind, idx0, 1000, B)
        b = synth.gen(stream, kind, idx0, 1000, B)
        assert a.tobytes() == b.tobytes(), kind


def test_generator_kat(orc):
    # SURVEY C-5 known-answer values for the generator
    assert orc.hash64(1, 0) == 0xce8ab6f93c07a171
    assert orc.hash64(1, 1) == 0x8b6fedbca0b19a3b
    assert orc.hash64(1, 1 << 32) == 0x9e15098546875521
    assert orc.hash64(2, 0) == 0x6d62f67cd2d30f24
    assert float(orc.gen_f32(1, "f32_unit", 0, 1)[0]) == 0.8068041205406189
    assert float(orc.gen_f32(1, "f32_signed", 0, 1)[0]) == 0.6136082410812378
    assert float(orc.gen_f32(1, "f32_int4", 0, 1)[0]) == 3.0
    assert int(orc.gen_i32(1, "i32_small", 0, 1, 1 << 20)[0]) == -346375
    assert int(orc.gen_i32(1, "i32_full", 0, 1)[0]) == -829769991


def test_generator_ranges():
    u = synth.gen(1, "f32_unit", 0, 1 << 16)
    assert (u > 0).all() and (u < 1).all()
    s = synth.gen(1, "f32_signed", 0, 1 << 16)
    assert (s > -1).all() and (s < 1).all() and (s != 0).all()
    assert set(np.unique(synth.gen(1, "f32_int4", 0, 4096))) == {0.0, 1.0, 2.0, 3.0}
    i = synth.gen(1, "i32_small", 0, 1 << 16, B=1 << 15)
    assert i.min() >= -(1 << 15) and i.max() < (1 << 15)


# ------------------------------------------------------------------ TMV / MV
def test_tmv_hand(orc):
    g = GOLD["tmv_hand"]
    y = orc.tmv(np.array(g["A"], np.float32), np.array(g["x"], np.float32))
    assert y.tolist() == g["y"]


def test_tmv_mv_kat(orc):
    # SURVEY C-5: h=4, w=3, f32_int4 (exact)
    A = synth.matrix(4, 3, "f32_int4")
    x4 = synth.vector(4, "f32_int4")
    x3 = synth.vector(3, "f32_int4")
    assert orc.tmv(A, x4).tolist() == [11, 6, 8]
    assert orc.mv(A, x3).tolist() == [9, 7, 1, 6]


def test_tmv_bruteforce_rational(orc):
    # exact rational sum, rounded once, on tiny non-square random inputs:
    # catches a transposed operand, a dropped term, a wrong index.
    for (h, w) in [(1, 1), (3, 5), (7, 2), (8, 8)]:
        A = synth.matrix(h, w, "f32_signed", seed=h * 100 + w)
        x = synth.vector(h, "f32_unit", seed=h * 100 + w)
        y = orc.tmv(A, x)
        for j in range(w):
            s = sum(Fraction(float(A[i, j])) * Fraction(float(x[i])) for i in range(h))
            assert y[j] == np.float32(float(s)), (h, w, j)


def test_mv_bruteforce_rational(orc):
    for (h, w) in [(1, 1), (5, 3), (2, 7), (8, 8)]:
        A = synth.matrix(h, w, "f32_signed", seed=h * 10 + w)
        x = synth.vector(w, "f32_unit", seed=h * 10 + w)
        y = orc.mv(A, x)
        for i in range(h):
            s = sum(Fraction(float(A[i, j])) * Fraction(float(x[j])) for j in range(w))
            assert y[i] == np.float32(float(s)), (h, w, i)


def test_tmv_closed_forms(orc):
    h, w = 37, 19
    x = synth.vector(h, "f32_unit")
    # A = all-ones: y_j = sum(x) (north star's example)
    y = orc.tmv(np.ones((h, w), np.float32), x)
    want = np.float32(float(sum(Fraction(float(v)) for v in x)))
    assert (y == want).all()
    # x = e_k: y = row k of A, bit-exact
    A = synth.matrix(h, w, "f32_signed")
    for k in [0, 5, h - 1]:
        e = np.zeros(h, np.float32)
        e[k] = 1
        assert orc.tmv(A, e).tobytes() == A[k].tobytes()
    # A = I: y = x
    xs = synth.vector(w, "f32_signed")
    assert orc.tmv(np.eye(w, dtype=np.float32), xs).tobytes() == xs.tobytes()
    # h = 0: empty sum
    assert (orc.tmv(np.zeros((0, 4), np.float32), np.zeros(0, np.float32)) == 0).all()


def test_mv_closed_forms(orc):
    h, w = 13, 41
    A = synth.matrix(h, w, "f32_signed")
    for k in [0, 7, w - 1]:
        e = np.zeros(w, np.float32)
        e[k] = 1
        assert orc.mv(A, e).tobytes() == np.ascontiguousarray(A[:, k]).tobytes()
    x = synth.vector(w, "f32_unit")
    y = orc.mv(np.ones((h, w), np.float32), x)
    assert (y == np.float32(float(sum(Fraction(float(v)) for v in x)))).all()


def test_tmv_equals_mv_of_transpose(orc):
    # second formulation: TMV(A) == MV(A^T), same summation order -> bit-exact
    A = synth.matrix(29, 23, "f32_signed")
    x = synth.vector(29, "f32_unit")
    assert orc.tmv(A, x).tobytes() == orc.mv(np.ascontiguousarray(A.T), x).tobytes()


def test_tmv_lda_padding_ignored(orc):
    h, w, lda = 9, 6, 8
    A = np.full((h, lda), np.nan, np.float32)
    A[:, :w] = synth.matrix(h, w, "f32_signed")
    x = synth.vector(h, "f32_unit")
    assert orc.tmv(A, x, w).tobytes() == orc.tmv(np.ascontiguousarray(A[:, :w]), x).tobytes()
    Am = np.full((w, lda), np.nan, np.float32)
    Am[:, :w] = synth.matrix(w, w, "f32_signed")
    xm = synth.vector(w, "f32_unit")
    assert orc.mv(Am, xm, w).tobytes() == orc.mv(np.ascontiguousarray(Am[:, :w]), xm).tobytes()


def test_tmv_exact_data_int(orc):
    # pin P3: integer-valued data -> exact integer result
    A = synth.matrix(300, 50, "f32_int4")
    x = synth.vector(300, "f32_int4")
    want = (A.astype(np.int64) * x.astype(np.int64)[:, None]).sum(0)
    assert (orc.tmv(A, x).astype(np.int64) == want).all()


def test_tmv_serial_is_fig2_rounding(orc):
    # the literal fp32 Fig 2 loop differs from the fp64 oracle only by rounding
    A = synth.matrix(4096, 8, "f32_unit")
    x = synth.vector(4096, "f32_unit")
    r, s = orc.tmv(A, x), orc.tmv_serial_f32(A, x)
    assert np.max(np.abs(r - s) / r) < 1e-5
    assert (orc.tmv(A[:1], x[:1]) == orc.tmv_serial_f32(A[:1], x[:1])).all()


def test_tmv_gen_matches_arrays(orc):
    h, w = 64, 40
    cols = [0, 1, 17, 39]
    A = synth.matrix(h, w, "f32_unit")
    x = synth.vector(h, "f32_unit")
    assert orc.tmv_gen(h, w, cols).tobytes() == orc.tmv(A, x)[cols].tobytes()
    rows = [0, 3, 63]
    xm = synth.vector(w, "f32_unit")
    assert orc.mv_gen(h, w, rows).tobytes() == orc.mv(A, xm)[rows].tobytes()


# ------------------------------------------------------------------ reduce
def test_reduce_closed_forms(orc):
    for L in [0, 1, 5, 32, 150, 1024]:
        ones = np.ones((3, L), np.int32)
        assert (orc.reduce(ones) == L).all()
        assert (orc.reduce(ones.astype(np.float32)) == L).all()
        iota = np.tile(np.arange(L, dtype=np.int32), (2, 1))
        assert (orc.reduce(iota) == L * (L - 1) // 2).all()
        assert (orc.reduce(iota.astype(np.float32)) == L * (L - 1) // 2).all()
        if L:
            perm = np.random.default_rng(L).permutation(L).astype(np.int32)[None, :]
            assert orc.reduce(perm, op=orc.MAX)[0] == L - 1
            assert orc.reduce(perm.astype(np.float32), op=orc.MAX)[0] == L - 1
    # L = 0: identity
    assert orc.reduce(np.zeros((2, 0), np.float32), op=orc.MAX)[0] == -np.inf
    assert orc.reduce(np.zeros((2, 0), np.int32), op=orc.MAX)[0] == np.iinfo(np.int32).min
    assert orc.reduce(np.zeros((2, 0), np.float32))[0] == 0


def test_reduce_i32_wrap(orc):
    assert orc.reduce(np.full((1, 8), 1 << 30, np.int32))[0] == 0
    g = GOLD["i32_wrap_hand"]
    assert orc.reduce(np.array([g["in"]], np.int32))[0] == g["sum"]
    x = synth.items(64, 77, "i32_full")
    want = [((sum(int(v) for v in row) + (1 << 31)) % (1 << 32)) - (1 << 31) for row in x]
    assert orc.reduce(x).tolist() == want


def test_reduce_kat(orc):
    # SURVEY C-5: i32_small(2^20), N=2, L=5
    x = synth.items(2, 5, "i32_small")
    assert x.tolist() == [[-346375, -4676, -224943, 706264, -303807],
                          [342190, 211657, -557527, -199899, 647748]]
    assert orc.reduce(x).tolist() == [-173537, 444169]
    assert orc.reduce(x, op=orc.MAX).tolist() == [706264, 647748]


def test_reduce_bruteforce(orc):
    x = synth.items(20, 37, "f32_signed")
    y = orc.reduce(x)
    for n in range(20):
        assert y[n] == np.float32(float(sum(Fraction(float(v)) for v in x[n])))
    # max: no rounding -> must equal numpy's max bit for bit
    assert orc.reduce(x, op=orc.MAX).tobytes() == x.max(1).tobytes()
    xi = synth.items(20, 37, "i32_full")
    assert orc.reduce(xi, op=orc.MAX).tobytes() == xi.max(1).tobytes()


def test_reduce_init(orc):
    x = synth.items(10, 9, "i32_small")
    ini = synth.init(10, "i32_small")
    assert (orc.reduce(x, init=ini) == orc.reduce(x) + ini).all()
    assert (orc.reduce(x, op=orc.MAX, init=ini) == np.maximum(x.max(1), ini)).all()
    xf = synth.items(10, 9, "f32_int4")
    inf_ = synth.init(10, "f32_int4")
    assert (orc.reduce(xf, init=inf_) == xf.sum(1) + inf_).all()


def test_reduce_gen_matches_arrays(orc):
    N, L = 50, 33
    items = [0, 7, 49]
    for dtype, kind, op in [(orc.F32, "f32_unit", orc.SUM), (orc.F32, "f32_signed", orc.MAX),
                            (orc.I32, "i32_small", orc.SUM), (orc.I32, "i32_full", orc.MAX)]:
        x = synth.items(N, L, kind)
        got = orc.reduce_gen(L, items, dtype, kind, op)
        assert got.tobytes() == orc.reduce(x, op=op)[items].tobytes()
        ini = synth.init(N, kind)
        got = orc.reduce_gen(L, items, dtype, kind, op, init_kind=kind)
        assert got.tobytes() == orc.reduce(x, op=op, init=ini)[items].tobytes()


# ------------------------------------------------------------------ scan
def test_scan_closed_forms(orc):
    for L in [1, 5, 64, 1024]:
        assert (orc.scan(np.ones((2, L), np.int32)) == np.arange(1, L + 1)).all()
        assert (orc.scan(np.ones((2, L), np.float32)) == np.arange(1, L + 1)).all()
        k = np.arange(L)
        io = np.tile(k.astype(np.int32), (2, 1))
        assert (orc.scan(io) == k * (k + 1) // 2).all()
    g = GOLD["scan_hand"]
    assert orc.scan(np.array([g["in"]], np.int32))[0].tolist() == g["out"]
    assert orc.scan(np.zeros((3, 0), np.int32)).shape == (3, 0)


def test_scan_bruteforce(orc):
    x = synth.items(6, 50, "f32_signed")
    y = orc.scan(x)
    for n in range(6):
        s = Fraction(0)
        for k in range(50):
            s += Fraction(float(x[n, k]))
            assert y[n, k] == np.float32(float(s))
    xi = synth.items(6, 50, "i32_full")
    yi = orc.scan(xi)
    for n in range(6):
        s = 0
        for k in range(50):
            s += int(xi[n, k])
            assert int(yi[n, k]) == ((s + (1 << 31)) % (1 << 32)) - (1 << 31)


def test_scan_kat_and_invariants(orc):
    x = synth.items(2, 5, "i32_small")
    y = orc.scan(x)
    assert y.tolist() == [[-346375, -351051, -575994, 130270, -173537],
                          [342190, 553847, -3680, -203579, 444169]]
    # last column of the inclusive scan is the reduction; first is the input
    x = synth.items(40, 33, "i32_full")
    ini = synth.init(40, "i32_full")
    y = orc.scan(x, init=ini)
    assert (y[:, -1] == orc.reduce(x, init=ini)).all()
    # differences recover the input (mod 2^32)
    d = np.diff(y.astype(np.int64), axis=1) % (1 << 32)
    assert (d == x[:, 1:].astype(np.int64) % (1 << 32)).all()


def test_scan_gen_matches_arrays(orc):
    N, L = 20, 31
    items = [0, 19, 4]
    for dtype, kind in [(orc.F32, "f32_unit"), (orc.I32, "i32_small")]:
        x = synth.items(N, L, kind)
        assert orc.scan_gen(L, items, dtype, kind).tobytes() == orc.scan(x)[items].tobytes()
        ini = synth.init(N, kind)
        assert (orc.scan_gen(L, items, dtype, kind, init_kind=kind).tobytes()
                == orc.scan(x, init=ini)[items].tobytes())


# ------------------------------------------------------------------ NP structure
def test_owner_map_paper_p426(orc):
    g = GOLD["owner_cyclic_L12_S8"]
    own = orc.owner_map(g["L"], g["S"], orc.CYCLIC, g["V"])
    assert own.tolist() == g["owner"]
    assert np.bincount(own, minlength=g["S"]).tolist() == g["counts"]


def test_owner_map_matches_paper_loop(orc):
    # second formulation: run the paper's loop `for (i=slave_id; i<N; i+=slave_size)`
    # and `n = ni*slave_size + slave_id` per slave
    for L in [0, 1, 3, 12, 31, 32, 33, 150, 1000]:
        for S in [1, 2, 4, 8, 16, 32]:
            want = np.full(L, -1)
            for s in range(S):
                i = s
                while i < L:
                    assert want[i] == -1
                    want[i] = s
                    i += S
            assert orc.owner_map(L, S, orc.CYCLIC, 1).tolist() == want.tolist()


def test_owner_map_vector_and_block(orc):
    assert orc.owner_map(12, 8, orc.CYCLIC, 4).tolist() == [0] * 4 + [1] * 4 + [2] * 4
    assert orc.owner_map(12, 8, orc.BLOCK, 1).tolist() == [0, 0, 1, 1, 2, 2, 3, 3, 4, 4, 5, 5]
    for L in [1, 7, 64, 150, 1023]:
        for S in [1, 2, 8, 32]:
            for V in [1, 4]:
                own = orc.owner_map(L, S, orc.BLOCK, V)
                # block: non-decreasing, contiguous per slave, chunk a multiple of V
                assert (np.diff(own) >= 0).all() and own.max() < S
                c = -(-L // S)
                c = -(-c // V) * V
                assert (np.bincount(own) <= c).all()
                assert (np.bincount(own)[:-1] == c).all()


def test_team_ids_paper_examples(orc):
    # shfl(var,0,4): the lane each lane reads is its master's lane
    g = GOLD["shfl_width_groups"]
    m, s = orc.team_ids(g["S"], orc.INTRA_WARP, 32)
    assert (np.arange(32) - s).tolist() == g["master_lane_of_lane"]
    # slave_size 4 intra-warp: 8 masters + 24 slaves per warp
    g = GOLD["intra_warp_S4_masters_per_warp"]
    assert len(set(m.tolist())) == g["masters_per_warp"] and int((s != 0).sum()) == g["slaves_per_warp"]
    # inter-warp 32x8: threads (1,0)..(1,7) form master 1's team
    g = GOLD["inter_warp_32x8"]
    bx, by = g["block"]
    m, s = orc.team_ids(g["S"], orc.INTER_WARP, bx * by)
    team = [(t % bx, t // bx) for t in range(bx * by) if m[t] == 1]
    assert sorted(team) == sorted(map(tuple, g["threads_of_master_1_xy"]))
    assert (s[m == 1] == np.arange(8)).all()
    # intra-warp with blockDim.x = slave_size = 8: (0,1)..(7,1) = master 1
    g = GOLD["intra_warp_8"]
    m, s = orc.team_ids(g["S"], orc.INTRA_WARP, 64)
    team = [(t % 8, t // 8) for t in range(64) if m[t] == 1]
    assert sorted(team) == sorted(map(tuple, g["threads_of_master_1_xy"]))


def test_team_ids_reject(orc):
    with pytest.raises(ValueError):
        orc.team_ids(3, orc.INTRA_WARP, 32)
    with pytest.raises(ValueError):
        orc.owner_map(4, 0, orc.CYCLIC)


# ------------------------------------------------------------------ ragged (f1)
def test_ragged_equal_lengths_is_batched_reduce(orc):
    # second formulation: equal segment lengths L reduce to the batched op
    N, L = 37, 13
    for kind, dt in [("f32_signed", np.float32), ("i32_full", np.int32)]:
        x = synth.items(N, L, kind)
        off = np.arange(N + 1, dtype=np.int64) * L
        for op in (orc.SUM, orc.MAX):
            assert orc.ragged_reduce(x.reshape(-1), off, op=op).tobytes() == orc.reduce(x, op=op).tobytes()


def test_ragged_bruteforce_and_empty(orc):
    lens = synth.lengths(60, 7)
    assert (lens == 0).any()
    off = synth.offsets_from_lengths(lens)
    x = synth.gen(1, "f32_signed", 0, int(off[-1]))
    y = orc.ragged_reduce(x, off)
    for n in range(60):
        s = sum((Fraction(float(v)) for v in x[off[n]:off[n + 1]]), Fraction(0))
        assert y[n] == np.float32(float(s))
    ym = orc.ragged_reduce(x, off, op=orc.MAX)
    for n in range(60):
        seg = x[off[n]:off[n + 1]]
        assert ym[n] == (seg.max() if len(seg) else -np.inf)
    ini = synth.init(60, "f32_int4")
    yi = orc.ragged_reduce(x, off, init=ini)
    assert (yi[lens == 0] == ini[lens == 0]).all()
    # decreasing offset pair -> empty loop
    off2 = np.array([0, 5, 3, 8], np.int64)
    xi = np.arange(8, dtype=np.int32)
    assert orc.ragged_reduce(xi, off2).tolist() == [10, 0, 3 + 4 + 5 + 6 + 7]


def test_ragged_lengths_distributions():
    u = synth.lengths(100000, 64, "uniform")
    assert u.min() == 0 and u.max() == 128 and abs(u.mean() - 64) < 1
    e = synth.lengths(100000, 64, "exp")
    assert e.min() == 0 and e.max() <= 16 * 64 and abs(e.mean() - 64) < 2


# ------------------------------------------------------------------ LE multi-section (f2)
def test_le_closed_forms(orc):
    # two-valued items a,b alternating (L even): ave=(a+b)/2, var=L((a-b)/2)^2, ep=0
    N, L = 5, 150
    a = np.arange(1, N + 1, dtype=np.float32)[:, None]
    x = np.where(np.arange(L)[None, :] % 2 == 0, a, 3 * a).astype(np.float32)
    g, ave, var, ep = orc.le_gicov(x, thr=0.0)
    assert (ave == 2 * a[:, 0]).all()
    assert (var == L * a[:, 0] ** 2).all()
    assert (ep == 0).all()
    assert (g == np.float32(2 * a[:, 0]) / np.sqrt(np.float32(L * a[:, 0] ** 2))).all()
    # constant items: var = 0 -> ratio inf > thr -> gicov = ave/0 = inf
    g, ave, var, ep = orc.le_gicov(np.full((3, 8), 0.25, np.float32), thr=1e30)
    assert (var == 0).all() and np.isinf(g).all()
    # a threshold no item passes leaves gicov untouched
    g, *_ = orc.le_gicov(x, thr=np.float32(1e30), gicov_fill=-7.0)
    assert (g == -7).all()


def test_le_bruteforce_and_layout(orc):
    x = synth.items(9, 23, "f32_signed")
    g, ave, var, ep = orc.le_gicov(x, thr=0.0)
    for n in range(9):
        s = sum(Fraction(float(v)) for v in x[n])
        a32 = np.float32(np.float32(float(s)) / np.float32(23))
        assert ave[n] == a32
        ts = [Fraction(float(v)) - Fraction(float(a32)) for v in x[n]]
        assert var[n] == np.float32(float(sum(t * t for t in ts)))
        assert ep[n] == np.float32(float(sum(ts)))
    # point-major layout of the transpose is the same computation
    g2, a2, v2, e2 = orc.le_gicov(np.ascontiguousarray(x.T), thr=0.0, layout=1)
    assert (a2 == ave).all() and (v2 == var).all() and (e2 == ep).all()
    assert np.array_equal(g2, g)


def test_parallel_oracle_equals_serial(orc):
    # the all-core CPU baseline splits outer items only: identical bits
    A = synth.matrix(200, 301, "f32_unit")
    x = synth.vector(200, "f32_unit")
    assert orc.tmv_parallel(A, x, 7).tobytes() == orc.tmv(A, x).tobytes()
    xm = synth.vector(301, "f32_unit")
    assert orc.mv_parallel(A, xm, 5).tobytes() == orc.mv(A, xm).tobytes()


# ------------------------------------------------------------------ randomised oracle invariants
from hypothesis import given, settings  # noqa: E402
from hypothesis import strategies as st  # noqa: E402


@settings(max_examples=60, deadline=None)
@given(N=st.integers(1, 30), L=st.integers(0, 40), seed=st.integers(0, 10**6))
def test_oracle_invariants_random(orc, N, L, seed):
    x = synth.items(N, L, "i32_full", seed=seed)
    ini = synth.init(N, "i32_full", seed=seed)
    r, sc = orc.reduce(x, init=ini), orc.scan(x, init=ini)
    exact = [((int(i) + sum(int(v) for v in row) + (1 << 31)) % (1 << 32)) - (1 << 31) for i, row in zip(ini, x)]
    assert r.tolist() == exact
    if L:
        assert (sc[:, -1] == r).all()
    xf = synth.items(N, L, "f32_int4", seed=seed)
    assert (orc.reduce(xf) == xf.astype(np.int64).sum(1)).all()
    assert (orc.reduce(xf, op=orc.MAX) == (xf.max(1) if L else -np.inf)).all()
    A = synth.matrix(N, L + 1, "f32_int4", seed=seed)
    xv = synth.vector(N, "f32_int4", seed=seed)
    assert orc.tmv(A, xv).tobytes() == orc.mv(np.ascontiguousarray(A.T), xv).tobytes()
