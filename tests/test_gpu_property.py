"""Randomised parity (hypothesis): random N, L, S, dist, map, dtype, op,
alignment and init against the oracle; integer data so every check is
bit-exact regardless of the summation order."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)
from hypothesis import HealthCheck, given, settings
from hypothesis import strategies as st

import oracle as O
import synth
from paper_conf_ppopp_yangz14_b200 import build as B
from paper_conf_ppopp_yangz14_b200 import cudanp as C
from test_gpu_parity import assert_exact, dev, host

pytestmark = pytest.mark.gpu
B.build()
C.load()

S_ = st.sampled_from(C.SLAVE_SIZES)
# + the inter-warp-only team sizes and the library's own choice
S_ALL = st.sampled_from(C.SLAVE_SIZES + C.INTER_ONLY_SIZES + (C.S_AUTO,))


def _map_for(S, map_):
    """A non-power-of-two S exists only as an inter-warp team."""
    return C.INTER_WARP if S in C.INTER_ONLY_SIZES and map_ == C.INTRA_WARP else map_
D_ = st.sampled_from([C.CYCLIC, C.BLOCK])
M_ = st.sampled_from([C.INTRA_WARP, C.INTER_WARP, C.AUTO])
CFG = settings(max_examples=150, deadline=None, suppress_health_check=list(HealthCheck))


@CFG
@given(N=st.integers(0, 700), L=st.integers(0, 300), S=S_ALL, dist=D_, map_=M_,
       op=st.sampled_from([C.SUM, C.MAX]), shift=st.integers(0, 3), use_init=st.booleans(),
       seed=st.integers(0, 10**6))
def test_reduce_random(N, L, S, dist, map_, op, shift, use_init, seed):
    map_ = _map_for(S, map_)
    x = synth.gen(1, "i32_full", 0, N * L + shift, seed=seed)
    xd = dev(x)[shift:].view(N, L) if N * L else dev(x)[: 0].view(N, L)
    ini = synth.init(N, "i32_full", seed=seed)
    ref = O.reduce(x[shift:].reshape(N, L), op=op, init=ini if use_init else None)
    got = host(C.cudanp_batched_loop_reduce(xd, dev(ini) if use_init and N else None, op=op,
                                            S=S, dist=dist, map=map_))
    assert_exact(got, ref, f"N={N} L={L} S={S} dist={dist} map={map_} op={op} shift={shift}")


@CFG
@given(N=st.integers(0, 400), L=st.integers(0, 300), S=S_ALL, dist=D_, map_=M_,
       shift=st.integers(0, 3), use_init=st.booleans(), seed=st.integers(0, 10**6))
def test_scan_random(N, L, S, dist, map_, shift, use_init, seed):
    map_ = _map_for(S, map_)
    x = synth.gen(1, "i32_small", 0, N * L + shift, B=1 << 15, seed=seed)
    xd = dev(x)[shift:].view(N, L) if N * L else dev(x)[: 0].view(N, L)
    ini = synth.init(N, "i32_small", B=1 << 15, seed=seed)
    ref = O.scan(x[shift:].reshape(N, L), init=ini if use_init else None)
    got = host(C.cudanp_batched_loop_scan(xd, dev(ini) if use_init and N else None, S=S, dist=dist,
                                          map=map_))
    assert_exact(got, ref, f"N={N} L={L} S={S} dist={dist} map={map_} shift={shift}")


@CFG
@given(h=st.integers(0, 300), w=st.integers(1, 300), pad=st.integers(0, 5), S=S_ALL, dist=D_,
       map_=M_, seed=st.integers(0, 10**6))
def test_matvec_random(h, w, pad, S, dist, map_, seed):
    map_ = _map_for(S, map_)
    lda = w + pad
    A = synth.matrix(h, lda, "f32_int4", seed=seed)
    xt, xm = synth.vector(h, "f32_int4", seed=seed), synth.vector(w, "f32_int4", seed=seed)
    Ad = dev(A)
    what = f"h={h} w={w} lda={lda} S={S} dist={dist} map={map_}"
    ref_t = O.tmv(A, xt, w) if h else np.zeros(w, np.float32)
    assert_exact(host(C.cudanp_tmv(Ad, dev(xt), S=S, dist=dist, map=map_, n_outer=w)), ref_t, "tmv " + what)
    if h:
        assert_exact(host(C.cudanp_mv(Ad, dev(xm), S=S, dist=dist, map=map_, n_inner=w)),
                     O.mv(A, xm, w), "mv " + what)


@CFG
@given(N=st.integers(1, 500), mean=st.integers(0, 80), S=S_, dist=D_, map_=M_,
       op=st.sampled_from([C.SUM, C.MAX]), shift=st.integers(0, 3), seed=st.integers(0, 10**6))
def test_ragged_random(N, mean, S, dist, map_, op, shift, seed):
    lens = synth.lengths(N, mean, "exp", seed=seed)
    off = synth.offsets_from_lengths(lens) + shift
    x = synth.gen(1, "i32_full", 0, int(off[-1]) + 1, seed=seed)
    got = host(C.cudanp_ragged_loop_reduce(dev(x), dev(off), op=op, S=S, dist=dist, map=map_))
    assert_exact(got, O.ragged_reduce(x, off, op=op), f"N={N} mean={mean} S={S} d={dist} m={map_}")


@CFG
@given(N=st.integers(0, 700), L4=st.integers(0, 80), S=S_, dist=D_, op=st.sampled_from([C.SUM, C.MAX]),
       use_init=st.booleans(), sb=st.sampled_from([0, 512, 8192]), seed=st.integers(0, 10**6))
def test_reduce_tma_random(N, L4, S, dist, op, use_init, sb, seed):
    L = 4 * L4
    x = synth.gen(1, "i32_full", 0, N * L, seed=seed).reshape(N, L)
    ini = synth.init(N, "i32_full", seed=seed)
    ref = O.reduce(x, op=op, init=ini if use_init else None)
    got = host(C.cudanp_batched_loop_reduce_tma(dev(x), dev(ini) if use_init and N else None, op=op,
                                                S=S, dist=dist, stage_bytes=sb))
    assert_exact(got, ref, f"TMA N={N} L={L} S={S} dist={dist} op={op} stage_bytes={sb}")


@CFG
@given(h=st.integers(0, 400), w4=st.integers(1, 80), pad4=st.integers(0, 2), S=S_, dist=D_,
       seed=st.integers(0, 10**6))
def test_tmv_tma_random(h, w4, pad4, S, dist, seed):
    w, lda = 4 * w4, 4 * (w4 + pad4)
    A = synth.matrix(h, lda, "f32_int4", seed=seed)
    x = synth.vector(h, "f32_int4", seed=seed)
    ref = O.tmv(A, x, w) if h else np.zeros(w, np.float32)
    got = host(C.cudanp_tmv(dev(A), dev(x), S=S, dist=dist, map=C.INTER_WARP_TMA, n_outer=w))
    assert_exact(got, ref, f"TMA h={h} w={w} lda={lda} S={S} dist={dist}")


BIG_ = st.sampled_from([64, 128, 256, 512, 1024, 2048, 4096, 8192])


@settings(max_examples=80, deadline=None, suppress_health_check=list(HealthCheck))
@given(N=st.integers(0, 300), L=st.integers(0, 20000), S=BIG_, dist=D_, shift=st.integers(0, 3),
       use_init=st.booleans(), seed=st.integers(0, 10**6))
def test_big_and_cluster_teams_random(N, L, S, dist, shift, use_init, seed):
    """Teams larger than a warp (S/32 warps) and than a CTA (a cluster of 8
    CTAs): reduce (sum and max), scan (the cluster scan is block-only) and MV."""
    x = synth.gen(1, "i32_small", 0, N * L + shift, B=1 << 15, seed=seed)
    xd = dev(x)[shift:].view(N, L) if N * L else dev(x)[: 0].view(N, L)
    xs = x[shift:].reshape(N, L)
    ini = synth.init(N, "i32_small", B=1 << 15, seed=seed)
    inid = dev(ini) if use_init and N else None
    what = f"N={N} L={L} S={S} dist={dist} shift={shift} init={use_init}"
    assert_exact(host(C.cudanp_batched_loop_reduce(xd, inid, S=S, dist=dist)),
                 O.reduce(xs, init=ini if use_init else None), "reduce " + what)
    assert_exact(host(C.cudanp_batched_loop_reduce(xd, None, op=C.MAX, S=S, dist=dist)),
                 O.reduce(xs, op=O.MAX), "reduce max " + what)
    assert_exact(host(C.cudanp_batched_loop_scan(xd, inid, S=S, dist=dist)),
                 O.scan(xs, init=ini if use_init else None), "scan " + what)
    if N and L:
        h, w = min(N, 64), min(L, 5000)
        A = synth.matrix(h, w, "f32_int4", seed=seed)
        xm = synth.vector(w, "f32_int4", seed=seed)
        assert_exact(host(C.cudanp_mv(dev(A), dev(xm), S=S, dist=dist)), O.mv(A, xm), "mv " + what)


@settings(max_examples=60, deadline=None, suppress_health_check=list(HealthCheck))
@given(h=st.integers(0, 3000), w=st.integers(1, 6000), pad=st.integers(0, 5), S=st.sampled_from([64, 128]),
       dist=D_, seed=st.integers(0, 10**6))
def test_narrow_tmv_big_teams_random(h, w, pad, S, dist, seed):
    """TMV S = 64 / 128: every CTA layout the call picks (V = 4 with 4 or 8
    column-masters, V = 1), the L2 prefetch before the dependency wait, any
    alignment of the row pitch."""
    lda = w + pad
    A = synth.matrix(h, lda, "f32_int4", seed=seed)
    x = synth.vector(h, "f32_int4", seed=seed)
    ref = O.tmv(A, x, w) if h else np.zeros(w, np.float32)
    got = host(C.cudanp_tmv(dev(A), dev(x), S=S, dist=dist, map=C.INTER_WARP, n_outer=w))
    assert_exact(got, ref, f"narrow TMV h={h} w={w} lda={lda} S={S} dist={dist}")
