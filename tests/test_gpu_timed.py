"""GPU parity for exactly what bench.py and the library's version selection
run, at the sizes they run it (VERDICT r1 "parity-test exactly what the bench
times"), plus the round-2 additions to the call surface:

  * every cudanp_autotune candidate for TMV and MV on the full C2 operands
    (16384 x 16384 fp32, the bench's workload), sampled against the oracle;
  * multi-warp teams (S = 64..1024) and cluster teams with more items than one
    persistent wave, so the grid-stride loops run (np_multi.cu, np_cluster.cu);
  * full-size C3 with the inter-warp map, C4 fp32 at L = 1024;
  * non-power-of-two inter-warp teams S = 3, 5, 10, 15 (Fig 12);
  * S = CUDANP_S_AUTO (the library's version choice) and MAP_AUTO's TMA choice;
  * the TMA TMV's fallbacks and its block distribution's ragged last tile.

Bars as in test_gpu_parity.py: bit-exact for int32, max and exact fp32 data
(pin P3); tol(L) relative error for fp32 sums on positive data (R17).
"""
import itertools
import math

import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import oracle as O
import synth
from paper_conf_ppopp_yangz14_b200 import build as B
from paper_conf_ppopp_yangz14_b200 import cudanp as C

pytestmark = pytest.mark.gpu

DISTS = (C.CYCLIC, C.BLOCK)
INTER_S = C.INTER_ONLY_SIZES


@pytest.fixture(scope="module", autouse=True)
def _lib():
    B.build()
    C.load()


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def host(t):
    torch.cuda.synchronize()
    return t.cpu().numpy()


def tol(L):
    return 1e-5 * max(1.0, math.sqrt(max(L, 1) / 4096.0))


def assert_rel(got, ref, L, what):
    got = np.asarray(got, np.float64)
    ref = np.asarray(ref, np.float64)
    assert got.shape == ref.shape, what
    if ref.size == 0:
        return
    err = np.max(np.abs(got - ref) / np.maximum(np.abs(ref), 1e-30))
    assert err <= tol(L), f"{what}: max rel err {err:.3e} > {tol(L):.3e}"


def assert_exact(got, ref, what):
    got, ref = np.asarray(got), np.asarray(ref)
    assert got.shape == ref.shape, what
    g = got.view(np.uint32) if got.dtype == np.float32 else got
    r = ref.view(np.uint32) if ref.dtype == np.float32 else ref
    if not np.array_equal(g, r):
        bad = np.argwhere(g != r)
        raise AssertionError(f"{what}: {len(bad)} mismatches, first at {bad[:3].tolist()}: "
                             f"got {got[tuple(bad[0])]} want {ref[tuple(bad[0])]}")


def run_or_unsupported(fn):
    """Run a call; None if the library reports the combination unsupported on
    this shape (the autotune skips those the same way)."""
    try:
        return fn()
    except C.CudanpError as e:
        if e.status == C.ERR_UNSUPPORTED:
            return None
        raise


# ------------------------------------------------------------------ C2: every autotune candidate
def _sample_idx(n, seed, k=256):
    rng = np.random.default_rng(seed)
    return np.unique(np.concatenate([rng.integers(0, n, k), [0, 1, 127, 128, n - 2, n - 1]]))


def test_full_size_C2_every_autotune_candidate():
    """The bench runs cudanp_autotune over these candidates on the C2 operands
    and times the fastest (e.g. TMA TMV S=8, multi-warp MV S=256): every one of
    them is checked here on the same operands, in the same launch shape."""
    n = 16384
    A = torch.empty(n, n, dtype=torch.float32, device="cuda")
    C.cudanp_generate(A, "f32_unit", stream_id=1)
    x = torch.empty(n, dtype=torch.float32, device="cuda")
    C.cudanp_generate(x, "f32_unit", stream_id=2)
    idx = _sample_idx(n, 10)
    ref_t, ref_m = O.tmv_gen(n, n, idx), O.mv_gen(n, n, idx)
    y = torch.empty(n, dtype=torch.float32, device="cuda")
    ran = {"tmv": 0, "mv": 0}
    for op, fn, ref in (("tmv", C.cudanp_tmv, ref_t), ("mv", C.cudanp_mv, ref_m)):
        for S, d, m in C.cudanp_autotune_candidates(op) + [(C.S_AUTO, C.CYCLIC, C.AUTO)]:
            y.fill_(float("nan"))
            if run_or_unsupported(lambda: fn(A, x, y, S=S, dist=d, map=m)) is None:
                continue
            ran[op] += 1
            assert_rel(host(y)[idx], ref, n, f"C2 {op} S={S} dist={d} map={m}")
    assert ran["tmv"] >= 30 and ran["mv"] >= 30, ran
    # exact data: every candidate gives the oracle's bits on every sampled output (P3)
    C.cudanp_generate(A, "f32_int4", stream_id=1)
    C.cudanp_generate(x, "f32_int4", stream_id=2)
    ref_t = O.tmv_gen(n, n, idx, "f32_int4", "f32_int4")
    ref_m = O.mv_gen(n, n, idx, "f32_int4", "f32_int4")
    for op, fn, ref in (("tmv", C.cudanp_tmv, ref_t), ("mv", C.cudanp_mv, ref_m)):
        for S, d, m in C.cudanp_autotune_candidates(op):
            if run_or_unsupported(lambda: fn(A, x, y, S=S, dist=d, map=m)) is None:
                continue
            assert_exact(host(y)[idx], ref, f"C2 {op} int4 S={S} dist={d} map={m}")
    del A
    torch.cuda.empty_cache()


def test_bench_timed_kernels_all_outputs_C2():
    """The two kernels the round-1 bench timed (TMA TMV S=8 cyclic, multi-warp
    MV S=256 cyclic) and the library's S_AUTO choice: every one of the 16384
    outputs, against the oracle on exact data (any dropped or doubled row of
    the persistent grid-stride loop changes a sum)."""
    n = 16384
    A = torch.empty(n, n, dtype=torch.float32, device="cuda")
    C.cudanp_generate(A, "f32_int4", stream_id=1)
    x = torch.empty(n, dtype=torch.float32, device="cuda")
    C.cudanp_generate(x, "f32_int4", stream_id=2)
    allidx = np.arange(n)
    ref_t = O.tmv_gen(n, n, allidx, "f32_int4", "f32_int4")
    ref_m = O.mv_gen(n, n, allidx, "f32_int4", "f32_int4")
    for S, d in ((8, C.CYCLIC), (8, C.BLOCK), (16, C.BLOCK), (32, C.CYCLIC)):
        assert_exact(host(C.cudanp_tmv(A, x, S=S, dist=d, map=C.INTER_WARP_TMA)), ref_t, f"tma S={S} d={d}")
    for S, d in ((256, C.CYCLIC), (128, C.CYCLIC), (512, C.CYCLIC), (256, C.BLOCK)):
        assert_exact(host(C.cudanp_mv(A, x, S=S, dist=d)), ref_m, f"mv multi S={S} d={d}")
    assert_exact(host(C.cudanp_tmv(A, x)), ref_t, "tmv S_AUTO")
    assert_exact(host(C.cudanp_mv(A, x)), ref_m, "mv S_AUTO")
    del A
    torch.cuda.empty_cache()


# ------------------------------------------------------------------ beyond one persistent wave
def _one_wave(op, L, S, dtype=C.F32):
    """Items one persistent wave of the multi-warp kernel holds (resident CTAs
    x teams per CTA), from the launch shape the library reports."""
    i = C.cudanp_launch_info(op, 1 << 30, L, dtype=dtype, S=S)
    return i["grid_ctas"] * max(1, i["block_threads"] // S)


def _beyond(op, L, S, dtype=C.F32, extra=3):
    """An item count of ~1.7 persistent waves plus a ragged remainder."""
    return int(1.7 * _one_wave(op, L, S, dtype)) + extra


@pytest.mark.parametrize("S", C.MULTI_WARP_SIZES)
def test_multi_warp_reduce_more_items_than_one_wave(S):
    for L, kind, dtype, op, exact in ((1000, "i32_full", C.I32, C.SUM, True),
                                      (999, "i32_full", C.I32, C.MAX, True),
                                      (640, "f32_unit", C.F32, C.SUM, False),
                                      (512, "f32_signed", C.F32, C.MAX, True)):
        N = _beyond("reduce", L, S, dtype, extra=L % 7)
        x = synth.items(N, L, kind, seed=S)
        ini = synth.init(N, kind, seed=S)
        ref = O.reduce(x, op=op, init=ini)
        for d in DISTS:
            got = host(C.cudanp_batched_loop_reduce(dev(x), dev(ini), op=op, S=S, dist=d))
            what = f"multi reduce S={S} N={N} L={L} {kind} op={op} dist={d}"
            assert_exact(got, ref, what) if exact else assert_rel(got, ref, L, what)


@pytest.mark.parametrize("S", C.MULTI_WARP_SIZES)
def test_multi_warp_scan_more_items_than_one_wave(S):
    # fp32 f32_unit too: the exclusive prefix of an S > 32 team is taken by a
    # shuffle, not incl - own, so it is within tol(L)
    for L, kind, exact in ((300, "i32_small", True), (257, "f32_int4", True),
                           (512, "f32_unit", False), (1024, "f32_unit", False)):
        N = _beyond("scan", L, S, C.I32, extra=L % 5)
        x = synth.items(N, L, kind, B=1 << 15, seed=S)
        ini = synth.init(N, kind, B=1 << 15, seed=S)
        ref = O.scan(x, init=ini)
        for d in DISTS:
            got = host(C.cudanp_batched_loop_scan(dev(x), dev(ini), S=S, dist=d))
            what = f"multi scan S={S} N={N} L={L} {kind} dist={d}"
            assert_exact(got, ref, what) if exact else assert_rel(got, ref, L, what)


@pytest.mark.parametrize("S", C.MULTI_WARP_SIZES)
def test_multi_warp_mv_more_rows_than_one_wave(S):
    for w, kind in ((1000, "f32_int4"), (999, "f32_int4"), (2048, "f32_unit")):
        h = _beyond("mv", w, S, extra=w % 3)
        A = synth.matrix(h, w, kind, seed=S)
        x = synth.vector(w, kind)
        ref = O.mv(A, x)
        for d in DISTS:
            got = host(C.cudanp_mv(dev(A), dev(x), S=S, dist=d))
            what = f"multi mv S={S} h={h} w={w} dist={d}"
            assert_exact(got, ref, what) if kind == "f32_int4" else assert_rel(got, ref, w, what)


@pytest.mark.parametrize("S", (64, 128, 256))
def test_multi_warp_ragged_more_segments_than_one_wave(S):
    N = 4 * _beyond("reduce", 700, S)
    lens = synth.lengths(N, 700, "exp", seed=S)
    off = synth.offsets_from_lengths(lens)
    x = synth.gen(1, "i32_full", 0, int(off[-1]))
    ref = O.ragged_reduce(x, off)
    for d in DISTS:
        got = host(C.cudanp_ragged_loop_reduce(dev(x), dev(off), S=S, dist=d))
        assert_exact(got, ref, f"multi ragged S={S} dist={d}")


@pytest.mark.parametrize("S", C.CLUSTER_SIZES)
def test_cluster_teams_more_items_than_resident_clusters(S):
    # launch_cluster strides clusters over items past 8 waves of resident clusters
    N, L = 3000, 4096 + 36
    x = synth.items(N, L, "i32_full", seed=S)
    ref = O.reduce(x)
    xs = synth.items(N, L, "f32_unit", seed=S)
    for d in DISTS:
        assert_exact(host(C.cudanp_batched_loop_reduce(dev(x), S=S, dist=d)), ref, f"cluster reduce S={S} d={d}")
        got = host(C.cudanp_batched_loop_scan(dev(xs), S=S, dist=d))
        assert_rel(got, O.scan(xs), L, f"cluster scan f32_unit S={S} d={d}")


# ------------------------------------------------------------------ full-size C3 inter / C4 fp32
def test_full_size_C3_inter_warp_sampled():
    N = 1 << 22
    items = _sample_idx(N, 3, 2048)
    for L in (32, 256):
        x = torch.empty(N, L, dtype=torch.float32, device="cuda")
        C.cudanp_generate(x, "f32_unit", stream_id=1)
        ref = O.reduce_gen(L, items, O.F32, "f32_unit")
        for S, d in itertools.product(C.SLAVE_SIZES + INTER_S, DISTS):
            got = host(C.cudanp_batched_loop_reduce(x, S=S, dist=d, map=C.INTER_WARP))
            assert_rel(got[items], ref, L, f"C3 inter L={L} S={S} dist={d}")
        del x
        xi = torch.empty(N, L, dtype=torch.int32, device="cuda")
        C.cudanp_generate(xi, "i32_small", stream_id=1)
        ref = O.reduce_gen(L, items, O.I32, "i32_small")
        for S, d in itertools.product(C.SLAVE_SIZES, DISTS):
            got = host(C.cudanp_batched_loop_reduce(xi, S=S, dist=d, map=C.INTER_WARP))
            assert_exact(got[items], ref, f"C3 inter i32 L={L} S={S} dist={d}")
        del xi
        torch.cuda.empty_cache()


def test_full_size_C4_fp32_L1024_sampled():
    N, L = 1 << 21, 1024
    items = _sample_idx(N, 4, 256)
    x = torch.empty(N, L, dtype=torch.float32, device="cuda")
    C.cudanp_generate(x, "f32_unit", stream_id=1)
    out = torch.empty_like(x)
    ref = O.scan_gen(L, items, O.F32, "f32_unit")
    sel = torch.from_numpy(items).cuda()
    for S, d, m in [(16, C.CYCLIC, C.INTRA_WARP), (32, C.CYCLIC, C.INTRA_WARP), (16, C.BLOCK, C.INTRA_WARP),
                    (8, C.CYCLIC, C.INTER_WARP), (64, C.CYCLIC, C.INTRA_WARP), (256, C.BLOCK, C.INTRA_WARP),
                    (C.S_AUTO, C.CYCLIC, C.AUTO)]:
        C.cudanp_batched_loop_scan(x, out=out, S=S, dist=d, map=m)
        assert_rel(host(out[sel]), ref, L, f"C4 f32 L=1024 S={S} dist={d} map={m}")
    del x, out
    torch.cuda.empty_cache()


# ------------------------------------------------------------------ non-power-of-two inter-warp S
@pytest.mark.parametrize("S", INTER_S)
def test_inter_warp_non_power_of_two_S(S):
    """Fig 12: inter-warp teams of 3, 5, 10, 15 for the four
    hot-path calls, both distributions, ragged tails; MAP_AUTO picks inter."""
    for h, w in ((1, 1), (37, 131), (300, 260), (129, 512), (1000, 1001)):
        A = synth.matrix(h, w, "f32_int4", seed=S)
        xt, xm = synth.vector(h, "f32_int4"), synth.vector(w, "f32_int4")
        for d, m in itertools.product(DISTS, (C.INTER_WARP, C.AUTO)):
            assert_exact(host(C.cudanp_tmv(dev(A), dev(xt), S=S, dist=d, map=m)), O.tmv(A, xt),
                         f"tmv S={S} h={h} w={w} d={d} m={m}")
            assert_exact(host(C.cudanp_mv(dev(A), dev(xm), S=S, dist=d, map=m)), O.mv(A, xm),
                         f"mv S={S} h={h} w={w} d={d} m={m}")
    Au, xu = synth.matrix(700, 900, "f32_unit"), synth.vector(700, "f32_unit")
    assert_rel(host(C.cudanp_tmv(dev(Au), dev(xu), S=S, map=C.INTER_WARP)), O.tmv(Au, xu), 700, "tmv unit")
    for N, L in ((1, 1), (33, 5), (70, 12), (300, 33), (129, 80), (200, 150), (97, 256), (1100, 64)):
        for kind, op, exact in (("i32_full", C.SUM, True), ("i32_full", C.MAX, True),
                                ("f32_signed", C.MAX, True), ("f32_unit", C.SUM, False)):
            x = synth.items(N, L, kind, seed=S)
            ini = synth.init(N, kind, seed=S)
            ref = O.reduce(x, op=op, init=ini)
            for d in DISTS:
                got = host(C.cudanp_batched_loop_reduce(dev(x), dev(ini), op=op, S=S, dist=d))
                what = f"reduce S={S} N={N} L={L} {kind} op={op} d={d}"
                assert_exact(got, ref, what) if exact else assert_rel(got, ref, L, what)
        for kind, exact in (("i32_small", True), ("f32_unit", False)):
            x = synth.items(N, L, kind, B=1 << 15, seed=S)
            ini = synth.init(N, kind, B=1 << 15, seed=S)
            ref = O.scan(x, init=ini)
            for d in DISTS:
                got = host(C.cudanp_batched_loop_scan(dev(x), dev(ini), S=S, dist=d))
                what = f"scan S={S} N={N} L={L} {kind} d={d}"
                assert_exact(got, ref, what) if exact else assert_rel(got, ref, L, what)
    with pytest.raises(C.CudanpError) as ei:
        C.cudanp_batched_loop_reduce(dev(synth.items(8, 8, "i32_full")), S=S, map=C.INTRA_WARP)
    assert ei.value.status == C.ERR_UNSUPPORTED


# ------------------------------------------------------------------ S_AUTO / MAP_AUTO
def test_auto_version_parity():
    """S = CUDANP_S_AUTO runs the (S, dist, map) cudanp_choose_version names,
    on every op, with results equal to the oracle's."""
    for h, w in ((1, 1), (300, 260), (129, 512), (1024, 1024), (2048, 4096), (300, 8192), (65, 12288)):
        A = synth.matrix(h, w, "f32_int4")
        xt, xm = synth.vector(h, "f32_int4"), synth.vector(w, "f32_int4")
        assert_exact(host(C.cudanp_tmv(dev(A), dev(xt))), O.tmv(A, xt), f"tmv auto {h}x{w}")
        assert_exact(host(C.cudanp_mv(dev(A), dev(xm))), O.mv(A, xm), f"mv auto {h}x{w}")
    for N, L in ((1, 1), (1000, 32), (257, 150), (64, 4096), (5000, 256), (3, 20000)):
        x = synth.items(N, L, "i32_full")
        assert_exact(host(C.cudanp_batched_loop_reduce(dev(x))), O.reduce(x), f"reduce auto {N}x{L}")
        xs = synth.items(N, L, "i32_small", B=1 << 12)
        assert_exact(host(C.cudanp_batched_loop_scan(dev(xs))), O.scan(xs), f"scan auto {N}x{L}")


# ------------------------------------------------------------------ TMA TMV: fallbacks and edges
def test_tma_tmv_misaligned_y_and_odd_width():
    """MAP_INTER_WARP_TMA / MAP_AUTO never fail on alignment: y at root +
    begin*4 (a fused gather's shard pointer) and widths that are not a
    multiple of 4 take TMA where it can run and the LDG kernel where not."""
    h, w = 777, 1001
    lda = 1004
    full = synth.matrix(h, lda, "f32_int4")
    A = dev(full)[:, :w]
    assert A.stride(0) == lda
    x = synth.vector(h, "f32_int4")
    ref = O.tmv(full, x, w)
    buf = torch.zeros(w + 3, dtype=torch.float32, device="cuda")
    for off in (0, 1, 2, 3):
        y = buf[off:off + w]
        for S, d, m in itertools.product((1, 4, 8, 32), DISTS, (C.INTER_WARP_TMA, C.AUTO)):
            y.fill_(float("nan"))
            C.cudanp_tmv(A, dev(x), y, S=S, dist=d, map=m)
            assert_exact(host(y), ref, f"tma off={off} S={S} d={d} m={m}")
        # the strict TMA entry point now accepts the unaligned y as well
        y.fill_(float("nan"))
        C.cudanp_tmv_tma(A, dev(x), y, S=8)
        assert_exact(host(y), ref, f"cudanp_tmv_tma off={off}")
    # a misaligned A cannot be described to TMA: MAP_INTER_WARP_TMA falls back
    flat = dev(np.concatenate([[0.0], full.reshape(-1)]).astype(np.float32))
    A1 = flat[1:].view(h, lda)[:, :w]
    assert A1.data_ptr() % 16 != 0
    y = torch.empty(w, dtype=torch.float32, device="cuda")
    C.cudanp_tmv(A1, dev(x), y, S=8, map=C.INTER_WARP_TMA)
    assert_exact(host(y), ref, "tma fallback misaligned A")
    with pytest.raises(C.CudanpError) as ei:
        C.cudanp_tmv_tma(A1, dev(x), y, S=8)
    assert ei.value.status == C.ERR_UNSUPPORTED


def test_tma_block_distribution_skips_the_next_slaves_rows():
    """Block distribution: a TMA box of RK rows may run past a slave's chunk
    into the next slave's rows.  Those rows are skipped, so an Inf there does
    not turn the previous slave's partial into NaN (0 * Inf) -- each column is
    +Inf exactly where the definition says (Inf in a row whose x > 0)."""
    for S, h in ((2, 37), (4, 101), (8, 1000), (16, 999), (32, 1003)):
        w = 256
        A = synth.matrix(h, w, "f32_unit")
        x = synth.vector(h, "f32_unit")          # all x > 0
        c = -(-h // S)                            # chunk of each slave
        rows = [min(k * c, h - 1) for k in range(1, S)]  # first row of slaves 1..S-1
        for j, r in enumerate(rows):
            A[r, (7 * j) % w] = np.inf
        ref = O.tmv(A, x)
        for rs in (-1, 0, 1, 2):
            got = host(C.cudanp_tmv_tma(dev(A), dev(x), S=S, dist=C.BLOCK, rows_sel=rs))
            assert not np.isnan(got).any(), f"NaN S={S} h={h} rows_sel={rs}"
            inf = np.isinf(ref)
            assert (np.isinf(got) == inf).all() and (got[inf] == ref[inf]).all(), f"S={S} h={h}"
            assert_rel(got[~inf], ref[~inf], h, f"finite S={S} h={h} rows_sel={rs}")


def test_binding_passes_row_stride_as_lda():
    """A column slice of a wider matrix is a row-strided view: the binding
    passes A.stride(0) as lda, so the kernels walk the right rows."""
    h, W, w = 300, 260, 197
    full = synth.matrix(h, W, "f32_int4")
    Ad = dev(full)[:, :w]
    xt, xm = synth.vector(h, "f32_int4"), synth.vector(w, "f32_int4")
    for S, m in ((1, C.AUTO), (8, C.INTER_WARP), (8, C.INTRA_WARP), (C.S_AUTO, C.AUTO)):
        assert_exact(host(C.cudanp_tmv(Ad, dev(xt), S=S, map=m)), O.tmv(full, xt, w), f"tmv view S={S}")
        assert_exact(host(C.cudanp_mv(Ad, dev(xm), S=S, map=m)), O.mv(full, xm, w), f"mv view S={S}")


# ------------------------------------------------------------------ tiled S = 1 baselines
def test_s1_tiled_baselines_parity():
    """CUDANP_IMPL_S1_TILED: one thread per item, rows through TMA-staged
    shared-memory tiles (the SMM-style no-NP baseline) -- the
    denominator of the NP speedups must compute the same thing.  Ragged row
    groups (h, N not multiples of the 64/128-row tiles), widths not multiples
    of the 32-column tile, multi-tile rows, init."""
    for h, w in ((1, 4), (37, 132), (300, 260), (129, 512), (1000, 1004), (4100, 68)):
        A = synth.matrix(h, w, "f32_int4", seed=w)
        xt, xm = synth.vector(h, "f32_int4"), synth.vector(w, "f32_int4")
        assert_exact(host(C.cudanp_mv_variant(C.S1_TILED, dev(A), dev(xm))), O.mv(A, xm), f"mv tiled {h}x{w}")
        assert_exact(host(C.cudanp_tmv_variant(C.S1_TILED, dev(A), dev(xt))), O.tmv(A, xt), f"tmv tiled {h}x{w}")
    Au, xu = synth.matrix(513, 2048, "f32_unit"), synth.vector(2048, "f32_unit")
    assert_rel(host(C.cudanp_mv_variant(C.S1_TILED, dev(Au), dev(xu))), O.mv(Au, xu), 2048, "mv tiled unit")
    # a padded row pitch (lda > w) through the binding's stride
    full = synth.matrix(200, 132, "f32_int4")
    xm = synth.vector(100, "f32_int4")
    assert_exact(host(C.cudanp_mv_variant(C.S1_TILED, dev(full)[:, :100], dev(xm))), O.mv(full, xm, 100),
                 "mv tiled lda")
    for N, L in ((1, 4), (33, 8), (129, 64), (1000, 100), (300, 1024), (5000, 36)):
        for kind, exact in (("i32_small", True), ("f32_int4", True), ("f32_unit", False)):
            x = synth.items(N, L, kind, B=1 << 15, seed=L)
            ini = synth.init(N, kind, B=1 << 15, seed=L)
            got = host(C.cudanp_batched_loop_scan_variant(C.S1_TILED, dev(x), dev(ini)))
            ref = O.scan(x, init=ini)
            what = f"scan tiled {kind} {N}x{L}"
            assert_exact(got, ref, what) if exact else assert_rel(got, ref, L, what)
            got = host(C.cudanp_batched_loop_scan_variant(C.S1_TILED, dev(x)))
            assert_exact(got, O.scan(x), what) if exact else assert_rel(got, O.scan(x), L, what)
        for kind, op in (("i32_full", C.SUM), ("i32_full", C.MAX), ("f32_signed", C.MAX), ("f32_int4", C.SUM)):
            x = synth.items(N, L, kind, seed=L)
            ini = synth.init(N, kind, seed=L)
            # max over all-negative-capable data: the zero-filled columns past L
            # must not take part
            assert_exact(host(C.cudanp_batched_loop_reduce_variant(C.S1_TILED, dev(x), op=op)),
                         O.reduce(x, op=op), f"reduce tiled {kind} op={op} {N}x{L}")
            assert_exact(host(C.cudanp_batched_loop_reduce_variant(C.S1_TILED, dev(x), dev(ini), op=op)),
                         O.reduce(x, op=op, init=ini), f"reduce tiled init {kind} op={op} {N}x{L}")
        xu = synth.items(N, L, "f32_unit", seed=L)
        assert_rel(host(C.cudanp_batched_loop_reduce_variant(C.S1_TILED, dev(xu))), O.reduce(xu), L,
                   f"reduce tiled f32_unit {N}x{L}")
    # preconditions: rows not a multiple of 4 elements, or x off 16-byte
    # alignment -> unsupported, not wrong
    with pytest.raises(C.CudanpError) as ei:
        C.cudanp_batched_loop_scan_variant(C.S1_TILED, dev(synth.items(10, 7, "i32_small")))
    assert ei.value.status == C.ERR_UNSUPPORTED
    A = dev(synth.matrix(40, 104, "f32_int4"))
    with pytest.raises(C.CudanpError) as ei:
        C.cudanp_mv_variant(C.S1_TILED, A[:, :101], dev(synth.vector(101, "f32_int4")))
    assert ei.value.status == C.ERR_UNSUPPORTED
    xb = torch.zeros(105, device="cuda")
    with pytest.raises(C.CudanpError) as ei:
        C.cudanp_mv_variant(C.S1_TILED, A, xb[1:])
    assert ei.value.status == C.ERR_UNSUPPORTED


def test_s1_tiled_full_size_C2_C4_sampled():
    """The tiled S = 1 kernels at the sizes the bench / sweep time them."""
    n = 16384
    A = torch.empty(n, n, dtype=torch.float32, device="cuda")
    C.cudanp_generate(A, "f32_unit", stream_id=1)
    x = torch.empty(n, dtype=torch.float32, device="cuda")
    C.cudanp_generate(x, "f32_unit", stream_id=2)
    idx = _sample_idx(n, 11)
    assert_rel(host(C.cudanp_mv_variant(C.S1_TILED, A, x))[idx], O.mv_gen(n, n, idx), n, "C2 mv tiled")
    assert_rel(host(C.cudanp_tmv_variant(C.S1_TILED, A, x))[idx], O.tmv_gen(n, n, idx), n, "C2 tmv tiled")
    del A
    torch.cuda.empty_cache()
    N = 1 << 21
    items = _sample_idx(N, 12, 256)
    sel = torch.from_numpy(items).cuda()
    for L in (64, 1024):
        xi = torch.empty(N, L, dtype=torch.int32, device="cuda")
        C.cudanp_generate(xi, "i32_small", stream_id=1, B=1 << 15)
        out = C.cudanp_batched_loop_scan_variant(C.S1_TILED, xi)
        assert_exact(host(out[sel]), O.scan_gen(L, items, O.I32, "i32_small", B=1 << 15), f"C4 tiled L={L}")
        del xi, out
        torch.cuda.empty_cache()
