"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle,
element by element, on the same seeded inputs.

Bar (BASELINE.json north_star):
  * int32 reduce / scan, every max, and fp32 on exactly-representable data
    (pin P3): bit-exact;
  * fp32 sums on positive data: max relative error <= tol(L) =
    1e-5 * max(1, sqrt(L/4096)) (reading R17), against the fp64 oracle.
Sizes span several tiles/waves and ragged tails; the full-size checks run in
the same launch configuration bench.py times, on sampled outputs the oracle
computes one by one.
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

SS = C.SLAVE_SIZES
DISTS = (C.CYCLIC, C.BLOCK)
MAPS = (C.INTRA_WARP, C.INTER_WARP)


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
    denom = np.maximum(np.abs(ref), 1e-30)
    err = np.max(np.abs(got - ref) / denom)
    assert err <= tol(L), f"{what}: max rel err {err:.3e} > {tol(L):.3e}"


def assert_exact(got, ref, what):
    got = np.asarray(got)
    ref = np.asarray(ref)
    assert got.shape == ref.shape, what
    if not np.array_equal(got.view(np.uint32) if got.dtype == np.float32 else got,
                          ref.view(np.uint32) if ref.dtype == np.float32 else ref):
        bad = np.argwhere(got != ref)
        raise AssertionError(f"{what}: {len(bad)} mismatches, first at {bad[:3].tolist()}: "
                             f"got {got[tuple(bad[0])]} want {ref[tuple(bad[0])]}")


# ------------------------------------------------------------------ infrastructure pins
def test_device_generator_matches_oracle_generator():
    # pin P8: three independent implementations of the generator agree
    for kind, n in [("f32_unit", 4099), ("f32_signed", 1000), ("f32_int4", 777)]:
        t = torch.empty(n, dtype=torch.float32, device="cuda")
        C.cudanp_generate(t, kind, stream_id=2, col0=(1 << 32) - 5)
        assert_exact(host(t), O.gen_f32(2, kind, (1 << 32) - 5, n), kind)
    for kind, B_ in [("i32_small", 1 << 20), ("i32_small", 1 << 15), ("i32_full", 1)]:
        t = torch.empty(5000, dtype=torch.int32, device="cuda")
        C.cudanp_generate(t, kind, stream_id=1, B=B_)
        assert_exact(host(t), O.gen_i32(1, kind, 0, 5000, B_), kind)
    # 2-D column shard of a wider matrix, with a padded leading dimension
    buf = torch.full((7, 12), -1.0, device="cuda")
    C.cudanp_generate(buf[:, :9], "f32_unit", row0=3, col0=20, w_global=50)
    want = synth.matrix(7, 9, "f32_unit", row0=3, col0=20, w_global=50)
    got = host(buf)
    assert_exact(got[:, :9], want, "2-D shard")
    assert (got[:, 9:] == -1).all()


def test_owner_map_is_the_papers_distribution():
    # the kernels' own Range code, run on the device, against the oracle's
    # restatement of P:166 / P:294 (cyclic) and reading R5 (block)
    for L in [0, 1, 3, 12, 31, 32, 33, 150, 1000, 4096]:
        for S in SS:
            for dist in DISTS:
                for V in (1, 4):
                    got = C.cudanp_debug_owner_map(L, S, dist, V)
                    assert_exact(got, O.owner_map(L, S, dist, V), f"L={L} S={S} dist={dist} V={V}")
    # loop count 12, slave_size 8 -> 4 slaves take 2 iterations, 4 take 1
    assert np.bincount(C.cudanp_debug_owner_map(12, 8, C.CYCLIC, 1)).tolist() == [2, 2, 2, 2, 1, 1, 1, 1]


def test_team_ids_match_paper_remap():
    for S in SS:
        m, s = C.cudanp_debug_team_ids(S, C.INTRA_WARP)
        om, os_ = O.team_ids(S, O.INTRA_WARP, len(m))
        assert_exact(m, om, f"intra master S={S}")
        assert_exact(s, os_, f"intra slave S={S}")
        m, s = C.cudanp_debug_team_ids(S, C.INTER_WARP)
        assert len(m) == 32 * S  # CTA = 32 masters x S slaves
        om, os_ = O.team_ids(S, O.INTER_WARP, len(m))
        assert_exact(m, om, f"inter master S={S}")
        assert_exact(s, os_, f"inter slave S={S}")


def test_read_from_master_broadcast():
    # every team member receives its master's value
    for S in SS:
        out = C.cudanp_debug_broadcast(S, C.INTRA_WARP)
        t = np.arange(len(out))
        assert_exact(out, (1000 * (t - t % S) + 7).astype(np.int32), f"intra S={S}")
        out = C.cudanp_debug_broadcast(S, C.INTER_WARP)
        t = np.arange(len(out))
        assert_exact(out, (1000 * (t % 32) + 7).astype(np.int32), f"inter S={S}")


# ------------------------------------------------------------------ batched reduce
REDUCE_SHAPES = [(0, 7), (1, 1), (3, 0), (33, 5), (70, 12), (257, 32), (300, 33), (129, 80),
                 (200, 150), (97, 256), (1100, 64)]


def _reduce_cases():
    # (dtype, op, kind, exact)
    return [(C.F32, C.SUM, "f32_unit", False), (C.F32, C.SUM, "f32_int4", True),
            (C.F32, C.MAX, "f32_signed", True), (C.I32, C.SUM, "i32_full", True),
            (C.I32, C.MAX, "i32_full", True)]


@pytest.mark.parametrize("case", _reduce_cases(), ids=lambda c: f"{c[0]}-{c[1]}-{c[2]}")
def test_reduce_parity(case):
    dtype, op, kind, exact = case
    for N, L in REDUCE_SHAPES:
        x = synth.items(N, L, kind)
        ini = synth.init(N, kind)
        ref = O.reduce(x, op=op)
        ref_i = O.reduce(x, op=op, init=ini)
        xd, inid = dev(x), dev(ini)
        for S, dist, map_ in itertools.product(SS, DISTS, MAPS):
            what = f"reduce {kind} op={op} N={N} L={L} S={S} dist={dist} map={map_}"
            got = host(C.cudanp_batched_loop_reduce(xd, op=op, S=S, dist=dist, map=map_))
            got_i = host(C.cudanp_batched_loop_reduce(xd, inid, op=op, S=S, dist=dist, map=map_))
            if exact:
                assert_exact(got, ref, what)
                assert_exact(got_i, ref_i, what + " init")
            else:
                assert_rel(got, ref, L, what)
                assert_rel(got_i, ref_i, L, what + " init")


def test_reduce_scalar_path_misaligned():
    # a base pointer off 16-byte alignment: intra-warp teams peel each row to
    # its 16-byte boundary (head/body/tail), inter-warp teams take the scalar path
    N, L = 300, 64
    x = synth.items(N + 1, L, "i32_full").reshape(-1)
    xd = dev(x)
    view = xd[1:1 + N * L].view(N, L)
    assert view.data_ptr() % 16 != 0
    ref = O.reduce(x[1:1 + N * L].reshape(N, L))
    for S, dist, map_ in itertools.product(SS, DISTS, MAPS):
        assert_exact(host(C.cudanp_batched_loop_reduce(view, S=S, dist=dist, map=map_)), ref,
                     f"misaligned S={S} dist={dist} map={map_}")


def test_reduce_peeled_rows_every_alignment():
    """Rows not 16-byte aligned (L % 4 != 0, or a base off by 1-3 elements):
    the intra-warp kernel peels a head of <= 3 elements, streams the aligned
    body in 128-bit units and finishes a tail of <= 3; every head/tail length
    and every (S, dist) against the oracle."""
    for L in (1, 2, 3, 5, 6, 7, 13, 150, 151, 1023):
        N = 203
        x = synth.items(N + 1, L, "i32_full", seed=L).reshape(-1)
        xf = synth.items(N + 1, L, "f32_int4", seed=L).reshape(-1)
        xd, xfd = dev(x), dev(xf)
        for sh in range(4):
            if sh * 1 + N * L > x.size:
                continue
            ref = O.reduce(x[sh:sh + N * L].reshape(N, L))
            ref_m = O.reduce(x[sh:sh + N * L].reshape(N, L), op=O.MAX)
            ref_f = O.reduce(xf[sh:sh + N * L].reshape(N, L))
            v, vf = xd[sh:sh + N * L].view(N, L), xfd[sh:sh + N * L].view(N, L)
            for S, dist in itertools.product(SS, DISTS):
                what = f"peel L={L} shift={sh} S={S} dist={dist}"
                assert_exact(host(C.cudanp_batched_loop_reduce(v, S=S, dist=dist, map=C.INTRA_WARP)), ref, what)
                assert_exact(host(C.cudanp_batched_loop_reduce(v, op=C.MAX, S=S, dist=dist, map=C.INTRA_WARP)),
                             ref_m, what + " max")
                assert_exact(host(C.cudanp_batched_loop_reduce(vf, S=S, dist=dist, map=C.INTRA_WARP)), ref_f,
                             what + " f32 exact data")


def test_reduce_int32_wrap_and_closed_forms():
    x = np.full((64, 8), 1 << 30, np.int32)
    for S in SS:
        assert (host(C.cudanp_batched_loop_reduce(dev(x), S=S)) == 0).all()
    ones = torch.ones(100, 256, dtype=torch.int32, device="cuda")
    for S in SS:
        assert (host(C.cudanp_batched_loop_reduce(ones, S=S)) == 256).all()
    # L = 0 -> init or the identity
    e = torch.empty(5, 0, dtype=torch.float32, device="cuda")
    assert (host(C.cudanp_batched_loop_reduce(e, op=C.MAX)) == -np.inf).all()
    ini = dev(np.arange(5, dtype=np.float32))
    assert (host(C.cudanp_batched_loop_reduce(e, ini)) == np.arange(5)).all()


# ------------------------------------------------------------------ batched scan
SCAN_SHAPES = [(0, 8), (1, 1), (33, 5), (70, 12), (100, 64), (41, 80), (37, 150), (64, 256),
               (20, 1024), (9, 1000)]


@pytest.mark.parametrize("case", [(C.I32, "i32_small", True), (C.F32, "f32_int4", True),
                                  (C.F32, "f32_unit", False)], ids=lambda c: c[1])
def test_scan_parity(case):
    dtype, kind, exact = case
    for N, L in SCAN_SHAPES:
        B_ = 1 << 15
        x = synth.items(N, L, kind, B=B_)
        ini = synth.init(N, kind, B=B_)
        ref = O.scan(x)
        ref_i = O.scan(x, init=ini)
        xd, inid = dev(x), dev(ini)
        for S, dist, map_ in itertools.product(SS, DISTS, MAPS):
            what = f"scan {kind} N={N} L={L} S={S} dist={dist} map={map_}"
            got = host(C.cudanp_batched_loop_scan(xd, S=S, dist=dist, map=map_))
            got_i = host(C.cudanp_batched_loop_scan(xd, inid, S=S, dist=dist, map=map_))
            if exact:
                assert_exact(got, ref, what)
                assert_exact(got_i, ref_i, what + " init")
            else:
                assert_rel(got, ref, L, what)
                assert_rel(got_i, ref_i, L, what + " init")


def test_scan_closed_forms_and_L0():
    for S in SS:
        ones = torch.ones(50, 1024, dtype=torch.int32, device="cuda")
        got = host(C.cudanp_batched_loop_scan(ones, S=S))
        assert (got == np.arange(1, 1025)).all()
    out = torch.full((4, 0), 7, dtype=torch.int32, device="cuda")
    C.cudanp_batched_loop_scan(torch.empty(4, 0, dtype=torch.int32, device="cuda"), out=out)


def test_scan_misaligned_output():
    N, L = 50, 64
    x = synth.items(N, L, "i32_small")
    xd = dev(x)
    buf = torch.zeros(N * L + 1, dtype=torch.int32, device="cuda")
    out = buf[1:].view(N, L)
    for S, dist, map_ in itertools.product(SS, DISTS, MAPS):
        C.cudanp_batched_loop_scan(xd, out=out, S=S, dist=dist, map=map_)
        assert_exact(host(out), O.scan(x), f"misaligned out S={S} dist={dist} map={map_}")


# ------------------------------------------------------------------ TMV / MV
MAT_SHAPES = [(0, 8), (8, 0), (1, 1), (3, 5), (37, 131), (300, 260), (129, 512), (1024, 1024)]


@pytest.mark.parametrize("kind", ["f32_unit", "f32_int4"])
def test_tmv_parity(kind):
    for h, w in MAT_SHAPES:
        A = synth.matrix(h, w, kind)
        x = synth.vector(h, kind)
        ref = O.tmv(A, x, w) if h else np.zeros(w, np.float32)
        Ad, xd = dev(A), dev(x)
        for S, dist, map_ in itertools.product(SS, DISTS, MAPS):
            what = f"tmv {kind} h={h} w={w} S={S} dist={dist} map={map_}"
            got = host(C.cudanp_tmv(Ad, xd, S=S, dist=dist, map=map_)) if w else np.zeros(0, np.float32)
            if kind == "f32_int4":
                assert_exact(got, ref, what)
            else:
                assert_rel(got, ref, h, what)


@pytest.mark.parametrize("kind", ["f32_unit", "f32_int4"])
def test_mv_parity(kind):
    for h, w in MAT_SHAPES:
        A = synth.matrix(h, w, kind)
        x = synth.vector(w, kind)
        ref = O.mv(A, x, w) if h else np.zeros(0, np.float32)
        Ad, xd = dev(A), dev(x)
        for S, dist, map_ in itertools.product(SS, DISTS, MAPS):
            what = f"mv {kind} h={h} w={w} S={S} dist={dist} map={map_}"
            got = host(C.cudanp_mv(Ad, xd, S=S, dist=dist, map=map_)) if h else np.zeros(0, np.float32)
            if kind == "f32_int4":
                assert_exact(got, ref, what)
            else:
                assert_rel(got, ref, w, what)


def test_matvec_padded_lda_and_scalar_path():
    h, w, lda = 70, 45, 52   # w % 4 != 0 -> scalar path; lda > w
    full = synth.matrix(h, lda, "f32_int4")
    A = full.copy()
    A[:, w:] = np.nan
    x_t = synth.vector(h, "f32_int4")
    x_m = synth.vector(w, "f32_int4")
    Ad = dev(A)
    for S, dist, map_ in itertools.product(SS, DISTS, MAPS):
        got = host(C.cudanp_tmv(Ad, dev(x_t), S=S, dist=dist, map=map_, n_outer=w))
        assert_exact(got, O.tmv(A, x_t, w), f"tmv lda S={S} dist={dist} map={map_}")
        got = host(C.cudanp_mv(Ad, dev(x_m), S=S, dist=dist, map=map_, n_inner=w))
        assert_exact(got, O.mv(A, x_m, w), f"mv lda S={S} dist={dist} map={map_}")


def test_tmv_closed_forms():
    h, w = 1024, 512
    x = synth.vector(h, "f32_unit")
    ones = torch.ones(h, w, device="cuda")
    ref = O.tmv(np.ones((h, w), np.float32), x)
    A = synth.matrix(h, w, "f32_signed")
    for S in SS:
        assert_rel(host(C.cudanp_tmv(ones, dev(x), S=S)), ref, h, f"ones S={S}")
        e = np.zeros(h, np.float32)
        e[77] = 1
        assert_exact(host(C.cudanp_tmv(dev(A), dev(e), S=S)), A[77], f"e_k S={S}")


# ------------------------------------------------------------------ comparison kernels
@pytest.mark.parametrize("impl", [C.S1_LITERAL, C.DP_THREAD, C.DP_BLOCK])
def test_variants_parity(impl):
    C.cudanp_dp_set_pending_launch_limit(1 << 16)
    C.cudanp_dp_error_count(reset=True)
    h, w = 300, 260
    A = synth.matrix(h, w, "f32_int4")
    xt, xm = synth.vector(h, "f32_int4"), synth.vector(w, "f32_int4")
    assert_exact(host(C.cudanp_tmv_variant(impl, dev(A), dev(xt))), O.tmv(A, xt), f"tmv impl={impl}")
    assert_exact(host(C.cudanp_mv_variant(impl, dev(A), dev(xm))), O.mv(A, xm), f"mv impl={impl}")
    Au = synth.matrix(h, w, "f32_unit")
    xu = synth.vector(h, "f32_unit")
    assert_rel(host(C.cudanp_tmv_variant(impl, dev(Au), dev(xu))), O.tmv(Au, xu), h, "tmv unit")
    for N, L in [(1, 1), (300, 33), (1000, 64), (77, 1000)]:
        for dtype, op, kind in [(C.I32, C.SUM, "i32_full"), (C.F32, C.MAX, "f32_signed"),
                                (C.I32, C.MAX, "i32_full")]:
            x = synth.items(N, L, kind)
            ini = synth.init(N, kind)
            got = host(C.cudanp_batched_loop_reduce_variant(impl, dev(x), dev(ini), op=op))
            assert_exact(got, O.reduce(x, op=op, init=ini), f"reduce impl={impl} N={N} L={L}")
        x = synth.items(N, L, "f32_unit")
        got = host(C.cudanp_batched_loop_reduce_variant(impl, dev(x)))
        assert_rel(got, O.reduce(x), L, f"reduce f32 impl={impl}")
        xi = synth.items(N, L, "i32_small")
        ini = synth.init(N, "i32_small")
        got = host(C.cudanp_batched_loop_scan_variant(impl, dev(xi), dev(ini)))
        assert_exact(got, O.scan(xi, init=ini), f"scan impl={impl} N={N} L={L}")
        x = synth.items(N, L, "f32_unit")
        assert_rel(host(C.cudanp_batched_loop_scan_variant(impl, dev(x))), O.scan(x), L, "scan f32")
    assert C.cudanp_dp_error_count(reset=True) == 0


# ------------------------------------------------------------------ full-size, bench configuration
def _gen_matrix(h, w, kind):
    A = torch.empty(h, w, dtype=torch.float32, device="cuda")
    C.cudanp_generate(A, kind, stream_id=1)
    return A


def _gen_vec(n, kind, stream_id=2, dtype=torch.float32):
    v = torch.empty(n, dtype=dtype, device="cuda")
    C.cudanp_generate(v, kind, stream_id=stream_id)
    return v


def test_full_size_C2_tmv_mv_sampled():
    """C2: 16384 x 16384 fp32, every S x dist x map (bench's sweep), sampled
    against the oracle computing each sampled output from the generator."""
    n = 16384
    A = _gen_matrix(n, n, "f32_unit")
    x = _gen_vec(n, "f32_unit")
    rng = np.random.default_rng(0)
    idx = np.unique(np.concatenate([rng.integers(0, n, 256), [0, 1, n - 2, n - 1]]))
    ref_t = O.tmv_gen(n, n, idx)
    ref_m = O.mv_gen(n, n, idx)
    for S, dist, map_ in itertools.product(SS, DISTS, MAPS):
        yt = host(C.cudanp_tmv(A, x, S=S, dist=dist, map=map_))
        assert_rel(yt[idx], ref_t, n, f"C2 tmv S={S} dist={dist} map={map_}")
        ym = host(C.cudanp_mv(A, x, S=S, dist=dist, map=map_))
        assert_rel(ym[idx], ref_m, n, f"C2 mv S={S} dist={dist} map={map_}")
    # exact-data invariant at full size: every variant gives identical bits (P3/P4)
    C.cudanp_generate(A, "f32_int4", stream_id=1)
    C.cudanp_generate(x, "f32_int4", stream_id=2)
    base = host(C.cudanp_tmv(A, x, S=1))
    assert_exact(base[idx], O.tmv_gen(n, n, idx, "f32_int4", "f32_int4"), "C2 tmv int4")
    for S, dist, map_ in itertools.product(SS, DISTS, MAPS):
        assert_exact(host(C.cudanp_tmv(A, x, S=S, dist=dist, map=map_)), base, f"P4 S={S}")
    del A
    torch.cuda.empty_cache()


def test_full_size_C1_tmv_all_outputs():
    n = 1024
    A = _gen_matrix(n, n, "f32_unit")
    x = _gen_vec(n, "f32_unit")
    # inputs regenerated by the oracle's own generator (never read back from the GPU)
    ref = O.tmv(O.gen_f32(1, "f32_unit", 0, n * n).reshape(n, n), O.gen_f32(2, "f32_unit", 0, n))
    for S, dist, map_ in itertools.product(SS, DISTS, MAPS):
        assert_rel(host(C.cudanp_tmv(A, x, S=S, dist=dist, map=map_)), ref, n, f"C1 S={S}")
    assert_rel(host(C.cudanp_tmv_variant(C.S1_LITERAL, A, x)), ref, n, "C1 literal")


def test_full_size_C3_reduce_sampled():
    N = 1 << 22
    rng = np.random.default_rng(1)
    items = np.unique(np.concatenate([rng.integers(0, N, 2048), [0, N - 1]]))
    for L in (32, 256):
        x = torch.empty(N, L, dtype=torch.float32, device="cuda")
        C.cudanp_generate(x, "f32_unit", stream_id=1)
        ref = O.reduce_gen(L, items, O.F32, "f32_unit")
        for S, dist in itertools.product(SS, DISTS):
            got = host(C.cudanp_batched_loop_reduce(x, S=S, dist=dist, map=C.INTRA_WARP))
            assert_rel(got[items], ref, L, f"C3 L={L} S={S} dist={dist}")
        del x
        xi = torch.empty(N, L, dtype=torch.int32, device="cuda")
        C.cudanp_generate(xi, "i32_full", stream_id=1)
        ref = O.reduce_gen(L, items, O.I32, "i32_full", op=O.MAX)
        for S in SS:
            got = host(C.cudanp_batched_loop_reduce(xi, op=C.MAX, S=S))
            assert_exact(got[items], ref, f"C3 i32 max L={L} S={S}")
        del xi
        torch.cuda.empty_cache()


def test_full_size_C4_scan_sampled():
    N, L = 1 << 21, 256
    rng = np.random.default_rng(2)
    items = np.unique(np.concatenate([rng.integers(0, N, 512), [0, N - 1]]))
    x = torch.empty(N, L, dtype=torch.int32, device="cuda")
    C.cudanp_generate(x, "i32_small", stream_id=1, B=1 << 15)
    ref = O.scan_gen(L, items, O.I32, "i32_small", B=1 << 15)
    out = torch.empty_like(x)
    for S, dist in itertools.product(SS, DISTS):
        C.cudanp_batched_loop_scan(x, out=out, S=S, dist=dist, map=C.INTRA_WARP)
        got = host(out[torch.from_numpy(items).cuda()])
        assert_exact(got, ref, f"C4 scan S={S} dist={dist}")
    del x, out
    torch.cuda.empty_cache()


# ------------------------------------------------------------------ Fig 16 ablation backends
@pytest.mark.parametrize("backend", [C.SHFL, C.SMEM, C.REDUX])
def test_reduce_backend_parity(backend):
    for N, L in [(1, 4), (70, 12), (300, 32), (97, 256), (1100, 64)]:
        for dtype, op, kind, exact in [(C.I32, C.SUM, "i32_full", True), (C.I32, C.MAX, "i32_full", True),
                                       (C.F32, C.MAX, "f32_signed", True), (C.F32, C.SUM, "f32_unit", False)]:
            x = synth.items(N, L, kind)
            ini = synth.init(N, kind)
            ref = O.reduce(x, op=op, init=ini)
            for S in SS:
                what = f"backend={backend} {kind} op={op} N={N} L={L} S={S}"
                if backend == C.REDUX and dtype == C.F32 and op == C.SUM:
                    with pytest.raises(C.CudanpError) as ei:
                        C.cudanp_batched_loop_reduce_backend(dev(x), dev(ini), op=op, S=S, backend=backend)
                    assert ei.value.status == C.ERR_UNSUPPORTED
                    continue
                got = host(C.cudanp_batched_loop_reduce_backend(dev(x), dev(ini), op=op, S=S, backend=backend))
                if exact:
                    assert_exact(got, ref, what)
                else:
                    assert_rel(got, ref, L, what)


# ------------------------------------------------------------------ edge shapes around team/tile sizes
def test_edge_shapes_per_S():
    """N around the masters per CTA / warp tile (31, 32, 33, tile +- 1) and L
    around S and 4S (S-1, S, S+1, 4S-1, 4S, 4S+1): every tail of the team,
    warp-tile and vector-unit logic (SURVEY §4 test plan item 2)."""
    for S in SS:
        tile = 8 * (32 // S) * 4  # intra-warp reduce: 8 warps x (32/S) items x K=4 tiles
        Ns = sorted({1, 31, 32, 33, tile - 1, tile, tile + 1})
        Ls = sorted({max(S - 1, 0), S, S + 1, 4 * S - 1, 4 * S, 4 * S + 1})
        for N in Ns:
            for L in Ls:
                x = synth.items(N, L, "i32_full", seed=N * 131 + L)
                ini = synth.init(N, "i32_full", seed=L)
                rr, rs = O.reduce(x, init=ini), O.scan(x, init=ini)
                xd, inid = dev(x), dev(ini)
                for dist, map_ in itertools.product(DISTS, MAPS):
                    what = f"edge S={S} N={N} L={L} dist={dist} map={map_}"
                    assert_exact(host(C.cudanp_batched_loop_reduce(xd, inid, S=S, dist=dist, map=map_)), rr, what)
                    assert_exact(host(C.cudanp_batched_loop_scan(xd, inid, S=S, dist=dist, map=map_)), rs, what)
        # TMV/MV widths around 32*V column strips and 8-master CTAs
        for w in (31, 32, 33, 127, 128, 129):
            h = 4 * S + 1
            A = synth.matrix(h, w, "f32_int4", seed=w)
            xt, xm = synth.vector(h, "f32_int4"), synth.vector(w, "f32_int4")
            for dist, map_ in itertools.product(DISTS, MAPS):
                what = f"edge matvec S={S} h={h} w={w} dist={dist} map={map_}"
                assert_exact(host(C.cudanp_tmv(dev(A), dev(xt), S=S, dist=dist, map=map_)), O.tmv(A, xt), what)
                assert_exact(host(C.cudanp_mv(dev(A), dev(xm), S=S, dist=dist, map=map_)), O.mv(A, xm), what)


def test_full_size_C5_single_gpu_sampled():
    """C5 at G=1: TMV 65536^2 (16 GiB) and the 64M-item reduce, sampled."""
    n = 65536
    A = _gen_matrix(n, n, "f32_unit")
    x = _gen_vec(n, "f32_unit")
    rng = np.random.default_rng(11)
    cols = np.unique(np.concatenate([rng.integers(0, n, 128), [0, n - 1]]))
    ref = O.tmv_gen(n, n, cols)
    for S, dist in itertools.product((8, 16, 32), DISTS):
        y = host(C.cudanp_tmv(A, x, S=S, dist=dist, map=C.INTER_WARP))
        assert_rel(y[cols], ref, n, f"C5 tmv S={S} dist={dist}")
    del A
    torch.cuda.empty_cache()
    N, L = 1 << 26, 64
    X = torch.empty(N, L, device="cuda")
    C.cudanp_generate(X, "f32_unit", stream_id=1)
    items = np.unique(np.concatenate([rng.integers(0, N, 2048), [0, N - 1]]))
    ref = O.reduce_gen(L, items, O.F32, "f32_unit")
    for S, dist in itertools.product((4, 8, 16), DISTS):
        got = host(C.cudanp_batched_loop_reduce(X, S=S, dist=dist, map=C.INTRA_WARP))
        assert_rel(got[items], ref, L, f"C5 reduce S={S} dist={dist}")
    del X
    torch.cuda.empty_cache()


# ------------------------------------------------------------------ TMA-staged TMV
def test_tmv_tma_parity():
    for h, w in [(1, 4), (37, 128), (300, 260), (1000, 516), (1024, 1024), (4097, 132)]:
        for kind in ("f32_int4", "f32_unit"):
            A = synth.matrix(h, w, kind)
            x = synth.vector(h, kind)
            ref = O.tmv(A, x)
            Ad, xd = dev(A), dev(x)
            for S, dist in itertools.product(SS, DISTS):
                got = host(C.cudanp_tmv_tma(Ad, xd, S=S, dist=dist))
                what = f"tma h={h} w={w} {kind} S={S} dist={dist}"
                # the same kernel through cudanp_tmv's map argument
                assert_exact(host(C.cudanp_tmv(Ad, xd, S=S, dist=dist, map=C.INTER_WARP_TMA)), got, what)
                if kind == "f32_int4":
                    assert_exact(got, ref, what)
                else:
                    assert_rel(got, ref, h, what)
    # padded lda, and the unsupported cases
    A = synth.matrix(50, 72, "f32_int4")
    xd = dev(synth.vector(50, "f32_int4"))
    got = host(C.cudanp_tmv_tma(dev(A), xd, S=4, n_outer=64))
    assert_exact(got, O.tmv(A, synth.vector(50, "f32_int4"), 64), "tma lda")
    with pytest.raises(C.CudanpError) as ei:
        C.cudanp_tmv_tma(dev(synth.matrix(5, 6, "f32_int4")), dev(synth.vector(5, "f32_int4")))
    assert ei.value.status == C.ERR_UNSUPPORTED


def test_tmv_tma_pinned_shapes_parity():
    # every strip width x rows-per-slave x ring depth, with rings that wrap
    # many times, ragged last strips and rows past h (zero-filled by TMA)
    for h, w in [(1000, 516), (2049, 1028)]:
        A = synth.matrix(h, w, "f32_int4")
        x = synth.vector(h, "f32_int4")
        ref = O.tmv(A, x)
        Ad, xd = dev(A), dev(x)
        ran = 0
        for S, dist, cols, rs, st in itertools.product(SS, DISTS, (32, 64, 128), (0, 1, 2), (2, 3)):
            try:
                got = host(C.cudanp_tmv_tma(Ad, xd, S=S, dist=dist, cols=cols, rows_sel=rs, stages=st))
            except C.CudanpError as e:   # this ring does not fit 227 KB
                assert e.status == C.ERR_INVALID
                continue
            ran += 1
            assert_exact(got, ref, f"tma h={h} w={w} S={S} dist={dist} cols={cols} rs={rs} st={st}")
        assert ran >= 180
    with pytest.raises(C.CudanpError) as ei:   # a ring larger than shared memory
        C.cudanp_tmv_tma(Ad, xd, S=32, cols=128, rows_sel=1, stages=64)
    assert ei.value.status == C.ERR_INVALID
    info = C.cudanp_launch_info("tmv_tma", 16384, 16384, S=8)
    # a producer warp beside the 8 slave warps; one CTA per strip of 32/64/128 columns
    assert info["block_threads"] == 32 * 8 + 32 and info["grid_ctas"] in (128, 256, 512)
    assert 0 < info["smem_bytes"] <= 227 * 1024


def test_tmv_tma_full_size_C2():
    n = 16384
    A = _gen_matrix(n, n, "f32_unit")
    x = _gen_vec(n, "f32_unit")
    cols = np.arange(0, n, 61)
    ref = O.tmv_gen(n, n, cols)
    for S, dist in itertools.product(SS, DISTS):
        assert_rel(host(C.cudanp_tmv_tma(A, x, S=S, dist=dist))[cols], ref, n, f"C2 tma S={S} d={dist}")
    del A
    torch.cuda.empty_cache()


# ------------------------------------------------------------------ teams larger than a warp
BIG_S = (64, 128, 256, 512, 1024)


def test_big_teams_parity():
    """S > 32: S/32 consecutive warps, shfl inside each warp + shared memory
    across them (the north star's "shared-memory fallback when S exceeds 32")."""
    for N, L in [(1, 1), (3, 0), (7, 1000), (70, 4096), (33, 333), (300, 64)]:
        x = synth.items(N, L, "i32_full", seed=L)
        ini = synth.init(N, "i32_full", seed=N)
        xs = synth.items(N, L, "i32_small", B=1 << 15, seed=L)
        xd, inid, xsd = dev(x), dev(ini), dev(xs)
        ref_s, ref_m = O.reduce(x, init=ini), O.reduce(x, op=O.MAX)
        ref_scan = O.scan(xs, init=ini)
        xf = synth.items(N, L, "f32_unit", seed=L)
        ref_f = O.reduce(xf)
        for S, dist in itertools.product(BIG_S, DISTS):
            what = f"big S={S} N={N} L={L} dist={dist}"
            assert_exact(host(C.cudanp_batched_loop_reduce(xd, inid, S=S, dist=dist)), ref_s, what)
            assert_exact(host(C.cudanp_batched_loop_reduce(xd, op=C.MAX, S=S, dist=dist)), ref_m, what)
            assert_exact(host(C.cudanp_batched_loop_scan(xsd, inid, S=S, dist=dist)), ref_scan, what)
            assert_rel(host(C.cudanp_batched_loop_reduce(dev(xf), S=S, dist=dist)), ref_f, L, what)
            with pytest.raises(C.CudanpError) as ei:
                C.cudanp_batched_loop_reduce(xd, S=S, dist=dist, map=C.INTER_WARP)
            assert ei.value.status == C.ERR_UNSUPPORTED
    for h, w in [(5, 4096), (64, 1000), (300, 260), (2, 65536)]:
        A = synth.matrix(h, w, "f32_int4", seed=w)
        xm, xt = synth.vector(w, "f32_int4"), synth.vector(h, "f32_int4")
        for S, dist in itertools.product(BIG_S, DISTS):
            assert_exact(host(C.cudanp_mv(dev(A), dev(xm), S=S, dist=dist)), O.mv(A, xm), f"mv big S={S}")
            if S <= 128:
                assert_exact(host(C.cudanp_tmv(dev(A), dev(xt), S=S, dist=dist)), O.tmv(A, xt),
                             f"tmv big S={S} h={h} w={w}")
    # TMV S = 64 / 128, every CTA layout the call picks (abi.cu tmv_vec): V = 4 with 4
    # column-masters (short or 16-column-rich matrices, C1), V = 4 with 8 (w >= 32 x SMs),
    # V = 1 (tall narrow or unaligned); ragged last CTAs; cold HBM via the L2 prefetch.
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    for h, w, mx_v in [(1024, 1024, (4, 4)), (1500, 2052, (4, 4)), (7, 1028, (4, 4)),
                       (300, 32 * sms + 64, (8, 4)), (3000, 1024, (8, 1)), (1024, 1022, (8, 1))]:
        A = synth.matrix(h, w, "f32_int4", seed=h + w)
        xt = synth.vector(h, "f32_int4")
        ref = O.tmv(A, xt)
        for S, dist in itertools.product((64, 128), DISTS):
            i = C.cudanp_launch_info("tmv", w, h, S=S, dist=dist, map=C.INTER_WARP, vec4=w % 4 == 0)
            assert (i["block_threads"] // S, -(-w // i["grid_ctas"])) == (mx_v[0], mx_v[0] * mx_v[1]), \
                f"layout h={h} w={w} S={S}: {i}"
            assert_exact(host(C.cudanp_tmv(dev(A), dev(xt), S=S, dist=dist, map=C.INTER_WARP)), ref,
                         f"tmv S={S} h={h} w={w} dist={dist} layout={mx_v}")
    # TMV with a cluster team per column group (S = 256 / 1024: 8 CTAs x 32 / 128 slave warps)
    for h, w in [(5, 4096), (64, 1000), (300, 260), (20000, 36), (70000, 3), (1, 1), (0, 7)]:
        A = synth.matrix(h, w, "f32_int4", seed=w)
        xt = synth.vector(h, "f32_int4")
        ref = O.tmv(A, xt) if h else np.zeros(w, np.float32)
        for S, dist in itertools.product((256, 1024), DISTS):
            assert_exact(host(C.cudanp_tmv(dev(A), dev(xt), S=S, dist=dist)), ref,
                         f"tmv cluster S={S} h={h} w={w} dist={dist}")


CLUSTER_S = (2048, 4096, 8192)


def test_cluster_teams_parity():
    """S > 1024: the team is a thread-block cluster of 8 CTAs (DSMEM partials
    into the master CTA, one cluster barrier per item); more items than
    resident clusters exercise the grid stride and the double-buffered slots."""
    for N, L in [(1, 1), (3, 0), (5, 8193), (40, 20000), (2500, 96), (9, 65536 + 4)]:
        x = synth.items(N, L, "i32_full", seed=L)
        ini = synth.init(N, "i32_full", seed=N)
        xd, inid = dev(x), dev(ini)
        ref_s, ref_m = O.reduce(x, init=ini), O.reduce(x, op=O.MAX)
        xf = synth.items(N, L, "f32_unit", seed=L)
        xfd = dev(xf)
        ref_f = O.reduce(xf)
        for S, dist in itertools.product(CLUSTER_S, DISTS):
            what = f"cluster S={S} N={N} L={L} dist={dist}"
            assert_exact(host(C.cudanp_batched_loop_reduce(xd, inid, S=S, dist=dist)), ref_s, what)
            assert_exact(host(C.cudanp_batched_loop_reduce(xd, op=C.MAX, S=S, dist=dist)), ref_m, what)
            assert_rel(host(C.cudanp_batched_loop_reduce(xfd, S=S, dist=dist)), ref_f, L, what)
            if L > 1:  # misaligned rows: scalar units
                v = xd.view(-1)[1:].view(-1)[: N * (L - 1)].view(N, L - 1)
                assert_exact(host(C.cudanp_batched_loop_reduce(v, S=S, dist=dist)),
                             O.reduce(x.reshape(-1)[1:1 + N * (L - 1)].reshape(N, L - 1)), what + " misaligned")
    with pytest.raises(C.CudanpError) as ei:
        C.cudanp_batched_loop_reduce(dev(synth.items(4, 64, "i32_full")), S=2048, map=C.INTER_WARP)
    assert ei.value.status == C.ERR_UNSUPPORTED
    # TMV has no cluster team (CUDANP_ERR_INVALID before launch)
    with pytest.raises(C.CudanpError) as ei:
        C.cudanp_tmv(dev(synth.matrix(8, 8, "f32_int4")), dev(synth.vector(8, "f32_int4")), S=2048)
    assert ei.value.status == C.ERR_INVALID
    # scan with a cluster per item (cyclic: chunked two-pass with per-round totals over DSMEM;
    # block: chunk sums), int32 bit-exact with carry-in, fp32 exact data
    for N, L in [(1, 1), (3, 0), (5, 8193), (40, 20000), (2500, 96), (9, 65540), (4, 5), (2, 600001), (3, 1 << 20)]:
        xs = synth.items(N, L, "i32_small", B=1 << 15, seed=L)
        ini = synth.init(N, "i32_small", seed=N)
        xf = synth.items(N, L, "f32_int4", seed=L)
        ref_s, ref_f = O.scan(xs, init=ini), O.scan(xf)
        xsd, inid, xfd = dev(xs), dev(ini), dev(xf)
        for S, dist in itertools.product(CLUSTER_S, DISTS):
            what = f"scan cluster S={S} N={N} L={L} dist={dist}"
            assert_exact(host(C.cudanp_batched_loop_scan(xsd, inid, S=S, dist=dist)), ref_s, what)
            assert_exact(host(C.cudanp_batched_loop_scan(xfd, S=S, dist=dist)), ref_f, what + " f32")
            if L > 1:  # misaligned rows: scalar units
                v = xsd.view(-1)[1:1 + N * (L - 1)].view(N, L - 1)
                assert_exact(host(C.cudanp_batched_loop_scan(v, inid, S=S, dist=dist)),
                             O.scan(xs.reshape(-1)[1:1 + N * (L - 1)].reshape(N, L - 1), init=ini),
                             what + " misaligned")
    i = C.cudanp_launch_info("reduce", 256, 65536, S=4096)
    assert i["block_threads"] == 512 and i["grid_ctas"] % 8 == 0
    # MV with a cluster per row (few long rows), exact data -> bit-exact
    for h, w in [(1, 5), (3, 0), (16, 65536), (300, 1000), (7, 4099)]:
        A = synth.matrix(h, w, "f32_int4", seed=w)
        xm = synth.vector(w, "f32_int4")
        for S, dist in itertools.product(CLUSTER_S, DISTS):
            assert_exact(host(C.cudanp_mv(dev(A), dev(xm), S=S, dist=dist)), O.mv(A, xm), f"mv cluster S={S} h={h} w={w}")


def test_launch_info_and_auto_map():
    """cudanp_launch_info reports the instantiation a call would launch; MAP_AUTO
    resolves per P:340-342 (TMV -> inter-warp, MV/reduce/scan -> intra-warp),
    TMV taking the TMA-staged inter-warp kernel on wide 16-byte aligned
    matrices and the LDG one on narrow or unaligned ones."""
    for op, auto in (("tmv", "inter_warp_tma"), ("mv", "intra_warp"), ("reduce", "intra_warp"),
                     ("scan", "intra_warp")):
        for S in SS:
            i = C.cudanp_launch_info(op, 1 << 14, 1 << 10, dtype=C.F32 if op != "scan" else C.I32, S=S)
            assert i["map"] == auto, (op, S, i)
    for S in SS:
        assert C.cudanp_launch_info("tmv", 1 << 10, 1 << 10, S=S)["map"] == "inter_warp"
        assert C.cudanp_launch_info("tmv", 1 << 14, 1 << 10, S=S, vec4=False)["map"] == "inter_warp"
    for op in ("tmv", "mv", "reduce", "scan"):
        for S in SS:
            i = C.cudanp_launch_info(op, 1 << 14, 1 << 10, dtype=C.F32 if op != "scan" else C.I32, S=S)
            assert i["block_threads"] > 0 and i["grid_ctas"] > 0 and i["regs_per_thread"] > 0
            assert i["block_threads"] <= 1024
        for m in (C.INTRA_WARP, C.INTER_WARP):
            i = C.cudanp_launch_info(op, 1000, 64, S=8, map=m)
            assert i["map"] == {C.INTRA_WARP: "intra_warp", C.INTER_WARP: "inter_warp"}[m]
    # inter-warp CTA = masters x S; big teams are S/32 warps of one CTA
    assert C.cudanp_launch_info("reduce", 1000, 64, S=8, map=C.INTER_WARP)["block_threads"] == 32 * 8
    assert C.cudanp_launch_info("reduce", 1000, 64, S=512)["block_threads"] == 512
    assert C.cudanp_launch_info("mv", 1000, 4096, S=1024)["block_threads"] == 1024


def test_autotune_picks_a_valid_fastest_version():
    # the paper's exhaustive version selection, run by the library
    A = torch.empty(2048, 2048, device="cuda")
    C.cudanp_generate(A, "f32_int4")
    x = torch.empty(2048, device="cuda")
    C.cudanp_generate(x, "f32_int4", stream_id=2)
    y = torch.empty(2048, device="cuda")
    tables = {}
    for op in ("tmv", "mv"):
        best, table = C.cudanp_autotune(op, A, x, y, lda=2048, n_outer=2048, n_inner=2048, reps=2)
        tables[op] = table
        finite = {k: v for k, v in table.items() if v != float("inf")}
        assert best in finite and finite[best] == min(finite.values())
        assert len(finite) >= 24
        S, d, m = best
        fn = C.cudanp_tmv if op == "tmv" else C.cudanp_mv
        ref = (O.tmv if op == "tmv" else O.mv)(host(A), host(x))
        assert_exact(host(fn(A, x, S=S, dist=d, map=m)), ref, f"autotuned {op} {best}")
    X = torch.empty(4096, 96, dtype=torch.int32, device="cuda")
    C.cudanp_generate(X, "i32_full")
    out = torch.empty(4096, dtype=torch.int32, device="cuda")
    best, table = C.cudanp_autotune("reduce", X, None, out, n_outer=4096, n_inner=96, dtype=C.I32, reps=2)
    assert_exact(host(out), O.reduce(host(X)), "autotune reduce: last run result")
    assert table[(64, C.CYCLIC, C.INTRA_WARP)] != float("inf")  # multi-warp reduce team
    # teams larger than both a warp and the 96-iteration loop are not timed
    assert table[(128, C.CYCLIC, C.INTRA_WARP)] == float("inf")
    assert table[(8192, C.CYCLIC, C.INTRA_WARP)] == float("inf")
    # TMV's candidate list only holds the built combinations (inter-warp for S > 32)
    assert (64, C.CYCLIC, C.INTRA_WARP) not in tables["tmv"]
    assert tables["tmv"][(64, C.CYCLIC, C.INTER_WARP)] != float("inf")


# ------------------------------------------------------------------ launch overlap (PDL)
def test_chained_calls_without_sync_see_their_predecessors():
    # The hot-path kernels are launched with programmatic dependent launch, so
    # each must wait for the previous kernel before reading its output (RAW)
    # or overwriting what it still reads (WAR).  Chain calls through shared
    # buffers with no host synchronisation in between and compare with the
    # oracle applied to the same chain.
    h = w = 1024
    A = synth.matrix(h, w, "f32_int4")
    x = synth.vector(h, "f32_int4")
    it = synth.items(3000, 96, "i32_small")
    Ad, xd, itd = dev(A), dev(x), dev(it)
    y1 = torch.empty(w, device="cuda")
    y2 = torch.empty(h, device="cuda")
    sc = torch.empty_like(itd)
    red = torch.empty(3000, dtype=torch.int32, device="cuda")
    for rep in range(20):
        S = (8, 16, 32, 64)[rep % 4]
        C.cudanp_tmv(Ad, xd, y1, S=min(S, 32), map=C.INTER_WARP_TMA if rep % 2 else C.INTER_WARP)
        C.cudanp_mv(Ad, y1, y2, S=S, map=C.INTRA_WARP)          # reads y1 (RAW)
        C.cudanp_tmv(Ad, y2, y1, S=S if S <= 32 else 64, map=C.INTER_WARP)  # overwrites y1 (WAR)
        C.cudanp_batched_loop_scan(itd, None, sc, S=S, map=C.INTRA_WARP)
        C.cudanp_batched_loop_reduce(sc, None, red, S=S, map=C.INTRA_WARP)
    ref_y2 = O.mv(A, O.tmv(A, x))           # integers < 2^24: exact in any order
    assert_exact(host(y2), ref_y2, "tmv -> mv chain")
    assert_rel(host(y1), O.tmv(A, ref_y2), h, "tmv -> mv -> tmv chain")
    assert_exact(host(red), O.reduce(O.scan(it)), "scan -> reduce chain")


def test_narrow_tmv_prefetch_sees_predecessor_writes():
    # The narrow (C1-shaped) TMV prefetches A and x into L2 BEFORE its
    # dependency wait.  Each round, the two kernels launched just before it
    # (no host sync) write NEW values into the very buffers it reads: A by a
    # scan, x by a reduce.  Every round's output must be that round's product.
    h = w = 1024
    Ad = torch.empty(h, w, device="cuda")
    xd = torch.empty(h, device="cuda")
    rounds = 6
    srcA = [synth.items(h, w, "f32_int4", seed=100 + k) for k in range(rounds)]
    srcx = [synth.items(h, 16, "f32_int4", seed=200 + k) for k in range(rounds)]
    dA, dx = [dev(a) for a in srcA], [dev(a) for a in srcx]
    ys = [torch.empty(w, device="cuda") for _ in range(rounds)]
    torch.cuda.synchronize()
    for k in range(rounds):
        S = (64, 128, 32)[k % 3]
        C.cudanp_batched_loop_scan(dA[k], None, Ad, S=8, map=C.INTRA_WARP)      # writes A
        C.cudanp_batched_loop_reduce(dx[k], None, xd, S=4, map=C.INTRA_WARP)    # writes x
        C.cudanp_tmv(Ad, xd, ys[k], S=S, dist=C.BLOCK if k % 2 else C.CYCLIC, map=C.INTER_WARP)
    for k in range(rounds):
        ref = O.tmv(O.scan(srcA[k]), O.reduce(srcx[k]))
        assert_rel(host(ys[k]), ref, h, f"round {k}")


# ------------------------------------------------------------------ TMA-staged reduce
def test_reduce_tma_parity_and_identity_with_ldg():
    # same per-lane order as the LDG intra-warp kernel -> bit-identical even on
    # fp32 data; and against the oracle (exact for int32 / max, tol for fp32 sums)
    for N, L in [(1, 4), (70, 36), (1000, 32), (3001, 64), (777, 256), (50, 1024), (9, 8192)]:
        for kind, dt in (("f32_unit", C.F32), ("i32_full", C.I32)):
            X = synth.items(N, L, kind)
            ini = synth.init(N, "f32_unit" if dt == C.F32 else "i32_small")
            Xd, inid = dev(X), dev(ini)
            for op in (C.SUM, C.MAX):
                ref = O.reduce(X, op=O.SUM if op == C.SUM else O.MAX, init=ini)
                for S, dist in itertools.product(SS, DISTS):
                    got = host(C.cudanp_batched_loop_reduce(Xd, inid, op=op, S=S, dist=dist,
                                                            map=C.INTRA_WARP_TMA))
                    ldg = host(C.cudanp_batched_loop_reduce(Xd, inid, op=op, S=S, dist=dist,
                                                            map=C.INTRA_WARP))
                    what = f"reduce_tma N={N} L={L} {kind} op={op} S={S} dist={dist}"
                    assert_exact(got, ldg, what + " vs LDG kernel")
                    if dt == C.I32 or op == C.MAX:
                        assert_exact(got, ref, what)
                    else:
                        assert_rel(got, ref, L, what)
    # ring shapes: tiny stages (one item per stage, many wraps) and 2-stage rings
    X = synth.items(513, 64, "i32_small")
    Xd = dev(X)
    for sb, st in ((256, 2), (256, 3), (4096, 2), (65536, 3)):
        got = host(C.cudanp_batched_loop_reduce_tma(Xd, S=8, stage_bytes=sb, stages=st))
        assert_exact(got, O.reduce(X), f"reduce_tma stage_bytes={sb} stages={st}")
    # L = 0 writes init; misaligned / L % 4 != 0 are unsupported (the plain call handles them)
    ini = synth.init(10, "i32_small")
    got = host(C.cudanp_batched_loop_reduce_tma(dev(np.zeros((10, 0), np.int32)), dev(ini)))
    assert_exact(got, ini, "reduce_tma L=0")
    with pytest.raises(C.CudanpError) as ei:
        C.cudanp_batched_loop_reduce_tma(dev(synth.items(10, 6, "i32_small")))
    assert ei.value.status == C.ERR_UNSUPPORTED
    info = C.cudanp_launch_info("reduce_tma", 1 << 22, 32, S=4)
    assert info["block_threads"] % 32 == 0 and info["grid_ctas"] <= 148
    assert 0 < info["smem_bytes"] <= 227 * 1024


def test_reduce_tma_full_size_C3_sampled():
    N, L = 1 << 22, 32
    X = torch.empty(N, L, dtype=torch.int32, device="cuda")
    C.cudanp_generate(X, "i32_small", stream_id=1, B=1 << 20)
    items = np.concatenate([np.arange(0, N, 9973), [N - 1]])
    ref = O.reduce_gen(L, items, O.I32, "i32_small")
    for S, dist in itertools.product((2, 4, 8), DISTS):
        got = host(C.cudanp_batched_loop_reduce(X, S=S, dist=dist, map=C.INTRA_WARP_TMA))
        assert_exact(got[items], ref, f"C3 reduce_tma S={S} dist={dist}")
    del X
    torch.cuda.empty_cache()
