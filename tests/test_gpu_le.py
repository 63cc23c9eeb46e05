"""GPU parity for the LE multi-section item (Figs 5-6)."""
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
from test_gpu_parity import assert_rel, dev, host

pytestmark = pytest.mark.gpu
INTER_S = (1, 2, 3, 4, 5, 8, 10, 15, 16, 32)
INTRA_S = (1, 2, 4, 8, 16, 32)


@pytest.fixture(scope="module", autouse=True)
def _lib():
    B.build()
    C.load()


def check(got, ref, x_items, L, thr, what):
    g, a, v, e = (host(t) for t in got)
    rg, ra, rv, re_ = ref
    assert_rel(a, ra, L, what + " ave")
    assert_rel(v, rv, L, what + " var")
    # ep is a cancelling sum: normwise bound against sum |Grad - ave|
    absum = np.abs(x_items.astype(np.float64) - ra[:, None].astype(np.float64)).sum(1)
    tol = 1e-5 * max(1.0, math.sqrt(L / 4096))
    assert (np.abs(e - re_) <= tol * absum + 1e-30).all(), what + " ep"
    with np.errstate(divide="ignore", invalid="ignore"):
        ratio = (ra.astype(np.float64) ** 2) / rv
        near = np.abs(ratio - thr) <= 1e-4 * thr
    stored_ref = rg != -1
    stored = g != -1
    assert ((stored == stored_ref) | near).all(), what + " branch"
    both = stored & stored_ref
    assert_rel(g[both], rg[both], L, what + " gicov")


@pytest.mark.parametrize("layout", [0, 1])
def test_le_parity(layout):
    for N, L in [(1, 1), (33, 7), (300, 150), (129, 64), (70, 1000)]:
        xi = synth.items(N, L, "f32_unit")              # (N, L) item view
        x = xi if layout == 0 else np.ascontiguousarray(xi.T)
        _, ra, rv, _ = O.le_gicov(x, 0.0, layout)
        with np.errstate(divide="ignore"):
            thr = float(np.median(ra.astype(np.float64) ** 2 / rv))
        ref = O.le_gicov(x, thr, layout)
        xd = dev(x)
        for S, d, m in itertools.product(INTER_S, (C.CYCLIC, C.BLOCK), (C.INTRA_WARP, C.INTER_WARP)):
            if m == C.INTRA_WARP and S not in INTRA_S:
                with pytest.raises(C.CudanpError) as ei:
                    C.cudanp_le_gicov(xd, thr, layout=layout, S=S, dist=d, map=m)
                assert ei.value.status == C.ERR_UNSUPPORTED
                continue
            got = C.cudanp_le_gicov(xd, thr, layout=layout, S=S, dist=d, map=m)
            check(got, ref, xi, L, thr, f"le layout={layout} N={N} L={L} S={S} d={d} m={m}")
        got = C.cudanp_le_gicov(xd, thr, layout=layout, literal=True)
        check(got, ref, xi, L, thr, f"le literal layout={layout} N={N} L={L}")


def test_le_full_size_sampled():
    N, L = 1 << 21, 150
    x = torch.empty(L, N, device="cuda")
    C.cudanp_generate(x, "f32_unit", stream_id=1)     # point-major: idx = i*N + n
    xs = O.gen_f32(1, "f32_unit", 0, N * L).reshape(L, N)
    rng = np.random.default_rng(9)
    items = np.unique(rng.integers(0, N, 1024))
    sub = np.ascontiguousarray(xs[:, items])
    _, ra, rv, _ = O.le_gicov(sub, 0.0, 1)
    thr = float(np.median(ra.astype(np.float64) ** 2 / rv))
    ref = O.le_gicov(sub, thr, 1)
    for S, d in itertools.product((3, 4, 5, 8, 10, 15, 16), (C.CYCLIC, C.BLOCK)):
        g, a, v, e = C.cudanp_le_gicov(x, thr, layout=1, S=S, dist=d, map=C.INTER_WARP)
        idx = torch.from_numpy(items).cuda()
        check((g[idx], a[idx], v[idx], e[idx]), ref, np.ascontiguousarray(sub.T), L, thr,
              f"full le S={S} d={d}")


def test_le_grad_placements_bit_identical():
    # Fig 6a/6b/6c: the home of Grad changes where loop 3 reads it, not the
    # order a slave visits its elements -> bit-identical to the register
    # partition, and within tolerance of the oracle
    for N, L in [(1, 4), (35, 8), (300, 150), (1001, 150), (64, 1000), (8, 4096)]:
        xi = synth.items(N, L, "f32_unit")
        _, ra, rv, _ = O.le_gicov(xi, 0.0, 0)
        with np.errstate(divide="ignore"):
            thr = float(np.median(ra.astype(np.float64) ** 2 / rv))
        ref = O.le_gicov(xi, thr, 0)
        xd = dev(xi)
        for S, d in itertools.product(INTRA_S, (C.CYCLIC, C.BLOCK)):
            base = [host(t) for t in C.cudanp_le_gicov(xd, thr, S=S, dist=d, map=C.INTRA_WARP)]
            check([torch.from_numpy(t) for t in base], ref, xi, L, thr, f"le regs N={N} L={L} S={S}")
            for pl in (C.GRAD_SHARED, C.GRAD_GLOBAL):
                got = [host(t) for t in C.cudanp_le_gicov(xd, thr, S=S, dist=d, map=C.INTRA_WARP,
                                                            placement=pl)]
                for gv, bv, name in zip(got, base, ("gicov", "ave", "var", "ep")):
                    assert np.array_equal(gv.view(np.uint32), bv.view(np.uint32)), \
                        f"placement {pl} N={N} L={L} S={S} d={d} {name}"
    # point-major: the global placement for both maps; the shared placement
    # (a TMA box of [32 items x L points] per group, Fig 6b) for inter-warp
    # teams of S <= 16, non-powers of two included
    x = np.ascontiguousarray(synth.items(200, 150, "f32_unit").T)
    xd = dev(x)
    for m in (C.INTRA_WARP, C.INTER_WARP):
        base = [host(t) for t in C.cudanp_le_gicov(xd, 0.02, layout=1, S=8, map=m)]
        got = [host(t) for t in C.cudanp_le_gicov(xd, 0.02, layout=1, S=8, map=m, placement=C.GRAD_GLOBAL)]
        for gv, bv in zip(got, base):
            assert np.array_equal(gv.view(np.uint32), bv.view(np.uint32))
    for N, L in [(4, 1), (36, 5), (200, 150), (1000, 150), (4100, 150), (64, 256)]:
        xi = synth.items(N, L, "f32_unit", seed=L)
        x = np.ascontiguousarray(xi.T)
        _, ra, rv, _ = O.le_gicov(xi, 0.0, 0)
        with np.errstate(divide="ignore"):
            thr = float(np.median(ra.astype(np.float64) ** 2 / rv))
        ref = O.le_gicov(xi, thr, 0)
        xd = dev(x)
        for S, d in itertools.product((1, 2, 3, 4, 5, 8, 10, 15, 16), (C.CYCLIC, C.BLOCK)):
            base = [host(t) for t in C.cudanp_le_gicov(xd, thr, layout=1, S=S, dist=d, map=C.INTER_WARP)]
            got = [host(t) for t in C.cudanp_le_gicov(xd, thr, layout=1, S=S, dist=d, map=C.INTER_WARP,
                                                        placement=C.GRAD_SHARED)]
            check([torch.from_numpy(t) for t in got], ref, xi, L, thr, f"le pm shared N={N} L={L} S={S}")
            for gv, bv, name in zip(got, base, ("gicov", "ave", "var", "ep")):
                assert np.array_equal(gv.view(np.uint32), bv.view(np.uint32)), \
                    f"pm shared placement N={N} L={L} S={S} d={d} {name}"
    for kw in ({"map": C.INTRA_WARP, "S": 8}, {"map": C.INTER_WARP, "S": 32}):
        with pytest.raises(C.CudanpError) as ei:
            C.cudanp_le_gicov(dev(np.ascontiguousarray(synth.items(200, 150, "f32_unit").T)), 0.02,
                              layout=1, placement=C.GRAD_SHARED, **kw)
        assert ei.value.status == C.ERR_UNSUPPORTED
    with pytest.raises(C.CudanpError) as ei:  # N % 4 != 0: the TMA row pitch
        C.cudanp_le_gicov(dev(np.ascontiguousarray(synth.items(203, 150, "f32_unit").T)), 0.02,
                          layout=1, S=8, map=C.INTER_WARP, placement=C.GRAD_SHARED)
    assert ei.value.status == C.ERR_UNSUPPORTED


def test_le_point_major_inter_many_groups_per_cta():
    # Point-major inter-warp with Grad in registers double-buffers loop 1
    # across groups (np_le.cu, DB): with N well past one persistent wave each
    # CTA alternates between its two register copies many times, an odd or
    # even number of groups, with a ragged last group.  Oracle parity, and
    # bit-identical to the re-read placement (Fig 6a, no double buffering).
    for N, L in [(300013, 40), (100003, 150)]:
        xi = synth.items(N, L, "f32_unit", seed=N)
        _, ra, rv, _ = O.le_gicov(xi, 0.0, 0)
        with np.errstate(divide="ignore"):
            thr = float(np.median(ra.astype(np.float64) ** 2 / rv))
        ref = O.le_gicov(xi, thr, 0)
        xd = dev(np.ascontiguousarray(xi.T))
        for S, d in itertools.product((3, 4, 5, 8, 10, 16, 32), (C.CYCLIC, C.BLOCK)):
            got = [host(t) for t in C.cudanp_le_gicov(xd, thr, layout=1, S=S, dist=d, map=C.INTER_WARP)]
            check([torch.from_numpy(t) for t in got], ref, xi, L, thr, f"le pm many N={N} L={L} S={S} d={d}")
            rr = [host(t) for t in C.cudanp_le_gicov(xd, thr, layout=1, S=S, dist=d, map=C.INTER_WARP,
                                                       placement=C.GRAD_GLOBAL)]
            for gv, bv, name in zip(got, rr, ("gicov", "ave", "var", "ep")):
                assert np.array_equal(gv.view(np.uint32), bv.view(np.uint32)), \
                    f"pm regs vs reread N={N} L={L} S={S} d={d} {name}"
