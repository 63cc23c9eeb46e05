"""GPU parity for the ragged loop-reduce against the oracle."""
import itertools

import numpy as np
import pytest

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("needs a CUDA device", allow_module_level=True)

import oracle as O
import synth
from paper_conf_ppopp_yangz14_b200 import build as B
from paper_conf_ppopp_yangz14_b200 import cudanp as C
from test_gpu_parity import assert_exact, assert_rel, dev, host

pytestmark = pytest.mark.gpu
SS = C.SLAVE_SIZES


@pytest.fixture(scope="module", autouse=True)
def _lib():
    B.build()
    C.load()


CASES = [(1, 5, "uniform"), (33, 1, "uniform"), (300, 13, "uniform"), (1000, 64, "exp"),
         (257, 150, "uniform"), (64, 700, "exp")]


@pytest.mark.parametrize("kind,op,exact", [("i32_full", C.SUM, True), ("i32_full", C.MAX, True),
                                           ("f32_signed", C.MAX, True), ("f32_int4", C.SUM, True),
                                           ("f32_unit", C.SUM, False)])
def test_ragged_parity(kind, op, exact):
    for N, mean, dist in CASES:
        lens = synth.lengths(N, mean, dist, seed=N + mean)
        off = synth.offsets_from_lengths(lens)
        total = int(off[-1]) + 3
        # shift by 0..3 elements: every head/tail alignment case
        for shift in (0, 1, 3):
            x = synth.gen(1, kind, 0, total)
            offs = off + shift
            ini = synth.init(N, kind)
            ref = O.ragged_reduce(x, offs, op=op)
            ref_i = O.ragged_reduce(x, offs, op=op, init=ini)
            xd, od, inid = dev(x), dev(offs), dev(ini)
            Lmax = int(lens.max()) if N else 0
            for S, d, m in itertools.product(SS, (C.CYCLIC, C.BLOCK), (C.INTRA_WARP, C.INTER_WARP)):
                what = f"ragged {kind} op={op} N={N} mean={mean} shift={shift} S={S} d={d} m={m}"
                got = host(C.cudanp_ragged_loop_reduce(xd, od, op=op, S=S, dist=d, map=m))
                got_i = host(C.cudanp_ragged_loop_reduce(xd, od, inid, op=op, S=S, dist=d, map=m))
                if exact:
                    assert_exact(got, ref, what)
                    assert_exact(got_i, ref_i, what + " init")
                else:
                    nz = lens > 0
                    assert_rel(got[nz], ref[nz], Lmax, what)
                    assert (got[~nz] == 0).all()
            got = host(C.cudanp_ragged_loop_reduce_literal(xd, od, inid, op=op))
            if exact:
                assert_exact(got, ref_i, "literal")


def test_ragged_decreasing_pair_is_empty():
    x = dev(np.arange(8, dtype=np.int32))
    off = dev(np.array([0, 5, 3, 8], np.int64))
    for S in SS:
        assert host(C.cudanp_ragged_loop_reduce(x, off, S=S)).tolist() == [10, 0, 25]


def test_ragged_full_size_sampled():
    N, mean = 1 << 22, 64
    lens = synth.lengths(N, mean, "exp")
    off = synth.offsets_from_lengths(lens)
    x = torch.empty(int(off[-1]), dtype=torch.int32, device="cuda")
    C.cudanp_generate(x, "i32_full", stream_id=1)
    od = dev(off)
    rng = np.random.default_rng(5)
    items = np.unique(rng.integers(0, N, 2048))
    xs = O.gen_i32(1, "i32_full", 0, int(off[-1]))  # the oracle's own copy of the input
    ref = O.ragged_reduce(xs, off)[items]
    for S, d in itertools.product(SS, (C.CYCLIC, C.BLOCK)):
        got = host(C.cudanp_ragged_loop_reduce(x, od, S=S, dist=d, map=C.INTRA_WARP))
        assert_exact(got[items], ref, f"full ragged S={S} d={d}")


def test_ragged_big_teams():
    """S > 32 multi-warp teams on few, long segments."""
    for N, mean in [(1, 5000), (37, 3000), (300, 700)]:
        lens = synth.lengths(N, mean, "exp", seed=N)
        for shift in (0, 2):
            off = synth.offsets_from_lengths(lens) + shift
            x = synth.gen(1, "i32_full", 0, int(off[-1]) + 1, seed=N)
            ref = O.ragged_reduce(x, off)
            refm = O.ragged_reduce(x, off, op=C.MAX)
            for S in (64, 128, 256, 512, 1024):
                for d in (C.CYCLIC, C.BLOCK):
                    what = f"ragged big N={N} S={S} d={d} shift={shift}"
                    assert_exact(host(C.cudanp_ragged_loop_reduce(dev(x), dev(off), S=S, dist=d)), ref, what)
                    assert_exact(host(C.cudanp_ragged_loop_reduce(dev(x), dev(off), op=C.MAX, S=S, dist=d)),
                                 refm, what)


@pytest.mark.parametrize("kind,op,exact", [("i32_full", C.SUM, True), ("i32_full", C.MAX, True),
                                           ("f32_signed", C.MAX, True), ("f32_unit", C.SUM, False)])
def test_ragged_adaptive_parity(kind, op, exact):
    """Team size chosen per segment: below the threshold the master alone, above
    it the whole warp; mixes of both in one warp, every alignment."""
    for N, mean, dist in CASES + [(3000, 90, "exp"), (40, 5000, "exp")]:
        lens = synth.lengths(N, mean, dist, seed=N + mean)
        off = synth.offsets_from_lengths(lens)
        for shift in (0, 1, 3):
            x = synth.gen(1, kind, 0, int(off[-1]) + 3)
            offs = off + shift
            ini = synth.init(N, kind)
            ref_i = O.ragged_reduce(x, offs, op=op, init=ini)
            xd, od, inid = dev(x), dev(offs), dev(ini)
            for th in (1, 7, 64, 128, 1 << 40):
                got = host(C.cudanp_ragged_loop_reduce_adaptive(xd, od, inid, op=op, threshold=th))
                what = f"adaptive {kind} op={op} N={N} mean={mean} shift={shift} th={th}"
                if exact:
                    assert_exact(got, ref_i, what)
                else:
                    assert_rel(got, ref_i, int(lens.max()) if N else 1, what)
    with pytest.raises(C.CudanpError):
        C.cudanp_ragged_loop_reduce_adaptive(dev(synth.gen(1, "i32_full", 0, 8)),
                                             dev(synth.offsets_from_lengths(np.array([3, 5]))), threshold=0)
