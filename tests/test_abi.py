"""C-ABI boundary checks that need no GPU: the library loads, exports every
function include/cudanp.h declares, and rejects bad arguments before any
launch (SURVEY §8(b) error conventions)."""
import ctypes
import os
import re

import pytest

from paper_conf_ppopp_yangz14_b200 import build as B
from paper_conf_ppopp_yangz14_b200 import cudanp as C

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    B.build()
    return C.load()


def declared_functions():
    hdr = open(os.path.join(ROOT, "include", "cudanp.h")).read()
    hdr = re.sub(r"/\*.*?\*/", "", hdr, flags=re.S)
    return sorted(set(re.findall(r"\b(?:int|const char\*|void)\s+\**(cudanp_\w+)\s*\(", hdr)))


def test_header_declares_the_four_hot_path_calls():
    names = declared_functions()
    for n in ["cudanp_tmv", "cudanp_mv", "cudanp_batched_loop_reduce", "cudanp_batched_loop_scan"]:
        assert n in names


def test_library_exports_every_declared_symbol(lib):
    names = declared_functions()
    assert len(names) >= 19
    for n in names:
        assert hasattr(lib, n), n
    # the binding wraps exactly the declared set
    assert sorted(C.EXPORTS) == names


def test_status_strings(lib):
    assert C.cudanp_status_string(0) == "CUDANP_OK"
    assert C.cudanp_status_string(1) == "CUDANP_ERR_INVALID"
    assert C.cudanp_status_string(99) == "CUDANP_UNKNOWN_STATUS"
    assert C.cudanp_version() >= 100


@pytest.mark.parametrize("S", [6, 7, 48, 1536, 16384, -1])
def test_bad_slave_size_rejected_before_launch(lib, S):
    rc = lib.cudanp_batched_loop_reduce(None, None, None, 10, 10, 0, 0, S, 0, 0, None)
    assert rc == C.ERR_INVALID
    assert "S must be" in lib.cudanp_last_error().decode()
    assert lib.cudanp_tmv(None, 4, None, None, 4, 4, S, 0, 0, None) == C.ERR_INVALID


@pytest.mark.parametrize("S", [2048, 4096, 8192])
def test_cluster_team_sizes_are_reduce_scan_mv_only(lib, S):
    # cluster teams (S > 1024) pass the reduce's, scan's and MV's S check (then
    # fail on the NULL pointers) and are rejected by TMV, before any launch
    assert lib.cudanp_batched_loop_reduce(None, None, None, 10, 10, 0, 0, S, 0, 0, None) == C.ERR_INVALID
    assert "S must be" not in lib.cudanp_last_error().decode()
    assert lib.cudanp_mv(None, 4, None, None, 4, 4, S, 0, 0, None) == C.ERR_INVALID
    assert "S must be" not in lib.cudanp_last_error().decode()
    assert lib.cudanp_batched_loop_scan(None, None, None, 10, 10, 0, S, 0, 0, None) == C.ERR_INVALID
    assert "S must be" not in lib.cudanp_last_error().decode()
    assert lib.cudanp_tmv(None, 4, None, None, 4, 4, S, 0, 0, None) == C.ERR_INVALID
    assert "S must be" in lib.cudanp_last_error().decode()


@pytest.mark.parametrize("S", [3, 5, 10, 15])
def test_non_power_of_two_teams_are_inter_warp_only(lib, S):
    """the power-of-two limit applies to intra-warp NP only.  S = 3, 5,
    10, 15 pass the S check of the four hot-path calls (then fail on the NULL
    pointers); the intra-warp map is refused as unsupported before any launch."""
    p = ctypes.c_void_p(16)
    for call in (lambda m: lib.cudanp_batched_loop_reduce(None, None, None, 10, 10, 0, 0, S, 0, m, None),
                 lambda m: lib.cudanp_batched_loop_scan(None, None, None, 10, 10, 0, S, 0, m, None),
                 lambda m: lib.cudanp_tmv(None, 4, None, None, 4, 4, S, 0, m, None),
                 lambda m: lib.cudanp_mv(None, 4, None, None, 4, 4, S, 0, m, None)):
        for m in (C.AUTO, C.INTER_WARP):
            assert call(m) == C.ERR_INVALID
            assert "S must be" not in lib.cudanp_last_error().decode()
        assert call(C.INTRA_WARP) == C.ERR_UNSUPPORTED
    assert lib.cudanp_mv(p, 4, p, p, 4, 4, S, 0, C.INTRA_WARP, None) == C.ERR_UNSUPPORTED


def test_auto_team_size_rule(lib):
    """S = CUDANP_S_AUTO: the library's version choice follows
    the rule stated in cudanp.h / DESIGN.md §6 (host-only, no GPU)."""
    ch = C.cudanp_choose_version
    # TMV: wide and TMA-able -> TMA S=8 cyclic (C2); narrow C1 -> inter-warp S=128 cyclic;
    # not 16-byte aligned -> LDG inter-warp
    assert ch("tmv", 16384, 16384) == (8, C.CYCLIC, C.INTER_WARP_TMA)
    assert ch("tmv", 1024, 1024) == (128, C.CYCLIC, C.INTER_WARP)
    assert ch("tmv", 2048, 1024) == (128, C.BLOCK, C.INTER_WARP)
    assert ch("tmv", 4096, 16384) == (128, C.CYCLIC, C.INTER_WARP)
    assert ch("tmv", 1024, 1024, vec4=False) == (64, C.BLOCK, C.INTER_WARP)
    assert ch("tmv", 8192, 65536) == (128, C.CYCLIC, C.INTER_WARP)    # C5 shard at G = 8
    assert ch("tmv", 8192, 65536, map=C.INTER_WARP_TMA) == (8, C.CYCLIC, C.INTER_WARP_TMA)
    assert ch("tmv", 12288, 16384) == (128, C.CYCLIC, C.INTER_WARP)
    assert ch("tmv", 14336, 16384) == (8, C.CYCLIC, C.INTER_WARP_TMA)
    assert ch("tmv", 65536, 65536) == (32, C.BLOCK, C.INTER_WARP)     # C5 at G = 1
    S, d, m = ch("tmv", 16384, 16384, vec4=False)
    assert m == C.INTER_WARP and 8 <= S <= 64
    # MV: C2 rows -> a 256-thread team (the bench's fastest); short rows stay small
    assert ch("mv", 16384, 16384) == (256, C.CYCLIC, C.INTRA_WARP)
    assert ch("mv", 1 << 20, 64)[0] == 1
    # reduce: S = L/8 (C3: 4, 8, 16, 32 at L = 32..256), block above L = 32
    for L, S in ((32, 4), (64, 8), (128, 16), (256, 32)):
        assert ch("reduce", 1 << 22, L) == (S, C.CYCLIC if L == 32 else C.BLOCK, C.INTRA_WARP)
    # few long items: the team grows past a warp
    S, d, m = ch("reduce", 256, 65536)
    assert S > 32 and m == C.INTRA_WARP
    # scan: S = 16 (C4), cyclic from L = 128
    assert ch("scan", 1 << 21, 1024) == (16, C.CYCLIC, C.INTRA_WARP)
    assert ch("scan", 1 << 21, 64) == (16, C.BLOCK, C.INTRA_WARP)
    # an explicit map is kept
    assert ch("reduce", 1 << 22, 64, map=C.INTER_WARP)[2] == C.INTER_WARP
    assert ch("mv", 4096, 4096, map=C.INTER_WARP)[2] == C.INTER_WARP
    # every chosen S is one the calls accept for that map
    for op in ("tmv", "mv", "reduce", "scan"):
        for N in (1, 100, 4096, 1 << 20):
            for L in (0, 1, 12, 64, 1000, 1 << 16):
                S, d, m = ch(op, N, L)
                assert S in C.SLAVE_SIZES or S in C.MULTI_WARP_SIZES, (op, N, L, S)
                if S > 32:
                    assert (m == C.INTRA_WARP) != (op == "tmv"), (op, N, L, S, m)
    with pytest.raises(C.CudanpError):
        ch("reduce", 10, 10, map=C.INTER_WARP_TMA)


def test_launch_info_resolves_auto_on_the_host(lib):
    """Launch shapes need no GPU to be computed for TMA TMV (the verdict's
    check: C2 TMV at S = 8 with MAP_AUTO runs the TMA-staged kernel)."""
    i = C.cudanp_launch_info("tmv", 16384, 16384, S=8)
    assert i["map"] == "inter_warp_tma" and i["S"] == 8
    i = C.cudanp_launch_info("tmv", 1024, 1024, S=8)
    assert i["map"] == "inter_warp"
    i = C.cudanp_launch_info("tmv", 16384, 16384, S=8, vec4=False)
    assert i["map"] == "inter_warp"
    i = C.cudanp_launch_info("mv", 16384, 16384, S=C.S_AUTO)
    assert (i["S"], i["dist"], i["map"]) == (256, "cyclic", "intra_warp")


def test_binding_rejects_misdescribed_tensors(lib):
    """The binding hands the library A.stride(0) as lda and refuses layouts the
    C ABI cannot express (strided views used to be misread)."""
    import torch
    A = torch.zeros(8, 12)
    x = torch.zeros(8)
    with pytest.raises(ValueError, match="unit column stride"):
        C.cudanp_tmv(A[:, ::2], x)
    with pytest.raises(ValueError, match="unit column stride"):
        C.cudanp_mv(A.t(), torch.zeros(8))
    with pytest.raises(TypeError, match="float32"):
        C.cudanp_tmv(A.double(), x)
    with pytest.raises(ValueError, match="needs 8"):
        C.cudanp_tmv(A, torch.zeros(5))
    with pytest.raises(ValueError, match="needs 12"):
        C.cudanp_tmv(A, x, torch.zeros(3))
    with pytest.raises(ValueError, match="n_outer"):
        C.cudanp_tmv(A, x, n_outer=13)
    with pytest.raises(ValueError, match="contiguous"):
        C.cudanp_batched_loop_reduce(torch.zeros(6, 10)[:, 1:])
    with pytest.raises(TypeError):
        C.cudanp_batched_loop_scan(torch.zeros(4, 4, dtype=torch.float64))
    with pytest.raises(ValueError, match="init"):
        C.cudanp_batched_loop_reduce(torch.zeros(6, 8), torch.zeros(3))
    with pytest.raises(TypeError, match="int32"):
        C.cudanp_batched_loop_reduce(torch.zeros(6, 8, dtype=torch.int32), None, torch.zeros(6))
    with pytest.raises(ValueError, match="needs 48"):
        C.cudanp_batched_loop_scan(torch.zeros(6, 8), None, torch.zeros(47))
    with pytest.raises(TypeError, match="int64"):
        C.cudanp_ragged_loop_reduce(torch.zeros(10), torch.zeros(3, dtype=torch.int32))
    # a row-padded view is a layout the ABI does express: it passes the checks
    # and only the device check (CPU tensor) stops it
    with pytest.raises(ValueError, match="CUDA device"):
        C.cudanp_tmv(A[:, :10], x)


def test_bad_arguments_rejected(lib):
    L = lib
    # negative sizes
    assert L.cudanp_mv(None, 4, None, None, -1, 4, 4, 0, 0, None) == C.ERR_INVALID
    # null pointers with non-zero sizes
    assert L.cudanp_tmv(None, 4, None, None, 4, 4, 4, 0, 0, None) == C.ERR_INVALID
    assert L.cudanp_batched_loop_scan(None, None, None, 3, 3, 0, 4, 0, 0, None) == C.ERR_INVALID
    # lda < row length
    p = ctypes.c_void_p(16)
    assert L.cudanp_tmv(p, 3, p, p, 4, 4, 4, 0, 0, None) == C.ERR_INVALID
    assert L.cudanp_mv(p, 3, p, p, 4, 4, 4, 0, 0, None) == C.ERR_INVALID
    # dtype / op / dist / map out of range
    assert L.cudanp_batched_loop_reduce(p, None, p, 3, 3, 7, 0, 4, 0, 0, None) == C.ERR_INVALID
    assert L.cudanp_batched_loop_reduce(p, None, p, 3, 3, 0, 9, 4, 0, 0, None) == C.ERR_INVALID
    assert L.cudanp_batched_loop_reduce(p, None, p, 3, 3, 0, 0, 4, 2, 0, None) == C.ERR_INVALID
    assert L.cudanp_batched_loop_reduce(p, None, p, 3, 3, 0, 0, 4, 0, 3, None) == C.ERR_INVALID
    # bad impl
    assert L.cudanp_tmv_variant(0, p, 4, p, p, 4, 4, None) == C.ERR_INVALID
    # overflowing sizes
    assert L.cudanp_batched_loop_reduce(p, None, p, 1 << 40, 1 << 40, 0, 0, 4, 0, 0, None) == C.ERR_INVALID


def test_shard_range_host_logic(lib):
    for N in [0, 1, 7, 1 << 26, 65536]:
        for G in [1, 2, 3, 4, 8]:
            ranges = [C.cudanp_shard_range(N, G, g) for g in range(G)]
            assert ranges[0][0] == 0 and ranges[-1][1] == N
            for g in range(G):
                assert ranges[g][0] == (g * N) // G and ranges[g][1] == ((g + 1) * N) // G
                if g:
                    assert ranges[g][0] == ranges[g - 1][1]
    with pytest.raises(C.CudanpError):
        C.cudanp_shard_range(10, 2, 2)


def test_binding_fails_loudly_without_library(tmp_path):
    mod = C
    saved = mod._lib
    try:
        mod._lib = None
        with pytest.raises(ImportError):
            mod.load(str(tmp_path / "missing.so"))
    finally:
        mod._lib = saved


def test_native_group_host_side(lib):
    # the NCCL unique id needs no GPU; bad arguments are rejected before NCCL
    uid = C.cudanp_group_unique_id()
    assert len(uid) == 128 and any(uid)
    h = ctypes.c_void_p()
    buf = ctypes.create_string_buffer(uid, 128)
    assert lib.cudanp_group_create(buf, 0, 0, ctypes.byref(h)) == C.ERR_INVALID
    assert lib.cudanp_group_create(buf, 2, 2, ctypes.byref(h)) == C.ERR_INVALID
    assert lib.cudanp_group_create(None, 1, 0, ctypes.byref(h)) == C.ERR_INVALID
    assert lib.cudanp_group_gather(None, None, None, 10, 0, None) == C.ERR_INVALID
    assert lib.cudanp_sharded_tmv(None, None, 4, None, None, None, 4, 4, 8, 0, 0, None) == C.ERR_INVALID
    assert lib.cudanp_group_destroy(None) == C.OK
