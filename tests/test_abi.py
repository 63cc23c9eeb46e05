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


@pytest.mark.parametrize("S", [0, 3, 5, 48, 1536, 16384, -1])
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
