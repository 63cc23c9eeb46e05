"""The boundary from plain C: tests/c_client/abi_client.c includes only
include/cudanp.h and the CUDA runtime, links libcudanp.so, and checks closed
forms of the four hot-path calls (SURVEY C-3 pin P2) on a stream it owns.

CPU: the client compiles and links as C99 against the header and the library
(the ABI has no C++ or torch types).  GPU: it runs and every check passes."""
import os
import shutil
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "tests", "c_client", "abi_client.c")
PKG = os.path.join(ROOT, "paper_conf_ppopp_yangz14_b200")
CUDA = "/usr/local/cuda"


def _build(tmp_path):
    from paper_conf_ppopp_yangz14_b200 import build as B
    B.build()
    cc = shutil.which("gcc") or shutil.which("cc")
    if cc is None:
        pytest.skip("no C compiler")
    exe = str(tmp_path / "abi_client")
    cmd = [cc, "-std=c99", "-O2", "-Wall", "-Werror", "-I" + os.path.join(ROOT, "include"),
           "-I" + os.path.join(CUDA, "include"), SRC, "-o", exe,
           "-L" + PKG, "-lcudanp", "-Wl,-rpath," + PKG,
           "-L" + os.path.join(CUDA, "lib64"), "-lcudart", "-Wl,-rpath," + os.path.join(CUDA, "lib64")]
    r = subprocess.run(cmd, capture_output=True, text=True)
    assert r.returncode == 0, r.stderr
    return exe


def test_c_client_compiles_against_the_abi(tmp_path):
    assert os.path.exists(_build(tmp_path))


@pytest.mark.gpu
def test_c_client_runs_closed_forms_on_gpu(tmp_path):
    exe = _build(tmp_path)
    r = subprocess.run([exe], capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stdout + r.stderr
    assert "abi_client: OK" in r.stdout
