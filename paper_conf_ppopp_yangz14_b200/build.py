"""Build libcudanp.so in-tree for sm_100a with nvcc (no torch extension).

    python -m paper_conf_ppopp_yangz14_b200.build [--force] [-j N]

NP kernels are compiled WITHOUT relocatable device code; only the
dynamic-parallelism translation unit (np_dp.cu) uses -rdc=true and is
device-linked against cudadevrt, so the NP kernels carry no
"dynamic-parallelism-enabled kernel overhead".  The CUDA
runtime is linked statically (the primary context is shared with torch's
runtime; no second libcudart.so is loaded).
"""
from __future__ import annotations

import argparse
import os
import shutil
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
BUILD = os.path.join(PKG, "_build")
LIB = os.path.join(PKG, "libcudanp.so")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVFLAGS = ["-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "--expt-relaxed-constexpr",
           "-Xptxas", "-warn-spills", "-I" + os.path.join(ROOT, "include")]
SOURCES = ["abi.cu", "np_reduce.cu", "np_scan.cu", "np_matvec.cu", "np_ragged.cu", "np_le.cu", "np_le_pm.cu", "np_tmv_tma.cu", "np_reduce_tma.cu", "np_le_tma.cu", "np_multi.cu", "np_cluster.cu", "np_s1_tiled.cu", "autotune.cu", "group.cu"]
RDC_SOURCES = ["np_dp.cu"]


def nvcc() -> str:
    for c in [os.environ.get("NVCC"), "/usr/local/cuda/bin/nvcc", shutil.which("nvcc")]:
        if c and os.path.exists(c):
            return c
    raise RuntimeError("nvcc not found: the CUDA extension cannot be built")


def _deps() -> list[str]:
    out = [os.path.join(ROOT, "include", "cudanp.h")]
    for f in os.listdir(CSRC):
        out.append(os.path.join(CSRC, f))
    out.append(os.path.abspath(__file__))
    return out


def stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(d) > t for d in _deps())


def _run(cmd: list[str]) -> None:
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError(f"command failed: {' '.join(cmd)}\n{r.stdout}\n{r.stderr}")
    if r.stderr.strip():
        sys.stderr.write(r.stderr)


def build(force: bool = False, jobs: int | None = None, verbose: bool = False,
          defines: tuple[str, ...] = (), out: str | None = None) -> str:
    """Build libcudanp.so.  `defines`/`out` build an experiment variant (e.g.
    -DCUDANP_TMV_U=4) into another file and build directory."""
    lib = out or LIB
    if not force and not defines and out is None and not stale():
        return LIB
    bdir = BUILD if not defines else BUILD + "_" + "_".join(d.replace("=", "") for d in defines)
    os.makedirs(bdir, exist_ok=True)
    dflags = ["-D" + d for d in defines]
    cc = nvcc()
    objs, cmds = [], []
    for s in SOURCES:
        o = os.path.join(bdir, s.replace(".cu", ".o"))
        objs.append(o)
        cmds.append([cc, *ARCH, *NVFLAGS, *dflags, "-c", os.path.join(CSRC, s), "-o", o])
    rdc_objs = []
    for s in RDC_SOURCES:
        o = os.path.join(bdir, s.replace(".cu", ".o"))
        rdc_objs.append(o)
        cmds.append([cc, *ARCH, *NVFLAGS, *dflags, "-rdc=true", "-c", os.path.join(CSRC, s), "-o", o])
    with ThreadPoolExecutor(max_workers=jobs or os.cpu_count() or 4) as ex:
        list(ex.map(_run, cmds))
    dlink = os.path.join(bdir, "dp_dlink.o")
    _run([cc, *ARCH, "-Xcompiler", "-fPIC", "-dlink", *rdc_objs, "-o", dlink, "-lcudadevrt"])
    tmp = lib + f".tmp{os.getpid()}"
    _run([cc, *ARCH, "-shared", "-Xcompiler", "-fPIC", "-o", tmp, *objs, *rdc_objs, dlink,
          "-lcudadevrt", "-cudart", "static", "-ldl"])
    os.replace(tmp, lib)
    if verbose:
        print("built", lib)
    return lib


def main() -> None:
    ap = argparse.ArgumentParser()
    ap.add_argument("--force", action="store_true")
    ap.add_argument("-j", type=int, default=None)
    ap.add_argument("-D", dest="defines", action="append", default=[])
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    build(force=a.force, jobs=a.j, verbose=True, defines=tuple(a.defines), out=a.out)


if __name__ == "__main__":
    main()
