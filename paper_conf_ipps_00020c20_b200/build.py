"""Build the sm_100a shared library in-tree (nvcc cross-compiles without a GPU).

    python -m paper_conf_ipps_00020c20_b200.build [--force] [--verbose]

Produces paper_conf_ipps_00020c20_b200/libhgemm.so exporting the C ABI of
include/hgemm.h.  Flags: -gencode arch=compute_100a,code=sm_100a (plain
sm_100 rejects tcgen05), -O3, -lineinfo (ncu source view), static cudart.
"""
from __future__ import annotations

import glob
import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
LIB = os.path.join(PKG, "libhgemm.so")
MB_LIB = os.path.join(PKG, "libhgemm_mb.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def sources():
    return sorted(glob.glob(os.path.join(CSRC, "*.cu")) + glob.glob(os.path.join(CSRC, "*.cuh"))
                  + [os.path.join(ROOT, "include", "hgemm.h")])


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in sources())


def build(force: bool = False, verbose: bool = False, defines=(), out: str | None = None) -> str:
    """Compile csrc/hgemm_api.cu into `out` (default: the in-tree libhgemm.so).
    `defines` adds -D flags (experiment variants are built to other paths)."""
    target = out or LIB
    if not force and out is None and not defines and not needs_build():
        return LIB
    tmp = target + f".tmp{os.getpid()}"
    # HGEMM_WATCHDOG_CYCLES > 0 builds a debug library whose pipeline waits trap after that
    # many cycles (a deadlock becomes a launch error instead of a hung GPU).
    watchdog = os.environ.get("HGEMM_WATCHDOG_CYCLES", "0")
    cmd = [NVCC, *ARCH, f"-DHGEMM_WATCHDOG_CYCLES={watchdog}ll", "-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC,-O3", "-shared",
           "-I", os.path.join(ROOT, "include"), "-o", tmp, os.path.join(CSRC, "hgemm_api.cu")]
    cmd[1:1] = [f"-D{d}" for d in defines]
    if verbose:
        cmd.insert(1, "-Xptxas=-v")
    subprocess.check_call(cmd)
    os.replace(tmp, target)
    return target


def build_microbench(force: bool = False) -> str:
    """The B200 micro-benchmark library (csrc/microbench.cu; NEXT-4, not on the GEMM path)."""
    src = os.path.join(CSRC, "microbench.cu")
    deps = [src] + glob.glob(os.path.join(CSRC, "*.cuh"))
    if not force and os.path.exists(MB_LIB) and all(os.path.getmtime(d) <= os.path.getmtime(MB_LIB) for d in deps):
        return MB_LIB
    tmp = MB_LIB + f".tmp{os.getpid()}"
    subprocess.check_call([NVCC, *ARCH, "-O3", "-std=c++17", "-lineinfo", "-Xcompiler", "-fPIC", "-shared",
                           "-o", tmp, src])
    os.replace(tmp, MB_LIB)
    return MB_LIB


def build_all(force: bool = False) -> None:
    build(force=force)
    build_microbench(force=force)


if __name__ == "__main__":
    defs = [a[2:] for a in sys.argv[1:] if a.startswith("-D")]
    outs = [a[6:] for a in sys.argv[1:] if a.startswith("--out=")]
    print(build(force="--force" in sys.argv, verbose="--verbose" in sys.argv, defines=defs,
                out=outs[0] if outs else None))
    if "--microbench" in sys.argv:
        print(build_microbench(force="--force" in sys.argv))
