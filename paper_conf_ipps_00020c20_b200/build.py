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


def units():
    """Translation units of libhgemm.so: the C ABI (hgemm_api.cu) and one TU per kernel
    family (hgemm_inst_*.cu), compiled in parallel and linked into one library."""
    return sorted(glob.glob(os.path.join(CSRC, "hgemm_*.cu")))


def needs_build() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    return any(os.path.getmtime(s) > t for s in sources())


def build(force: bool = False, verbose: bool = False, defines=(), out: str | None = None) -> str:
    """Compile the TUs of csrc/ into `out` (default: the in-tree libhgemm.so), one nvcc
    process per TU in parallel.  `defines` adds -D flags (experiment variants are built
    to other paths)."""
    from concurrent.futures import ThreadPoolExecutor
    import tempfile
    target = out or LIB
    if not force and out is None and not defines and not needs_build():
        return LIB
    tmp = target + f".tmp{os.getpid()}"
    # HGEMM_WATCHDOG_CYCLES > 0 builds a debug library whose pipeline waits trap after that
    # many cycles (a deadlock becomes a launch error instead of a hung GPU).
    watchdog = os.environ.get("HGEMM_WATCHDOG_CYCLES", "0")
    flags = [*ARCH, *[f"-D{d}" for d in defines], f"-DHGEMM_WATCHDOG_CYCLES={watchdog}ll", "-O3", "-std=c++17",
             "-lineinfo", "-Xcompiler", "-fPIC,-O3", "-I", os.path.join(ROOT, "include")]
    if verbose:
        flags.append("-Xptxas=-v")
    with tempfile.TemporaryDirectory(prefix="hgemm_build_") as td:
        objs = []

        def compile_one(src):
            obj = os.path.join(td, os.path.basename(src)[:-3] + ".o")
            subprocess.check_call([NVCC, *flags, "-c", "-o", obj, src])
            return obj
        with ThreadPoolExecutor(max_workers=max(1, min(len(units()), os.cpu_count() or 1))) as ex:
            objs = list(ex.map(compile_one, units()))
        # export the C ABI only (the hgi:: internals shared between the TUs stay local)
        vs = os.path.join(td, "exports.map")
        with open(vs, "w") as f:
            f.write("{ global: hgemm*; local: *; };\n")
        subprocess.check_call([NVCC, *ARCH, "-shared", "-Xlinker", f"--version-script={vs}", "-o", tmp, *objs])
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
