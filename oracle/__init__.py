"""CPU FP64 oracle for C = alpha*op(A)*op(B) + beta*C (FP16 in, FP16/FP32 out).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py`` (its ``cpu_baseline`` leg and ``--impl reference``) may import
this package.  It shares no code with the CUDA path and never imports it.

The arithmetic lives in ``oracle/hgemm_ref.c`` (plain C, see its header for
the paper passages it follows: Alg. 1 P:246-272,
BASELINE.json north_star (4)).  This module only marshals numpy arrays.

Storage convention (reading R2): column-major, BLAS ``op()``.
Arrays passed in are flat (or Fortran-ordered) buffers of raw FP16 bits
(``numpy.uint16``) or ``numpy.float16`` (viewed as bits).

Parity pins: ``tests/test_oracle_pins.py``.  No function here is
"parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "hgemm_ref.c")
_LIB_PATH = os.path.join(_HERE, "libhgemm_ref.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle (gcc -O2, no -ffast-math, OpenMP) in-tree."""
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fno-fast-math", "-ffp-contract=off", "-fopenmp",
                               "-fPIC", "-shared", "-Wall", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        i64, f32, vp, c = ctypes.c_int64, ctypes.c_float, ctypes.c_void_p, ctypes.c_char
        lib.hgemm_ref.argtypes = [i64, i64, i64, f32, vp, i64, vp, i64, f32, vp, i64, c, c,
                                  ctypes.c_int, vp, vp, vp, ctypes.c_int]
        lib.hgemm_ref.restype = ctypes.c_int
        lib.hgemm_ref_entries.argtypes = [i64, i64, i64, f32, vp, i64, vp, i64, f32, vp, i64, c, c,
                                          ctypes.c_int, vp, vp, i64, vp, vp, vp, ctypes.c_int]
        lib.hgemm_ref_entries.restype = ctypes.c_int
        lib.hgemm_ref_f16_to_f64.argtypes = [ctypes.c_uint16]
        lib.hgemm_ref_f16_to_f64.restype = ctypes.c_double
        lib.hgemm_ref_f64_to_f16.argtypes = [ctypes.c_double]
        lib.hgemm_ref_f64_to_f16.restype = ctypes.c_uint16
        lib.hgemm_ref_max_threads.restype = ctypes.c_int
        _lib = lib
    return _lib


def max_threads() -> int:
    return int(_load().hgemm_ref_max_threads())


def f16_to_f64(bits: int) -> float:
    """Step 1 (exact decode) for one binary16 bit pattern."""
    return float(_load().hgemm_ref_f16_to_f64(int(bits) & 0xFFFF))


def f64_to_f16(x: float) -> int:
    """Step 4 (single RN-even rounding) for one double; returns the bit pattern."""
    return int(_load().hgemm_ref_f64_to_f16(float(x)))


def _bits(a) -> np.ndarray:
    a = np.asarray(a)
    if a.dtype == np.float16:
        a = a.view(np.uint16)
    if a.dtype != np.uint16:
        raise TypeError("oracle inputs must be float16 or uint16 bit patterns")
    return np.ascontiguousarray(a.reshape(-1, order="F") if a.ndim > 1 else a)


def _ptr(a):
    return a.ctypes.data_as(ctypes.c_void_p) if a is not None else None


def hgemm_ref(m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, transA="N", transB="N",
              out_dtype="f16", nthreads=1, want_r=True):
    """Full reference.  Returns (C_out, r, absab).

    C_out has C's storage (flat length ldc*n, dtype uint16 bits for f16 or
    float32 for f32); r and absab are float64 (m, n) Fortran-ordered arrays.
    """
    out_f32 = 1 if out_dtype in ("f32", np.float32, "float32") else 0
    Ab, Bb = _bits(A), _bits(B)
    if C is not None:
        Cin = np.ascontiguousarray(np.asarray(C).reshape(-1, order="F"))
        if out_f32:
            Cin = Cin.astype(np.float32, copy=False)
        else:
            Cin = Cin.view(np.uint16) if Cin.dtype == np.float16 else Cin.astype(np.uint16, copy=False)
    else:
        Cin = None
    size = ldc * n if n > 0 else 0
    C_out = np.zeros(max(size, 1), dtype=np.float32 if out_f32 else np.uint16)
    if Cin is not None:
        cnt = min(size, Cin.size)
        C_out[:cnt] = Cin[:cnt]              # untouched padding rows keep their input bytes
    r = np.zeros((m, n), dtype=np.float64, order="F") if want_r else None
    ab = np.zeros((m, n), dtype=np.float64, order="F") if want_r else None
    rc = _load().hgemm_ref(m, n, k, float(alpha), _ptr(Ab), lda, _ptr(Bb), ldb, float(beta),
                           _ptr(Cin), ldc, transA.encode(), transB.encode(), out_f32,
                           _ptr(C_out), _ptr(r), _ptr(ab), int(nthreads))
    if rc != 0:
        raise ValueError(f"hgemm_ref rejected its arguments (rc={rc})")
    return C_out[:size], r, ab


def hgemm_ref_entries(m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, transA, transB,
                      out_dtype, idx_i, idx_j, nthreads=1):
    """Sampled reference: entries (idx_i[t], idx_j[t]).  Returns (c_out, r, absab)."""
    out_f32 = 1 if out_dtype in ("f32", np.float32, "float32") else 0
    Ab, Bb = _bits(A), _bits(B)
    Cin = None
    if C is not None:
        Cin = np.ascontiguousarray(np.asarray(C).reshape(-1, order="F"))
        if out_f32:
            Cin = Cin.astype(np.float32, copy=False)
        else:
            Cin = Cin.view(np.uint16) if Cin.dtype == np.float16 else Cin.astype(np.uint16, copy=False)
    ii = np.ascontiguousarray(idx_i, dtype=np.int64)
    jj = np.ascontiguousarray(idx_j, dtype=np.int64)
    cnt = ii.size
    c_out = np.zeros(max(cnt, 1), dtype=np.float32 if out_f32 else np.uint16)
    r = np.zeros(max(cnt, 1), dtype=np.float64)
    ab = np.zeros(max(cnt, 1), dtype=np.float64)
    rc = _load().hgemm_ref_entries(m, n, k, float(alpha), _ptr(Ab), lda, _ptr(Bb), ldb, float(beta),
                                   _ptr(Cin), ldc, transA.encode(), transB.encode(), out_f32,
                                   _ptr(ii), _ptr(jj), cnt, _ptr(c_out), _ptr(r), _ptr(ab),
                                   int(nthreads))
    if rc != 0:
        raise ValueError(f"hgemm_ref_entries rejected its arguments (rc={rc})")
    return c_out[:cnt], r[:cnt], ab[:cnt]
