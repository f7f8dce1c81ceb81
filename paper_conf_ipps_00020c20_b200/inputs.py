"""Seeded synthetic input generators shared by tests, smoke() and bench.py.

This module holds NONE of the method's arithmetic: it only draws random
numbers and lays matrices out in memory.  Both the CUDA path's callers and
the oracle's callers take their inputs from here; neither the oracle nor the
CUDA binding imports it.

Input recipe (BASELINE.json north_star (4),
SURVEY 8(d)):
  * random operands: uniform[-1, 1) drawn in float32 by a seeded generator,
    rounded to FP16 (numpy's float32->float16 cast, RN-even);
  * integer operands: uniform integers in [lo, hi] (exactly representable);
  * storage is column-major (BLAS) with a leading dimension ld >= rows; any
    padding rows are filled with a sentinel (NaN by default) so that a read
    of padding is visible in the result.
"""
from __future__ import annotations

import numpy as np

SENTINEL_F16 = np.float16(np.nan)


def rng(seed: int) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(int(seed)))


def uniform_f16(rows: int, cols: int, seed: int, lo: float = -1.0, hi: float = 1.0) -> np.ndarray:
    """(rows, cols) float16, Fortran order, uniform[lo, hi) rounded to FP16."""
    g = rng(seed)
    x = g.uniform(lo, hi, size=(cols, rows)).astype(np.float32)
    return np.asfortranarray(x.T.astype(np.float16))


def integer_f16(rows: int, cols: int, seed: int, lo: int = -8, hi: int = 8) -> np.ndarray:
    """(rows, cols) float16 with integer values in [lo, hi], Fortran order."""
    g = rng(seed)
    x = g.integers(lo, hi + 1, size=(cols, rows))
    return np.asfortranarray(x.T.astype(np.float16))


def uniform_f16_blocked(rows: int, cols: int, seed: int, block: int = 4096, lo: float = -1.0,
                        hi: float = 1.0, col0: int = 0, ncols: int | None = None) -> np.ndarray:
    """Columns [col0, col0 + ncols) of a (rows, cols) uniform[lo, hi) FP16 matrix whose
    column block b (columns [b*block, (b+1)*block)) is drawn by rng(seed * 100003 + b)
    (SURVEY 8(e) "Inputs": the global matrix is defined block by block, so any slab of
    it -- a rank's share at any world size -- is reproduced without drawing the rest).
    Returns a Fortran-ordered (rows, ncols) array."""
    ncols = cols - col0 if ncols is None else ncols
    out = np.empty((rows, ncols), dtype=np.float16, order="F")
    b0, b1 = col0 // block, (col0 + ncols + block - 1) // block
    for b in range(b0, b1):
        c0, c1 = b * block, min(cols, (b + 1) * block)
        x = rng(seed * 100003 + b).random(size=(c1 - c0, rows), dtype=np.float32)
        x *= np.float32(hi - lo)
        x += np.float32(lo)
        s0, s1 = max(c0, col0), min(c1, col0 + ncols)
        out[:, s0 - col0:s1 - col0] = x[s0 - c0:s1 - c0].T.astype(np.float16)
    return out


def integer_f16_blocked(rows: int, cols: int, seed: int, lo: int, hi: int, block: int = 4096, col0: int = 0,
                        ncols: int | None = None) -> np.ndarray:
    """As uniform_f16_blocked, with integer values in [lo, hi] (exactly representable)."""
    ncols = cols - col0 if ncols is None else ncols
    out = np.empty((rows, ncols), dtype=np.float16, order="F")
    b0, b1 = col0 // block, (col0 + ncols + block - 1) // block
    for b in range(b0, b1):
        c0, c1 = b * block, min(cols, (b + 1) * block)
        x = rng(seed * 100003 + b).integers(lo, hi + 1, size=(c1 - c0, rows), dtype=np.int8)
        s0, s1 = max(c0, col0), min(c1, col0 + ncols)
        out[:, s0 - col0:s1 - col0] = x[s0 - c0:s1 - c0].T.astype(np.float16)
    return out


def to_colmajor(mat: np.ndarray, ld: int, fill=SENTINEL_F16) -> np.ndarray:
    """Flat column-major buffer of length ld*cols holding ``mat`` (rows <= ld)."""
    rows, cols = mat.shape
    if ld < max(rows, 1):
        raise ValueError("ld < rows")
    buf = np.full((ld, max(cols, 0)), fill, dtype=mat.dtype, order="F")
    buf[:rows, :] = mat
    return buf.reshape(-1, order="F")


def from_colmajor(buf: np.ndarray, rows: int, cols: int, ld: int) -> np.ndarray:
    return np.asarray(buf).reshape(ld, cols, order="F")[:rows, :]


def stored_shape(op_rows: int, op_cols: int, trans: str):
    """Shape of the stored matrix whose op() is op_rows x op_cols."""
    return (op_cols, op_rows) if trans in ("T", "t") else (op_rows, op_cols)


def store_op(op_mat: np.ndarray, trans: str, ld: int | None = None, fill=SENTINEL_F16):
    """Store the logical op(X) as the column-major buffer X for flag ``trans``.

    Returns (flat buffer, ld)."""
    stored = op_mat.T if trans in ("T", "t") else op_mat
    rows = stored.shape[0]
    if ld is None:
        ld = max(rows, 1)
    return to_colmajor(np.asfortranarray(stored), ld, fill), ld


def accumulator_width_case(m: int, n: int, k: int, base: float = 64.0):
    """op(A) (m x k) and op(B) (k x n) whose exact product is k/16 - 2 everywhere.

    SURVEY 8(c) "accumulator-width test": a large first product base*base,
    one unit product in every 16-wide K chunk strictly between, and
    -base*base at p = k-1.  An FP32 accumulator (24-bit significand) keeps
    the unit terms; an FP16 accumulator (11-bit) rounds them away (result 0).
    Requires k % 16 == 0 and k >= 48.
    """
    if k % 16 or k < 48:
        raise ValueError("k must be a multiple of 16 and >= 48")
    a = np.zeros((m, k), dtype=np.float16)
    b = np.zeros((k, n), dtype=np.float16)
    a[:, 0] = base
    b[0, :] = base
    ones = np.arange(16, k - 16, 16)
    a[:, ones] = 1
    b[ones, :] = 1
    a[:, k - 1] = -base
    b[k - 1, :] = base
    return np.asfortranarray(a), np.asfortranarray(b), float(k // 16 - 2)


# BASELINE.json configs as concrete synthetic workloads.
# (m, n, k, transA, transB, alpha, beta, out_dtype) in the column-major ABI.
WORKLOADS = {
    "cfg1_256_NN_f32": (256, 256, 256, "N", "N", 1.0, 0.0, "f32"),
    "cfg2_8192_TN_f16": (8192, 8192, 8192, "T", "N", 1.0, 0.0, "f16"),
    "cfg2_8192_NN_f16": (8192, 8192, 8192, "N", "N", 1.0, 0.0, "f16"),
    "cfg2_8192_NT_f16": (8192, 8192, 8192, "N", "T", 1.0, 0.0, "f16"),
    "cfg2_8192_TN_f32": (8192, 8192, 8192, "T", "N", 1.0, 0.0, "f32"),
    "cfg3_bert_ffn1_4096": (4096, 4096, 1024, "T", "N", 1.0, 1.0, "f16"),
    "cfg3_bert_ffn1_16384": (16384, 4096, 1024, "T", "N", 1.0, 1.0, "f16"),
    "cfg3_bert_ffn2_4096": (4096, 1024, 4096, "T", "N", 1.0, 1.0, "f16"),
    "cfg3_lstm_b64": (64, 4096, 2048, "T", "N", 1.0, 1.0, "f16"),
    "cfg3_lstm_b256": (256, 4096, 2048, "T", "N", 1.0, 1.0, "f16"),
    "cfg3_lstm_b1024": (1024, 4096, 2048, "T", "N", 1.0, 1.0, "f16"),
    "cfg4_skinny_n64": (16384, 64, 4096, "T", "N", 1.0, 0.0, "f16"),
    "cfg4_skinny_n128": (16384, 128, 4096, "T", "N", 1.0, 0.0, "f16"),
    "cfg4_skinny_n256": (16384, 256, 4096, "T", "N", 1.0, 0.0, "f16"),
    # config 5: the GLOBAL 32768^3 problem, N-slab sharded over the ranks (strong scaling)
    "cfg5_sharded_32768": (32768, 32768, 32768, "T", "N", 1.0, 0.0, "f16"),
}
STRONG_SCALING = {"cfg5_sharded_32768"}

# Square sweep of the paper's evaluation: W = 1024..16384 step 256.
SQUARE_SWEEP = list(range(1024, 16384 + 1, 256))
# ... as bench workloads "sq_<W>" (BASELINE.json configs[1], paper layout TN, FP16 out)
for _w in SQUARE_SWEEP:
    WORKLOADS[f"sq_{_w}"] = (_w, _w, _w, "T", "N", 1.0, 0.0, "f16")
