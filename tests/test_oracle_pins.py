"""Pins for the CPU oracle (oracle/hgemm_ref.c) against things other than itself.

Every check here compares the oracle with something the paper or mathematics
fixes (SURVEY 8(c) "What pins each part"):
  * exhaustive FP16 decode vs numpy's float16 -> float64 conversion;
  * FP64 -> FP16 RN-even encode vs numpy's float64 -> float16 cast (a single
    correct rounding) and vs hand-derived ties in tests/golden/;
  * the FP64 sum vs exact rational arithmetic (fractions.Fraction) on tiny
    shapes, and vs numpy's float64 matmul;
  * closed forms: identity, permutation, integer-valued inputs, alpha/beta,
    k == 0, alpha == 0, beta == 0 with NaN in C, accumulator-width test;
  * the worked examples in tests/golden/hand_examples.json.
A plausible bug (dropped term, sign, transposed operand, wrong ld, wrong
rounding direction, double rounding) fails at least one of them.
"""
import json
import math
import os
from fractions import Fraction

import numpy as np
import pytest

from paper_conf_ipps_00020c20_b200 import inputs

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "hand_examples.json")
TRANS = [("N", "N"), ("N", "T"), ("T", "N"), ("T", "T")]


def _num(v):
    if isinstance(v, str):
        if v in ("nan", "inf", "-inf"):
            return float(v)
        return float.fromhex(v)
    return float(v)


def _run(oracle, opA, opB, tA, tB, alpha=1.0, beta=0.0, C=None, out="f16", pad=0, nthreads=1):
    """Store op(A), op(B) for the given flags (with ld padding) and call the oracle."""
    m, k = opA.shape
    n = opB.shape[1]
    sa = inputs.stored_shape(m, k, tA)
    sb = inputs.stored_shape(k, n, tB)
    A, lda = inputs.store_op(np.asarray(opA, dtype=np.float16), tA, ld=max(sa[0], 1) + pad)
    B, ldb = inputs.store_op(np.asarray(opB, dtype=np.float16), tB, ld=max(sb[0], 1) + pad)
    ldc = max(m, 1) + pad
    cdt = np.float32 if out == "f32" else np.float16
    if C is None:
        Cbuf = inputs.to_colmajor(np.full((m, n), np.nan, dtype=cdt), ldc, fill=cdt(np.nan))
    else:
        Cbuf = inputs.to_colmajor(np.asarray(C, dtype=cdt), ldc, fill=cdt(np.nan))
    c_out, r, ab = oracle.hgemm_ref(m, n, k, alpha, A, lda, B, ldb, beta, Cbuf, ldc, tA, tB, out,
                                    nthreads=nthreads)
    if out == "f16":
        c_out = c_out.view(np.float16)
    co = inputs.from_colmajor(c_out, m, n, ldc)
    pad_part = np.asarray(c_out).reshape(ldc, n, order="F")[m:, :] if n else None
    return co, r, ab, pad_part


# ---------------------------------------------------------------- step 1 / 4

def test_decode_exhaustive(oracle_mod):
    bits = np.arange(65536, dtype=np.uint16)
    ref = bits.view(np.float16).astype(np.float64)
    got = np.array([oracle_mod.f16_to_f64(int(b)) for b in bits])
    nan = np.isnan(ref)
    assert np.array_equal(np.isnan(got), nan)
    assert np.array_equal(got[~nan], ref[~nan])
    # sign of zero
    assert math.copysign(1.0, oracle_mod.f16_to_f64(0x8000)) == -1.0


def test_encode_roundtrip_all_finite(oracle_mod):
    bits = np.arange(65536, dtype=np.uint16)
    vals = bits.view(np.float16)
    for b, v in zip(bits, vals):
        if np.isfinite(v):
            assert oracle_mod.f64_to_f16(float(v)) == int(b)


def test_encode_vs_numpy_random_and_edges(oracle_mod):
    g = np.random.Generator(np.random.PCG64(7))
    x = np.concatenate([
        g.uniform(-1, 1, 20000),
        g.standard_normal(20000) * 3000.0,
        np.ldexp(g.uniform(-1, 1, 20000), g.integers(-30, 17, 20000)),
        np.array([1 + 2.0**-11, 1 + 3 * 2.0**-11, 65504.0, 65519.99, 65520.0, -65520.0,
                  2.0**-24, 2.0**-25, 1.5 * 2.0**-25, 2.0**-14, 2.0**-14 - 2.0**-25,
                  2.0**-14 - 2.0**-26, 0.0, -0.0, 1e300, -1e300, 1e-300]),
    ])
    with np.errstate(over="ignore"):
        ref = x.astype(np.float16).view(np.uint16)
    got = np.array([oracle_mod.f64_to_f16(float(v)) for v in x], dtype=np.uint16)
    assert np.array_equal(got, ref), np.nonzero(got != ref)


# ---------------------------------------------------------------- golden

def _golden_cases():
    with open(GOLDEN) as f:
        return json.load(f)["cases"]


def _dense(case, key):
    if key in case:
        return np.array([[_num(v) for v in row] for row in case[key]])
    sp = case[key + "_sparse"]
    shape = (sp["m"], sp["k"]) if key == "A" else (sp["k"], sp["n"])
    d = np.zeros(shape)
    for i, j, v in sp["nz"]:
        d[i, j] = v
    return d


@pytest.mark.parametrize("case", _golden_cases(), ids=lambda c: c["name"])
@pytest.mark.parametrize("tA,tB", TRANS)
def test_golden_hand_examples(oracle_mod, case, tA, tB):
    A = _dense(case, "A")
    B = _dense(case, "B")
    C = _dense(case, "C") if "C" in case else None
    expect = np.array([[_num(v) for v in row] for row in case["expect"]])
    bits = np.array([[int(v, 16) for v in row] for row in case["expect_f16_bits"]], dtype=np.uint16)
    co, r, _, _ = _run(oracle_mod, A, B, tA, tB, case["alpha"], case["beta"], C=C, out="f16")
    assert np.array_equal(r, expect)
    assert np.array_equal(co.view(np.uint16), bits)
    co32, r32, _, _ = _run(oracle_mod, A, B, tA, tB, case["alpha"], case["beta"],
                           C=None if C is None else C.astype(np.float32), out="f32")
    assert np.array_equal(co32, expect.astype(np.float32))


# ---------------------------------------------------------------- step 2: the sum

@pytest.mark.parametrize("m,n,k", [(1, 1, 1), (2, 3, 7), (3, 2, 8), (7, 5, 15), (8, 8, 16), (5, 9, 17), (4, 3, 33)])
@pytest.mark.parametrize("tA,tB", TRANS)
def test_brute_force_exact_rational(oracle_mod, m, n, k, tA, tB):
    opA = inputs.uniform_f16(m, k, seed=m * 100 + k)
    opB = inputs.uniform_f16(k, n, seed=n * 100 + k + 1)
    _, r, ab, _ = _run(oracle_mod, opA, opB, tA, tB, pad=3, out="f32")
    for i in range(m):
        for j in range(n):
            exact = sum(Fraction(float(opA[i, p])) * Fraction(float(opB[p, j])) for p in range(k))
            absab = sum(abs(Fraction(float(opA[i, p])) * Fraction(float(opB[p, j]))) for p in range(k))
            # FP64 summation error bound k * 2^-53 * sum|a||b|
            assert abs(Fraction(r[i, j]) - exact) <= Fraction(k, 2**53) * absab
            assert ab[i, j] == float(absab)


@pytest.mark.parametrize("tA,tB", TRANS)
@pytest.mark.parametrize("out", ["f16", "f32"])
def test_vs_numpy_matmul(oracle_mod, tA, tB, out):
    m, n, k = 67, 45, 130
    opA = inputs.uniform_f16(m, k, seed=11)
    opB = inputs.uniform_f16(k, n, seed=12)
    co, r, ab, pad = _run(oracle_mod, opA, opB, tA, tB, pad=5, out=out, nthreads=4)
    ref = opA.astype(np.float64) @ opB.astype(np.float64)
    absref = np.abs(opA.astype(np.float64)) @ np.abs(opB.astype(np.float64))
    assert np.all(np.abs(r - ref) <= 1e-12 * absref)
    assert np.allclose(ab, absref, rtol=1e-13, atol=0)
    if out == "f16":
        assert np.array_equal(co.view(np.uint16), r.astype(np.float16).view(np.uint16))
    else:
        assert np.array_equal(co, r.astype(np.float32))
    # rows of C beyond m (the ld padding) keep their input bytes
    assert np.all(np.isnan(pad.astype(np.float32)))


# ---------------------------------------------------------------- closed forms

@pytest.mark.parametrize("tA,tB", TRANS)
@pytest.mark.parametrize("out", ["f16", "f32"])
def test_identity_left_and_right(oracle_mod, tA, tB, out):
    k = 40
    X = inputs.uniform_f16(k, 23, seed=5)
    co, _, _, _ = _run(oracle_mod, np.eye(k), X, tA, tB, pad=2, out=out)
    assert np.array_equal(co.astype(np.float64), X.astype(np.float64))
    Y = inputs.uniform_f16(19, k, seed=6)
    co, _, _, _ = _run(oracle_mod, Y, np.eye(k), tA, tB, pad=1, out=out)
    assert np.array_equal(co.astype(np.float64), Y.astype(np.float64))


@pytest.mark.parametrize("tA,tB", TRANS)
def test_permutation(oracle_mod, tA, tB):
    k = 37
    perm = np.random.Generator(np.random.PCG64(3)).permutation(k)
    P = np.eye(k)[perm]
    X = inputs.uniform_f16(k, 11, seed=9)
    co, _, _, _ = _run(oracle_mod, P, X, tA, tB, out="f16")
    assert np.array_equal(co.view(np.uint16), X[perm].view(np.uint16))
    co, _, _, _ = _run(oracle_mod, X.T.copy(), P.T.copy(), tA, tB, out="f16")
    assert np.array_equal(co.view(np.uint16), X.T[:, perm].view(np.uint16))


@pytest.mark.parametrize("tA,tB", TRANS)
@pytest.mark.parametrize("alpha,beta", [(1.0, 0.0), (2.0, 1.0), (-0.5, -1.0), (1.0, 0.5)])
def test_integer_exact(oracle_mod, tA, tB, alpha, beta):
    m, n, k = 29, 31, 96
    opA = inputs.integer_f16(m, k, seed=21)
    opB = inputs.integer_f16(k, n, seed=22)
    C = inputs.integer_f16(m, n, seed=23, lo=-100, hi=100).astype(np.float32)
    exact = opA.astype(np.int64) @ opB.astype(np.int64)
    want = alpha * exact.astype(np.float64) + beta * C.astype(np.float64)
    co, r, _, _ = _run(oracle_mod, opA, opB, tA, tB, alpha, beta, C=C, out="f32", pad=4)
    assert np.array_equal(r, want)
    assert np.array_equal(co, want.astype(np.float32))


def test_k_zero_and_alpha_zero(oracle_mod):
    m, n = 5, 4
    C = inputs.integer_f16(m, n, seed=1)
    for tA, tB in TRANS:
        co, r, ab, _ = _run(oracle_mod, np.zeros((m, 0)), np.zeros((0, n)), tA, tB, 1.0, 2.0, C=C)
        assert np.array_equal(r, 2.0 * C.astype(np.float64))
        assert np.all(ab == 0)
        A = np.full((m, 3), np.inf)
        co, r, _, _ = _run(oracle_mod, A, np.ones((3, n)), tA, tB, 0.0, -1.0, C=C)
        assert np.array_equal(r, -C.astype(np.float64))
        co, r, _, _ = _run(oracle_mod, A, np.ones((3, n)), tA, tB, 0.0, 0.0, C=C)
        assert np.array_equal(r, np.zeros((m, n)))


def test_beta_zero_never_reads_C(oracle_mod):
    opA = inputs.uniform_f16(9, 12, seed=1)
    opB = inputs.uniform_f16(12, 7, seed=2)
    co, r, _, _ = _run(oracle_mod, opA, opB, "N", "N", 1.0, 0.0, C=np.full((9, 7), np.nan))
    assert not np.any(np.isnan(r))
    assert not np.any(np.isnan(co.astype(np.float32)))


@pytest.mark.parametrize("k", [64, 256, 4096])
def test_accumulator_width_closed_form(oracle_mod, k):
    a, b, expect = inputs.accumulator_width_case(3, 2, k)
    for tA, tB in TRANS:
        co, r, _, _ = _run(oracle_mod, a, b, tA, tB, out="f16")
        assert np.all(r == expect)
        assert np.all(co.astype(np.float64) == expect)


def test_entries_match_full(oracle_mod):
    m, n, k = 50, 40, 70
    opA = inputs.uniform_f16(m, k, seed=31)
    opB = inputs.uniform_f16(k, n, seed=32)
    C = inputs.uniform_f16(m, n, seed=33)
    for tA, tB in TRANS:
        A, lda = inputs.store_op(opA, tA, ld=inputs.stored_shape(m, k, tA)[0] + 2)
        B, ldb = inputs.store_op(opB, tB)
        Cb = inputs.to_colmajor(C, m + 1)
        full, r, ab = oracle_mod.hgemm_ref(m, n, k, 0.75, A, lda, B, ldb, -1.5, Cb, m + 1, tA, tB, "f16")
        g = np.random.Generator(np.random.PCG64(4))
        ii = g.integers(0, m, 300)
        jj = g.integers(0, n, 300)
        c2, r2, ab2 = oracle_mod.hgemm_ref_entries(m, n, k, 0.75, A, lda, B, ldb, -1.5, Cb, m + 1,
                                                   tA, tB, "f16", ii, jj, nthreads=3)
        assert np.array_equal(r2, r[ii, jj])
        assert np.array_equal(ab2, ab[ii, jj])
        assert np.array_equal(c2, full.reshape(m + 1, n, order="F")[ii, jj])


def test_rejects_bad_arguments(oracle_mod):
    A = np.zeros(4, dtype=np.uint16)
    with pytest.raises(ValueError):
        oracle_mod.hgemm_ref(2, 2, 2, 1.0, A, 2, A, 2, 0.0, None, 1, "N", "N", "f16")
    with pytest.raises(ValueError):
        oracle_mod.hgemm_ref_entries(2, 2, 2, 1.0, A, 2, A, 2, 0.0, None, 2, "N", "N", "f16",
                                     [2], [0])
