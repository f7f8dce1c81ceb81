"""GPU parity of the FP16-accumulate compute type (hgemm_ex, HGEMM_COMPUTE_F16).

The paper's kernel accumulates in FP16 (HMMA.1688.F16, SIV-A; its
register budget only fits FP16 accumulators, SVI-A.3); the B200 build
offers it as an opt-in compute type (tcgen05.mma kind::f16 with c_format = F16,
SURVEY 8(f) NEXT-4).  FP16 accumulation has no exact plain definition (the
order and rounding of the partial sums inside the tensor core are unspecified),
so it is checked against what is fixed:

* random inputs in [-1,1): the BASELINE.json north_star (4) bound against the
  exact FP64 oracle, and a diagnostic showing the accumulator really is FP16
  (error well above what FP32 accumulation gives);
* integer inputs whose every partial sum is an integer of magnitude <= 2048:
  exact in FP16 in any order, so bit-exact against the oracle;
* the accumulator-width case: a 4096 = 64*64 head, one unit
  product per 16-deep K step, -4096 at the end.  An FP16 accumulator (ulp 4 at
  4096) drops every unit, so the closed-form result is exactly 0; FP32 gives
  k/16 - 2 (tests/test_gpu_parity.py);
* the accumulator probe (informational): base 2048*2048 = 2^22 with FP32
  accumulation is exact with a 24-bit significand, 0 with 22 bits.
"""
import numpy as np
import pytest

from paper_conf_ipps_00020c20_b200 import inputs

from .gpu_util import GpuCase, assert_within_tolerance

pytestmark = pytest.mark.gpu

TRANS = [("N", "N"), ("N", "T"), ("T", "N"), ("T", "T")]
TILES = [("auto", 0), ("tc2", 512), ("tc2", 256), ("simt", 0)]


@pytest.fixture(autouse=True)
def _reset_config():
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config()
    yield
    binding.set_config()


def _use(kernel, bn):
    from paper_conf_ipps_00020c20_b200 import binding
    if kernel == "auto":
        binding.set_config()
    else:
        binding.set_config(kernel, block_n=bn)


@pytest.mark.parametrize("kernel,bn", TILES)
@pytest.mark.parametrize("tA,tB", TRANS)
def test_acc16_accumulator_width_is_zero(kernel, bn, tA, tB):
    _use(kernel, bn)
    for k in (1024, 4096):
        a, b, fp32_exact = inputs.accumulator_width_case(300, 264, k)
        case = GpuCase(a, b, tA, tB, out="f16")
        got = case.view(case.run_gpu(compute="f16")).astype(np.float64)
        assert np.all(got == 0.0), (k, np.unique(got)[:5])
        if kernel != "simt":
            assert case.stats["last_kernel"] == "tc2", case.stats
        # the same inputs through the FP32 compute type keep every unit term
        got32 = case.view(case.run_gpu(compute="f32")).astype(np.float64)
        assert np.all(got32 == fp32_exact)


@pytest.mark.parametrize("kernel,bn", TILES)
@pytest.mark.parametrize("tA,tB", TRANS)
@pytest.mark.parametrize("alpha,beta", [(1.0, 0.0), (2.0, 1.0), (1.0, -1.0)])
def test_acc16_integer_bit_exact(oracle_mod, kernel, bn, tA, tB, alpha, beta):
    _use(kernel, bn)
    m, n, k = 300, 520, 512          # every partial sum |.| <= 512 * 4 = 2048: exact in FP16
    opA = inputs.integer_f16(m, k, 31, -2, 2)
    opB = inputs.integer_f16(k, n, 32, -2, 2)
    C = inputs.integer_f16(m, n, 33, -8, 8)
    case = GpuCase(opA, opB, tA, tB, alpha=alpha, beta=beta, C=C, out="f16", pad=(8, 16, 8))
    got = case.run_gpu(compute="f16")
    c_ref, r, _ = case.oracle(oracle_mod)
    # the accumulator is exact (integer partial sums |.| <= 2048); the epilogue
    # alpha*acc + beta*c is exact in FP32 and rounded once to FP16, like the oracle's r
    assert np.array_equal(case.view(got).astype(np.float64), case.view(c_ref).astype(np.float64))  # IEEE ==
    small = np.abs(r) <= 2048
    assert np.array_equal(case.view(got).astype(np.float64)[small], r[small])
    assert np.all(np.isnan(case.padding(got).astype(np.float32)))   # ld padding never written


@pytest.mark.parametrize("kernel,bn", TILES)
@pytest.mark.parametrize("tA,tB", TRANS)
@pytest.mark.parametrize("beta", [0.0, 1.0])
def test_acc16_random_within_bound(oracle_mod, kernel, bn, tA, tB, beta):
    _use(kernel, bn)
    m, n, k = 333, 520, 1000
    C = inputs.uniform_f16(m, n, 43) if beta else None
    case = GpuCase(inputs.uniform_f16(m, k, 41), inputs.uniform_f16(k, n, 42), tA, tB, beta=beta, C=C, out="f16")
    got = case.run_gpu(compute="f16")
    _, r, ab = case.oracle(oracle_mod)
    rel = assert_within_tolerance(case, got, r, ab)
    # FP16 accumulation is visible: FP32 accumulation stays below 1e-5 of |A||B| (test_gpu_parity)
    assert 1e-5 < rel < 1e-3, rel


def test_acc16_full_size_sampled(oracle_mod):
    """8192^3 TN (the metric shape) with FP16 accumulation: sampled entries and tile edges."""
    import torch
    from paper_conf_ipps_00020c20_b200 import binding
    from .test_gpu_large import _device_inputs, _sample_indices
    from .gpu_util import tolerance
    m = n = k = 8192
    (hA, lda), (hB, ldb), hC, dA, dB, dC = _device_inputs(m, n, k, "T", "N", 500, 0.0, "f16")
    binding.hgemm_ex(m, n, k, 1.0, dA, lda, dB, ldb, 0.0, dC, m, "T", "N", "f16", compute="f16")
    torch.cuda.synchronize()
    assert binding.get_stats()["last_kernel"] == "tc2"
    got = dC.cpu().numpy().view(np.float16)
    ii, jj = _sample_indices(m, n, seed=500)
    _, r, ab = oracle_mod.hgemm_ref_entries(m, n, k, 1.0, hA, lda, hB, ldb, 0.0, None, m, "T", "N", "f16", ii, jj,
                                            nthreads=oracle_mod.max_threads())
    g = got[ii + jj * m].astype(np.float64)
    bound = tolerance(r, ab, 1.0, 0.0, None, "f16", g)
    assert np.all(np.abs(g - r) <= bound)


def test_acc16_invalid_arguments():
    import torch
    from paper_conf_ipps_00020c20_b200 import binding
    A = torch.zeros(64, 64, dtype=torch.float16, device="cuda")
    C32 = torch.zeros(64, 64, dtype=torch.float32, device="cuda")
    with pytest.raises(binding.HgemmError):     # FP16 accumulation needs FP16 output
        binding.hgemm_ex(64, 64, 64, 1.0, A, 64, A, 64, 0.0, C32, 64, "T", "N", "f32", compute="f16")
    with pytest.raises(binding.HgemmError):     # unknown compute type
        binding.hgemm_ex(64, 64, 64, 1.0, A, 64, A, 64, 0.0, A, 64, "T", "N", "f16", compute=7)


@pytest.mark.parametrize("compute", ["f32", "f16"])
def test_accumulator_probe_informational(compute, capsys):
    """Base 2048*2048 = 2^22 (SURVEY 8(c) "accumulator probe"): with FP32 accumulation the
    result is k/16 - 2 if the tensor core keeps a 24-bit significand (0 with 22 bits); with
    FP16 accumulation 2^22 overflows FP16 (max 65504), so the result is not finite or 0.
    Recorded, not asserted beyond the FP32 case's two admissible values."""
    k = 4096
    a, b, exact = inputs.accumulator_width_case(128, 128, k, base=2048.0)
    case = GpuCase(a, b, "T", "N", out="f16" if compute == "f16" else "f32")
    got = case.view(case.run_gpu(compute=compute)).astype(np.float64)
    vals = np.unique(got)
    print(f"accumulator probe ({compute} accumulate, base 2^11, k={k}): values {vals[:4]} (exact {exact})")
    if compute == "f32":
        assert set(vals.tolist()) <= {exact, 0.0}
