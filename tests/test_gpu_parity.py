"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Rules (BASELINE.json north_star (4)):
  * random inputs in [-1,1): |C_gpu - r| <= 1e-3*(|alpha||A||B| + |beta||C|)_ij,
    + one FP16 ulp for FP16 output;
  * integer-valued, identity, permutation and accumulator-width inputs:
    bit-exact in value (IEEE ==);
  * beta == 0 never reads C; quick returns; ld padding never read/written.
Shapes span several tiles plus ragged tails in every dimension.
"""
import numpy as np
import pytest

from paper_conf_ipps_00020c20_b200 import inputs

from .gpu_util import GpuCase, assert_within_tolerance, ulp16

pytestmark = pytest.mark.gpu

TRANS = [("N", "N"), ("N", "T"), ("T", "N"), ("T", "T")]
KERNELS = [("tc2", 512), ("tc2", 256), ("tc1", 256), ("tc1", 128), ("splitk", 64), ("splitk", 128), ("simt", 0)]
TC_KERNELS = KERNELS[:4]   # same K order inside the tensor core -> bitwise identical results


@pytest.fixture(autouse=True)
def _reset_config():
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config()
    yield
    binding.set_config()


def _use(kernel, bn):
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config(kernel, block_n=bn)


def _expect_kernel(case, kernel, bn=0):
    if kernel != "auto":
        assert case.stats["last_kernel"] == kernel, case.stats
    if bn:
        assert case.stats["block_n"] == bn, case.stats


@pytest.mark.parametrize("kernel,bn", KERNELS)
@pytest.mark.parametrize("tA,tB", TRANS)
@pytest.mark.parametrize("out", ["f16", "f32"])
def test_random_ragged(oracle_mod, kernel, bn, tA, tB, out):
    m, n, k = 300, 520, 200          # 2-3 tiles + ragged tails in m, n and k
    _use(kernel, bn)
    case = GpuCase(inputs.uniform_f16(m, k, 1), inputs.uniform_f16(k, n, 2), tA, tB, out=out, pad=(8, 16, 8))
    got = case.run_gpu()
    _expect_kernel(case, kernel, bn)
    c_ref, r, ab = case.oracle(oracle_mod)
    rel = assert_within_tolerance(case, got, r, ab)
    if out == "f32":   # diagnostic: FP32 accumulation error is ~1e-7 of |A||B|
        assert rel < 1e-5, f"precision regression: max err/absab = {rel}"
    else:              # FP16 output: same diagnostic plus one FP16 ulp of output rounding
        g = case.view(got).astype(np.float64)
        assert np.all(np.abs(g - r) <= 1e-5 * ab + ulp16(np.maximum(np.abs(g), np.abs(r))))
    # padding rows of C are never written
    assert np.all(np.isnan(case.padding(got).astype(np.float32)))


@pytest.mark.parametrize("kernel,bn", KERNELS)
@pytest.mark.parametrize("tA,tB", TRANS)
@pytest.mark.parametrize("out", ["f16", "f32"])
def test_integer_bit_exact(oracle_mod, kernel, bn, tA, tB, out):
    m, n, k = 257, 391, 1000
    _use(kernel, bn)
    opA = inputs.integer_f16(m, k, 3, -4, 4)
    opB = inputs.integer_f16(k, n, 4, -4, 4)
    if out == "f16":  # keep |C| <= 2048 so FP16 output is exact
        opA = (opA.astype(np.float32) / 2).round().astype(np.float16)
    case = GpuCase(opA, opB, tA, tB, out=out)
    got = case.run_gpu()
    _expect_kernel(case, kernel)
    c_ref, r, _ = case.oracle(oracle_mod)
    if out == "f16":
        assert np.max(np.abs(r)) <= 2048
    assert np.array_equal(case.view(got).astype(np.float64), r)
    assert np.array_equal(case.view(got), case.view(c_ref))


@pytest.mark.parametrize("kernel,bn", KERNELS)
@pytest.mark.parametrize("tA,tB", TRANS)
def test_identity_and_permutation(oracle_mod, kernel, bn, tA, tB):
    _use(kernel, bn)
    k = 384
    X = inputs.uniform_f16(k, 200, 5)
    case = GpuCase(np.eye(k, dtype=np.float16), X, tA, tB, out="f16")
    got = case.run_gpu()
    assert np.array_equal(case.view(got).view(np.uint16), X.view(np.uint16))
    perm = np.random.Generator(np.random.PCG64(8)).permutation(k)
    P = np.eye(k, dtype=np.float16)[perm]
    Y = inputs.uniform_f16(150, k, 6)
    case = GpuCase(Y, P.T.copy(), tA, tB, out="f32")
    got = case.run_gpu()
    assert np.array_equal(case.view(got), Y[:, perm].astype(np.float32))


@pytest.mark.parametrize("kernel,bn", KERNELS)
@pytest.mark.parametrize("k", [4096, 8192])
def test_accumulator_width(oracle_mod, kernel, bn, k):
    """FP32 accumulation gets k/16 - 2 exactly; an FP16 accumulator returns 0."""
    _use(kernel, bn)
    a, b, expect = inputs.accumulator_width_case(256, 256, k)
    for tA, tB in TRANS:
        case = GpuCase(a, b, tA, tB, out="f32")
        got = case.view(case.run_gpu())
        assert np.all(got == expect), (tA, tB, np.unique(got)[:5])


@pytest.mark.parametrize("kernel,bn", KERNELS)
@pytest.mark.parametrize("alpha,beta", [(1.0, 0.0), (2.0, 1.0), (-0.5, -1.0), (1.0, 0.5), (0.25, 2.0)])
@pytest.mark.parametrize("out", ["f16", "f32"])
def test_alpha_beta_integer(oracle_mod, kernel, bn, alpha, beta, out):
    _use(kernel, bn)
    m, n, k = 200, 300, 128
    opA = inputs.integer_f16(m, k, 9, -3, 3)
    opB = inputs.integer_f16(k, n, 10, -3, 3)
    C = inputs.integer_f16(m, n, 11, -64, 64)
    case = GpuCase(opA, opB, "T", "N", alpha, beta, C=C, out=out, pad=(0, 0, 8))
    got = case.run_gpu()
    c_ref, r, _ = case.oracle(oracle_mod)
    assert np.array_equal(case.view(got).astype(np.float64), r)


# (kernel, block_n, max_ctas): few persistent clusters, so every CTA runs several
# tiles in a row and the staging boxes that carry C (TMA-loaded, combined in place,
# TMA-stored) rotate across tiles and accumulator halves.
BETA_CASES = [("tc2", 512, 4), ("tc2", 256, 4), ("tc1", 256, 3), ("tc1", 128, 5), ("tc2", 512, 0), ("tc1", 128, 0)]


@pytest.mark.parametrize("kernel,bn,max_ctas", BETA_CASES)
@pytest.mark.parametrize("tA,tB", [("T", "N"), ("N", "T")])
@pytest.mark.parametrize("out", ["f16", "f32"])
@pytest.mark.parametrize("m", [600, 597])   # 597: N (= m) not a multiple of 16 B -> chunked path
def test_beta_random_multi_tile(oracle_mod, kernel, bn, max_ctas, tA, tB, out, m):
    """beta != 0 on random inputs, several tiles per CTA, ragged m/n/k, ld padding."""
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config(kernel, block_n=bn, max_ctas=max_ctas, stream_k=1)
    n, k = 1100, 200
    C = inputs.uniform_f16(m, n, 17).astype(np.float32 if out == "f32" else np.float16)
    case = GpuCase(inputs.uniform_f16(m, k, 15), inputs.uniform_f16(k, n, 16), tA, tB, 0.75, -1.25, C=C,
                   out=out, pad=(8, 16, 8))
    got = case.run_gpu()
    _expect_kernel(case, kernel, bn)
    _, r, ab = case.oracle(oracle_mod)
    assert_within_tolerance(case, got, r, ab)
    assert np.all(np.isnan(case.padding(got).astype(np.float32)))


@pytest.mark.parametrize("kernel,bn", KERNELS)
@pytest.mark.parametrize("out", ["f16", "f32"])
def test_beta_zero_never_reads_C(oracle_mod, kernel, bn, out):
    _use(kernel, bn)
    m, n, k = 130, 270, 96
    case = GpuCase(inputs.uniform_f16(m, k, 1), inputs.uniform_f16(k, n, 2), "N", "N", 1.0, 0.0,
                   out=out, c_fill=np.nan)
    got = case.view(case.run_gpu())
    assert not np.any(np.isnan(got.astype(np.float32)))


def test_quick_returns(oracle_mod):
    m, n = 100, 70
    C = inputs.uniform_f16(m, n, 3)
    for out in ("f16", "f32"):
        # k == 0 -> C = beta*C
        case = GpuCase(np.zeros((m, 0), np.float16), np.zeros((0, n), np.float16), "N", "N", 1.0, 2.0,
                       C=C, out=out)
        got = case.view(case.run_gpu()).astype(np.float64)
        assert np.array_equal(got, (2.0 * C.astype(np.float64)).astype(np.float16 if out == "f16" else np.float32))
        # alpha == 0 with inf in A -> C = beta*C, A*B not evaluated
        A = np.full((m, 5), np.inf, np.float16)
        case = GpuCase(A, np.ones((5, n), np.float16), "N", "N", 0.0, -1.0, C=C, out=out)
        got = case.view(case.run_gpu()).astype(np.float64)
        assert np.array_equal(got, -C.astype(np.float64))
        # alpha == 0, beta == 0 -> zeros without reading a NaN C
        case = GpuCase(A, np.ones((5, n), np.float16), "N", "N", 0.0, 0.0, out=out, c_fill=np.nan)
        got = case.view(case.run_gpu()).astype(np.float64)
        assert np.all(got == 0)


def test_degenerate_shapes(oracle_mod):
    for (m, n, k) in [(1, 1, 1), (1, 300, 70), (300, 1, 70), (7, 9, 1), (129, 257, 63), (16, 16, 16)]:
        for tA, tB in TRANS:
            case = GpuCase(inputs.uniform_f16(m, k, m + k), inputs.uniform_f16(k, n, n + 7 * k), tA, tB, out="f32")
            got = case.run_gpu()
            _, r, ab = case.oracle(oracle_mod)
            assert_within_tolerance(case, got, r, ab)


def test_unaligned_falls_back_to_simt(oracle_mod):
    m, n, k = 130, 70, 77
    case = GpuCase(inputs.uniform_f16(m, k, 1), inputs.uniform_f16(k, n, 2), "T", "N", out="f16", pad=(3, 5, 1),
                   align=False)
    got = case.run_gpu()
    assert case.stats["last_kernel"] == "simt"
    _, r, ab = case.oracle(oracle_mod)
    assert_within_tolerance(case, got, r, ab)


def test_overflow_to_inf(oracle_mod):
    opA = np.full((128, 64), 16.0, np.float16)
    opB = np.full((64, 128), 64.0, np.float16)      # 64 * 1024 = 65536 -> inf
    for kernel, bn in KERNELS:
        _use(kernel, bn)
        case = GpuCase(opA, opB, "T", "N", out="f16")
        got = case.view(case.run_gpu())
        assert np.all(np.isposinf(got.astype(np.float32)))


def test_deterministic(oracle_mod):
    m, n, k = 1000, 700, 1500
    case = GpuCase(inputs.uniform_f16(m, k, 1), inputs.uniform_f16(k, n, 2), "T", "N", out="f32")
    a, b = case.run_gpu(repeat=2)
    assert np.array_equal(a.view(np.uint32), b.view(np.uint32))


def test_all_kernels_agree_on_random(oracle_mod):
    """Different tile shapes only change which CTA computes an element, not the K
    order inside the tensor core, so tc1/tc2 results are bitwise identical."""
    m, n, k = 700, 900, 640
    base = None
    from paper_conf_ipps_00020c20_b200 import binding
    for kernel, bn in TC_KERNELS:
        binding.set_config(kernel, block_n=bn, stream_k=1)   # whole tiles: no k split anywhere
        case = GpuCase(inputs.uniform_f16(m, k, 1), inputs.uniform_f16(k, n, 2), "T", "N", out="f32")
        got = case.run_gpu()
        if base is None:
            base = got
        else:
            assert np.array_equal(got.view(np.uint32), base.view(np.uint32)), kernel


# (kernel, block_n, max_ctas): cluster counts that give stream-K ranges of
# 40 / 24 k-blocks (two segments per split tile), 12 (three segments: tiles
# fewer than clusters) and whole data-parallel waves before the stream-K part.
SK_CASES = [("tc2", 256, 8), ("tc2", 256, 32), ("tc1", 256, 8), ("tc1", 128, 12), ("tc1", 128, 40),
            ("tc1", 128, 4), ("tc2", 512, 8), ("tc2", 512, 4), ("tc2", 512, 12)]


@pytest.mark.parametrize("kernel,bn,max_ctas", SK_CASES)
@pytest.mark.parametrize("tA,tB", TRANS)
@pytest.mark.parametrize("out,beta", [("f16", 0.0), ("f16", 1.0), ("f32", 0.5)])
def test_stream_k(oracle_mod, kernel, bn, max_ctas, tA, tB, out, beta):
    """Stream-K: tiles split in k between clusters and summed through the FP32
    workspace in k order -- within tolerance, deterministic across launches
    (the flags return to 0 after every launch), padding untouched."""
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config(kernel, block_n=bn, max_ctas=max_ctas, stream_k=2)
    m, n, k = 300, 520, 2000
    C = inputs.uniform_f16(m, n, 7).astype(np.float32 if out == "f32" else np.float16)
    case = GpuCase(inputs.uniform_f16(m, k, 5), inputs.uniform_f16(k, n, 6), tA, tB, 1.0, beta, C=C, out=out,
                   pad=(8, 16, 8))
    a, b, c = case.run_gpu(repeat=3)
    assert case.stats["last_kernel"] == kernel and case.stats["stream_k"] == 2, case.stats
    u = np.uint32 if out == "f32" else np.uint16
    assert np.array_equal(a.view(u), b.view(u)) and np.array_equal(a.view(u), c.view(u))
    _, r, ab = case.oracle(oracle_mod)
    assert_within_tolerance(case, a, r, ab)
    assert np.all(np.isnan(case.padding(a).astype(np.float32)))


@pytest.mark.parametrize("kernel,bn,max_ctas", SK_CASES)
def test_stream_k_integer_exact(oracle_mod, kernel, bn, max_ctas):
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config(kernel, block_n=bn, max_ctas=max_ctas, stream_k=2)
    opA = inputs.integer_f16(300, 1984, 3, -4, 4)
    opB = inputs.integer_f16(1984, 520, 4, -4, 4)
    case = GpuCase(opA, opB, "T", "N", out="f32")
    got = case.view(case.run_gpu())
    assert case.stats["stream_k"] == 2, case.stats
    _, r, _ = case.oracle(oracle_mod)
    assert np.array_equal(got.astype(np.float64), r)
    a, b, expect = inputs.accumulator_width_case(300, 520, 2048)
    case = GpuCase(a, b, "N", "T", out="f32")
    assert np.all(case.view(case.run_gpu()) == expect)


@pytest.mark.parametrize("kernel,bn,max_ctas", [("tc2", 256, 8), ("tc2", 256, 32), ("tc1", 128, 12)])
@pytest.mark.parametrize("out,beta", [("f16", 1.0), ("f32", 0.0)])
def test_stream_k_kgroup(oracle_mod, kernel, bn, max_ctas, out, beta):
    """Stream-K with k-group stages (256-wide pair tiles, TN, k % 128 == 0): work items split at
    even k-blocks (units of two), summed through the workspace in k order -- within tolerance,
    deterministic across launches; integer inputs exact."""
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config(kernel, block_n=bn, max_ctas=max_ctas, stream_k=2)
    m, n, k = 300, 520, 2048
    C = inputs.uniform_f16(m, n, 7).astype(np.float32 if out == "f32" else np.float16)
    case = GpuCase(inputs.uniform_f16(m, k, 5), inputs.uniform_f16(k, n, 6), "T", "N", 1.0, beta, C=C, out=out,
                   pad=(8, 16, 8))
    a, b, c = case.run_gpu(repeat=3)
    assert case.stats["stream_k"] == 2 and case.stats["splits"] == 2, case.stats
    u = np.uint32 if out == "f32" else np.uint16
    assert np.array_equal(a.view(u), b.view(u)) and np.array_equal(a.view(u), c.view(u))
    _, r, ab = case.oracle(oracle_mod)
    assert_within_tolerance(case, a, r, ab)
    opA, opB = inputs.integer_f16(m, k, 3, -4, 4), inputs.integer_f16(k, n, 4, -4, 4)
    case = GpuCase(opA, opB, "T", "N", out="f32")
    got = case.view(case.run_gpu())
    assert case.stats["stream_k"] == 2 and case.stats["splits"] == 2, case.stats
    _, r, _ = case.oracle(oracle_mod)
    assert np.array_equal(got.astype(np.float64), r)


def test_stream_k_graph_capture(oracle_mod):
    """Stream-K inside a captured CUDA graph: the workspace is created by an
    eager call on the stream first; replays reuse it (flags reset each launch)."""
    import torch
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config("tc2", block_n=256, max_ctas=8, stream_k=2)
    m, n, k = 300, 520, 2000
    case = GpuCase(inputs.uniform_f16(m, k, 1), inputs.uniform_f16(k, n, 2), "T", "N", 1.0, 0.0, out="f32")
    dA = torch.from_numpy(case.A.view(np.int16).copy()).cuda()
    dB = torch.from_numpy(case.B.view(np.int16).copy()).cuda()
    dC = torch.full((case.ldc * n,), float("nan"), dtype=torch.float32, device="cuda")
    s = torch.cuda.Stream()
    args = (m, n, k, 1.0, dA, case.lda, dB, case.ldb, 0.0, dC, case.ldc, "T", "N", "f32", s.cuda_stream)
    with torch.cuda.stream(s):
        binding.hgemm(*args)
    torch.cuda.synchronize()
    eager = dC.cpu().numpy().copy()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.stream(s):
        with torch.cuda.graph(g, stream=s):
            binding.hgemm(*args)
    assert binding.get_stats()["stream_k"] == 2
    for _ in range(3):
        dC.fill_(float("nan"))
        g.replay()
        torch.cuda.synchronize()
        assert np.array_equal(dC.cpu().numpy().view(np.uint32), eager.view(np.uint32))
    _, r, ab = case.oracle(oracle_mod)
    assert_within_tolerance(case, eager, r, ab)


@pytest.mark.parametrize("splits", [2, 4, 8])
@pytest.mark.parametrize("bn", [64, 128])
@pytest.mark.parametrize("tA,tB", TRANS)
def test_splitk_splits(oracle_mod, splits, bn, tA, tB):
    """Split-K over a cluster: every split count, ragged K ranges (some splits empty);
    k = 1024 (16 k-blocks) takes the 2-k-block stages (3-D Ak view) for a K-major op(B)^T."""
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config("splitk", block_n=bn, splits=splits)
    for (m, n, k) in [(200, 300, 1000), (64, 4096, 448), (130, 257, 100), (72, 1000, 1024)]:
        case = GpuCase(inputs.uniform_f16(m, k, 7), inputs.uniform_f16(k, n, 8), tA, tB, 1.0, 0.5,
                       C=inputs.uniform_f16(m, n, 9), out="f16")
        got = case.run_gpu()
        assert case.stats["last_kernel"] == "splitk" and case.stats["splits"] == splits, case.stats
        _, r, ab = case.oracle(oracle_mod)
        assert_within_tolerance(case, got, r, ab)
        a, b = case.run_gpu(repeat=2)
        assert np.array_equal(a.view(np.uint16), b.view(np.uint16))   # deterministic reduction order
    for kk in (640, 2048):
        opA = inputs.integer_f16(90, kk, 3, -4, 4)
        opB = inputs.integer_f16(kk, 70, 4, -4, 4)
        case = GpuCase(opA, opB, tA, tB, out="f32")
        got = case.view(case.run_gpu())
        _, r, _ = case.oracle(oracle_mod)
        assert np.array_equal(got.astype(np.float64), r)


def test_splitk_auto_for_underfilled(oracle_mod):
    """LSTM-gate shape (m=64 batch, n=4096, k=2048) in NN layout (no streaming kernel):
    automatic selection splits K."""
    m, n, k = 64, 4096, 2048
    case = GpuCase(inputs.uniform_f16(m, k, 1), inputs.uniform_f16(k, n, 2), "N", "N", 1.0, 1.0,
                   C=inputs.uniform_f16(m, n, 3), out="f16")
    got = case.run_gpu()
    assert case.stats["last_kernel"] == "splitk", case.stats
    _, r, ab = case.oracle(oracle_mod)
    assert_within_tolerance(case, got, r, ab)


@pytest.mark.parametrize("w,tA,tB,out,spl", [(256, "N", "N", "f32", 4), (384, "T", "N", "f16", 4),
                                              (512, "N", "N", "f32", 4), (768, "T", "N", "f16", 2),
                                              (333, "T", "T", "f16", 4), (200, "T", "T", "f16", 4),
                                              (250, "N", "T", "f32", 4), (130, "T", "N", "f16", 2)])
def test_splitk_auto_small_problems(oracle_mod, w, tA, tB, out, spl):
    """Small problems (K <= 1024, one wave of 128 x 64 split tiles) go to the 64-wide split-K
    kernel automatically (BJ config 1 among them; W <= 256 with 64-row "HM" tiles): random
    inputs within the BJ bound and integer inputs bit-exact, ragged sizes included."""
    for integer in (False, True):
        if integer:
            opA, opB = inputs.integer_f16(w, w, 5, -2, 2), inputs.integer_f16(w, w, 6, -2, 2)
        else:
            opA, opB = inputs.uniform_f16(w, w, 5), inputs.uniform_f16(w, w, 6)
        case = GpuCase(opA, opB, tA, tB, out=out)
        got = case.run_gpu()
        st = case.stats
        assert st["last_kernel"] == "splitk" and st["block_n"] == 64 and st["splits"] == spl, st
        c_ref, r, ab = case.oracle(oracle_mod)
        if integer:
            assert out == "f32" or np.max(np.abs(r)) <= 2048  # exact in FP16
            assert np.array_equal(case.view(got).astype(np.float64), r)
        else:
            assert_within_tolerance(case, got, r, ab)


@pytest.mark.parametrize("kernel,bn", [("tc2", 256), ("tc1", 128)])
@pytest.mark.parametrize("m,n,k", [(520, 600, 1024), (300, 1100, 384), (1000, 700, 2048)])
@pytest.mark.parametrize("out", ["f16", "f32"])
@pytest.mark.parametrize("beta", [0.0, 1.0])
def test_tc_kgroup_stages(oracle_mod, kernel, bn, m, n, k, out, beta):
    """256-wide CTA-pair tiles and 1-SM 128 x 128 tiles with two k-blocks per ring stage (3-D
    TMA boxes; layout TN, k % 128 == 0, stream-K off): random inputs within the BJ bound,
    integer inputs bit-exact, ragged m / n."""
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config(kernel, block_n=bn, stream_k=1)
    for integer in (False, True):
        if integer:
            opA, opB = inputs.integer_f16(m, k, 21, -2, 2), inputs.integer_f16(k, n, 22, -2, 2)
            C = inputs.integer_f16(m, n, 23, -16, 16)
        else:
            opA, opB, C = inputs.uniform_f16(m, k, 21), inputs.uniform_f16(k, n, 22), inputs.uniform_f16(m, n, 23)
        case = GpuCase(opA, opB, "T", "N", 1.0, beta, C=C, out=out)
        got = case.run_gpu()
        assert case.stats["last_kernel"] == kernel and case.stats["block_n"] == bn, case.stats
        assert case.stats["splits"] == 2, case.stats   # k-group stages
        c_ref, r, ab = case.oracle(oracle_mod)
        if integer:
            assert out == "f32" or np.max(np.abs(r)) <= 2048
            assert np.array_equal(case.view(got).astype(np.float64), r)
        else:
            assert_within_tolerance(case, got, r, ab)


def test_tc_kgroup_accumulator_width(oracle_mod):
    """k-group stages keep the FP32 accumulator: k/16 - 2 exactly (512 x 512, k = 4096, TN)."""
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config("tc2", block_n=256, stream_k=1)
    a, b, expect = inputs.accumulator_width_case(512, 512, 4096)
    case = GpuCase(a, b, "T", "N", out="f32")
    got = case.view(case.run_gpu())
    assert case.stats["splits"] == 2, case.stats
    assert np.all(got == expect), np.unique(got)[:5]


def test_cuda_graph_capture_and_replay(oracle_mod):
    """hgemm() is asynchronous and allocation-free, so it can be captured in a CUDA graph."""
    import torch
    from paper_conf_ipps_00020c20_b200 import binding
    m, n, k = 384, 640, 512
    case = GpuCase(inputs.uniform_f16(m, k, 1), inputs.uniform_f16(k, n, 2), "T", "N", 1.0, 0.0, out="f32")
    dA = torch.from_numpy(case.A.view(np.int16).copy()).cuda()
    dB = torch.from_numpy(case.B.view(np.int16).copy()).cuda()
    dC = torch.full((case.ldc * n,), float("nan"), dtype=torch.float32, device="cuda")
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    with torch.cuda.stream(s):
        with torch.cuda.graph(g, stream=s):
            binding.hgemm(m, n, k, 1.0, dA, case.lda, dB, case.ldb, 0.0, dC, case.ldc, "T", "N", "f32",
                          s.cuda_stream)
    dC.fill_(float("nan"))
    g.replay()
    torch.cuda.synchronize()
    _, r, ab = case.oracle(oracle_mod)
    assert_within_tolerance(case, dC.cpu().numpy(), r, ab)


@pytest.mark.parametrize("tA,tB", TRANS)
@pytest.mark.parametrize("out,beta", [("f16", 0.0), ("f16", 1.0), ("f32", 0.5)])
def test_hgemm_host_buffers(oracle_mod, tA, tB, out, beta):
    """Host-buffer entry point: panelled H2D / GEMM / D2H pipeline gives the same C."""
    import torch
    from paper_conf_ipps_00020c20_b200 import binding
    m, n, k = 300, 2600, 520            # several column panels + ragged tails; host ld padding
    case = GpuCase(inputs.uniform_f16(m, k, 1), inputs.uniform_f16(k, n, 2), tA, tB, 1.0, beta,
                   C=inputs.uniform_f16(m, n, 3), out=out, pad=(3, 5, 7), align=False)
    hA = torch.from_numpy(case.A.view(np.int16).copy()).pin_memory()
    hB = torch.from_numpy(case.B.view(np.int16).copy()).pin_memory()
    cv = case.C_in.view(np.int16) if out == "f16" else case.C_in
    hC = torch.from_numpy(cv.copy()).pin_memory()
    ws_bytes = binding.host_workspace_size(m, n, k, tA, tB, out)
    ws = torch.empty(ws_bytes, dtype=torch.uint8, device="cuda")
    binding.hgemm_host(m, n, k, 1.0, hA, case.lda, hB, case.ldb, beta, hC, case.ldc, tA, tB, out, ws)
    got = hC.numpy()
    if out == "f16":
        got = got.view(np.float16)
    _, r, ab = case.oracle(oracle_mod)
    assert_within_tolerance(case, got, r, ab)
    # the host padding rows of C are untouched
    pad = case.padding(got).astype(np.float32)
    assert np.all(np.isnan(pad))


@pytest.mark.parametrize("tA,tB", [("T", "N"), ("N", "T")])
def test_hgemm_host_row_pieces(oracle_mod, tA, tB):
    """m >= 4096: the first column panel's GEMM runs in row pieces of op(A) (started as their
    rows arrive), the last panel in slices; beta = 1 so every element is written exactly once."""
    import torch
    from paper_conf_ipps_00020c20_b200 import binding
    m, n, k = 4100, 2600, 264
    case = GpuCase(inputs.integer_f16(m, k, 61, -2, 2), inputs.integer_f16(k, n, 62, -2, 2), tA, tB, 1.0, 1.0,
                   C=inputs.integer_f16(m, n, 63, -4, 4), out="f32", pad=(3, 5, 7), align=False)
    hA = torch.from_numpy(case.A.view(np.int16).copy()).pin_memory()
    hB = torch.from_numpy(case.B.view(np.int16).copy()).pin_memory()
    hC = torch.from_numpy(case.C_in.copy()).pin_memory()
    ws = torch.empty(binding.host_workspace_size(m, n, k, tA, tB, "f32"), dtype=torch.uint8, device="cuda")
    binding.hgemm_host(m, n, k, 1.0, hA, case.lda, hB, case.ldb, 1.0, hC, case.ldc, tA, tB, "f32", ws)
    _, r, _ = case.oracle(oracle_mod)
    assert np.array_equal(case.view(hC.numpy()).astype(np.float64), r)
    assert np.all(np.isnan(case.padding(hC.numpy())))


# ------------------------------------------------------------------ HBM-streaming kernel (skinny, TN)
@pytest.mark.parametrize("n", [64, 100, 128, 200, 256])
@pytest.mark.parametrize("cw,max_ctas", [(48, 0), (112, 3), (16, 5), (128, 0)])
@pytest.mark.parametrize("out,beta", [("f16", 0.0), ("f16", 0.5), ("f32", 0.0), ("f32", -1.5)])
def test_stream_kernel(oracle_mod, n, cw, max_ctas, out, beta):
    """Streaming kernel: chunks of cw rows of op(A) per persistent CTA (max_ctas
    forces several chunks per CTA -> both TMEM accumulator buffers), 1 or 2
    M-subtiles (n <= 128 / <= 256), ragged m, n and k, ld padding untouched."""
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config("stream", block_n=cw, max_ctas=max_ctas)
    m, k = 1003, 330
    C = inputs.uniform_f16(m, n, 27).astype(np.float32 if out == "f32" else np.float16)
    case = GpuCase(inputs.uniform_f16(m, k, 25), inputs.uniform_f16(k, n, 26), "T", "N", 1.25, beta, C=C,
                   out=out, pad=(8, 16, 8))
    got = case.run_gpu()
    assert case.stats["last_kernel"] == "stream", case.stats
    assert case.stats["block_n"] == (min(cw, 128) if n > 128 else cw), case.stats
    _, r, ab = case.oracle(oracle_mod)
    assert_within_tolerance(case, got, r, ab)
    if out == "f32":
        rel = np.max(np.abs(case.view(got).astype(np.float64) - r) / np.maximum(ab + np.abs(beta) * np.abs(case.Cmat), 1e-30))
        assert rel < 1e-5, rel
    assert np.all(np.isnan(case.padding(got).astype(np.float32)))


@pytest.mark.parametrize("n", [64, 256])
def test_stream_kernel_integer_exact(oracle_mod, n):
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config("stream", block_n=64)
    opA = inputs.integer_f16(2000, 1024, 31, -4, 4)
    opB = inputs.integer_f16(1024, n, 32, -4, 4)
    case = GpuCase(opA, opB, "T", "N", out="f32")
    got = case.view(case.run_gpu())
    assert case.stats["last_kernel"] == "stream", case.stats
    _, r, _ = case.oracle(oracle_mod)
    assert np.array_equal(got.astype(np.float64), r)
    a, b, expect = inputs.accumulator_width_case(2000, n, 4096)
    case = GpuCase(a, b, "T", "N", out="f32")
    assert np.all(case.view(case.run_gpu()) == expect)
    assert case.stats["last_kernel"] == "stream", case.stats


@pytest.mark.parametrize("n", [64, 100, 128])
@pytest.mark.parametrize("k,g", [(640, 2), (704, 1), (4096, 2)])
@pytest.mark.parametrize("cw,max_ctas", [(112, 0), (48, 5)])
@pytest.mark.parametrize("out,beta", [("f16", 0.5), ("f32", 0.0)])
def test_stream_kernel_kgroup(oracle_mod, n, k, g, cw, max_ctas, out, beta):
    """Streaming kernel with K a multiple of 64: G = 2 consecutive k-blocks per stage
    through the 3-D op(A) tensor map when G divides the k-block count (640, 4096),
    G = 1 through the 2-D map when it does not (704 = 11 k-blocks); ragged m, several
    chunks per CTA (max_ctas), k rotation across CTAs."""
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config("stream", block_n=cw, max_ctas=max_ctas)
    m = 1003
    C = inputs.uniform_f16(m, n, 57).astype(np.float32 if out == "f32" else np.float16)
    case = GpuCase(inputs.uniform_f16(m, k, 55), inputs.uniform_f16(k, n, 56), "T", "N", 0.75, beta, C=C,
                   out=out, pad=(8, 16, 8))
    got = case.run_gpu()
    assert case.stats["last_kernel"] == "stream", case.stats
    assert case.stats["splits"] == g, case.stats
    _, r, ab = case.oracle(oracle_mod)
    assert_within_tolerance(case, got, r, ab)
    assert np.all(np.isnan(case.padding(got).astype(np.float32)))


def test_stream_routing_by_n(oracle_mod):
    """Automatic choice on the skinny TN shapes: n <= 128 streams, n in (128, 256] takes
    the 2-SM tile kernel (faster there); both against the oracle on sampled entries."""
    m, k = 16384, 512
    for n, expect in ((96, "stream"), (128, "stream"), (192, "tc2"), (256, "tc2")):
        case = GpuCase(inputs.uniform_f16(m, k, 61), inputs.uniform_f16(k, n, 62), "T", "N", out="f16")
        got = case.run_gpu()
        assert case.stats["last_kernel"] == expect, (n, case.stats)
        rows = np.arange(0, m, 89)
        ii, jj = np.meshgrid(rows, np.arange(n), indexing="ij")
        _, r, ab = oracle_mod.hgemm_ref_entries(m, n, k, 1.0, case.A, case.lda, case.B, case.ldb, 0.0, None,
                                                case.ldc, "T", "N", "f16", ii.ravel(), jj.ravel())
        g = case.view(got)[ii.ravel(), jj.ravel()].astype(np.float64)
        assert np.all(np.abs(g - r) <= 1e-3 * ab + ulp16(np.maximum(np.abs(g), np.abs(r))))


def test_stream_kernel_auto_and_fallback(oracle_mod):
    """Automatic choice: the skinny TN shape of BJ configs[3] takes the streaming
    kernel; the same shape in NN layout takes the tile kernels (still correct)."""
    m, n, k = 16384, 64, 512
    for tA, tB, expect in (("T", "N", "stream"), ("N", "N", None)):
        case = GpuCase(inputs.uniform_f16(m, k, 41), inputs.uniform_f16(k, n, 42), tA, tB, out="f16")
        got = case.run_gpu()
        if expect:
            assert case.stats["last_kernel"] == expect, case.stats
        else:
            assert case.stats["last_kernel"] != "stream", case.stats
        rows = np.arange(0, m, 97)
        cols = np.arange(n)
        ii, jj = np.meshgrid(rows, cols, indexing="ij")
        _, r, ab = oracle_mod.hgemm_ref_entries(m, n, k, 1.0, case.A, case.lda, case.B, case.ldb, 0.0, None,
                                                case.ldc, tA, tB, "f16", ii.ravel(), jj.ravel())
        g = case.view(got)[ii.ravel(), jj.ravel()].astype(np.float64)
        assert np.all(np.abs(g - r) <= 1e-3 * ab + ulp16(np.maximum(np.abs(g), np.abs(r))))


# Half-tile tail (forced with hgemm_config_t.half_tail = 2):
# with 512-wide tiles, a last wave of r <= clusters/2 tiles runs as 2r 256-wide items.  (m, n, max_ctas): kernel tiles =
# ceil(n/256) x ceil(m/512); clusters = max_ctas/2.
#   (1500, 1100, 12): 5 x 3 = 15 tiles on 6 clusters -> 2 whole waves + 3 split tiles
#   (1100, 1100, 12): same grid, the last tile column is 76 wide: its second half is
#                     entirely outside N (loads zero-filled, stores clipped)
#   (1100,  700,  0): 3 x 3 = 9 tiles on 74 clusters -> every tile split
#   (1497, 1100, 22): 15 tiles on 11 clusters -> 1 wave + 4 split tiles; N = 1497 is
#                     not a multiple of 16 B -> chunked epilogue
HALF_CASES = [(1500, 1100, 12), (1100, 1100, 12), (1100, 700, 0), (1497, 1100, 22)]


@pytest.mark.parametrize("m,n,max_ctas", HALF_CASES)
@pytest.mark.parametrize("tA,tB", [("T", "N"), ("N", "T")])
@pytest.mark.parametrize("out,beta", [("f16", 0.0), ("f16", 1.0), ("f32", 0.5)])
def test_half_tile_tail(oracle_mod, m, n, max_ctas, tA, tB, out, beta):
    """512-wide tiles with the split tail: within tolerance of the oracle and bitwise
    equal to the 256-wide kernel (same K order per element)."""
    from paper_conf_ipps_00020c20_b200 import binding
    k = 520
    C = inputs.uniform_f16(m, n, 27).astype(np.float32 if out == "f32" else np.float16)
    opA, opB = inputs.uniform_f16(m, k, 25), inputs.uniform_f16(k, n, 26)
    binding.set_config("tc2", block_n=512, max_ctas=max_ctas, stream_k=1, half_tail=2)
    case = GpuCase(opA, opB, tA, tB, 1.0, beta, C=C, out=out, pad=(8, 16, 8))
    got, again = case.run_gpu(repeat=2)
    _expect_kernel(case, "tc2", 512)
    assert case.stats["half_tail"] == 2, case.stats
    binding.set_config("tc2", block_n=256, max_ctas=max_ctas, stream_k=1)
    ref256 = GpuCase(opA, opB, tA, tB, 1.0, beta, C=C, out=out, pad=(8, 16, 8)).run_gpu()
    u = np.uint32 if out == "f32" else np.uint16
    assert np.array_equal(got.view(u), again.view(u))
    assert np.array_equal(got.view(u), ref256.view(u))
    _, r, ab = case.oracle(oracle_mod)
    assert_within_tolerance(case, got, r, ab)
    assert np.all(np.isnan(case.padding(got).astype(np.float32)))


def test_half_tile_tail_integer_exact(oracle_mod):
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config("tc2", block_n=512, max_ctas=12, stream_k=1, half_tail=2)
    opA = inputs.integer_f16(1500, 1024, 3, -4, 4)
    opB = inputs.integer_f16(1024, 1100, 4, -4, 4)
    case = GpuCase(opA, opB, "T", "N", out="f32")
    got = case.view(case.run_gpu())
    _, r, _ = case.oracle(oracle_mod)
    assert np.array_equal(got.astype(np.float64), r)


def test_half_tile_tail_regression_slow_epilogue(oracle_mod):
    """The case that exposed a tmem_full parity alias (a half item as a CTA's third
    work item, beta != 0, entirely outside N), run repeatedly."""
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config("tc2", block_n=512, max_ctas=12, stream_k=1, half_tail=2)
    m, n, k = 1100, 1100, 520
    C = inputs.uniform_f16(m, n, 27).astype(np.float16)
    case = GpuCase(inputs.uniform_f16(m, k, 25), inputs.uniform_f16(k, n, 26), "T", "N", 1.0, 1.0, C=C, out="f16")
    outs = case.run_gpu(repeat=20)
    assert case.stats["half_tail"] == 2
    assert all(np.array_equal(o.view(np.uint16), outs[0].view(np.uint16)) for o in outs)
    _, r, ab = case.oracle(oracle_mod)
    assert_within_tolerance(case, outs[0], r, ab)


# Streaming kernel with swapped operands (small m, long n; TN; forced with the "stream"
# kernel choice): op(A) resident, op(B) streamed, C stored transposed from the
# accumulator.
@pytest.mark.parametrize("m,n", [(1, 2400), (64, 4096), (100, 4100), (256, 2500)])
@pytest.mark.parametrize("out,beta", [("f16", 0.0), ("f16", 1.0), ("f32", -0.5)])
def test_stream_swapped(oracle_mod, m, n, out, beta):
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config("stream")   # forced: not chosen automatically (slower than split-K here)
    k = 520
    C = inputs.uniform_f16(m, n, 37).astype(np.float32 if out == "f32" else np.float16)
    case = GpuCase(inputs.uniform_f16(m, k, 35), inputs.uniform_f16(k, n, 36), "T", "N", 1.5, beta, C=C,
                   out=out, pad=(8, 16, 8))
    got = case.run_gpu()
    assert case.stats["last_kernel"] == "stream" and case.stats["group_m"] == 1, case.stats
    _, r, ab = case.oracle(oracle_mod)
    assert_within_tolerance(case, got, r, ab)
    assert np.all(np.isnan(case.padding(got).astype(np.float32)))


def test_stream_swapped_integer_exact(oracle_mod):
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config("stream")
    opA = inputs.integer_f16(64, 2048, 33, -4, 4)
    opB = inputs.integer_f16(2048, 4096, 34, -4, 4)
    case = GpuCase(opA, opB, "T", "N", out="f32")
    got = case.view(case.run_gpu())
    assert case.stats["last_kernel"] == "stream" and case.stats["group_m"] == 1, case.stats
    _, r, _ = case.oracle(oracle_mod)
    assert np.array_equal(got.astype(np.float64), r)


@pytest.mark.parametrize("tile_n", [128, 144, 160, 192, 240])
@pytest.mark.parametrize("tA,tB", [("T", "N"), ("T", "T")])   # flexible widths need a K-major op(A)
@pytest.mark.parametrize("out,beta", [("f16", 0.0), ("f32", 0.0), ("f16", 1.0), ("f32", -0.5)])
def test_flexible_tile_width(oracle_mod, tile_n, tA, tB, out, beta):
    """CTA-pair kernel with tiles of tile_n columns: chunks
    that cross a tile end are stored directly, never by a TMA box running into the next tile."""
    from paper_conf_ipps_00020c20_b200 import binding
    binding.set_config("tc2", block_n=256, tile_n=tile_n)
    m, n, k = 1000, 600, 328           # several tiles of every width + ragged m / n / k
    C = inputs.uniform_f16(m, n, 23) if beta else None
    case = GpuCase(inputs.uniform_f16(m, k, 21), inputs.uniform_f16(k, n, 22), tA, tB, beta=beta, C=C, out=out,
                   pad=(8, 16, 8))
    got = case.run_gpu()
    assert case.stats["last_kernel"] == "tc2" and case.stats["tile_n"] == tile_n % 256, case.stats
    _, r, ab = case.oracle(oracle_mod)
    assert_within_tolerance(case, got, r, ab)
    assert np.all(np.isnan(case.padding(got).astype(np.float32)))
    # integer inputs: bit-exact, and every element written exactly once (beta = 1 over an integer C)
    opA = inputs.integer_f16(m, k, 24, -2, 2)
    opB = inputs.integer_f16(k, n, 25, -2, 2)
    Ci = inputs.integer_f16(m, n, 26, -4, 4)
    case = GpuCase(opA, opB, tA, tB, beta=1.0, C=Ci, out="f32")
    got = case.run_gpu()
    _, r, _ = case.oracle(oracle_mod)
    assert np.array_equal(case.view(got).astype(np.float64), r)


@pytest.mark.parametrize("w", [1792, 2304, 2560])
def test_flexible_tile_width_auto_mid_square(oracle_mod, w):
    """The automatic choice at mid-size squares of the paper sweep, sampled against the oracle."""
    from .test_gpu_large import _check_sampled
    got, stats = _check_sampled(oracle_mod, w, w, w, "T", "N", 1.0, 0.0, "f16", seed=700)
    assert stats["last_kernel"] in ("tc2", "tc1", "splitk"), stats
