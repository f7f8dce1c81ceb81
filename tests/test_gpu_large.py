"""GPU parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (automatic kernel selection), on sampled outputs the oracle computes one
by one: random entries plus full rows and columns at tile edges."""
import numpy as np
import pytest

from paper_conf_ipps_00020c20_b200 import inputs

from .gpu_util import tolerance

pytestmark = pytest.mark.gpu


def _device_inputs(m, n, k, tA, tB, seed, beta, out):
    """Seeded inputs generated on the host (inputs.py) and copied to the device."""
    import torch
    sa = inputs.stored_shape(m, k, tA)
    sb = inputs.stored_shape(k, n, tB)
    A = inputs.uniform_f16(sa[0], sa[1], seed)          # stored matrices (column-major, ld = rows)
    B = inputs.uniform_f16(sb[0], sb[1], seed + 1)
    C = inputs.uniform_f16(m, n, seed + 2) if beta != 0 else None
    cdt = np.float32 if out == "f32" else np.float16
    hA = A.reshape(-1, order="F")
    hB = B.reshape(-1, order="F")
    hC = (C.astype(cdt).reshape(-1, order="F") if C is not None else np.zeros(m * n, cdt))
    dA = torch.from_numpy(hA.view(np.int16)).cuda()
    dB = torch.from_numpy(hB.view(np.int16)).cuda()
    dC = torch.from_numpy(hC.view(np.int16) if out == "f16" else hC).cuda()
    return (hA, sa[0]), (hB, sb[0]), hC, dA, dB, dC


def _sample_indices(m, n, tile=256, count=4096, seed=0):
    g = np.random.Generator(np.random.PCG64(seed))
    ii = list(g.integers(0, m, count))
    jj = list(g.integers(0, n, count))
    edge_rows = sorted({0, min(127, m - 1), min(128, m - 1), min(tile - 1, m - 1), min(tile, m - 1), m - 1})
    edge_cols = sorted({0, min(127, n - 1), min(128, n - 1), min(tile - 1, n - 1), min(tile, n - 1), n - 1})
    for i in edge_rows:                     # full rows at tile edges
        ii += [i] * n
        jj += list(range(n))
    for j in edge_cols:                     # full columns at tile edges
        ii += list(range(m))
        jj += [j] * m
    return np.array(ii, np.int64), np.array(jj, np.int64)


def _check_sampled(oracle_mod, m, n, k, tA, tB, alpha, beta, out, seed=100):
    import torch
    from paper_conf_ipps_00020c20_b200 import binding
    (hA, lda), (hB, ldb), hC, dA, dB, dC = _device_inputs(m, n, k, tA, tB, seed, beta, out)
    binding.set_config()
    binding.hgemm(m, n, k, alpha, dA, lda, dB, ldb, beta, dC, m, tA, tB, out)
    torch.cuda.synchronize()
    got = dC.cpu().numpy()
    if out == "f16":
        got = got.view(np.float16)
    ii, jj = _sample_indices(m, n, seed=seed)
    _, r, ab = oracle_mod.hgemm_ref_entries(m, n, k, alpha, hA, lda, hB, ldb, beta, hC, m, tA, tB, out, ii, jj,
                                            nthreads=oracle_mod.max_threads())
    g = got[ii + jj * m].astype(np.float64)
    cvals = hC[ii + jj * m].astype(np.float64) if beta != 0 else None
    bound = tolerance(r, ab, alpha, beta, cvals, out, g)
    bad = ~(np.abs(g - r) <= bound)
    assert not bad.any(), f"{bad.sum()} sampled entries out of tolerance"
    if out == "f32":
        rel = float(np.max(np.abs(g - r) / np.maximum(ab, 1e-30)))
        assert rel < 1e-5, rel
    return got, binding.get_stats()


@pytest.mark.slow
@pytest.mark.parametrize("tA,tB,out", [("T", "N", "f16"), ("N", "N", "f16"), ("N", "T", "f16"), ("T", "N", "f32")])
def test_metric_config_8192(oracle_mod, tA, tB, out):
    got, stats = _check_sampled(oracle_mod, 8192, 8192, 8192, tA, tB, 1.0, 0.0, out)
    assert stats["last_kernel"] == "tc2"


@pytest.mark.slow
@pytest.mark.parametrize("name", ["cfg1_256_NN_f32", "cfg3_bert_ffn1_4096", "cfg3_bert_ffn1_16384", "cfg3_bert_ffn2_4096",
                                  "cfg3_lstm_b64", "cfg3_lstm_b256", "cfg3_lstm_b1024", "cfg4_skinny_n64",
                                  "cfg4_skinny_n128", "cfg4_skinny_n256"])
def test_baseline_configs(oracle_mod, name):
    m, n, k, tA, tB, alpha, beta, out = inputs.WORKLOADS[name]
    _check_sampled(oracle_mod, m, n, k, tA, tB, alpha, beta, out, seed=200)


@pytest.mark.slow
@pytest.mark.parametrize("w,beta,out", [(7168, 0.0, "f16"), (6400, 1.0, "f16"), (7680, 0.0, "f32")])
def test_half_tile_tail_full_size(oracle_mod, w, beta, out):
    """Square sizes of the paper sweep where the automatic choice runs 512-wide tiles
    with the half-tile tail: sampled entries, tile edges."""
    got, stats = _check_sampled(oracle_mod, w, w, w, "T", "N", 1.0, beta, out, seed=300)
    assert stats["last_kernel"] == "tc2" and stats["block_n"] == 512 and stats["half_tail"] == 2, stats


@pytest.mark.slow
def test_vs_cublas_full_matrix():
    """Whole-matrix cross-check against cuBLAS (torch.mm, FP32 accumulation forced)."""
    import torch
    from paper_conf_ipps_00020c20_b200 import hgemm_torch
    torch.backends.cuda.matmul.allow_fp16_reduced_precision_reduction = False
    g = torch.Generator(device="cuda").manual_seed(5)
    A = (torch.rand(4096, 4096, generator=g, device="cuda") * 2 - 1).half()
    W = (torch.rand(4096, 4096, generator=g, device="cuda") * 2 - 1).half()
    ours = hgemm_torch(A, W.t(), out_dtype=torch.float32)
    ref = torch.mm(A.float(), W.float().t())
    absab = torch.mm(A.float().abs(), W.float().abs().t())
    assert torch.all((ours - ref).abs() <= 2e-3 * absab)


def test_hgemm_torch_layouts(oracle_mod):
    import torch
    from paper_conf_ipps_00020c20_b200 import hgemm_torch
    M, N, K = 333, 517, 264
    a = inputs.uniform_f16(M, K, 1)
    b = inputs.uniform_f16(K, N, 2)
    exact = a.astype(np.float64) @ b.astype(np.float64)
    absab = np.abs(a.astype(np.float64)) @ np.abs(b.astype(np.float64))
    A = torch.from_numpy(np.ascontiguousarray(a)).cuda()
    B = torch.from_numpy(np.ascontiguousarray(b)).cuda()
    for Aop in (A, A.t().contiguous().t()):
        for Bop in (B, B.t().contiguous().t()):
            C = hgemm_torch(Aop, Bop, out_dtype=torch.float32)
            assert np.all(np.abs(C.cpu().numpy() - exact) <= 1e-3 * absab)
    C0 = torch.from_numpy(np.ascontiguousarray(inputs.uniform_f16(M, N, 3))).cuda()
    C = C0.clone()
    hgemm_torch(A, B, C, alpha=0.5, beta=2.0)
    want = 0.5 * exact + 2.0 * C0.double().cpu().numpy()
    bound = 1e-3 * (0.5 * absab + 2 * np.abs(C0.double().cpu().numpy())) + 2.0**-9 * np.abs(want) + 2**-24
    assert np.all(np.abs(C.double().cpu().numpy() - want) <= bound)


# ---------------------------------------------------------------- BJ config 5: 32768^3, N-sharded
def _cfg5_case(oracle_mod, n0, n1, *, integer=False, out="f16", seed=600, n_glob=32768):
    """One rank's N-slab [n0, n1) of BASELINE.json configs[4] (m = n = k = 32768, TN, FP16 out),
    generated block by block (inputs.uniform_f16_blocked) so the slab is exactly those
    columns of the global B, run through hgemm() with the automatic choice (what
    bench.py times per rank), checked on sampled entries + tile-edge rows/columns
    against the oracle."""
    import torch
    from paper_conf_ipps_00020c20_b200 import binding
    m = k = 32768
    ns = n1 - n0
    if integer:   # |C| <= ~6 sigma = 6*sqrt(k*4/9) ~ 720 < 2048: exact in FP32 and in FP16
        At = inputs.integer_f16_blocked(k, m, seed, -1, 1)                       # stored A: k x m (op(A)^T)
        Bs = inputs.integer_f16_blocked(k, n_glob, seed + 1, -1, 1, col0=n0, ncols=ns)
    else:
        At = inputs.uniform_f16_blocked(k, m, seed)
        Bs = inputs.uniform_f16_blocked(k, n_glob, seed + 1, col0=n0, ncols=ns)
    hA = At.reshape(-1, order="F")
    hB = Bs.reshape(-1, order="F")
    dA = torch.from_numpy(hA.view(np.int16)).cuda()
    dB = torch.from_numpy(hB.view(np.int16)).cuda()
    cdt = torch.float32 if out == "f32" else torch.float16
    dC = torch.full((ns, m), float("nan"), dtype=cdt, device="cuda")
    binding.set_config()
    binding.hgemm(m, ns, k, 1.0, dA, k, dB, k, 0.0, dC, m, "T", "N", out)
    torch.cuda.synchronize()
    stats = binding.get_stats()
    got = dC.cpu().numpy()
    del dA, dB, dC
    torch.cuda.empty_cache()
    if out == "f16":
        got = got.view(np.float16)
    got = got.reshape(-1)                      # column-major C slab, ldc = m
    ii, jj = _sample_indices(m, ns, count=2048, seed=seed)
    _, r, ab = oracle_mod.hgemm_ref_entries(m, ns, k, 1.0, hA, k, hB, k, 0.0, None, m, "T", "N", out, ii, jj,
                                            nthreads=oracle_mod.max_threads())
    g = got[ii + jj * m].astype(np.float64)
    if integer:
        assert np.array_equal(g, r), f"{np.sum(g != r)} sampled entries differ (integer inputs must be exact)"
    else:
        bound = tolerance(r, ab, 1.0, 0.0, None, out, g)
        bad = ~(np.abs(g - r) <= bound)
        assert not bad.any(), f"{bad.sum()} sampled entries out of tolerance"
        rel = float(np.max(np.abs(g - r) / np.maximum(ab, 1e-30)))
        assert rel < 1e-5 + (2.0 ** -10 if out == "f16" else 0.0), rel
    return stats


@pytest.mark.slow
@pytest.mark.parametrize("out", ["f16", "f32"])
def test_cfg5_full_32768_one_gpu(oracle_mod, out):
    """The whole 32768^3 problem on one GPU (the G = 1 point of config 5)."""
    stats = _cfg5_case(oracle_mod, 0, 32768, out=out)
    assert stats["last_kernel"] == "tc2", stats


@pytest.mark.slow
@pytest.mark.parametrize("g", [0, 7])
def test_cfg5_g8_slab(oracle_mod, g):
    """Rank g's slab at G = 8 (32768 x 4096 x 32768): the per-GPU problem of the 8-GPU run."""
    stats = _cfg5_case(oracle_mod, 4096 * g, 4096 * (g + 1))
    assert stats["last_kernel"] == "tc2", stats


@pytest.mark.slow
def test_cfg5_g8_slab_integer_exact(oracle_mod):
    """Integer inputs in [-1, 1] at k = 32768 through the automatic multi-wave persistent path:
    every partial sum is an integer < 2^24, so the sampled entries must be bit-exact."""
    _cfg5_case(oracle_mod, 4096 * 3, 4096 * 4, integer=True)


@pytest.mark.slow
def test_cfg5_full_integer_exact(oracle_mod):
    _cfg5_case(oracle_mod, 0, 32768, integer=True, out="f32")
