"""Sharded path on one GPU (world size 1): the slab/panel bookkeeping around the
CUDA kernels gives bitwise the single-call result (same per-element K order), and
that result agrees with the CPU oracle on sampled entries (north_star (4))."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _setup(m, n, k, seed=0):
    from .test_gpu_allgather import _inputs
    A, B, C0 = _inputs(m, n, k, k, "f16", 1.0, seed)   # host-drawn (inputs.py), copied to the device
    return A, B, C0


@pytest.mark.parametrize("beta", [0.0, 1.0])
def test_sharded_world1_equals_single_call(oracle_mod, beta):
    import torch
    from paper_conf_ipps_00020c20_b200 import binding, hgemm_sharded, hgemm_sharded_overlapped
    m, n, k = 2048, 1536, 1024
    A, B, C0 = _setup(m, n, k)
    binding.set_config("tc2", block_n=256, stream_k=1)   # whole tiles: the bitwise claim needs one k order
    try:
        ref = C0.clone()
        binding.hgemm(m, n, k, 1.0, A, k, B, k, beta, ref, m, "T", "N", "f16")
        c1 = C0.clone()
        assert hgemm_sharded(m, n, k, 1.0, A, k, B, k, beta, c1, m, "T", "N", "f16") == (0, n)
        c2 = C0.clone()
        assert hgemm_sharded_overlapped(m, n, k, 1.0, A, k, B, k, beta, c2, m, "T", "N", "f16", panels=4) == (0, n)
        torch.cuda.synchronize()
    finally:
        binding.set_config()
    r = ref.cpu().numpy().view(np.uint16)
    assert np.array_equal(c1.cpu().numpy().view(np.uint16), r)
    assert np.array_equal(c2.cpu().numpy().view(np.uint16), r)
    from .test_gpu_allgather import oracle_check
    oracle_check(oracle_mod, m, n, k, A, k, B, k, beta, C0, c1, "f16")
