"""Fused all-gather of op(A) + GEMM on one B200 (include/hgemm.h hgemm_allgather_a).

Only one GPU is available, so the ranks are either
* "virtual": W gather buffers on the same device, each holding only its
  rank's rows of op(A) (the rest NaN), the call for rank r pulling the others
  with the kernel's copy warps (from the same HBM instead of over NVLink); or
* real processes: two processes on cuda:0 exchanging CUDA IPC handles over a
  gloo group (sharded.FusedAllGatherA, the code path of a multi-GPU run).
Every result must be bitwise equal to hgemm() on the full A (whole tiles, one
k order per element), and the gather buffer must end equal to the full A; the
fused result is also checked against the CPU oracle on sampled entries and
tile-edge rows/columns (north_star (4) bound), so the sharded path is anchored
to the paper's definition and not only to hgemm().  Inputs are drawn on the
host by inputs.py (the generators the oracle's callers use) and copied over.
A test checks that the kernel waits for its copy warps: with k = 32768 (one
64 KB row per copy unit, 7/8 of the rows remote) the tiles of peer chunks are
scheduled long before their rows are all in place, and the result must still
be exact.
"""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _dev(x):
    import torch
    return torch.from_numpy(np.ascontiguousarray(x)).cuda()


def _inputs(m, n, k, lda, out, beta, seed=0):
    """Host-drawn seeded inputs (inputs.py) on the device: A (m, lda) with row i = op(A)
    row i (the 'T' layout: stored k x m column-major), B (n, k) = stored k x n ('N'),
    C0 (n, m) = column-major C."""
    import torch
    from paper_conf_ipps_00020c20_b200 import inputs
    A = torch.full((m, lda), float("nan"), dtype=torch.float16, device="cuda")
    A[:, :k] = _dev(inputs.uniform_f16(m, k, 10 * seed + 1))
    B = _dev(inputs.uniform_f16(n, k, 10 * seed + 2))
    cdt = torch.float32 if out == "f32" else torch.float16
    C0 = _dev(inputs.uniform_f16(n, m, 10 * seed + 3)).to(cdt) if beta != 0 else \
        torch.full((n, m), float("nan"), dtype=cdt, device="cuda")
    return A, B, C0


def oracle_check(oracle_mod, m, n, k, A, lda, B, ldb, beta, C0, C, out, count=1024, seed=0):
    """Sampled entries + tile-edge rows/columns of the column-major C (m x n, ldc = m)
    against the oracle, north_star (4) bound.  A: (.., lda) rows = op(A) rows ('T');
    B: (n, ldb) rows = op(B) columns ('N')."""
    from .gpu_util import tolerance
    from .test_gpu_large import _sample_indices

    def bits(t):
        h = t.cpu().numpy().reshape(-1)
        return h.view(np.uint16) if h.dtype == np.float16 else h
    hA, hB = bits(A), bits(B)
    hC0 = bits(C0) if beta != 0 else None
    ii, jj = _sample_indices(m, n, count=count, seed=seed)
    _, r, ab = oracle_mod.hgemm_ref_entries(m, n, k, 1.0, hA, lda, hB, ldb, beta, hC0, m, "T", "N", out, ii, jj,
                                            nthreads=oracle_mod.max_threads())
    got = C.cpu().numpy().reshape(-1)[ii + jj * m].astype(np.float64)
    cv = C0.cpu().numpy().reshape(-1)[ii + jj * m].astype(np.float64) if beta != 0 else None
    bound = tolerance(r, ab, 1.0, beta, cv, out, got)
    bad = ~(np.abs(got - r) <= bound)
    assert not bad.any(), f"{bad.sum()} of {ii.size} sampled entries outside the north_star (4) bound"


def _reference(m, n, k, A, lda, B, beta, C0, out):
    from paper_conf_ipps_00020c20_b200 import binding
    ref = C0.clone()
    binding.set_config(stream_k=1)
    try:
        binding.hgemm(m, n, k, 1.0, A, lda, B, k, beta, ref, m, "T", "N", out)
    finally:
        binding.set_config()
    return ref


def _bits(t):
    return t.cpu().numpy().view(np.uint16 if t.element_size() == 2 else np.uint32)


def _virtual(m, n, k, world, chunk_rows, out="f16", beta=0.0, lda=None, calls=1, expect_fused=True, oracle_mod=None):
    import torch
    from paper_conf_ipps_00020c20_b200 import binding
    from paper_conf_ipps_00020c20_b200.sharded import slab_bounds
    lda = lda or k + (-k) % 8
    A, B, C0 = _inputs(m, n, k, lda, out, beta)
    ref = _reference(m, n, k, A, lda, B, beta, C0, out)
    rs = [slab_bounds(m, world, q, align=chunk_rows)[0] for q in range(world)] + [m]
    ws = torch.full((2 + m // chunk_rows,), 12345, dtype=torch.int32, device="cuda")   # zeroed by the call
    for rank in range(world):
        bufs = []
        for q in range(world):
            b = torch.full_like(A, float("nan"))
            b[rs[q]:rs[q + 1]] = A[rs[q]:rs[q + 1]]
            bufs.append(b)
        for it in range(calls):
            C = C0.clone()
            for q in range(world):        # the peers' rows must be fetched again by every call
                if q != rank:
                    bufs[rank][rs[q]:rs[q + 1]] = float("nan")
            l0 = binding.get_stats()["launches"]
            binding.hgemm_allgather_a(m, n, k, 1.0, bufs[rank], lda, bufs, rs, rank, B, k, beta, C, m, "N", out,
                                      workspace=ws, chunk_rows=chunk_rows)
            torch.cuda.synchronize()
            st = binding.get_stats()
            if expect_fused:
                assert st["launches"] - l0 == 1 and st["last_kernel"] == "tc2"   # one kernel did both
            assert np.array_equal(_bits(C), _bits(ref)), f"rank {rank} call {it}: C differs from hgemm()"
            assert np.array_equal(_bits(bufs[rank][:, :k]), _bits(A[:, :k])), f"rank {rank}: gather incomplete"
    if oracle_mod is not None:   # the last rank's fused result against the paper's definition
        oracle_check(oracle_mod, m, n, k, A, lda, B, k, beta, C0, C, out)


@pytest.mark.parametrize("m,n,k,world,chunk_rows,out,beta", [
    (2048, 1024, 512, 1, 512, "f16", 0.0),
    (4096, 1536, 1024, 2, 1024, "f16", 0.0),     # chunk-aligned: one raster group per chunk, rotated
    (4096, 768, 640, 4, 512, "f32", 1.0),
    (3000, 700, 328, 3, 512, "f16", -1.0),       # ragged m / n / k, partial last chunk
    (2560, 1000, 256, 2, 384, "f16", 0.0),       # chunk not a multiple of the tile: no rotation
])
def test_virtual_ranks_bitwise(oracle_mod, m, n, k, world, chunk_rows, out, beta):
    _virtual(m, n, k, world, chunk_rows, out, beta, oracle_mod=oracle_mod)


def test_kernel_waits_for_its_copy_warps(oracle_mod):
    # k = 32768: one 64 KB row per copy unit, 7 of 8 chunks remote, large enough that
    # the first tiles of every remote chunk are scheduled before their rows are in
    _virtual(4096, 4096, 32768, 8, 512, oracle_mod=oracle_mod)


def test_repeated_calls():
    _virtual(2048, 1024, 512, 2, 512, calls=3)


def test_unaligned_lda_falls_back_unfused():
    # lda % 8 != 0 breaks the TMA preconditions: copies on the stream first, then hgemm()
    _virtual(1024, 512, 256, 2, 256, lda=259, expect_fused=False)


def test_unaligned_shards_fall_back_unfused():
    import torch
    from paper_conf_ipps_00020c20_b200 import binding
    m, n, k = 1000, 384, 256
    A, B, C0 = _inputs(m, n, k, k, "f16", 0.0)
    ref = _reference(m, n, k, A, k, B, 0.0, C0, "f16")
    rs = [0, 300, 1000]                                # not on 256-row chunk boundaries
    bufs = [torch.full_like(A, float("nan")) for _ in range(2)]
    for q in range(2):
        bufs[q][rs[q]:rs[q + 1]] = A[rs[q]:rs[q + 1]]
    ws = torch.zeros(8, dtype=torch.int32, device="cuda")
    C = C0.clone()
    binding.hgemm_allgather_a(m, n, k, 1.0, bufs[1], k, bufs, rs, 1, B, k, 0.0, C, m, "N", "f16",
                              workspace=ws, chunk_rows=256)
    torch.cuda.synchronize()
    assert np.array_equal(_bits(C), _bits(ref))
    assert np.array_equal(_bits(bufs[1]), _bits(A))


def test_invalid_arguments():
    import torch
    from paper_conf_ipps_00020c20_b200 import binding
    A = torch.zeros(64, 64, dtype=torch.float16, device="cuda")
    C = torch.zeros(64, 64, dtype=torch.float16, device="cuda")
    ws = torch.zeros(2, dtype=torch.int32, device="cuda")
    with pytest.raises(binding.HgemmError):       # peer pointer missing
        binding.hgemm_allgather_a(64, 64, 64, 1.0, A, 64, [A, None], [0, 32, 64], 0, A, 64, 0.0, C, 64,
                                  workspace=ws, chunk_rows=64)
    with pytest.raises(binding.HgemmError):       # workspace too small (1 + 2 chunks)
        binding.hgemm_allgather_a(64, 64, 64, 1.0, A, 64, [A], [0, 64], 0, A, 64, 0.0, C, 64,
                                  workspace=ws, chunk_rows=32)
    with pytest.raises(binding.HgemmError):       # rank out of range
        binding.hgemm_allgather_a(64, 64, 64, 1.0, A, 64, [A], [0, 64], 1, A, 64, 0.0, C, 64,
                                  workspace=ws, chunk_rows=64)


# ------------------------------------------------------------------ two processes, real CUDA IPC
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _ipc_worker(rank, world, port, m, n, k, tmp):
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_00020c20_b200.sharded import FusedAllGatherA, slab_bounds
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    g = torch.Generator(device="cuda").manual_seed(5)
    A = (torch.rand(m, k, generator=g, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, generator=g, device="cuda") * 2 - 1).half()
    ag = FusedAllGatherA(m, k, chunk_rows=512)
    ag.A.fill_(float("nan"))
    r0, r1 = ag.own_rows
    ag.own_view().copy_(A[r0:r1])
    torch.cuda.synchronize()
    dist.barrier()
    n0, n1 = slab_bounds(n, world, rank)
    Bs = B[n0:n1].contiguous()
    C = torch.full((n1 - n0, m), float("nan"), dtype=torch.float16, device="cuda")
    ag(n1 - n0, 1.0, Bs, k, 0.0, C, m, "N", "f16")
    torch.cuda.synchronize()
    dist.barrier()
    np.save(os.path.join(tmp, f"slab{rank}.npy"), C.cpu().numpy().view(np.uint16))
    np.save(os.path.join(tmp, f"gathered{rank}.npy"), ag.A[:, :k].cpu().numpy().view(np.uint16))
    ag.close()
    dist.barrier()
    dist.destroy_process_group()


def test_two_processes_cuda_ipc(tmp_path):
    import torch
    import torch.multiprocessing as mp
    from paper_conf_ipps_00020c20_b200 import binding
    m, n, k = 2048, 1024, 768
    world = 2
    mp.spawn(_ipc_worker, args=(world, _free_port(), m, n, k, str(tmp_path)), nprocs=world, join=True)
    g = torch.Generator(device="cuda").manual_seed(5)
    A = (torch.rand(m, k, generator=g, device="cuda") * 2 - 1).half()
    B = (torch.rand(n, k, generator=g, device="cuda") * 2 - 1).half()
    ref = torch.empty(n, m, dtype=torch.float16, device="cuda")
    binding.set_config(stream_k=1)
    try:
        binding.hgemm(m, n, k, 1.0, A, k, B, k, 0.0, ref, m, "T", "N", "f16")
    finally:
        binding.set_config()
    cat = np.concatenate([np.load(os.path.join(tmp_path, f"slab{r}.npy")) for r in range(world)], axis=0)
    assert np.array_equal(cat, ref.cpu().numpy().view(np.uint16))
    for r in range(world):
        assert np.array_equal(np.load(os.path.join(tmp_path, f"gathered{r}.npy")), A.cpu().numpy().view(np.uint16))


def test_fused_allgather_long_k_many_waves(oracle_mod):
    """>= 8 whole waves and K >= 8192: the fused kernel runs with the wave barrier (DESIGN.md
    "Wave barrier") while its copy warps pull the peer's rows; bitwise equal to hgemm()."""
    _virtual(8192, 16384, 8192, 2, 4096, oracle_mod=oracle_mod)
