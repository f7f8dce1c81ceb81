"""Fused all-gather of op(A) + GEMM (include/hgemm.h hgemm_allgather_a) on CPU.

* The copy schedule is the library's own (hgemm_allgather_plan, a host-only
  C-ABI call): every row of op(A) is copied exactly once, from its owner, the
  records of a chunk are consecutive, and the local chunks come first followed
  by the owners rank+1, rank+2, ... (so at any moment the ranks pull from
  different peers).
* The Python layer (sharded.FusedAllGatherA) runs over gloo with world size 2
  and 3: handle exchange, shard bookkeeping and epochs are the product code;
  only CUDA IPC (replaced by file-backed shared tensors) and the GPU call
  (replaced by a host emulation that executes the library's plan and then the
  oracle) are injected.  The gathered buffer must equal the full A and the
  slab must equal the oracle on the full A, bitwise.
"""
import os
import random
import socket

import numpy as np
import pytest

from paper_conf_ipps_00020c20_b200 import binding, inputs
from paper_conf_ipps_00020c20_b200.sharded import FusedAllGatherA, default_chunk_rows, slab_bounds


def _check_plan(m, rs, rank, cr):
    world = len(rs) - 1
    ops = binding.allgather_plan(m, rs, rank, cr)
    seen = np.zeros(m, dtype=np.int64)
    owner = np.empty(m, dtype=np.int64)
    for q in range(world):
        owner[rs[q]:rs[q + 1]] = q
    chunks_done = set()
    prev_chunk = None
    for c, src, r0, r1 in ops:
        assert 0 <= r0 < r1 <= m
        assert c * cr <= r0 and r1 <= min(m, (c + 1) * cr)          # inside its chunk
        assert np.all(owner[r0:r1] == src)                            # copied from its owner
        seen[r0:r1] += 1
        if c != prev_chunk:
            assert c not in chunks_done                               # a chunk's records are consecutive
            if prev_chunk is not None:
                chunks_done.add(prev_chunk)
            prev_chunk = c
    assert np.all(seen == 1)                                          # every row exactly once
    # chunk order: by the owner of the chunk's first row, rotated to start at `rank`
    firsts = []
    for c, src, r0, r1 in ops:
        if not firsts or firsts[-1][0] != c:
            firsts.append((c, owner[c * cr]))
    dist = [(o - rank) % world for _, o in firsts]
    assert dist == sorted(dist)
    return ops


def test_plan_small_example():
    # rows 0..9, rank 0 owns 0..3, rank 1 owns 4..9, chunks of 3 rows
    assert binding.allgather_plan(10, [0, 4, 10], 1, 3) == [
        (2, 1, 6, 9), (3, 1, 9, 10), (0, 0, 0, 3), (1, 0, 3, 4), (1, 1, 4, 6)]
    assert binding.allgather_plan(10, [0, 4, 10], 0, 3) == [
        (0, 0, 0, 3), (1, 0, 3, 4), (1, 1, 4, 6), (2, 1, 6, 9), (3, 1, 9, 10)]


def test_plan_random_cover():
    rng = random.Random(7)
    for _ in range(300):
        world = rng.randint(1, 8)
        m = rng.choice([0, 1, 7, 100, 513, 4096, 32768])
        cuts = sorted(rng.randint(0, m) for _ in range(world - 1))
        rs = [0] + cuts + [m]
        cr = rng.choice([1, 3, 64, 512, 2048, 100000])
        for rank in range(world):
            _check_plan(m, rs, rank, cr)


def test_plan_sharded_32768():
    world, m = 8, 32768
    cr = default_chunk_rows(m, world)
    assert cr == 4096
    rs = [slab_bounds(m, world, q, align=cr)[0] for q in range(world)] + [m]
    for rank in range(world):
        ops = _check_plan(m, rs, rank, cr)
        assert len(ops) == m // cr                    # chunk-aligned shards: one record per chunk
        assert ops[0][1] == rank and ops[0][2] == rs[rank]


@pytest.mark.parametrize("bad", [
    dict(m=10, rs=[0, 4, 9], rank=0, cr=3),     # splits do not end at m
    dict(m=10, rs=[1, 4, 10], rank=0, cr=3),    # splits do not start at 0
    dict(m=10, rs=[0, 6, 4, 10], rank=0, cr=3),  # decreasing
    dict(m=10, rs=[0, 4, 10], rank=2, cr=3),    # rank out of range
    dict(m=10, rs=[0, 4, 10], rank=0, cr=0),    # chunk_rows < 1
])
def test_plan_invalid(bad):
    with pytest.raises(binding.HgemmError):
        binding.allgather_plan(bad["m"], bad["rs"], bad["rank"], bad["cr"])


# ------------------------------------------------------------------ gloo, world 2 and 3
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, case, tmp):
    import torch
    import torch.distributed as dist

    import oracle
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    m, n, k, cr, beta, out = case
    lda = k + (-k) % 8

    def alloc(mm, ld, nws):
        path = os.path.join(tmp, f"A{rank}.bin")
        A = torch.from_file(path, shared=True, size=mm * ld, dtype=torch.float16).view(mm, ld)
        A.fill_(float("nan"))                    # rows not yet gathered read as NaN
        return A, torch.zeros(nws, dtype=torch.int32)

    def get_handle(A):
        return os.path.join(tmp, f"A{rank}.bin").encode()

    def open_(h):
        return torch.from_file(h.decode(), shared=True, size=m * lda, dtype=torch.float16).view(m, lda)

    calls = []

    def emulate(m_, n_, k_, alpha, A, lda_, peers, row_splits, rank_, B, ldb, beta_, C, ldc, transB, out_dtype, *,
                workspace, chunk_rows, stream):
        assert workspace.numel() >= 1 + -(-m_ // chunk_rows)
        # the copies in the library's chunk order ...
        for c, src, r0, r1 in binding.allgather_plan(m_, row_splits, rank_, chunk_rows):
            if src != rank_:
                A[r0:r1, :k_] = peers[src][r0:r1, :k_]
        # ... then the GEMM on the gathered buffer (transA = 'T': stored k x m with lda)
        a = A.numpy().view(np.uint16).reshape(-1)
        c_out, _, _ = oracle.hgemm_ref(m_, n_, k_, alpha, a, lda_, B, ldb, beta_, C, ldc, "T", transB, out_dtype,
                                       want_r=False)
        if out_dtype == "f32":
            C[:] = c_out
        else:
            C.view(np.uint16)[:] = c_out
        calls.append(1)

    ag = FusedAllGatherA(m, k, lda=lda, chunk_rows=cr, alloc=alloc, ipc=(get_handle, open_, lambda p: None))
    assert ag.row_splits[0] == 0 and ag.row_splits[-1] == m
    r0, r1 = ag.own_rows
    allsplits = [None] * world
    dist.all_gather_object(allsplits, ag.row_splits)
    assert all(s == ag.row_splits for s in allsplits)        # every rank agrees on the ownership
    A_full = inputs.uniform_f16(m, k, 21)                      # op(A), row-major m x k
    n0, n1 = slab_bounds(n, world, rank)
    B_full = inputs.uniform_f16(k, n, 22)                      # op(B) k x n, transB 'N'
    Bl = np.asfortranarray(B_full[:, n0:n1]).reshape(-1, order="F").view(np.uint16)
    cdt = np.float32 if out == "f32" else np.float16
    C0 = inputs.uniform_f16(m, n, 23).astype(cdt)[:, n0:n1]
    for it in range(2):                                        # two calls, A changes in between
        ag.own_view()[:] = torch.from_numpy(A_full[r0:r1] * (1 if it == 0 else -1))
        dist.barrier()                                         # peers' own rows complete
        C = np.asfortranarray(C0).reshape(-1, order="F").copy()
        ag(n1 - n0, 1.0, Bl, k, beta, C, m, "N", out, gemm=emulate)
        dist.barrier()                                         # nobody rewrites rows still being pulled
        full = A_full * (1 if it == 0 else -1)
        assert np.array_equal(ag.A[:, :k].numpy().view(np.uint16), full.view(np.uint16))
        aT = np.asfortranarray(full.T).reshape(-1, order="F").view(np.uint16)   # stored k x m
        ref, _, _ = oracle.hgemm_ref(m, n1 - n0, k, 1.0, aT, k, Bl, k, beta,
                                     np.asfortranarray(C0).reshape(-1, order="F").copy(), m, "T", "N", out,
                                     want_r=False)
        assert np.array_equal(C.view(np.uint8), ref.view(np.uint8))
    assert calls == [1, 1]
    ag.close()
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,case", [
    (2, (96, 40, 24, 16, 0.0, "f16")),
    (2, (100, 33, 40, 32, 1.0, "f32")),     # ragged last chunk
    (3, (130, 20, 16, 8, -1.0, "f16")),
])
def test_fused_allgather_gloo(tmp_path, world, case, oracle_mod):
    import torch.multiprocessing as mp
    mp.spawn(_worker, args=(world, _free_port(), case, str(tmp_path)), nprocs=world, join=True)
