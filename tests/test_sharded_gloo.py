"""N-slab sharded path on CPU: world_size 2 over gloo.

The slab bookkeeping, the broadcast of A and the pointer offsets of the
sharded path (paper_conf_ipps_00020c20_b200/sharded.py) run exactly as on the
B200 box; only the per-rank GEMM is injected (the oracle on host buffers,
since this container has no GPU).  The concatenated slabs must be bitwise
equal to the single-process result (no split-K => same per-element
arithmetic).  The same invariant is checked on the GPU by bench.py --gpus N.
"""
import os
import socket

import numpy as np
import pytest

from paper_conf_ipps_00020c20_b200 import inputs
from paper_conf_ipps_00020c20_b200.sharded import (hgemm_sharded, hgemm_sharded_overlapped, slab_bounds,
                                                   slab_offsets)


def test_slab_bounds_cover_and_align():
    for n in (0, 1, 7, 8, 100, 1000, 8192, 32768, 12345):
        for world in (1, 2, 3, 4, 8):
            spans = [slab_bounds(n, world, r) for r in range(world)]
            assert spans[0][0] == 0 and spans[-1][1] == n
            for (a0, a1), (b0, b1) in zip(spans, spans[1:]):
                assert a1 == b0 and a0 <= a1
            for a0, a1 in spans[:-1]:
                assert a1 % 8 == 0 or a1 == n
            widths = [b - a for a, b in spans]
            assert max(widths) - min(widths) <= 16   # one align unit + the ragged last unit
    assert slab_bounds(32768, 8, 3) == (12288, 16384)


def test_slab_offsets():
    assert slab_offsets(16, 100, 50, "N", 2, 2) == (16 * 100 * 2, 16 * 50 * 2)
    assert slab_offsets(16, 100, 50, "T", 2, 4) == (16 * 2, 16 * 50 * 4)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _split(obj):
    if hasattr(obj, "base") and hasattr(obj, "off"):
        return obj.base, obj.off
    return obj, 0


def _oracle_gemm(m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, tA, tB, out, stream):
    """Host stand-in for the CUDA hgemm with the same argument list (tests only)."""
    import oracle
    At, aoff = _split(A)
    Bt, boff = _split(B)
    Ct, coff = _split(C)
    a = At.numpy().view(np.uint16).reshape(-1)[aoff // 2:]
    b = Bt.numpy().view(np.uint16).reshape(-1)[boff // 2:]
    esz = 4 if out == "f32" else 2
    cflat = Ct.numpy().reshape(-1)
    cview = cflat.view(np.float32 if out == "f32" else np.uint16)[coff // esz:]
    need_b = ((k - 1) + (n - 1) * ldb + 1) if tB == "N" else ((n - 1) + (k - 1) * ldb + 1)
    need_c = (m - 1) + (n - 1) * ldc + 1
    c_out, _, _ = oracle.hgemm_ref(m, n, k, alpha, a, lda, b[:need_b], ldb, beta,
                                   cview[:need_c].copy(), ldc, tA, tB, out, want_r=False)
    cview[:need_c] = c_out[:need_c]


def _worker(rank, world, port, case, result_dir):
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    m, n, k, tA, tB, alpha, beta, out, local = case[:9]
    overlap = len(case) > 9 and case[9]
    sa = inputs.stored_shape(m, k, tA)
    sb = inputs.stored_shape(k, n, tB)
    A_full = inputs.uniform_f16(sa[0], sa[1], 11)
    B_full = inputs.uniform_f16(sb[0], sb[1], 12)
    C_full = inputs.uniform_f16(m, n, 13).astype(np.float32 if out == "f32" else np.float16)
    # only the source rank holds A before the broadcast
    A = torch.from_numpy(A_full.reshape(-1, order="F").copy())          # float16 (gloo has no int16)
    if rank != 0:
        A.zero_()
    lda, ldb, ldc = sa[0], sb[0], m
    n0, n1 = slab_bounds(n, world, rank)
    cv = np.int16 if out == "f16" else np.float32
    if local:
        if tB == "N":
            Bl = B_full[:, n0:n1]
        else:
            Bl = B_full[n0:n1, :]
        # local slab storage keeps the global leading dimension
        Bbuf = np.zeros(ldb * (Bl.shape[1] if tB == "N" else k), dtype=np.float16)
        Bbuf_2d = Bbuf.reshape(ldb, -1, order="F")
        Bbuf_2d[:Bl.shape[0], :Bl.shape[1]] = Bl
        B = torch.from_numpy(Bbuf.view(np.int16))
        C = torch.from_numpy(np.ascontiguousarray(C_full[:, n0:n1]).reshape(-1, order="F").view(cv).copy())
    else:
        B = torch.from_numpy(B_full.reshape(-1, order="F").view(np.int16).copy())
        C = torch.from_numpy(C_full.reshape(-1, order="F").view(cv).copy())
    if overlap:
        got = hgemm_sharded_overlapped(m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, tA, tB, out, panels=3,
                                       local_slabs=local, gemm=_oracle_gemm)
    else:
        got = hgemm_sharded(m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, tA, tB, out,
                            local_slabs=local, gemm=_oracle_gemm)
    assert got == (n0, n1)
    # A was replicated
    assert np.array_equal(A.numpy().view(np.uint16), A_full.reshape(-1, order="F").view(np.uint16))
    cn = C.numpy().view(np.float16 if out == "f16" else np.float32)
    slab = (cn.reshape(m, -1, order="F") if local else cn.reshape(m, n, order="F")[:, n0:n1])
    np.save(os.path.join(result_dir, f"slab{rank}.npy"), np.ascontiguousarray(slab))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("case", [
    (37, 70, 45, "T", "N", 1.0, 0.0, "f16", False),
    (37, 70, 45, "N", "T", 0.5, 1.0, "f32", False),
    (29, 53, 33, "T", "T", 1.0, -1.0, "f16", True),
    (16, 8, 64, "N", "N", 1.0, 0.0, "f32", True),
    (41, 70, 45, "T", "N", 1.0, 0.5, "f16", False, True),     # NEXT-2: panel-pipelined broadcast
    (64, 33, 80, "T", "T", -1.0, 0.0, "f32", True, True),
])
def test_sharded_gloo_world2_bitwise(tmp_path, case, oracle_mod):
    import torch.multiprocessing as mp
    world = 2
    mp.spawn(_worker, args=(world, _free_port(), case, str(tmp_path)), nprocs=world, join=True)
    m, n, k, tA, tB, alpha, beta, out = case[:8]
    slabs = [np.load(os.path.join(tmp_path, f"slab{r}.npy")) for r in range(world)]
    cat = np.concatenate(slabs, axis=1)
    # single-process reference on the same seeded inputs
    sa = inputs.stored_shape(m, k, tA)
    sb = inputs.stored_shape(k, n, tB)
    A = inputs.uniform_f16(sa[0], sa[1], 11).reshape(-1, order="F")
    B = inputs.uniform_f16(sb[0], sb[1], 12).reshape(-1, order="F")
    Cin = inputs.uniform_f16(m, n, 13).astype(np.float32 if out == "f32" else np.float16).reshape(-1, order="F")
    c_out, _, _ = oracle_mod.hgemm_ref(m, n, k, alpha, A, sa[0], B, sb[0], beta, Cin, m, tA, tB, out)
    ref = c_out.view(np.float16) if out == "f16" else c_out
    ref = ref.reshape(m, n, order="F")
    assert cat.shape == ref.shape
    assert np.array_equal(cat.view(np.uint16 if out == "f16" else np.uint32),
                          ref.view(np.uint16 if out == "f16" else np.uint32))
