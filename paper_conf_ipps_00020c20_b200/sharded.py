"""N-slab sharded multi-GPU HGEMM (BASELINE.json north_star (3)).

GPU g of G owns the output columns [n0, n1) of C and the matching slab of
op(B); A is replicated.  In the column-major ABI both slabs are pointer
offsets with unchanged leading dimensions:
    op(B)[:, n0:n1]  ->  B + n0*ldb   (transB 'N')   or   B + n0   (transB 'T')
    C[:, n0:n1]      ->  C + n0*ldc
No reduction is needed because K is not split, so each rank's slab is
computed with exactly the single-GPU per-element arithmetic: the
concatenation of the slabs is bitwise equal to the single-GPU result.

The one exchange step is the replication of A: an NCCL broadcast from the
source rank over NVLink/NVSwitch (torch.distributed, backend "nccl" on
B200; "gloo" in the CPU tests).  It is timed and reported separately from
the GEMM (north_star (3)).
"""
from __future__ import annotations


def slab_bounds(n: int, world: int, rank: int, align: int = 8):
    """Contiguous, balanced column slab [n0, n1) of rank `rank` out of `world`.

    Boundaries are multiples of `align` columns (keeps C + n0*ldc 16-byte
    aligned for FP16 when ldc % 8 == 0) except the last one, which is n."""
    if world <= 0 or not (0 <= rank < world):
        raise ValueError("bad world/rank")
    units = (n + align - 1) // align
    base, rem = divmod(units, world)
    u0 = rank * base + min(rank, rem)
    u1 = u0 + base + (1 if rank < rem else 0)
    return min(u0 * align, n), min(u1 * align, n)


def slab_offsets(n0: int, ldb: int, ldc: int, transB: str, elem_b: int = 2, elem_c: int = 2):
    """Byte offsets of the slab starting at column n0 inside B and C."""
    off_b = (n0 * ldb if transB in ("N", "n") else n0) * elem_b
    off_c = n0 * ldc * elem_c
    return off_b, off_c


def hgemm_sharded(m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, transA="N", transB="N",
                  out_dtype="f16", *, group=None, src=0, broadcast_A=True, gemm=None, stream=None):
    """Sharded C = alpha*op(A)*op(B) + beta*C over the ranks of `group`.

    A: the full A tensor on every rank (its contents on rank `src` are
    broadcast to the others when `broadcast_A`).  B, C: tensors holding the
    FULL-size column-major storage on this rank (only this rank's slab is
    read/written), or flat tensors; the slab is addressed by pointer offset.
    `gemm` defaults to the CUDA hgemm (binding.hgemm); the CPU tests inject
    another callable with the same signature.  Returns (n0, n1)."""
    import torch.distributed as dist

    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    if broadcast_A and world > 1:
        dist.broadcast(A, src=src, group=group)
    n0, n1 = slab_bounds(n, world, rank)
    if gemm is None:
        from .binding import hgemm as gemm
    f32 = str(out_dtype) in ("f32", "float32", "torch.float32", "1")
    off_b, off_c = slab_offsets(n0, ldb, ldc, transB, 2, 4 if f32 else 2)
    if n1 > n0:
        gemm(m, n1 - n0, k, alpha, A, lda, _offset(B, off_b), ldb, beta, _offset(C, off_c), ldc,
             transA, transB, out_dtype, stream)
    return n0, n1


class _Offset:
    """A (tensor, byte offset) pair that the binding's pointer marshalling accepts."""

    def __init__(self, base, off):
        self.base, self.off = base, off

    def data_ptr(self):
        return int(self.base.data_ptr()) + self.off


def _offset(t, off):
    if isinstance(t, int):
        return t + off
    return _Offset(t, off)
