"""N-slab sharded multi-GPU HGEMM (BASELINE.json north_star (3)).

GPU g of G owns the output columns [n0, n1) of C and the matching slab of
op(B); A is replicated.  In the column-major ABI both slabs are pointer
offsets with unchanged leading dimensions:
    op(B)[:, n0:n1]  ->  B + n0*ldb   (transB 'N')   or   B + n0   (transB 'T')
    C[:, n0:n1]      ->  C + n0*ldc
No reduction is needed because K is not split, so each rank's slab is
computed with the single-GPU per-element arithmetic of whatever kernel the
slab's shape selects.  The concatenation of the slabs is bitwise equal to
the single-GPU result when every call runs the same tile kernel with whole
tiles (e.g. hgemm_config_t kernel = tc2, a fixed block_n, stream_k = 1):
with the automatic choice a narrow slab or a short panel can select split-K,
the streaming kernel or stream-K, which sum the k-blocks of an element in a
different grouping (results then agree within the north_star (4) bound, not
bitwise).

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
    if n < 0:
        raise ValueError("n < 0")
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


def _world_rank(group):
    import torch.distributed as dist
    if not dist.is_initialized():
        return 1, 0
    return dist.get_world_size(group), dist.get_rank(group)


def broadcast_A(A, *, group=None, src=0):
    """Replicate A from rank `src` (the sharded path's one collective)."""
    import torch.distributed as dist
    world, _ = _world_rank(group)
    if world > 1:
        dist.broadcast(A, src=src, group=group)


def order_after_current_stream(stream):
    """Make `stream` wait for the work queued so far on torch's current CUDA stream.

    torch.distributed's wait() (a synchronous broadcast, or Work.wait() of an async
    one) orders the collective before later work on the CURRENT stream only; the
    GEMM is enqueued on `stream`, which may be another stream, so it must wait on an
    event recorded there.  `stream`: None (the current stream: nothing to do), an int
    handle or a torch.cuda.Stream.  No-op without CUDA (the CPU tests)."""
    if stream is None:
        return
    import torch
    if not torch.cuda.is_available():
        return
    cur = torch.cuda.current_stream()
    handle = int(stream) if isinstance(stream, int) else int(stream.cuda_stream)
    if handle == int(cur.cuda_stream):
        return
    ev = torch.cuda.Event()
    ev.record(cur)
    target = torch.cuda.ExternalStream(handle) if isinstance(stream, int) else stream
    target.wait_event(ev)


def hgemm_sharded(m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, transA="N", transB="N",
                  out_dtype="f16", *, group=None, src=0, broadcast=True, local_slabs=False,
                  gemm=None, stream=None):
    """Sharded C = alpha*op(A)*op(B) + beta*C over the ranks of `group`.

    n is the GLOBAL number of columns.  A: the full A on every rank (rank
    `src`'s copy is broadcast first when `broadcast`).  B and C either hold
    the full-size column-major storage on every rank (local_slabs=False; this
    rank's slab is addressed by pointer offset) or only this rank's slab
    (local_slabs=True; the slab starts at the buffer start, same ld).
    `gemm` defaults to the CUDA hgemm of the C ABI; the CPU tests inject
    another callable with the same signature.  Returns this rank's (n0, n1)."""
    world, rank = _world_rank(group)
    if broadcast:
        broadcast_A(A, group=group, src=src)
        if world > 1:
            order_after_current_stream(stream)   # the GEMM's stream sees the broadcast A
    n0, n1 = slab_bounds(n, world, rank)
    if gemm is None:
        from .binding import hgemm as gemm
    f32 = str(out_dtype) in ("f32", "float32", "torch.float32", "1")
    if local_slabs:
        off_b = off_c = 0
    else:
        off_b, off_c = slab_offsets(n0, ldb, ldc, transB, 2, 4 if f32 else 2)
    if n1 > n0:
        gemm(m, n1 - n0, k, alpha, A, lda, _offset(B, off_b), ldb, beta, _offset(C, off_c), ldc,
             transA, transB, out_dtype, stream)
    return n0, n1


def hgemm_sharded_overlapped(m, n, k, alpha, A, lda, B, ldb, beta, C, ldc, transA="T", transB="N",
                             out_dtype="f16", *, panels=4, group=None, src=0, local_slabs=False, gemm=None,
                             stream=None):
    """Sharded GEMM with the broadcast of A pipelined against the GEMM.

    op(A) is split into `panels` row panels (m ranges).  With transA = 'T'
    (A stored k x m, the paper's layout) row panel [m0, m1) of op(A) is the
    contiguous column range A[:, m0:m1] = A + m0*lda, so each panel is one
    contiguous NCCL broadcast.  All broadcasts are enqueued asynchronously
    (in order on the communicator's stream); the GEMM of panel i
    (C[m0:m1, slab] = op(A)[m0:m1, :] op(B)[:, slab], a pointer offset into C)
    waits only for broadcast i, so it overlaps broadcasts i+1, i+2, ...
    Each panel is its own hgemm() call: with a fixed tile kernel and whole tiles
    (hgemm_config_t tc2 / block_n / stream_k = 1) every element is bitwise the
    unpipelined result; with the automatic choice a short panel may select another
    kernel (same north_star (4) bound, possibly different last bits).
    Returns this rank's (n0, n1)."""
    import torch.distributed as dist
    if transA not in ("T", "t"):
        raise ValueError("row panels of op(A) are contiguous only for transA='T'")
    world, rank = _world_rank(group)
    n0, n1 = slab_bounds(n, world, rank)
    if gemm is None:
        from .binding import hgemm as gemm
    f32 = str(out_dtype) in ("f32", "float32", "torch.float32", "1")
    esz_c = 4 if f32 else 2
    off_b, off_c = (0, 0) if local_slabs else slab_offsets(n0, ldb, ldc, transB, 2, esz_c)
    bounds = [(m * i) // panels for i in range(panels + 1)]
    bounds = [b - b % 8 if 0 < b < m else b for b in bounds]   # 16-B aligned panel starts
    works = []
    if world > 1:
        flat = A.view(-1)
        for i in range(panels):
            p0, p1 = bounds[i], bounds[i + 1]
            if p1 > p0:
                works.append(dist.broadcast(flat[p0 * lda:p1 * lda], src=src, group=group, async_op=True))
            else:
                works.append(None)
    for i in range(panels):
        p0, p1 = bounds[i], bounds[i + 1]
        if world > 1 and works[i] is not None:
            works[i].wait()          # torch's current stream waits for panel i only ...
            order_after_current_stream(stream)   # ... and so does the GEMM's stream
        if p1 > p0 and n1 > n0:
            gemm(p1 - p0, n1 - n0, k, alpha, _offset(A, p0 * lda * 2), lda, _offset(B, off_b), ldb, beta,
                 _offset(C, off_c + p0 * esz_c), ldc, transA, transB, out_dtype, stream)
    return n0, n1


class _Offset:
    """A (tensor, byte offset) pair that the binding's pointer marshalling accepts."""

    def __init__(self, base, off):
        self.base, self.off = base, off

    def data_ptr(self):
        return int(self.base.data_ptr()) + self.off


def _offset(t, off):
    if off == 0:
        return t
    if isinstance(t, int):
        return t + off
    return _Offset(t, off)


def default_chunk_rows(m: int, world: int, bn: int = 512) -> int:
    """Chunk of op(A) rows per counter of the fused all-gather: one shard (m/world),
    rounded down to the 512-wide tile.  The kernel rasters one group of tiles per
    chunk, and every group re-reads all of op(B)'s slab, so fewer, larger chunks
    cut L2/HBM traffic (8192^3 with 8 virtual ranks: 512-row chunks +11% over
    hgemm, shard-sized chunks see profiles/r01b); the local shard's tiles, which
    need no transfer, cover the wait for the first remote one."""
    shard = m // max(1, world)
    return max(bn, shard - shard % bn)


class FusedAllGatherA:
    """A replicated by an all-gather fused with the GEMM (hgemm_allgather_a, NEXT-2).

    Rank q owns rows [row_splits[q], row_splits[q+1]) of op(A) (transA = 'T',
    the paper's layout: A stored k x m, row i of op(A) = A + i*lda).  Every rank
    allocates a full-size gather buffer `self.A` (a (m, lda) float16 tensor whose
    row i is op(A) row i) and writes its own rows there; the buffers are mapped
    into every peer with CUDA IPC once (handles exchanged over the process
    group).  Each call is ONE kernel: a copy warp per CTA pulls the peers' rows
    over NVLink while the persistent GEMM of this rank's C slab consumes each
    chunk of rows as soon as it is complete, so the exchange overlaps the MMAs
    tile by tile.  The result is bitwise that of hgemm() on the gathered A.

    The caller synchronises the ranks around a call (a barrier after writing its
    own rows, and before rewriting them while a peer may still be reading).
    `ipc` = (get_handle, open, close) and `alloc` are injection points for the
    CPU (gloo) tests of the exchange logic; the defaults are the C ABI and torch."""

    def __init__(self, m: int, k: int, *, lda: int | None = None, group=None, chunk_rows: int | None = None,
                 device=None, ipc=None, alloc=None):
        import torch
        import torch.distributed as dist
        self.world, self.rank = _world_rank(group)
        self.m, self.k = int(m), int(k)
        self.lda = int(lda) if lda is not None else max(1, self.k + (-self.k) % 8)
        self.chunk_rows = int(chunk_rows) if chunk_rows else default_chunk_rows(self.m, self.world)
        # shards on chunk boundaries: every chunk has one owner (the fused kernel's precondition)
        self.row_splits = [slab_bounds(self.m, self.world, q, align=self.chunk_rows)[0] for q in range(self.world)]
        self.row_splits.append(self.m)
        nws = 1 + max(1, -(-self.m // self.chunk_rows))
        if alloc is None:
            dev = device if device is not None else torch.device("cuda", torch.cuda.current_device())
            self.A = torch.empty((self.m, self.lda), dtype=torch.float16, device=dev)
            self.workspace = torch.zeros(nws, dtype=torch.int32, device=dev)
        else:
            self.A, self.workspace = alloc(self.m, self.lda, nws)
        if ipc is None:
            from . import binding
            ipc = (binding.ipc_get_handle, binding.ipc_open, binding.ipc_close)
        self._get_handle, self._open, self._close = ipc
        self.peers = [None] * self.world
        self._opened = []
        if self.world > 1:
            mine = self._get_handle(self.A)
            allh = [None] * self.world
            dist.all_gather_object(allh, mine, group=group)
            for q, h in enumerate(allh):
                if q != self.rank:
                    self.peers[q] = self._open(h)
                    self._opened.append(self.peers[q])

    @property
    def own_rows(self):
        return self.row_splits[self.rank], self.row_splits[self.rank + 1]

    def own_view(self):
        """This rank's rows of op(A) inside the gather buffer, to be written by the caller."""
        r0, r1 = self.own_rows
        return self.A[r0:r1, :self.k]

    def __call__(self, n, alpha, B, ldb, beta, C, ldc, transB="N", out_dtype="f16", *, stream=None, gemm=None):
        """C (m x n slab) = alpha * op(A) * op(B) + beta * C with op(A) gathered on the fly."""
        if gemm is None:
            from .binding import hgemm_allgather_a as gemm
        gemm(self.m, n, self.k, alpha, self.A, self.lda, self.peers, self.row_splits, self.rank, B, ldb, beta, C,
             ldc, transB, out_dtype, workspace=self.workspace, chunk_rows=self.chunk_rows, stream=stream)

    def close(self):
        for p in self._opened:
            self._close(p)
        self._opened = []
        self.peers = [None] * self.world
