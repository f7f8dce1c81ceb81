/*
 * include/hgemm.h -- C ABI of the B200-native (sm_100a) half-precision GEMM.
 *
 * Operation (SII-A, "C = alpha*A*B + beta*C"; FP16 inputs,
 * P:401; accumulation in FP32 and FP16 or FP32 output per BASELINE.json
 * north_star (1)):
 *
 *      C <- alpha * op(A) * op(B) + beta * C
 *
 * Storage is COLUMN-MAJOR with BLAS/cuBLAS semantics (readings R1,
 * R2: the paper's "A m x k, B n x k, A row-major, B column-major" benchmark
 * layout, is transA='T', transB='N' here):
 *   op(A) is m x k:  transA 'N' -> A is m x k, lda >= max(1,m)
 *                    transA 'T' -> A is k x m, lda >= max(1,k)
 *   op(B) is k x n:  transB 'N' -> B is k x n, ldb >= max(1,k)
 *                    transB 'T' -> B is n x k, ldb >= max(1,n)
 *   C is m x n, ldc >= max(1,m); element (i,j) at C[i + j*ldc].
 * A and B hold IEEE binary16 values (__half).  C holds __half when
 * out_dtype == HGEMM_OUT_F16 and float when HGEMM_OUT_F32; it is read (when
 * beta != 0) and written in that same type.  Products are accumulated in
 * FP32 on the tensor cores; the epilogue computes alpha*acc + beta*c in FP32
 * and rounds once to the output type (round-to-nearest-even, overflow to inf).
 *
 * Ownership and lifetime: A, B and C are DEVICE pointers owned by the
 * caller, who keeps them alive until the work enqueued on `stream`
 * completes.  The library allocates nothing on the call path and keeps no
 * pointer after returning.  C must not overlap A or B.
 *
 * Asynchrony and errors: hgemm() enqueues on `stream` (0 = legacy default
 * stream) and returns without synchronising.  Argument errors are detected
 * synchronously: the call returns HGEMM_ERR_INVALID_VALUE, enqueues nothing
 * and leaves C untouched.  Launch/encode failures return HGEMM_ERR_CUDA with
 * the CUDA error left readable by cudaGetLastError().  Device faults surface
 * at the caller's next synchronisation, as for any CUDA kernel.
 *
 * BLAS quick returns: m == 0 or n == 0 -> no-op.  k == 0 or alpha == 0 ->
 * C = beta*C.  beta == 0 -> C is never read (NaN/Inf in C do not propagate).
 *
 * Fast path (tcgen05 tensor cores + TMA): A and B 16-byte aligned, lda and
 * ldb multiples of 8 elements, C 16-byte aligned and ldc*sizeof(out) a
 * multiple of 16 bytes.  Anything else runs a slower CUDA-core kernel with
 * the same semantics (never an error; n > 65535*64 runs as several launches
 * over column ranges).  All indexing is 64-bit.
 *
 * Thread safety: hgemm() is reentrant; per-device properties and per-kernel
 * launch setup are cached (initialised once per device, std::call_once).
 * hgemm_set_config() is process-global and meant for tests and benchmarks.
 *
 * Co-residency: the persistent tile kernels size their grid to the clusters
 * the GPU holds at once.  Two features make CTAs of one launch wait for each
 * other and so assume that all of them become resident: the stream-K fix-up
 * (heads wait for the partials of later clusters) and the wave barrier
 * (launches with >= 8 whole waves and K >= 8192: the producers meet before
 * each wave).  On a GPU shared with other work a not-yet-resident cluster
 * only delays the others; under MPS / green contexts with fewer SMs than
 * the device reports, disable them (hgemm_config_t.stream_k = 1, environment
 * HGEMM_WSYNC=0).
 */
#ifndef HGEMM_H_
#define HGEMM_H_

#include <stdint.h>
#include <cuda_runtime_api.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum { HGEMM_OUT_F16 = 0, HGEMM_OUT_F32 = 1 } hgemm_dtype_t;

typedef enum {
    HGEMM_SUCCESS = 0,
    HGEMM_ERR_INVALID_VALUE = 1, /* m,n,k < 0; bad trans char; ld too small;
                                    NULL pointer with a nonzero extent; bad out_dtype */
    HGEMM_ERR_ARCH = 2,          /* current device is not compute capability 10.0 */
    HGEMM_ERR_CUDA = 3           /* CUDA runtime/driver failure (launch, tensor-map encode) */
} hgemm_status_t;

/* C <- alpha*op(A)*op(B) + beta*C (see above).  transA/transB in {'N','n','T','t'}. */
hgemm_status_t hgemm(int64_t m, int64_t n, int64_t k,
                     float alpha, const void *A, int64_t lda,
                     const void *B, int64_t ldb,
                     float beta, void *C, int64_t ldc,
                     char transA, char transB, hgemm_dtype_t out_dtype,
                     cudaStream_t stream);

/* Accumulation type of hgemm_ex (like cublasGemmEx's computeType).
 *   HGEMM_COMPUTE_F32: products accumulated in FP32 (what hgemm() does; BASELINE.json
 *                      north_star (1)).
 *   HGEMM_COMPUTE_F16: products accumulated in FP16 on the tensor cores
 *                      (tcgen05.mma kind::f16 with an FP16 accumulator, c_format = F16):
 *                      the paper's own precision mode, HMMA.1688.F16 (SIV-A;
 *                      its register budget only fits FP16 accumulators, SVI-A.3).
 *                      The epilogue still computes alpha*acc + beta*c in FP32 and rounds
 *                      once to FP16.  Requires out_dtype == HGEMM_OUT_F16.  Accuracy:
 *                      the FP16 accumulator loses the low bits of partial sums above 2048
 *                      (11-bit significand); integer sums stay exact only while every
 *                      partial sum is an integer of magnitude <= 2048. */
typedef enum { HGEMM_COMPUTE_F32 = 0, HGEMM_COMPUTE_F16 = 1 } hgemm_compute_t;

/* hgemm() with an explicit accumulation type; same arguments, layout, ownership,
 * asynchrony, quick returns and fallback rules as hgemm().  Errors as hgemm(),
 * plus HGEMM_ERR_INVALID_VALUE for an unknown compute type or HGEMM_COMPUTE_F16
 * with out_dtype != HGEMM_OUT_F16.  The fast path uses the CTA-pair tile kernels
 * (whole tiles, no stream-K / split-K / streaming kernels); the CUDA-core
 * fallback rounds its accumulator to FP16 after every product. */
hgemm_status_t hgemm_ex(int64_t m, int64_t n, int64_t k,
                        float alpha, const void *A, int64_t lda,
                        const void *B, int64_t ldb,
                        float beta, void *C, int64_t ldc,
                        char transA, char transB, hgemm_dtype_t out_dtype,
                        hgemm_compute_t compute, cudaStream_t stream);

/* Host-buffer variant: A, B and C are HOST pointers (page-locked memory gives
 * full copy/compute overlap; pageable memory works but serialises the copies),
 * same meaning, layout and quick-return rules as hgemm().  The call is
 * SYNCHRONOUS: it returns after C has been written back to host memory.
 * `workspace` is caller-owned DEVICE memory of at least
 * hgemm_host_workspace_size(...) bytes (it holds the device copies of A, B
 * and C).  The problem is processed in column panels of op(B)/C: panel j's
 * host->device copy, GEMM and device->host copy run on three internal
 * streams so the transfers of one panel overlap the GEMM of another; the
 * first panel's GEMM is cut into row pieces of op(A) that start as soon as
 * their rows of A have arrived.  Calls on one device are serialised (the
 * pipeline streams are per device); calls on different devices run
 * concurrently.  `stream` orders the whole call after prior work on it
 * (0 = legacy stream).
 * Errors: HGEMM_ERR_INVALID_VALUE as for hgemm(), also for a NULL or too
 * small workspace; HGEMM_ERR_CUDA for copy/launch failures.  An error after
 * the first copy was enqueued returns only once the internal streams have
 * drained, so no copy touches the caller's host buffers afterwards. */
size_t hgemm_host_workspace_size(int64_t m, int64_t n, int64_t k, char transA, char transB,
                                 hgemm_dtype_t out_dtype);
hgemm_status_t hgemm_host(int64_t m, int64_t n, int64_t k,
                          float alpha, const void *A, int64_t lda,
                          const void *B, int64_t ldb,
                          float beta, void *C, int64_t ldc,
                          char transA, char transB, hgemm_dtype_t out_dtype,
                          void *workspace, size_t workspace_bytes, cudaStream_t stream);

/* Static, NUL-terminated description of a status code (never NULL). */
const char *hgemm_status_string(hgemm_status_t s);

/* Kernel selection, for tests and benchmarks.  0 fields mean "automatic". */
typedef enum {
    HGEMM_KERNEL_AUTO = 0,
    HGEMM_KERNEL_SIMT = 1,       /* CUDA-core fallback (always available) */
    HGEMM_KERNEL_TC_1SM = 2,     /* tcgen05 cta_group::1, tile 128 x block_n */
    HGEMM_KERNEL_TC_2SM = 3,     /* tcgen05 cta_group::2 (CTA pair), tile 256 x block_n (256 or 512); 256-wide
                                    tiles in layout TN with k % 128 == 0 and n > 256 load two k-blocks per
                                    ring stage through 3-D TMA boxes (hgemm_get_last_config: splits = 2) */
    HGEMM_KERNEL_SPLITK = 4,     /* tcgen05 cta_group::1, tile 128 x block_n (64 or 128), K split over a
                                    cluster of `splits` CTAs, reduced through distributed shared memory */
    HGEMM_KERNEL_STREAM = 5      /* HBM-streaming tcgen05 kernel for skinny shapes: n <= 256, transA 'T',
                                    transB 'N' (both operands K-contiguous); one persistent CTA per SM,
                                    each owning column chunks of C^T of block_n (multiple of 16) rows of op(A);
                                    with n > 256 and m <= 256 the operands are swapped (op(B) streamed,
                                    C stored transposed; reported with group_m = 1);
                                    other shapes/layouts fall back to the automatic choice.  The
                                    automatic choice takes it for n <= 128 and m >= 64 x #SMs
                                    (16384 x 256 runs faster on the 2-SM tile kernel).  With K a
                                    multiple of 64 a stage holds G consecutive k-blocks of op(A)
                                    fetched by one 3-D TMA load; hgemm_get_last_config reports G in
                                    `splits` */
} hgemm_kernel_t;

typedef struct {
    int32_t kernel;    /* hgemm_kernel_t */
    int32_t block_n;   /* tile width along the output's contiguous dim: 128, 256 (1-SM, 2-SM) or
                          512 (2-SM only); HGEMM_KERNEL_STREAM: chunk width, a multiple of 16 in
                          [16, 256] (n <= 128) or [16, 128] (n <= 256); 0 = auto */
    int32_t group_m;   /* L2 raster group height in tiles (0 = auto) */
    int32_t max_ctas;  /* cap on persistent CTAs (0 = all SMs) */
    int32_t splits;    /* HGEMM_KERNEL_SPLITK: K splits per tile, 2, 4 or 8 (0 = auto) */
    int32_t stream_k;  /* tensor-core tile kernels: 0 = auto, 1 = never, 2 = whenever the
                          tile count is not a multiple of the persistent cluster count.  Stream-K cuts
                          the k-blocks of the last tiles into equal contiguous ranges, one per cluster;
                          a tile split between clusters is summed in k order through a library-owned
                          FP32 workspace (per device and stream, allocated on first use, never during
                          stream capture), so results are deterministic for a given device. */
    int32_t half_tail; /* 512-wide 2-SM tiles: 0 = auto (when r tiles are left for a last wave after
                          at least 4 whole waves and r <= clusters/2, those r tiles are processed as
                          2r 256-wide items), 1 = never, 2 = whenever r <= clusters/2.  Same per-element
                          arithmetic as whole tiles.  hgemm_get_last_config reports 2 if it was used,
                          1 if not (tile kernels). */
    int32_t tile_n;    /* HGEMM_KERNEL_TC_2SM with block_n 256 only: flexible tile width, a multiple of
                          16 in [128, 256] (0 = block_n).  Tiles of tile_n columns of the output's
                          contiguous dimension (m), so that the tile count fills whole waves; needs a
                          K-major op(A) (transA 'T'), otherwise block_n is used.  The automatic choice
                          does not use it (measured slower than 256-wide tiles with stream-K at every
                          mid-size shape tried; environment HGEMM_FLEX=1 lets its wave model consider
                          it); hgemm_get_last_config reports the width used (0 = block_n).  Whole
                          tiles, no stream-K. */
} hgemm_config_t;

/* Set (cfg != NULL) or reset to automatic (cfg == NULL) the process-global
 * selection.  Returns HGEMM_ERR_INVALID_VALUE for an unknown kernel or
 * block_n.  A forced tensor-core kernel whose preconditions do not hold
 * still falls back to SIMT. */
hgemm_status_t hgemm_set_config(const hgemm_config_t *cfg);

/* The configuration used by the most recent successful hgemm() call in
 * this process (kernel == HGEMM_KERNEL_AUTO if none, or if it was a quick
 * return).  `out` must not be NULL. */
hgemm_status_t hgemm_get_last_config(hgemm_config_t *out);

/* Number of kernel launches hgemm() has enqueued in this process. */
int64_t hgemm_launch_count(void);

/* Diagnostic clock probe.  When `device_buf` is non-NULL (device memory of
 * at least 4 x 8 bytes, owned by the caller), every tensor-core launch makes
 * its CTA 0 write {clock64 at start, %globaltimer ns at start, clock64 at
 * end, %globaltimer ns at end}; the SM clock during the kernel is
 * (clk1-clk0)/(ns1-ns0) GHz.  NULL (the default) disables it.  Process-global. */
hgemm_status_t hgemm_set_probe(unsigned long long *device_buf);

/* ------------------------------------------------------------------------
 * Sharded path: all-gather of op(A) fused with the GEMM
 * (BASELINE.json north_star (3): "N-column slabs of B and C are sharded per
 * GPU with A replicated"; the paper itself
 * is single-GPU, its C = alpha*A*B + beta*C is P:47, SII-A).
 *
 * Rank q of `world` owns rows [row_splits[q], row_splits[q+1]) of op(A)
 * (row_splits: host array of world+1 values, 0 = row_splits[0] <= ... <=
 * row_splits[world] = m).  Every rank holds a full-size GATHER BUFFER `A`
 * in the paper's layout, transA = 'T' (A stored k x m column-major, lda >= k,
 * so row i of op(A) is the contiguous run A + i*lda of k FP16 values), in
 * which its own rows are already written.  A_peers (host array of `world`
 * device pointers) holds every other rank's gather buffer as mapped into this
 * process (hgemm_ipc_open below; for ranks on one device, plain pointers);
 * A_peers[rank] is ignored.  The caller must make the peers' own rows
 * complete before the call (e.g. a barrier after writing them).
 *
 * ONE persistent tcgen05 kernel on `stream` does both steps: an extra copy
 * warp in every CTA pulls the peers' rows of op(A) with 16-B loads from the
 * P2P-mapped peer buffers (NVLink/NVSwitch) into `A`, in copy units of ~64 KB
 * of rows taken from a shared work index in the order owners rank+1, rank+2,
 * ... (mod world), and counts each finished unit in its chunk's counter; the
 * TMA producer of each CTA waits, before the first load of a tile, until
 * every chunk of op(A) rows the tile reads is complete (local chunks never
 * wait), and tiles are scheduled chunk by chunk starting with the local rows,
 * so the transfer overlaps the MMAs tile by tile.  Chunk c is rows
 * [c*chunk_rows, (c+1)*chunk_rows) of op(A).  The result is C = alpha*op(A)*
 * op(B) + beta*C (m x n, same meaning as hgemm() with transA = 'T'), bitwise
 * identical to hgemm() on the gathered A, and `A` ends holding all m rows.
 * `workspace`: caller-owned device memory of workspace_ints >= 1 +
 * ceil(m/chunk_rows) int32, zeroed by the call (stream-ordered memset); one
 * call at a time per workspace.
 * The fused kernel needs world <= 8, shard boundaries on chunk boundaries,
 * k % 8 == 0, 16-B aligned A, peers, B and C and the hgemm() tensor-core
 * preconditions; otherwise (or for a quick return) the peers' rows are copied
 * on `stream` first (cudaMemcpy2DAsync) and hgemm() runs unfused.  Asynchronous
 * like hgemm().
 * Errors (synchronous, nothing enqueued): HGEMM_ERR_INVALID_VALUE for the
 * hgemm() argument errors, world < 1, rank outside [0, world), bad
 * row_splits, chunk_rows < 1, workspace too small, NULL workspace / A / a
 * needed peer pointer; HGEMM_ERR_ARCH; HGEMM_ERR_CUDA. */
hgemm_status_t hgemm_allgather_a(int64_t m, int64_t n, int64_t k, float alpha,
                                 void *A, int64_t lda, const void *const *A_peers,
                                 const int64_t *row_splits, int32_t world, int32_t rank,
                                 const void *B, int64_t ldb, float beta, void *C, int64_t ldc,
                                 char transB, hgemm_dtype_t out_dtype,
                                 int32_t *workspace, int64_t workspace_ints, int64_t chunk_rows,
                                 cudaStream_t stream);

/* The chunk order of hgemm_allgather_a (the unfused copies follow it, the
 * fused kernel's work index and tile raster follow the same owner rotation),
 * as data (host only, no GPU needed).
 * Writes up to max_ops records of 4 int64 {chunk, src_rank, row0, row1} to
 * `ops` in issue order and the total count to *num_ops.  The records of one
 * chunk are consecutive.  A record
 * with src_rank == rank covers rows already local (no copy).  Every row of
 * [0, m) appears in exactly one record, with its owner as src_rank.
 * ops may be NULL (count only).  Errors: HGEMM_ERR_INVALID_VALUE as above. */
hgemm_status_t hgemm_allgather_plan(int64_t m, const int64_t *row_splits, int32_t world, int32_t rank,
                                    int64_t chunk_rows, int64_t *ops, int64_t max_ops, int64_t *num_ops);

/* CUDA IPC of device buffers (cudaIpcGetMemHandle / cudaIpcOpenMemHandle),
 * for interior pointers of an allocation: the handle carries the offset of
 * `dptr` from its allocation base (cuMemGetAddressRange).  The handle is
 * plain bytes: exchange it between processes by any means (the Python
 * layer uses torch.distributed.all_gather_object).  hgemm_ipc_open maps a
 * peer's buffer into this process (peer access enabled lazily) and returns
 * the pointer matching the peer's dptr; hgemm_ipc_close unmaps it.
 * Errors: HGEMM_ERR_INVALID_VALUE (NULL arguments, unknown pointer),
 * HGEMM_ERR_CUDA. */
typedef struct {
    unsigned char handle[64];  /* cudaIpcMemHandle_t */
    int64_t offset;            /* dptr - allocation base, bytes */
} hgemm_ipc_handle_t;
hgemm_status_t hgemm_ipc_get_handle(const void *dptr, hgemm_ipc_handle_t *out);
hgemm_status_t hgemm_ipc_open(const hgemm_ipc_handle_t *h, void **dptr);
hgemm_status_t hgemm_ipc_close(void *dptr);

#ifdef __cplusplus
}
#endif

#endif /* HGEMM_H_ */
