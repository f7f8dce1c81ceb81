// CUDA-core kernels that complete the ABI outside the tensor-core fast path:
//   * hgemm_simt_kernel : C = alpha*op(A)*op(B) + beta*C for any alignment /
//     leading dimension (the TMA preconditions of include/hgemm.h do not hold).
//     FP32 accumulation, same epilogue rounding as the tcgen05 path.
//   * hgemm_scale_kernel: the BLAS quick return C = beta*C (k == 0 or alpha == 0),
//     writing zeros without reading C when beta == 0.
// Column-major ABI indexing (include/hgemm.h).
#pragma once
#include <cuda_fp16.h>

namespace hg {

template <bool OUT_F32>
__device__ __forceinline__ float load_c(const void *C, int64_t idx) {
  if constexpr (OUT_F32) return static_cast<const float *>(C)[idx];
  else return __half2float(static_cast<const __half *>(C)[idx]);
}
template <bool OUT_F32>
__device__ __forceinline__ void store_c(void *C, int64_t idx, float v) {
  if constexpr (OUT_F32) static_cast<float *>(C)[idx] = v;
  else static_cast<__half *>(C)[idx] = __float2half_rn(v);
}

// 64 x 64 output tile per 256-thread block, 4 x 4 outputs per thread, K step 16.
// ACC16 (hgemm_ex HGEMM_COMPUTE_F16, FP16 output): an FP16 accumulator (the paper's
// FP16-accumulate mode, P:98 / P:350) updated once per 16-deep K step, like one
// tcgen05.mma kind::f16 K = 16 step: the step's 16 products are summed in FP32 and
// the accumulator is rounded to FP16 after adding them.
template <bool OUT_F32, bool ACC16 = false>
__global__ void __launch_bounds__(256) hgemm_simt_kernel(int64_t m, int64_t n, int64_t k, float alpha,
                                                         const __half *__restrict__ A, int64_t lda,
                                                         const __half *__restrict__ B, int64_t ldb, float beta,
                                                         void *C, int64_t ldc, int transA, int transB) {
  __shared__ float As[16][64 + 1];  // As[p][i] = opA(i0+i, p0+p)
  __shared__ float Bs[16][64 + 1];  // Bs[p][j] = opB(p0+p, j0+j)
  const int64_t i0 = static_cast<int64_t>(blockIdx.x) * 64;
  const int64_t j0 = static_cast<int64_t>(blockIdx.y) * 64;
  const int tx = threadIdx.x & 15, ty = threadIdx.x >> 4;
  float acc[4][4] = {};
  for (int64_t p0 = 0; p0 < k; p0 += 16) {
    float acc0[4][4];  // ACC16: the accumulator before this K step
    if constexpr (ACC16) {
#pragma unroll
      for (int r = 0; r < 4; ++r)
#pragma unroll
        for (int c = 0; c < 4; ++c) {
          acc0[r][c] = acc[r][c];
          acc[r][c] = 0.f;
        }
    }
    for (int e = threadIdx.x; e < 16 * 64; e += 256) {
      const int pp = transA ? (e & 15) : (e >> 6);
      const int ii = transA ? (e >> 4) : (e & 63);
      const int64_t gi = i0 + ii, gp = p0 + pp;
      float v = 0.f;
      if (gi < m && gp < k) v = __half2float(transA ? A[gp + gi * lda] : A[gi + gp * lda]);
      As[pp][ii] = v;
      const int pb = transB ? (e >> 6) : (e & 15);
      const int jb = transB ? (e & 63) : (e >> 4);
      const int64_t gj = j0 + jb, gq = p0 + pb;
      float w = 0.f;
      if (gj < n && gq < k) w = __half2float(transB ? B[gj + gq * ldb] : B[gq + gj * ldb]);
      Bs[pb][jb] = w;
    }
    __syncthreads();
#pragma unroll
    for (int pp = 0; pp < 16; ++pp) {
      float a[4], b[4];
#pragma unroll
      for (int r = 0; r < 4; ++r) a[r] = As[pp][tx + 16 * r];
#pragma unroll
      for (int c = 0; c < 4; ++c) b[c] = Bs[pp][ty + 16 * c];
#pragma unroll
      for (int r = 0; r < 4; ++r)
#pragma unroll
        for (int c = 0; c < 4; ++c) acc[r][c] = fmaf(a[r], b[c], acc[r][c]);
    }
    if constexpr (ACC16) {
#pragma unroll
      for (int r = 0; r < 4; ++r)
#pragma unroll
        for (int c = 0; c < 4; ++c) acc[r][c] = __half2float(__float2half_rn(acc0[r][c] + acc[r][c]));
    }
    __syncthreads();
  }
#pragma unroll
  for (int r = 0; r < 4; ++r)
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      const int64_t gi = i0 + tx + 16 * r, gj = j0 + ty + 16 * c;
      if (gi < m && gj < n) {
        const int64_t idx = gi + gj * ldc;
        float o = alpha * acc[r][c];
        if (beta != 0.0f) o = fmaf(beta, load_c<OUT_F32>(C, idx), o);
        store_c<OUT_F32>(C, idx, o);
      }
    }
}

template <bool OUT_F32>
__global__ void hgemm_scale_kernel(int64_t m, int64_t n, float beta, void *C, int64_t ldc) {
  const int64_t total = m * n;
  for (int64_t e = blockIdx.x * static_cast<int64_t>(blockDim.x) + threadIdx.x; e < total;
       e += static_cast<int64_t>(gridDim.x) * blockDim.x) {
    const int64_t i = e % m, j = e / m;
    const int64_t idx = i + j * ldc;
    const float o = (beta != 0.0f) ? beta * load_c<OUT_F32>(C, idx) : 0.0f;
    store_c<OUT_F32>(C, idx, o);
  }
}

}  // namespace hg
