/*
 * oracle/hgemm_ref.c -- CPU FP64 reference for C = alpha*op(A)*op(B) + beta*C.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference legs may load or call this.
 * It shares no code, header, table or helper with the CUDA path
 * (paper_conf_ipps_00020c20_b200/csrc) and neither side includes the other.
 *
 * What it computes (the plain definition; PAPER.md = /root/reference/PAPER.md):
 *   P:47  (SII-A)  "C = alpha*A*B + beta*C, where A, B and C are m x k, n x k and
 *                  m x n matrices" -- read as BLAS op(A) m x k, op(B) k x n,
 *                  column-major storage (readings R1, R2).
 *   P:49  (SII-A)  m x n x k notation.
 *   P:401 (SVII)   FP16 inputs (and FP16 output).
 *   P:246-272 (Alg. 1) the blocked method only reorders the K summation, so the
 *                  result the method reaches is the plain triple loop below.
 *   BASELINE.json north_star (4): "FP16 -> FP64 naive triple loop".
 * Steps, in order (DESIGN.md section "Oracle"):
 *   1. decode every FP16 input exactly to FP64 by bit manipulation (IEEE 754
 *      binary16: 1 sign, 5 exponent (bias 15), 10 fraction bits, subnormals,
 *      inf, NaN) -- not through a compiler half type;
 *   2. s_ij = sum_{p=0}^{k-1} opA(i,p)*opB(p,j) in FP64, p increasing
 *      (FP16 x FP16 products are exact in FP64);
 *   3. r_ij = alpha*s_ij + beta*c_ij, with BLAS quick-return semantics:
 *      beta == 0 -> C is never read; alpha == 0 or k == 0 -> r = beta*c
 *      (reading R6);
 *   4. round r ONCE to the output type: FP32 by C's (float) conversion
 *      (round-to-nearest-even), FP16 by f64_to_f16 below (RN-even, overflow
 *      to +-inf, subnormals kept; reading R4).
 * It also returns the unrounded r_ij and absab_ij = sum_p |opA(i,p)|*|opB(p,j)|,
 * the scale of the north_star (4) tolerance 1e-3*(|A||B|)_ij.
 *
 * Parity pins for every function here: tests/test_oracle_pins.py
 * (exhaustive decode, RN-even encode incl. hand-derived ties in
 * tests/golden/, numpy float64 matmul cross-check, identity / permutation /
 * integer closed forms, accumulator-width closed form).
 */
#include <math.h>
#include <stdint.h>
#include <stddef.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* Step 1: IEEE binary16 bits -> exact double. */
double hgemm_ref_f16_to_f64(uint16_t h)
{
    int sign = (h >> 15) & 1;
    int e = (h >> 10) & 0x1f;
    int f = h & 0x3ff;
    double v;
    if (e == 0) {
        v = ldexp((double)f, -24);                 /* subnormal: f * 2^-24 */
    } else if (e == 31) {
        v = (f == 0) ? INFINITY : NAN;             /* inf / NaN */
    } else {
        v = ldexp((double)(1024 + f), e - 25);     /* (1.f) * 2^(e-15) */
    }
    return sign ? -v : v;
}

/* Step 4 (FP16 output): double -> binary16, one rounding, nearest-even. */
uint16_t hgemm_ref_f64_to_f16(double x)
{
    uint16_t sign = signbit(x) ? 0x8000u : 0u;
    double a = fabs(x);
    if (isnan(x)) return (uint16_t)(sign | 0x7e00u);
    if (isinf(a)) return (uint16_t)(sign | 0x7c00u);
    if (a == 0.0) return sign;
    int e;
    (void)frexp(a, &e);          /* a = f * 2^e, f in [0.5,1)  =>  floor(log2 a) = e-1 */
    int E = e - 1;
    if (E < -14) {
        /* subnormal range: quantum 2^-24; rint() rounds half to even */
        double q = rint(ldexp(a, 24));
        /* q == 1024 is the smallest normal, whose bit pattern is 0x0400 */
        return (uint16_t)(sign | (uint16_t)q);
    }
    double q = rint(ldexp(a, 10 - E));   /* significand in [1024, 2048] */
    if (q == 2048.0) { q = 1024.0; E += 1; }
    if (E > 15) return (uint16_t)(sign | 0x7c00u);   /* |x| >= 65520 -> inf */
    return (uint16_t)(sign | (uint16_t)((E + 15) << 10) | (uint16_t)((int)q - 1024));
}

static inline int is_trans(char t) { return t == 'T' || t == 't'; }

/* opA(i,p), opB(p,j) for column-major storage. */
static inline uint16_t opA_bits(const uint16_t *A, int64_t lda, char tA, int64_t i, int64_t p)
{
    return is_trans(tA) ? A[p + i * lda] : A[i + p * lda];
}
static inline uint16_t opB_bits(const uint16_t *B, int64_t ldb, char tB, int64_t p, int64_t j)
{
    return is_trans(tB) ? B[j + p * ldb] : B[p + j * ldb];
}

/* Step 3: r = alpha*s + beta*c with BLAS quick-return semantics. */
static double finish_entry(int64_t i, int64_t j, int64_t k, float alpha, double s,
                           float beta, const void *C, int64_t ldc, int out_f32, double *absab)
{
    double c = 0.0;
    if (beta != 0.0f) {                                /* beta == 0: C never read */
        c = out_f32 ? (double)((const float *)C)[i + j * ldc]
                    : hgemm_ref_f16_to_f64(((const uint16_t *)C)[i + j * ldc]);
    }
    if (alpha == 0.0f || k == 0) {                     /* BLAS quick return */
        *absab = 0.0;
        return (beta != 0.0f) ? (double)beta * c : 0.0;
    }
    double r = (double)alpha * s;
    if (beta != 0.0f) r += (double)beta * c;
    return r;
}

static void one_entry(int64_t i, int64_t j, int64_t k, float alpha,
                      const uint16_t *A, int64_t lda, const uint16_t *B, int64_t ldb,
                      float beta, const void *C, int64_t ldc, char tA, char tB, int out_f32,
                      double *r_out, double *absab_out, void *C_out, int64_t out_index)
{
    double s = 0.0, absab = 0.0;
    for (int64_t p = 0; p < k; ++p) {                  /* steps 1-2, p increasing */
        double a = hgemm_ref_f16_to_f64(opA_bits(A, lda, tA, i, p));
        double b = hgemm_ref_f16_to_f64(opB_bits(B, ldb, tB, p, j));
        s += a * b;
        absab += fabs(a) * fabs(b);
    }
    double r = finish_entry(i, j, k, alpha, s, beta, C, ldc, out_f32, &absab);
    if (r_out) r_out[out_index] = r;
    if (absab_out) absab_out[out_index] = absab;
    if (C_out) {                                       /* step 4 */
        if (out_f32) ((float *)C_out)[out_index] = (float)r;
        else ((uint16_t *)C_out)[out_index] = hgemm_ref_f64_to_f16(r);
    }
}

/*
 * Full reference.  Same argument order as the product ABI (include/hgemm.h),
 * but host pointers, raw FP16 bits, and a separate output buffer:
 *   C      : input C (read only when beta != 0), column-major, ldc
 *   C_out  : m x n output, column-major with leading dimension ldc (may be NULL;
 *            may equal C only when beta == 0)
 *   r_out, absab_out : optional (NULL) m x n column-major with leading dim m
 *   nthreads : OpenMP threads over output columns (1 = single thread)
 * Returns 0, or -1 on invalid arguments.
 */
int hgemm_ref(int64_t m, int64_t n, int64_t k, float alpha,
              const uint16_t *A, int64_t lda, const uint16_t *B, int64_t ldb,
              float beta, const void *C, int64_t ldc, char transA, char transB,
              int out_f32, void *C_out, double *r_out, double *absab_out, int nthreads)
{
    if (m < 0 || n < 0 || k < 0) return -1;
    if (ldc < (m > 1 ? m : 1)) return -1;
    int nt = nthreads > 0 ? nthreads : 1;
    /* Step 1: decode every input once: Ad[i*k + p] = opA(i,p), Bd[j*k + p] = opB(p,j). */
    double *Ad = (double *)malloc(sizeof(double) * (size_t)(m * k > 0 ? m * k : 1));
    double *Bd = (double *)malloc(sizeof(double) * (size_t)(n * k > 0 ? n * k : 1));
    if (!Ad || !Bd) { free(Ad); free(Bd); return -2; }
    int64_t i0, j0;
#pragma omp parallel for num_threads(nt)
    for (i0 = 0; i0 < m; ++i0)
        for (int64_t p = 0; p < k; ++p)
            Ad[i0 * k + p] = hgemm_ref_f16_to_f64(opA_bits(A, lda, transA, i0, p));
#pragma omp parallel for num_threads(nt)
    for (j0 = 0; j0 < n; ++j0)
        for (int64_t p = 0; p < k; ++p)
            Bd[j0 * k + p] = hgemm_ref_f16_to_f64(opB_bits(B, ldb, transB, p, j0));
    /* Steps 2-4 per output entry. */
    int64_t jj;
#pragma omp parallel for schedule(dynamic, 1) num_threads(nt)
    for (jj = 0; jj < n; ++jj) {
        for (int64_t i = 0; i < m; ++i) {
            double s = 0.0, absab = 0.0;
            const double *a = Ad + i * k, *b = Bd + jj * k;
            for (int64_t p = 0; p < k; ++p) {          /* step 2, p increasing */
                s += a[p] * b[p];
                absab += fabs(a[p]) * fabs(b[p]);
            }
            double r = finish_entry(i, jj, k, alpha, s, beta, C, ldc, out_f32, &absab);
            if (r_out) r_out[i + jj * m] = r;
            if (absab_out) absab_out[i + jj * m] = absab;
            if (C_out) {
                if (out_f32) ((float *)C_out)[i + jj * ldc] = (float)r;
                else ((uint16_t *)C_out)[i + jj * ldc] = hgemm_ref_f64_to_f16(r);
            }
        }
    }
    free(Ad);
    free(Bd);
    return 0;
}

/*
 * Sampled reference for large shapes: entries (idx_i[t], idx_j[t]), t < count.
 * Outputs are dense length-count arrays (any of them may be NULL).
 */
int hgemm_ref_entries(int64_t m, int64_t n, int64_t k, float alpha,
                      const uint16_t *A, int64_t lda, const uint16_t *B, int64_t ldb,
                      float beta, const void *C, int64_t ldc, char transA, char transB,
                      int out_f32, const int64_t *idx_i, const int64_t *idx_j, int64_t count,
                      void *C_out, double *r_out, double *absab_out, int nthreads)
{
    if (m < 0 || n < 0 || k < 0 || count < 0) return -1;
    for (int64_t t = 0; t < count; ++t)
        if (idx_i[t] < 0 || idx_i[t] >= m || idx_j[t] < 0 || idx_j[t] >= n) return -1;
    (void)nthreads;
    int64_t t;
#pragma omp parallel for schedule(dynamic, 16) num_threads(nthreads > 0 ? nthreads : 1)
    for (t = 0; t < count; ++t)
        one_entry(idx_i[t], idx_j[t], k, alpha, A, lda, B, ldb, beta, C, ldc, transA, transB,
                  out_f32, r_out, absab_out, C_out, t);
    return 0;
}

int hgemm_ref_max_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
