/* Oracle O5: plain triple-loop matrix product.  TEST INFRASTRUCTURE ONLY
 * (see oracle/__init__.py) -- never linked into the product library.
 *
 * PAPER.md P:15 / P:18: the blocked column-based algorithm computes C = A x B,
 * each iteration adding the rank-b product of the pivot column A(b) and the
 * pivot row B(b) ("Ci += A(b) x B(b)").  Summed over all N/b iterations that is
 * exactly the plain product, so the oracle is the plain product:
 *
 *     C[i][j] = sum_k A[i][k] * B[k][j]
 *
 * i-k-j loop order, FP64 accumulation (FP32 inputs are widened exactly),
 * OpenMP over rows i only (each row's sum is computed sequentially in k, so the
 * result does not depend on the thread count).  No BLAS, no blocking.
 * Build: gcc -O2 -fopenmp -fno-fast-math -ffp-contract=off -shared -fPIC.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

/* C (M x N, ldc) = A (M x K, lda) * B (K x N, ldb); float inputs, double out. */
void oracle_gemm_f32in(int64_t M, int64_t N, int64_t K,
                       const float* A, int64_t lda,
                       const float* B, int64_t ldb,
                       double* C, int64_t ldc)
{
    int64_t i;
#pragma omp parallel for schedule(static)
    for (i = 0; i < M; ++i) {
        double* c = C + i * ldc;
        for (int64_t j = 0; j < N; ++j) c[j] = 0.0;
        for (int64_t k = 0; k < K; ++k) {
            const double a = (double)A[i * lda + k];
            const float* b = B + k * ldb;
            for (int64_t j = 0; j < N; ++j) c[j] += a * (double)b[j];
        }
    }
}

/* Same definition with double inputs (FP64 configuration, BASELINE config 1). */
void oracle_gemm_f64in(int64_t M, int64_t N, int64_t K,
                       const double* A, int64_t lda,
                       const double* B, int64_t ldb,
                       double* C, int64_t ldc)
{
    int64_t i;
#pragma omp parallel for schedule(static)
    for (i = 0; i < M; ++i) {
        double* c = C + i * ldc;
        for (int64_t j = 0; j < N; ++j) c[j] = 0.0;
        for (int64_t k = 0; k < K; ++k) {
            const double a = A[i * lda + k];
            const double* b = B + k * ldb;
            for (int64_t j = 0; j < N; ++j) c[j] += a * b[j];
        }
    }
}

int oracle_num_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}

/* Thread count of the OpenMP loops above (timing only; the result does not
 * depend on it).  bench.py's reference arm runs on rank 0 alone under
 * torchrun, which exports OMP_NUM_THREADS=1. */
void oracle_set_num_threads(int n)
{
#ifdef _OPENMP
    if (n > 0) omp_set_num_threads(n);
#else
    (void)n;
#endif
}
