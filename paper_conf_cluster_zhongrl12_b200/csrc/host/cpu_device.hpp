// Host-CPU devices (§III, §V: a socket of c cores running
// the GEMM kernel simultaneously, speed function s_c(x) with problem size x/c
// per core).  A CPU device is a team of worker threads
// pinned to c host cores; its rectangle of the column-based arrangement is
// updated by the product-side FP32 / FP64 GEMM below (packed, cache-blocked,
// AVX-512 or AVX2 FMA micro-kernels), rows split evenly across the cores.
//
// This is a device of the partition, chosen by the caller (pmm_create_local
// with cuda_devices[i] = FPM_CPU_DEVICE), never a fallback for GPU work: a GPU
// device's update always runs on the GPU, and the library has no code path that
// moves it here.  No CUDA types in this header.
#pragma once

#include <cstdint>
#include <vector>

namespace fpm {
namespace cpu {

struct Team;

// Host cores this process may run on (sched_getaffinity), ascending.
std::vector<int> allowed_cores();
// Worker threads pinned one per core (cores empty: `n` unpinned threads).
Team* team_create(const std::vector<int>& cores, int n = 0);
void team_destroy(Team* t);
// Instruction set of the micro-kernels in use: "avx512", "avx2" or "generic".
const char* isa();

// C (M x N, ldc) (+)= A (M x K) * B (K x N, ldb), row-major; A stored in
// K-segments of `seg` columns: A(i, k) = A[(k / seg) * seg_stride + i * lda + k % seg]
// (seg = K, seg_stride = 0: an ordinary row-major A).  accumulate = false
// overwrites C.  FP32 accumulates in FP32 FMA over K-blocks of 256 and adds each
// block's sum to C (SGEMM arithmetic, "implemented by the GEMM routine");
// FP64 likewise in FP64.  Rows of C are split across the team's threads.
void gemm_f32(Team* t, int64_t M, int64_t N, int64_t K, const float* A, int64_t lda, int64_t seg, int64_t seg_stride,
              const float* B, int64_t ldb, float* C, int64_t ldc, bool accumulate);
void gemm_f64(Team* t, int64_t M, int64_t N, int64_t K, const double* A, int64_t lda, int64_t seg, int64_t seg_stride,
              const double* B, int64_t ldb, double* C, int64_t ldc, bool accumulate);

// The shared counter-based generator (synth/__init__.py) on the host: rows
// [r0, r0 + rows) x cols [c0, c0 + cols) of the global N x N matrix into dst
// (row stride ld), dist 0 = U[-1, 1), 1 = integers in [-8, 8].
void fill_synthetic(Team* t, void* dst, bool f64, int64_t ld, uint64_t seed, int64_t N, int64_t r0, int64_t c0,
                    int64_t rows, int64_t cols, int dist);

}  // namespace cpu
}  // namespace fpm
