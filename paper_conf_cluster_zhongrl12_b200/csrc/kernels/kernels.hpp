// Internal launcher interface of the sm_100a kernels (C++ only, not the ABI).
#pragma once

#include <cuda_runtime.h>

#include <cstdint>

#include "../common.hpp"

namespace fpm {

// How an FP32 operand is represented on the tensor cores (reading Q15).
enum class SplitScheme : int {
    F16X3 = 0,   // x 2^e = h0 + h1 in fp16, per-row power-of-two scale, 3 x kind::f16
    TF32X3 = 1,  // x = hi + lo in tf32, 3 x kind::tf32
    I8PROBE = 2, // timing probe only (kernel-level entry): int8 operands, 3 x kind::i8, s32 accumulator
    F16I8 = 3,   // x 2^e = h0 + h1; h0 h0' in kind::f16 + 32 (q l' + l q') in kind::i8 (update_f32.cu)
};

// The next update group's F16X3 staging, run by a staging warp of
// the chunked update kernel (variants 7 / 8) while its MMAs run: the persistent
// update holds every SM, so standalone staging kernels could only run between
// two updates (measured: 0.44 ms per group at c5, 1.9 % of the step).  The
// arithmetic is the standalone kernels' (split_math.cuh), so the staged
// operands are the same bits.  A: pieces of the device's rows, each nseg
// segments of K elements (segment j of row r at src + j seg_stride + r lda),
// written to rows row_off.. of a_hi / a_lo (row stride ld_out) with their
// inverse scales in sa.  B: the block-row(s) b_src (Kb x W, row stride ldb)
// transposed into b_hi / b_lo (W x Kb, row stride Kb), column maxima in bmax,
// inverse scales in sb (b_src null: no B -- the device reads another device's
// staged B operand).  ctr: two zeroed counters for the grid barrier between the
// maxima and the split of B (the kernel leaves them zeroed).
constexpr int kMaxStagePieces = 16;
struct StagePiece {
    const float* src;
    int64_t seg_stride, row_off, rows;
};
struct StageJob {
    int active = 0;
    int npieces = 0;
    int nseg = 1;
    int64_t K = 0, lda = 0, ld_out = 0;
    StagePiece a[kMaxStagePieces] = {};
    void* a_hi = nullptr;
    void* a_lo = nullptr;
    float* sa = nullptr;
    const float* b_src = nullptr;
    int64_t ldb = 0, Kb = 0, W = 0;
    void* b_hi = nullptr;
    void* b_lo = nullptr;
    float* sb = nullptr;
    unsigned* bmax = nullptr;
    unsigned* ctr = nullptr;
    // streamed inputs (pmm_run): progress flags of the devices holding this
    // group's pieces (own, local or IPC peer memory) that must reach `need`
    // ((epoch << 16) | (last pivot + 1)) before the staging reads them
    int nwait = 0;
    const unsigned long long* wait_flag[kMaxStagePieces + 1] = {};
    unsigned long long need = 0;
};

struct UpdateArgs {
    const void* a_hi;   // M x K, K-major (row-major, ld = K), fp16 or tf32-in-fp32
    const void* a_lo;
    const void* bt_hi;  // Nc x K, K-major
    const void* bt_lo;
    const float* sa;    // per-row inverse scale of A (F16X3), M floats
    const float* sb;    // per-row inverse scale of Bt (F16X3), Nc floats
    float* C;           // M x Nc, ld = ldc
    int64_t M, Nc, K, ldc;
    SplitScheme scheme;
    int cta_group;      // 1 or 2
    int num_sms;        // SMs the persistent grid may use
    bool accumulate = true;  // false: C = A . Bt^T (no read of C)
    int raster_group = 16;   // tile-rows per raster group (L2 reuse)
    int l2_hint_b = 0;       // B^T tile L2 policy: 0 evict_normal, 1 evict_first, 2 evict_last
    bool raster_snake = false;  // variants 7 / 8: odd raster groups walk the columns backwards
    int variant = -1;        // smem split (cta_group 2): -1 auto (= 8), 4 = SW128 x 2 + 4 C chunks,
                             // 0 = SW128 x 3 stages + 2 C chunks, 1 = SW64 x 4 + 6,
                             // 2 = SW128 x 2 + 6, 3 = SW64 x 5 + 4,
                             // 7 = chunked accumulation (below), 3 stages, C by TMA reduce-add,
                             // 8 = the same with 2 stages (leaves shared memory for NCCL kernels)
    int chunk_k = 0;         // variants 7 / 8: K per TMEM accumulation (0 auto = 512); each chunk's
                             // sum is drained and added to a per-thread FP32 register sum, so the
                             // tensor-core accumulation error stays that of a short K (DESIGN Q15c)
    StageJob stage;          // variants 7 / 8, F16X3: the next group's staging (inactive by default)
};

// C += A . Bt^T  (the rank-b update)
// Diagnostic counters of the F16I8 MMA issuer: op 1 = reset + enable, 0 = disable,
// 2 = read the 4 counters (current device) into out.
void update_prof(int op, unsigned long long* out);
void launch_update_f32(const UpdateArgs& a, cudaStream_t st);

// Split an FP32 panel (rows x K, row stride ld) into the two operand halves.
// F16X3: hi/lo are __half[rows*K], inv_scale[rows] written.
// TF32X3: hi/lo are float[rows*K], inv_scale untouched (may be null).
void launch_split_rows(const float* src, int64_t ld, int64_t rows, int64_t K, SplitScheme s, void* hi,
                       void* lo, float* inv_scale, cudaStream_t st);

// Fused pivots: row r of the operand is nseg segments of K elements, segment j
// at src + j*seg_stride + r*ld; output row stride ld_out (>= nseg*K); the F16X3
// scale is taken over the whole fused row.
// With given_max (F16X3), the row maxima are taken from it (bits of non-negative
// floats, e.g. from launch_rowmax_seg over a wider K) instead of this panel.
void launch_split_rows_seg(const float* src, int64_t ld, int64_t seg_stride, int nseg, int64_t rows, int64_t K,
                           int64_t ld_out, SplitScheme s, void* hi, void* lo, float* inv_scale, cudaStream_t st,
                           const unsigned* given_max = nullptr);

// B pivot row src (K x W, row stride ld) -> split halves of its transpose
// (W x K, K-major), per-row (= per-column of src) inverse scales for F16X3.
// ld_out: row stride of the output (default K); given_max as above (per column).
void launch_split_cols(const float* src, int64_t ld, int64_t K, int64_t W, SplitScheme s, void* hi, void* lo,
                       float* inv_scale, cudaStream_t st, int64_t ld_out = -1, const unsigned* given_max = nullptr);

// m_bits[r] = max(m_bits[r], bits of max |x| over row r of the (fused) panel)
// -- atomicMax on the bit patterns of non-negative floats; zero m_bits first.
void launch_rowmax_seg(const float* src, int64_t ld, int64_t seg_stride, int nseg, int64_t rows, int64_t K,
                       unsigned* m_bits, cudaStream_t st);
// m_bits[c] = max(m_bits[c], bits of max |x| over column c of a K x W block-row)
void launch_colmax(const float* src, int64_t ld, int64_t K, int64_t W, unsigned* m_bits, cudaStream_t st);

// dst (cols x rows, K-major) = transpose of src (rows x cols, ld).
void launch_transpose_f32(const float* src, int64_t ld, int64_t rows, int64_t cols, float* dst,
                          cudaStream_t st);
void launch_transpose_f64(const double* src, int64_t ld, int64_t rows, int64_t cols, double* dst,
                          cudaStream_t st);

// C (M x Nc, ldc) += A (M x K, lda) . Bt^T, Bt (Nc x K), FP64 on DMMA.  With
// seg > 0, A is K / seg panels of M x seg (row stride lda) seg_stride elements
// apart (the pivots of a fused group); seg <= 0: one M x K matrix.
void launch_update_f64(const double* A, int64_t lda, const double* Bt, double* C, int64_t M, int64_t Nc,
                       int64_t K, int64_t ldc, bool accumulate, int num_sms, cudaStream_t st, int64_t seg = 0,
                       int64_t seg_stride = 0);

// Seeded counter-based generator (same bits as synth/__init__.py).
void launch_fill_synthetic(void* dst, bool f64, int64_t ld, uint64_t seed, int64_t N, int64_t r0, int64_t c0,
                           int64_t rows, int64_t cols, int dist, cudaStream_t st);

// Panel copy (rows x cols elements of `elem` bytes) between strided buffers.
void launch_zero(void* dst, size_t bytes, cudaStream_t st);

}  // namespace fpm
