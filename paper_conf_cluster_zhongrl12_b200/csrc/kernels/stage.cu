// Pivot staging kernels: the FP32 operand split for the tensor
// cores, the B pivot-row transpose to a K-major panel, the FP64 update on DMMA,
// and the seeded synthetic-input generator.  All HBM-bound except the FP64
// update; vectorised, coalesced, grid sized in multiples of the SM count.
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>

#include "kernels.hpp"
#include "split_math.cuh"

namespace fpm {

namespace {

__device__ __forceinline__ float tf32_rna(float x) {
    uint32_t r;
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
    return __uint_as_float(r);
}


// F16I8 codes of a scaled element xs = x 2^s (update_f32.cu): h0 = fp16_rn(xs),
// q = clamp(rint(xs / 256), +-127), l = rint(8 (xs - h0)) (|l| <= 64).
__device__ __forceinline__ __half f16i8_codes(float xs, int& qc, int& lc) {
    const __half h = __float2half_rn(xs);
    qc = min(127, max(-127, __float2int_rn(xs * (1.0f / 256.0f))));
    lc = __float2int_rn((xs - __half2float(h)) * 8.0f);
    return h;
}
__device__ __forceinline__ uint32_t pack4_s8(int a, int b, int c, int d) {
    return (uint32_t)(a & 0xff) | ((uint32_t)(b & 0xff) << 8) | ((uint32_t)(c & 0xff) << 16) |
           ((uint32_t)(d & 0xff) << 24);
}

// One warp per row.  A row of the operand is nseg segments of K elements, segment
// j at src + j * seg_stride + row * ld (the panels of nseg consecutive pivots
// fused into one update); it is written to out + row * ld_out + j * K.
// F16X3: choose 2^s with the maximum of the whole (fused) row scaled into
// [2^14, 2^15), h0 = fp16(x 2^s), h1 = fp16(x 2^s - h0); inv_scale = 2^-s.
// With `given` set, the row maximum is given[row] (bits of a non-negative float,
// from rowmax_k over a wider K range) and the first pass is skipped.
__device__ __forceinline__ float row_absmax(const float* src, int64_t ld, int64_t seg_stride, int nseg, int64_t row,
                                            int64_t K, int lane) {
    const int64_t n4 = K / 4;
    float m = 0.0f;
    for (int j = 0; j < nseg; ++j) {
        const float4* s4 = reinterpret_cast<const float4*>(src + j * seg_stride + row * ld);
        for (int64_t i = lane; i < n4; i += 32) {
            const float4 v = s4[i];
            m = fmaxf(m, fmaxf(fmaxf(fabsf(v.x), fabsf(v.y)), fmaxf(fabsf(v.z), fabsf(v.w))));
        }
    }
    return warp_max(m);
}

// I8 (F16I8): `lo` holds the int8 codes instead of h1, as 128-byte rows per
// 64-wide k-block: [q of the 64 | l of the 64] (K % 64 == 0).
template <bool I8>
__global__ void __launch_bounds__(256) split_rows_f16(const float* __restrict__ src, int64_t ld, int64_t seg_stride,
                                                      int nseg, int64_t rows, int64_t K, int64_t ld_out,
                                                      __half* __restrict__ hi, __half* __restrict__ lo,
                                                      float* __restrict__ inv_scale,
                                                      const unsigned* __restrict__ given) {
    const int64_t row = (int64_t)blockIdx.x * 8 + threadIdx.x / 32;
    const int lane = threadIdx.x % 32;
    if (row >= rows) return;
    const int64_t n4 = K / 4;
    const float m = given ? __uint_as_float(given[row]) : row_absmax(src, ld, seg_stride, nseg, row, K, lane);
    const int s = f16x3_shift(m);
    const float scale = ldexpf(1.0f, s);
    if (lane == 0) inv_scale[row] = ldexpf(1.0f, -s);
    for (int j = 0; j < nseg; ++j) {
        const float4* s4 = reinterpret_cast<const float4*>(src + j * seg_stride + row * ld);
        __half2* h2 = reinterpret_cast<__half2*>(hi + row * ld_out + j * K);
        __half2* l2 = reinterpret_cast<__half2*>(lo + row * ld_out + j * K);
        for (int64_t i = lane; i < n4; i += 32) {
            const float4 v = s4[i];
            const float x[4] = {v.x * scale, v.y * scale, v.z * scale, v.w * scale};
            __half h[4], l[4];
            int qc[4], lc[4];
#pragma unroll
            for (int q = 0; q < 4; ++q) {
                if constexpr (I8) {
                    h[q] = f16i8_codes(x[q], qc[q], lc[q]);
                } else {
                    f16x3_split((&v.x)[q], scale, h[q], l[q]);
                }
            }
            h2[2 * i] = __halves2half2(h[0], h[1]);
            h2[2 * i + 1] = __halves2half2(h[2], h[3]);
            if constexpr (I8) {
                const int64_t k = 4 * i;
                uint8_t* b8 = reinterpret_cast<uint8_t*>(l2) + (k / 64) * 128 + (k % 64);
                *reinterpret_cast<uint32_t*>(b8) = pack4_s8(qc[0], qc[1], qc[2], qc[3]);
                *reinterpret_cast<uint32_t*>(b8 + 64) = pack4_s8(lc[0], lc[1], lc[2], lc[3]);
            } else {
                l2[2 * i] = __halves2half2(l[0], l[1]);
                l2[2 * i + 1] = __halves2half2(l[2], l[3]);
            }
        }
    }
}

__global__ void __launch_bounds__(256) split_rows_tf32(const float* __restrict__ src, int64_t ld, int64_t seg_stride,
                                                       int nseg, int64_t rows, int64_t K, int64_t ld_out,
                                                       float* __restrict__ hi, float* __restrict__ lo) {
    const int64_t n4 = K / 4;
    const int64_t per_row = nseg * n4;
    const int64_t total = rows * per_row;
    for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = idx / per_row, rem = idx - r * per_row;
        const int64_t j = rem / n4, c = rem - j * n4;
        const float4 v = reinterpret_cast<const float4*>(src + j * seg_stride + r * ld)[c];
        float4 h, l;
        h.x = tf32_rna(v.x); l.x = tf32_rna(v.x - h.x);
        h.y = tf32_rna(v.y); l.y = tf32_rna(v.y - h.y);
        h.z = tf32_rna(v.z); l.z = tf32_rna(v.z - h.z);
        h.w = tf32_rna(v.w); l.w = tf32_rna(v.w - h.w);
        reinterpret_cast<float4*>(hi + r * ld_out + j * K)[c] = h;
        reinterpret_cast<float4*>(lo + r * ld_out + j * K)[c] = l;
    }
}

// B pivot row (K rows x W cols, row stride ld) -> K-major operand halves of its
// transpose (W rows x K, row stride ld_out), split as in split_rows_*.
// Three launches: column maxima (colmax_tile_k), the split + transpose
// (split_cols_t), then the inverse scales (scale_from_max_k); with `given`
// maxima (the fused tail) the first and last are skipped.  Both main kernels
// are spread over the whole grid of (32 columns) x (K chunks), and use no
// shared memory: kernels with shared memory were measured NOT to co-reside with
// the persistent update kernel (they waited for it to finish, even with the
// max-shared carveout and ~34 KB left per SM), while these must run under it.
// A warp reads 8 rows x 32 columns (128 B coalesced per row; lane = column),
// each lane writes its column's 8 values as 16 B of output row `column`; the 4
// warps of a CTA fill 64 B of each output row, merged into full sectors in L2.
// The split runs in CTAs of 128 threads: it needs ~60 registers per thread, and
// the persistent update (320 threads x 168 registers) leaves 11 776 registers
// of an SM free -- 4 warps fit beside it, 8 did not, so a 256-thread split
// waited for the update to finish (measured: 0.41 ms exposed per update group
// at c5, pmm_group_times).
constexpr int kColTileK = 32;     // rows of B (= K of the output) per CTA: 4 warps x 8 rows
constexpr int kColThreads = 128;
constexpr int kColMaxRows = 256;  // rows per CTA of the maxima pass: 8 warps x 32 rows
constexpr int kColsPerCta = 128;  // 32 lanes x 4 columns (float4 loads)

// m_bits[c] = max(m_bits[c], bits of max |src[r][c]|): each warp 32 rows of 128
// columns (a float4 per lane and row), one atomicMax per column per warp.
__global__ void __launch_bounds__(256) colmax_tile_k(const float* __restrict__ src, int64_t ld, int64_t K,
                                                     int64_t W, unsigned* __restrict__ m_bits) {
    const int lane = threadIdx.x % 32, warp = threadIdx.x / 32;
    const int64_t col = (int64_t)blockIdx.x * kColsPerCta + 4 * lane;
    const int64_t r0 = (int64_t)blockIdx.y * kColMaxRows + warp * 32;
    if (col >= W || r0 >= K) return;  // W % 4 == 0: four columns are all in or all out
    float4 m = make_float4(0.f, 0.f, 0.f, 0.f);
    const int rows = K - r0 < 32 ? (int)(K - r0) : 32;
#pragma unroll 8
    for (int i = 0; i < rows; ++i) {
        const float4 v = *reinterpret_cast<const float4*>(src + (r0 + i) * ld + col);
        m.x = fmaxf(m.x, fabsf(v.x));
        m.y = fmaxf(m.y, fabsf(v.y));
        m.z = fmaxf(m.z, fabsf(v.z));
        m.w = fmaxf(m.w, fabsf(v.w));
    }
    atomicMax(m_bits + col + 0, __float_as_uint(m.x));
    atomicMax(m_bits + col + 1, __float_as_uint(m.y));
    atomicMax(m_bits + col + 2, __float_as_uint(m.z));
    atomicMax(m_bits + col + 3, __float_as_uint(m.w));
}

// Split + transpose: warp w of a CTA reads rows kk .. kk+7 (kk = k0 + 8 w) of 128
// columns (a float4 per lane and row); each lane then writes, for each of its 4
// columns, the 8 values as 16 B of output row `column`.
// I8 (F16I8): `lo` holds int8 codes as 128-byte rows per 64-wide k-block:
// [l of the 64 | q of the 64] (the B side of the cross-term product).
template <bool F16, bool I8 = false>
__global__ void __launch_bounds__(kColThreads) split_cols_t(const float* __restrict__ src, int64_t ld, int64_t K, int64_t W,
                                                    int64_t ld_out, void* __restrict__ hi, void* __restrict__ lo,
                                                    const unsigned* __restrict__ m_bits,
                                                    float* __restrict__ inv_scale) {
    const int lane = threadIdx.x % 32, warp = threadIdx.x / 32;
    const int64_t col = (int64_t)blockIdx.x * kColsPerCta + 4 * lane;
    const int64_t kk = (int64_t)blockIdx.y * kColTileK + warp * 8;
    if (col >= W || kk >= K) return;  // K % 8 == 0, W % 4 == 0: chunks are all in or all out
    float x[4][8];
#pragma unroll
    for (int i = 0; i < 8; ++i) {
        const float4 v = *reinterpret_cast<const float4*>(src + (kk + i) * ld + col);
        x[0][i] = v.x;
        x[1][i] = v.y;
        x[2][i] = v.z;
        x[3][i] = v.w;
    }
#pragma unroll
    for (int c = 0; c < 4; ++c) {
        const int64_t orow = (col + c) * ld_out + kk;
        if constexpr (F16) {
            const int s = f16x3_shift(__uint_as_float(m_bits[col + c]));
            const float scale = ldexpf(1.0f, s);
            if (inv_scale != nullptr && kk == 0) inv_scale[col + c] = ldexpf(1.0f, -s);
            __align__(16) __half h[8], l[8];
            int qc[8], lc[8];
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                const float xs = x[c][i] * scale;
                if constexpr (I8) {
                    h[i] = f16i8_codes(xs, qc[i], lc[i]);
                } else {
                    f16x3_split(x[c][i], scale, h[i], l[i]);
                }
            }
            *reinterpret_cast<uint4*>(static_cast<__half*>(hi) + orow) = *reinterpret_cast<uint4*>(h);
            if constexpr (I8) {
                uint8_t* b8 = reinterpret_cast<uint8_t*>(static_cast<__half*>(lo) + (col + c) * ld_out) +
                              (kk / 64) * 128 + (kk % 64);
                *reinterpret_cast<uint2*>(b8) =
                    make_uint2(pack4_s8(lc[0], lc[1], lc[2], lc[3]), pack4_s8(lc[4], lc[5], lc[6], lc[7]));
                *reinterpret_cast<uint2*>(b8 + 64) =
                    make_uint2(pack4_s8(qc[0], qc[1], qc[2], qc[3]), pack4_s8(qc[4], qc[5], qc[6], qc[7]));
            } else {
                *reinterpret_cast<uint4*>(static_cast<__half*>(lo) + orow) = *reinterpret_cast<uint4*>(l);
            }
        } else {
            __align__(16) float h[8], l[8];
#pragma unroll
            for (int i = 0; i < 8; ++i) {
                h[i] = tf32_rna(x[c][i]);
                l[i] = tf32_rna(x[c][i] - h[i]);
            }
            float4* hp = reinterpret_cast<float4*>(static_cast<float*>(hi) + orow);
            float4* lp = reinterpret_cast<float4*>(static_cast<float*>(lo) + orow);
            hp[0] = *reinterpret_cast<float4*>(h);
            hp[1] = *reinterpret_cast<float4*>(h + 4);
            lp[0] = *reinterpret_cast<float4*>(l);
            lp[1] = *reinterpret_cast<float4*>(l + 4);
        }
    }
}

// In place: maxima bits -> inverse F16X3 scales 2^-s (the buffer is inv_scale).
__global__ void __launch_bounds__(256) scale_from_max_k(float* __restrict__ buf, int64_t W) {
    const int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (c < W) buf[c] = ldexpf(1.0f, -f16x3_shift(buf[c]));
}

// Maxima |x| of the rows of a (fused) panel / the columns of a block-row, merged
// into m_bits with atomicMax on the bit patterns (non-negative floats order like
// their bits): the common F16X3 scale of an operand staged in several pieces.
__global__ void __launch_bounds__(256) rowmax_k(const float* __restrict__ src, int64_t ld, int64_t seg_stride,
                                                int nseg, int64_t rows, int64_t K, unsigned* __restrict__ m_bits) {
    const int64_t row = (int64_t)blockIdx.x * 8 + threadIdx.x / 32;
    const int lane = threadIdx.x % 32;
    if (row >= rows) return;
    const float m = row_absmax(src, ld, seg_stride, nseg, row, K, lane);
    if (lane == 0) atomicMax(m_bits + row, __float_as_uint(m));
}

template <class T>
__global__ void __launch_bounds__(256) transpose_k(const T* __restrict__ src, int64_t ld, int64_t rows,
                                                   int64_t cols, T* __restrict__ dst) {
    __shared__ T tile[32][33];
    const int64_t r0 = (int64_t)blockIdx.y * 32, c0 = (int64_t)blockIdx.x * 32;
    for (int j = threadIdx.y; j < 32; j += 8) {
        const int64_t r = r0 + j, c = c0 + threadIdx.x;
        if (r < rows && c < cols) tile[j][threadIdx.x] = src[r * ld + c];
    }
    __syncthreads();
    for (int j = threadIdx.y; j < 32; j += 8) {
        const int64_t c = c0 + j, r = r0 + threadIdx.x;
        if (r < rows && c < cols) dst[c * rows + r] = tile[threadIdx.x][j];
    }
}

// ---- seeded generator: identical bits to synth/__init__.py
__device__ __forceinline__ uint64_t synth_hash(uint64_t seed, uint64_t idx) {
    uint64_t z = seed * 0xD1B54A32D192ED03ull + (idx + 1ull) * 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

template <class T>
__global__ void __launch_bounds__(256) fill_k(T* dst, int64_t ld, uint64_t seed, int64_t N, int64_t r0, int64_t c0,
                                              int64_t rows, int64_t cols, int dist) {
    const int64_t total = rows * cols;
    for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < total;
         idx += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = idx / cols, c = idx - r * cols;
        const uint64_t z = synth_hash(seed, (uint64_t)(r0 + r) * (uint64_t)N + (uint64_t)(c0 + c));
        double x;
        if (dist == FPM_DIST_PM1) x = (double)(z >> 40) * (1.0 / 8388608.0) - 1.0;
        else x = (double)((z >> 32) % 17ull) - 8.0;
        dst[r * ld + c] = (T)x;
    }
}

// ---- FP64 rank-b update on the FP64 tensor path (mma.sync m8n8k4 f64 ->
// SASS DMMA.8x8x4).  One persistent CTA per SM holds two independent groups of
// 8 warps; each group walks its own sequence of 64 x 128 C tiles (warp tiles
// 32 x 32: 4 x 4 DMMA tiles, 32 accumulators per lane) with its own 3-stage
// cp.async ring (K chunks of 16) and its own named barrier, so one group's
// epilogue (the C read-modify-write) overlaps the other's main loop -- what two
// co-resident CTAs would do, without letting the hardware spread them over
// more SMs than the device's cap.  Smem rows are padded to 20 doubles so the
// fragment loads (lane -> row lane/4, column lane%4) are conflict-free per
// half-warp.  Measured (ncu, L = 8192, K = 512): the previous 128 x 128
// single-group design kept the DMMA pipe 73 % busy.
// K per cp.async chunk: 32 (2 stages, one group barrier per 32 K) measured 31.2
// vs 30.4 TFLOP/s at L = 8192, K = 512 (config 1's fused K) and 20.7 vs 21.4 at
// K = 64; 16 (3 stages) kept selectable.
#ifndef FPM_F64_BK
#define FPM_F64_BK 32
#endif
#if FPM_F64_BK == 32
constexpr int F64_BM = 64, F64_BN = 128, F64_BK = 32, F64_LD = 36, F64_ST = 2, F64_GROUPS = 2;
#else
constexpr int F64_BM = 64, F64_BN = 128, F64_BK = 16, F64_LD = 20, F64_ST = 3, F64_GROUPS = 2;
#endif
// Warps per group and warp tile width: 8 warps of 32 x 32 (FPM_F64_WIDE 0, the
// default) or 4 warps of 32 x 64 (1: 32 independent DMMAs per k-step per warp;
// measured the same, 31.1 vs 31.2 TFLOP/s at L = 8192, K = 512).
#ifndef FPM_F64_WIDE
#define FPM_F64_WIDE 0
#endif
constexpr int F64_WTN = FPM_F64_WIDE ? 64 : 32, F64_GW = FPM_F64_WIDE ? 4 : 8;
constexpr int F64_GT = F64_GW * 32, F64_THREADS = F64_GROUPS * F64_GT, F64_NJ = F64_WTN / 8;
constexpr int F64_GROUP_DOUBLES = F64_ST * (F64_BM + F64_BN) * F64_LD;
constexpr int F64_SMEM = F64_GROUPS * F64_GROUP_DOUBLES * 8;  // 184320 B (BK 16) / 221184 B (BK 32)

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem, bool valid) {
    const uint32_t s = static_cast<uint32_t>(__cvta_generic_to_shared(smem));
    const int n = valid ? 16 : 0;  // src-size 0 -> zero fill
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(s), "l"(gmem), "r"(n) : "memory");
}

// named barrier 1 + grp with immediate operands (a register id would reserve
// all 16 barriers of the CTA and keep other kernels off the SM)
__device__ __forceinline__ void group_bar(int grp) {
    if (grp == 0)
        asm volatile("bar.sync 1, %0;" ::"n"(F64_GT) : "memory");
    else
        asm volatile("bar.sync 2, %0;" ::"n"(F64_GT) : "memory");
}

// A may be segmented along K (fused pivots, each pivot's H x b panel stored on
// its own): element (r, k) at A + (k / seg) * seg_stride + r * lda + k % seg.
// seg is even, so the two consecutive k of a 16-byte copy share a segment.
__global__ void __launch_bounds__(F64_THREADS, 1) update_f64_k(const double* __restrict__ A, int64_t lda, int64_t seg,
                                                       int64_t seg_stride, const double* __restrict__ Bt,
                                                       double* __restrict__ C, int64_t M, int64_t Nc, int64_t K,
                                                       int64_t ldc, int accumulate) {
    extern __shared__ double sm64[];
    const int grp = threadIdx.x / F64_GT, gtid = threadIdx.x % F64_GT;
    double* As = sm64 + grp * F64_GROUP_DOUBLES;       // [ST][BM][LD]
    double* Bs = As + F64_ST * F64_BM * F64_LD;        // [ST][BN][LD]
    const int warp = gtid / 32, lane = threadIdx.x % 32;
    constexpr int WARPS_N = F64_BN / F64_WTN;
    const int wm = (warp / WARPS_N) * 32, wn = (warp % WARPS_N) * F64_WTN;
    const int64_t tiles_n = (Nc + F64_BN - 1) / F64_BN;
    const int64_t tiles = ((M + F64_BM - 1) / F64_BM) * tiles_n;
    const int64_t nk = (K + F64_BK - 1) / F64_BK;
    // persistent over tiles (the grid is capped at the device's SM cap); the
    // two groups of a CTA take alternate tiles
    const int64_t first = 2 * (int64_t)blockIdx.x + grp, stride = 2 * (int64_t)gridDim.x;

    // load cursor: (tile lt, chunk lkb) runs ST-1 chunks ahead of the compute
    int64_t lt = first, lkb = 0;
    int slot_l = 0;
    auto advance_load = [&]() {
        if (lt < tiles) {
            const int64_t m0 = (lt / tiles_n) * F64_BM, n0 = (lt % tiles_n) * F64_BN, k0 = lkb * F64_BK;
            // A: 64 rows x BK doubles (BK / 2 16-B chunks per row); B: 128 rows
            constexpr int CPR = F64_BK / 2, A_IT = F64_BM * CPR / F64_GT, B_IT = F64_BN * CPR / F64_GT;
#pragma unroll
            for (int it = 0; it < A_IT + B_IT; ++it) {
                const int idx = gtid + it * F64_GT;
                const bool isA = it < A_IT;
                const int j = isA ? idx : idx - A_IT * F64_GT;
                const int r = j / CPR, c2 = (j % CPR) * 2;
                const int64_t gk = k0 + c2;
                const bool ka = gk < K;  // K even: a 2-element chunk is all in or all out
                if (isA) {
                    const int64_t gm = m0 + r;
                    const int64_t off = (gk / seg) * seg_stride + gm * lda + gk % seg;
                    cp_async16(As + (slot_l * F64_BM + r) * F64_LD + c2, A + (ka && gm < M ? off : 0), ka && gm < M);
                } else {
                    const int64_t gn = n0 + r;
                    cp_async16(Bs + (slot_l * F64_BN + r) * F64_LD + c2, Bt + (ka && gn < Nc ? gn * K + gk : 0),
                               ka && gn < Nc);
                }
            }
            if (++lkb == nk) {
                lkb = 0;
                lt += stride;
            }
        }
        asm volatile("cp.async.commit_group;" ::: "memory");  // (empty past the last tile)
        slot_l = slot_l + 1 == F64_ST ? 0 : slot_l + 1;
    };
#pragma unroll
    for (int s = 0; s < F64_ST - 1; ++s) advance_load();

    int slot_c = 0;
    for (int64_t t = first; t < tiles; t += stride) {
        const int64_t m0 = (t / tiles_n) * F64_BM, n0 = (t % tiles_n) * F64_BN;
        double acc[4][F64_NJ][2];
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int j = 0; j < F64_NJ; ++j) acc[i][j][0] = acc[i][j][1] = 0.0;

        for (int64_t kb = 0; kb < nk; ++kb) {
            asm volatile("cp.async.wait_group %0;" ::"n"(F64_ST - 2) : "memory");
            group_bar(grp);  // chunk visible to the group; the slot refilled next is free
            advance_load();
            const double* as = As + slot_c * F64_BM * F64_LD;
            const double* bs = Bs + slot_c * F64_BN * F64_LD;
#pragma unroll
            for (int kk = 0; kk < F64_BK; kk += 4) {
                double a[4], b[F64_NJ];
#pragma unroll
                for (int i = 0; i < 4; ++i) a[i] = as[(wm + i * 8 + lane / 4) * F64_LD + kk + lane % 4];
#pragma unroll
                for (int j = 0; j < F64_NJ; ++j) b[j] = bs[(wn + j * 8 + lane / 4) * F64_LD + kk + lane % 4];
#pragma unroll
                for (int i = 0; i < 4; ++i)
#pragma unroll
                    for (int j = 0; j < F64_NJ; ++j)
                        asm volatile(
                            "mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0, %1}, {%2}, {%3}, {%0, %1};"
                            : "+d"(acc[i][j][0]), "+d"(acc[i][j][1])
                            : "d"(a[i]), "d"(b[j]));
            }
            slot_c = slot_c + 1 == F64_ST ? 0 : slot_c + 1;
        }
        // epilogue: this group's next chunks are already in flight, the other
        // group keeps the DMMA pipe busy.  Interior tiles: the four C loads of
        // a DMMA row are issued together (one global round trip per row, not
        // one per element); edge tiles take the guarded path.
        const bool interior = m0 + F64_BM <= M && n0 + F64_BN <= Nc && (ldc & 1) == 0 &&
                              (reinterpret_cast<uintptr_t>(C) & 15) == 0;
        if (interior) {
#pragma unroll
            for (int i = 0; i < 4; ++i) {
                double2* rowp = reinterpret_cast<double2*>(C + (m0 + wm + i * 8 + lane / 4) * ldc + n0 + wn +
                                                           2 * (lane % 4));
                double2 c[F64_NJ];
#pragma unroll
                for (int j = 0; j < F64_NJ; ++j) c[j] = accumulate ? __ldcs(rowp + 4 * j) : make_double2(0.0, 0.0);
#pragma unroll
                for (int j = 0; j < F64_NJ; ++j) {
                    c[j].x += acc[i][j][0];
                    c[j].y += acc[i][j][1];
                    __stcs(rowp + 4 * j, c[j]);
                }
            }
            continue;
        }
#pragma unroll
        for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int j = 0; j < F64_NJ; ++j) {
                const int64_t gm = m0 + wm + i * 8 + lane / 4;
                const int64_t gn = n0 + wn + j * 8 + 2 * (lane % 4);
                if (gm >= M) continue;
                double* cp = C + gm * ldc + gn;
                if (gn + 1 < Nc && (reinterpret_cast<uintptr_t>(cp) & 15) == 0) {
                    double2 c = accumulate ? *reinterpret_cast<double2*>(cp) : make_double2(0.0, 0.0);
                    c.x += acc[i][j][0];
                    c.y += acc[i][j][1];
                    *reinterpret_cast<double2*>(cp) = c;
                } else {
#pragma unroll
                    for (int h = 0; h < 2; ++h)
                        if (gn + h < Nc) cp[h] = (accumulate ? cp[h] : 0.0) + acc[i][j][h];
                }
            }
    }  // tile loop
    asm volatile("cp.async.wait_group 0;" ::: "memory");
}

int grid_for(int64_t work, int threads) {
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    int64_t blocks = (work + threads - 1) / threads;
    const int64_t cap = (int64_t)sms * 8;  // 8 resident 256-thread CTAs per SM
    if (blocks > cap) blocks = cap;
    return (int)(blocks < 1 ? 1 : blocks);
}

void check_launch(const char* what) {
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) fail(FPM_ECUDA, "%s launch: %s", what, cudaGetErrorString(e));
}

}  // namespace

void launch_split_rows_seg(const float* src, int64_t ld, int64_t seg_stride, int nseg, int64_t rows, int64_t K,
                           int64_t ld_out, SplitScheme s, void* hi, void* lo, float* inv_scale, cudaStream_t st,
                           const unsigned* given_max) {
    if (rows <= 0 || K <= 0 || nseg <= 0) return;
    FPM_CHECK_ARG(K % 4 == 0 && ld % 4 == 0 && seg_stride % 4 == 0 && ld_out % 4 == 0 && ld_out >= nseg * K,
                  "split: K, ld, seg_stride, ld_out must be multiples of 4 and ld_out >= nseg*K");
    if (s == SplitScheme::F16X3 || s == SplitScheme::F16I8) {
        const int64_t blocks = (rows + 7) / 8;
        if (s == SplitScheme::F16I8) {
            FPM_CHECK_ARG(K % 64 == 0 && ld_out % 64 == 0, "F16I8 split: K and ld_out multiples of 64");
            split_rows_f16<true><<<(unsigned)blocks, 256, 0, st>>>(src, ld, seg_stride, nseg, rows, K, ld_out,
                                                                   static_cast<__half*>(hi), static_cast<__half*>(lo),
                                                                   inv_scale, given_max);
        } else {
            split_rows_f16<false><<<(unsigned)blocks, 256, 0, st>>>(src, ld, seg_stride, nseg, rows, K, ld_out,
                                                                    static_cast<__half*>(hi),
                                                                    static_cast<__half*>(lo), inv_scale, given_max);
        }
        check_launch("split_rows_f16");
    } else {
        split_rows_tf32<<<grid_for(rows * nseg * K / 4, 256), 256, 0, st>>>(
            src, ld, seg_stride, nseg, rows, K, ld_out, static_cast<float*>(hi), static_cast<float*>(lo));
        check_launch("split_rows_tf32");
    }
}

void launch_split_rows(const float* src, int64_t ld, int64_t rows, int64_t K, SplitScheme s, void* hi, void* lo,
                       float* inv_scale, cudaStream_t st) {
    launch_split_rows_seg(src, ld, 0, 1, rows, K, K, s, hi, lo, inv_scale, st);
}

void launch_split_cols(const float* src, int64_t ld, int64_t K, int64_t W, SplitScheme s, void* hi, void* lo,
                       float* inv_scale, cudaStream_t st, int64_t ld_out, const unsigned* given_max) {
    if (K <= 0 || W <= 0) return;
    if (ld_out < 0) ld_out = K;
    FPM_CHECK_ARG(K % 8 == 0 && ld_out % 8 == 0 && ld_out >= K, "split_cols: K, ld_out multiples of 8, ld_out >= K");
    FPM_CHECK_ARG(W % 4 == 0 && ld % 4 == 0 && (reinterpret_cast<uintptr_t>(src) & 15) == 0,
                  "split_cols: W and ld multiples of 4, src 16-byte aligned");
    const dim3 grid((unsigned)((W + kColsPerCta - 1) / kColsPerCta), (unsigned)((K + kColTileK - 1) / kColTileK));
    if (s == SplitScheme::F16X3 || s == SplitScheme::F16I8) {
        FPM_CHECK_ARG(inv_scale != nullptr, "F16X3 / F16I8 need inv_scale");
        const bool i8 = s == SplitScheme::F16I8;
        if (i8) FPM_CHECK_ARG(K % 64 == 0 && ld_out % 64 == 0, "F16I8 split: K and ld_out multiples of 64");
        auto kern = i8 ? split_cols_t<true, true> : split_cols_t<true, false>;
        if (given_max) {
            kern<<<grid, kColThreads, 0, st>>>(src, ld, K, W, ld_out, hi, lo, given_max, inv_scale);
        } else {  // maxima into inv_scale (as bits), split, then bits -> inverse scales in place
            unsigned* bits = reinterpret_cast<unsigned*>(inv_scale);
            const cudaError_t e = cudaMemsetAsync(bits, 0, (size_t)W * sizeof(unsigned), st);
            if (e != cudaSuccess) fail(FPM_ECUDA, "split_cols memset: %s", cudaGetErrorString(e));
            launch_colmax(src, ld, K, W, bits, st);
            kern<<<grid, kColThreads, 0, st>>>(src, ld, K, W, ld_out, hi, lo, bits, nullptr);
            check_launch("split_cols");
            scale_from_max_k<<<(unsigned)((W + 255) / 256), 256, 0, st>>>(inv_scale, W);
        }
    } else {
        split_cols_t<false><<<grid, kColThreads, 0, st>>>(src, ld, K, W, ld_out, hi, lo, nullptr, nullptr);
    }
    check_launch("split_cols");
}

void launch_rowmax_seg(const float* src, int64_t ld, int64_t seg_stride, int nseg, int64_t rows, int64_t K,
                       unsigned* m_bits, cudaStream_t st) {
    if (rows <= 0 || K <= 0 || nseg <= 0) return;
    FPM_CHECK_ARG(K % 4 == 0 && ld % 4 == 0 && seg_stride % 4 == 0, "rowmax: K, ld, seg_stride multiples of 4");
    rowmax_k<<<(unsigned)((rows + 7) / 8), 256, 0, st>>>(src, ld, seg_stride, nseg, rows, K, m_bits);
    check_launch("rowmax");
}

void launch_colmax(const float* src, int64_t ld, int64_t K, int64_t W, unsigned* m_bits, cudaStream_t st) {
    if (K <= 0 || W <= 0) return;
    FPM_CHECK_ARG(K % 8 == 0 && W % 4 == 0 && ld % 4 == 0 && (reinterpret_cast<uintptr_t>(src) & 15) == 0,
                  "colmax: K multiple of 8, W and ld multiples of 4, src 16-byte aligned");
    const dim3 grid((unsigned)((W + kColsPerCta - 1) / kColsPerCta), (unsigned)((K + kColMaxRows - 1) / kColMaxRows));
    colmax_tile_k<<<grid, 256, 0, st>>>(src, ld, K, W, m_bits);
    check_launch("colmax");
}

void launch_transpose_f32(const float* src, int64_t ld, int64_t rows, int64_t cols, float* dst, cudaStream_t st) {
    if (rows <= 0 || cols <= 0) return;
    dim3 grid((unsigned)((cols + 31) / 32), (unsigned)((rows + 31) / 32));
    transpose_k<float><<<grid, dim3(32, 8), 0, st>>>(src, ld, rows, cols, dst);
    check_launch("transpose_f32");
}

void launch_transpose_f64(const double* src, int64_t ld, int64_t rows, int64_t cols, double* dst,
                          cudaStream_t st) {
    if (rows <= 0 || cols <= 0) return;
    dim3 grid((unsigned)((cols + 31) / 32), (unsigned)((rows + 31) / 32));
    transpose_k<double><<<grid, dim3(32, 8), 0, st>>>(src, ld, rows, cols, dst);
    check_launch("transpose_f64");
}

void launch_update_f64(const double* A, int64_t lda, const double* Bt, double* C, int64_t M, int64_t Nc,
                       int64_t K, int64_t ldc, bool accumulate, int num_sms, cudaStream_t st, int64_t seg,
                       int64_t seg_stride) {
    if (M <= 0 || Nc <= 0 || K <= 0) return;
    if (seg <= 0) {  // one contiguous row of K per A row
        seg = K;
        seg_stride = 0;
    }
    FPM_CHECK_ARG(K % 8 == 0 && lda % 2 == 0 && seg % 2 == 0 && seg_stride % 2 == 0 && (seg >= K || lda >= seg),
                  "FP64 update: K % 8 == 0, even lda / seg / seg_stride, lda >= seg for segmented A");
    FPM_CHECK_ARG((reinterpret_cast<uintptr_t>(A) & 15) == 0 && (reinterpret_cast<uintptr_t>(Bt) & 15) == 0,
                  "FP64 update: A and Bt must be 16-byte aligned");
    static uint64_t attr_done = 0;  // one bit per CUDA device
    int dev = 0;
    cudaGetDevice(&dev);
    if (!(attr_done & (1ull << dev))) {
        cudaError_t e = cudaFuncSetAttribute(update_f64_k, cudaFuncAttributeMaxDynamicSharedMemorySize, F64_SMEM);
        if (e != cudaSuccess) fail(FPM_ECUDA, "cudaFuncSetAttribute(update_f64): %s", cudaGetErrorString(e));
        attr_done |= 1ull << dev;
    }
    const int64_t tiles = ((Nc + F64_BN - 1) / F64_BN) * ((M + F64_BM - 1) / F64_BM);
    int sms = num_sms;
    if (sms <= 0) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    const unsigned grid = (unsigned)std::min<int64_t>((tiles + 1) / 2, std::max(1, sms));  // 1 CTA (2 tile groups) per SM
    update_f64_k<<<grid, F64_THREADS, F64_SMEM, st>>>(A, lda, seg, seg_stride, Bt, C, M, Nc, K, ldc, accumulate ? 1 : 0);
    check_launch("update_f64");
}

void launch_fill_synthetic(void* dst, bool f64, int64_t ld, uint64_t seed, int64_t N, int64_t r0, int64_t c0,
                           int64_t rows, int64_t cols, int dist, cudaStream_t st) {
    if (rows <= 0 || cols <= 0) return;
    FPM_CHECK_ARG(dist == FPM_DIST_PM1 || dist == FPM_DIST_INT, "unknown dist %d", dist);
    const int g = grid_for(rows * cols, 256);
    if (f64) fill_k<double><<<g, 256, 0, st>>>(static_cast<double*>(dst), ld, seed, N, r0, c0, rows, cols, dist);
    else fill_k<float><<<g, 256, 0, st>>>(static_cast<float*>(dst), ld, seed, N, r0, c0, rows, cols, dist);
    check_launch("fill_synthetic");
}

void launch_zero(void* dst, size_t bytes, cudaStream_t st) {
    cudaError_t e = cudaMemsetAsync(dst, 0, bytes, st);
    if (e != cudaSuccess) fail(FPM_ECUDA, "cudaMemsetAsync: %s", cudaGetErrorString(e));
}

}  // namespace fpm
