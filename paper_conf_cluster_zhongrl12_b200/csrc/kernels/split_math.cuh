// F16X3 operand-split arithmetic (reading Q15), shared by the
// standalone staging kernels (stage.cu) and the staging warp of the update
// kernel (update_f32.cu) so both produce the same bits by construction.
#pragma once

#include <cuda_fp16.h>

#include <cstdint>

namespace fpm {

__device__ __forceinline__ float warp_max(float v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v = fmaxf(v, __shfl_xor_sync(0xffffffffu, v, o));
    return v;
}

// Power-of-two F16X3 scale 2^s that puts the maximum m in [2^14, 2^15).
__device__ __forceinline__ int f16x3_shift(float m) {
    int e = 0;
    if (m > 0.0f) frexpf(m, &e);  // m < 2^e
    int s = (m > 0.0f) ? 15 - e : 0;
    return s < -126 ? -126 : (s > 127 ? 127 : s);
}

// x 2^s = h + l: h = fp16_rn(x 2^s), l = fp16_rn(x 2^s - h)  (scale = 2^s)
__device__ __forceinline__ void f16x3_split(float x, float scale, __half& h, __half& l) {
    const float xs = x * scale;
    h = __float2half_rn(xs);
    l = __float2half_rn(xs - __half2float(h));
}

}  // namespace fpm
