// pack.cuh — operand packing for the tensor-core path.
//
// The boundary takes Caffe NCHW fp32 blobs (P87, network-agnostic contract P262).  TMA needs
// 16-byte-aligned strides and the implicit GEMM wants channels innermost, so activations are
// transposed once to NHWC with the channel pitch padded to a 16-byte multiple, applying the math
// mode's operand rounding (TF32: cvt.rna; BF16: round-to-nearest-even).  The dy pack also emits
// the per-(sample, pixel-tile, channel) partial sums of the bias gradient, each reduced by a
// fixed shuffle tree so db is deterministic.
#pragma once
#include <cuda_bf16.h>

#include "ptx.cuh"

namespace glp {

template <int ELEM>
struct PackOut;
template <>
struct PackOut<2> {
  __device__ __forceinline__ static void store4(void *dst, size_t idx, float a, float b, float c,
                                                float d) {
    __nv_bfloat162 lo = __floats2bfloat162_rn(a, b), hi = __floats2bfloat162_rn(c, d);
    uint2 u;
    u.x = *reinterpret_cast<uint32_t *>(&lo);
    u.y = *reinterpret_cast<uint32_t *>(&hi);
    *reinterpret_cast<uint2 *>(static_cast<__nv_bfloat16 *>(dst) + idx) = u;
  }
  __device__ __forceinline__ static void store1(void *dst, size_t idx, float a) {
    static_cast<__nv_bfloat16 *>(dst)[idx] = __float2bfloat16_rn(a);
  }
};
template <>
struct PackOut<4> {
  __device__ __forceinline__ static void store4(void *dst, size_t idx, float a, float b, float c,
                                                float d) {
    uint4 u = make_uint4(f32_to_tf32_rna(a), f32_to_tf32_rna(b), f32_to_tf32_rna(c),
                         f32_to_tf32_rna(d));
    *reinterpret_cast<uint4 *>(static_cast<float *>(dst) + idx) = u;
  }
  __device__ __forceinline__ static void store1(void *dst, size_t idx, float a) {
    static_cast<uint32_t *>(dst)[idx] = f32_to_tf32_rna(a);
  }
};

// NCHW fp32 [N][C][HW] -> NHWC [N][HW][Cp] (rounded), zero for c >= C.  Tile 32 ch x 32 px.
// grid (ceil(HW/32), ceil(Cp/32), N), block 256.  db_part (optional): [N][ceil(HW/32)][C].
template <int ELEM>
__global__ void __launch_bounds__(256) pack_nchw_to_nhwc(const float *__restrict__ src,
                                                         void *__restrict__ dst, int C, int HW,
                                                         int Cp, float *__restrict__ db_part) {
  __shared__ float tile[32][33];
  const int n = blockIdx.z, c0 = blockIdx.y * 32, p0 = blockIdx.x * 32;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const float *s = src + (size_t)n * C * HW;
#pragma unroll
  for (int cc = warp; cc < 32; cc += 8) {
    const int c = c0 + cc, px = p0 + lane;
    float v = 0.f;
    if (c < C && px < HW) v = __ldg(s + (size_t)c * HW + px);
    tile[cc][lane] = v;
    if (db_part != nullptr && c < C) {
      float t = v;
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
      if (lane == 0) db_part[((size_t)n * gridDim.x + blockIdx.x) * C + c] = t;
    }
  }
  __syncthreads();
  const int pp = threadIdx.x >> 3, cq = threadIdx.x & 7;
  const int px = p0 + pp, c = c0 + 4 * cq;
  if (px < HW && c < Cp) {
    const size_t o = ((size_t)n * HW + px) * Cp + c;
    PackOut<ELEM>::store4(dst, o, tile[4 * cq][pp], tile[4 * cq + 1][pp], tile[4 * cq + 2][pp],
                          tile[4 * cq + 3][pp]);
  }
}

// W [Co][C][Kh][Kw] -> forward B operand Wp[co][tap*Cp + c] with row length Kpad (zero padded).
template <int ELEM>
__global__ void pack_w_fwd(const float *__restrict__ w, void *__restrict__ out, int Co, int C,
                           int taps, int Cp, int Kpad) {
  const size_t total = (size_t)Co * Kpad;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < total;
       i += (size_t)gridDim.x * blockDim.x) {
    const int co = (int)(i / Kpad), k = (int)(i % Kpad);
    const int t = k / Cp, c = k % Cp;
    float v = 0.f;
    if (t < taps && c < C) v = __ldg(w + ((size_t)co * C + c) * taps + t);
    PackOut<ELEM>::store1(out, i, v);
  }
}

// W [Co][C][Kh][Kw] -> backward-data B operand Wt[ci][tap*Cop + co] (row length Kpad).
template <int ELEM>
__global__ void pack_w_dgrad(const float *__restrict__ w, void *__restrict__ out, int Co, int C,
                             int taps, int Cop, int Kpad) {
  const size_t total = (size_t)C * Kpad;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < total;
       i += (size_t)gridDim.x * blockDim.x) {
    const int ci = (int)(i / Kpad), k = (int)(i % Kpad);
    const int t = k / Cop, co = k % Cop;
    float v = 0.f;
    if (t < taps && co < Co) v = __ldg(w + ((size_t)co * C + ci) * taps + t);
    PackOut<ELEM>::store1(out, i, v);
  }
}

}  // namespace glp
