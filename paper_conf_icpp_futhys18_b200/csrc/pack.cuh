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

// NCHW fp32 [N][C][HW] -> NHWC [N][HW][Cp] (rounded), zero for c >= C.
// Tile 32 channels x PACK_PT pixels per 256-thread block: 16 independent coalesced loads per
// thread, conflict-free transposed smem reads, 16-byte stores.
// grid (ceil(HW/PACK_PT), ceil(Cp/32), N).  db_part (optional): [N][ceil(HW/PACK_PT)][C], each
// entry the sum of one channel over one pixel tile in a fixed order (lane-sequential over the 4
// pixel quarters, then a xor-shuffle tree).
constexpr int PACK_PT = 128;

// Padded destination (Wd != Ws): the pixels are written on a wider Hd x Wd grid (row q = h*Wd + w,
// HWd = Hd*Wd rows per image), zeros at the positions outside the Hs x Ws source image — the
// dy operand of the halo filter gradient (hwgrad.cuh).  Blocks then run over destination rows.
template <int ELEM>
__global__ void __launch_bounds__(256) pack_nchw_to_nhwc(const float *__restrict__ src,
                                                         void *__restrict__ dst, int C, int HW,
                                                         int Cp, float *__restrict__ db_part,
                                                         unsigned int *__restrict__ tickets,
                                                         int n_tickets, int Ws, int Wd, int HWd) {
  __shared__ float tile[32][PACK_PT + 1];
  pdl_launch_dependents();
  pdl_wait();
  const int n = blockIdx.z, c0 = blockIdx.y * 32, p0 = blockIdx.x * PACK_PT;
  const bool padded = Wd != Ws;
  const int Hs = padded ? HW / Ws : 0;
  // arm the completion tickets of the deterministic db reduction that consumes db_part
  if (tickets != nullptr && (blockIdx.x | blockIdx.y | blockIdx.z) == 0)
    for (int i = threadIdx.x; i < n_tickets; i += blockDim.x) tickets[i] = 0u;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const float *s = src + (size_t)n * C * HW;
  // source pixel of each of this lane's 4 destination rows (one division per thread; the rows
  // are 32 apart, so the padded column advances by 32 with at most one wrap when Wd > 32)
  int spx[4];
  bool sok[4];
  {
    const int q0 = p0 + lane;
    int h = padded ? q0 / Wd : 0, w = padded ? q0 - h * Wd : 0;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      if (padded) {
        sok[q] = h < Hs && w < Ws;
        spx[q] = h * Ws + w;
        w += 32;
        while (w >= Wd) {
          w -= Wd;
          ++h;
        }
      } else {
        spx[q] = q0 + q * 32;
        sok[q] = spx[q] < HW;
      }
    }
  }
  float v[4][4];
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const int c = c0 + warp + 8 * k;
#pragma unroll
    for (int q = 0; q < 4; ++q)
      v[k][q] = (c < C && sok[q]) ? __ldg(s + (size_t)c * HW + spx[q]) : 0.f;
  }
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const int cc = warp + 8 * k;
#pragma unroll
    for (int q = 0; q < 4; ++q) tile[cc][q * 32 + lane] = v[k][q];
    if (db_part != nullptr && c0 + cc < C) {
      float t = ((v[k][0] + v[k][1]) + (v[k][2] + v[k][3]));
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) t += __shfl_xor_sync(0xffffffffu, t, o);
      if (lane == 0) db_part[((size_t)n * gridDim.x + blockIdx.x) * C + c0 + cc] = t;
    }
  }
  __syncthreads();
  // 16-byte chunks: lanes cover consecutive chunks of a pixel's 32-channel row (64 B bf16 /
  // 128 B fp32), so each warp store instruction writes whole contiguous row segments.
  constexpr int CPT = 16 / ELEM;            // channels per 16-byte chunk
  constexpr int CPP = 32 / CPT;             // chunks per pixel row of the tile
  constexpr int PPP = 256 / CPP;            // pixels per pass
#pragma unroll
  for (int pass = 0; pass < PACK_PT / PPP; ++pass) {
    const int pp = pass * PPP + threadIdx.x / CPP, j = threadIdx.x % CPP;
    const int px = p0 + pp, cl = j * CPT, c = c0 + cl;
    if (px < HWd && c < Cp) {
      const size_t o = ((size_t)n * HWd + px) * Cp + c;
#pragma unroll
      for (int u = 0; u < CPT; u += 4)
        PackOut<ELEM>::store4(dst, o + u, tile[cl + u][pp], tile[cl + u + 1][pp],
                              tile[cl + u + 2][pp], tile[cl + u + 3][pp]);
    }
  }
}

// Small channel counts (Cp <= 16): one thread per pixel, loads coalesced across pixels.
template <int ELEM>
__global__ void __launch_bounds__(256) pack_nchw_to_nhwc_small(const float *__restrict__ src,
                                                               void *__restrict__ dst, int N, int C,
                                                               int HW, int Cp) {
  pdl_launch_dependents();
  pdl_wait();
  const size_t total = (size_t)N * HW;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < total;
       i += (size_t)gridDim.x * blockDim.x) {
    const size_t n = i / HW, px = i % HW;
    const float *s = src + n * C * HW + px;
    for (int c = 0; c < Cp; c += 4) {
      float a[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) a[u] = (c + u < C) ? __ldg(s + (size_t)(c + u) * HW) : 0.f;
      PackOut<ELEM>::store4(dst, i * Cp + c, a[0], a[1], a[2], a[3]);
    }
  }
}

// Space-to-depth pack for strided convolutions with few input channels:
//   x'[n][h'][w'][c'] = x[n][c][S*h' + dh - P][S*w' + dw - P]  (0 outside),  c' = (dh*S + dw)*C + c
// turns a stride-S, K x K conv into a stride-1, ceil(K/S) x ceil(K/S) conv over S*S*C channels
// with the same output, so the implicit GEMM runs unit-stride im2col TMA on a dense channel axis.
// One block per (n, h'): the S source rows are staged in shared memory (coalesced reads), then the
// output row is written with 16-byte stores.  Dynamic smem = S*C*W floats.
template <int ELEM>
__global__ void __launch_bounds__(256) pack_s2d(const float *__restrict__ x, void *__restrict__ dst,
                                                int C, int H, int W, int S, int P, int Hs, int Ws,
                                                int Cps) {
  extern __shared__ float rows[];   // [S*C][W] source rows (row r = dh*C + c)
  pdl_launch_dependents();
  pdl_wait();
  const int hs = blockIdx.x, n = blockIdx.y;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, nwarps = blockDim.x >> 5;
  // one warp per source row, 8 independent coalesced loads in flight per lane (no per-element
  // index division: the row is fixed per warp iteration)
  // (a trailing partial warp, blockDim % 32 != 0, takes no rows)
  for (int r = warp; warp < nwarps && r < S * C; r += nwarps) {
    const int dh = r / C, c = r - dh * C;
    const int ih = S * hs + dh - P;
    const bool rin = ih >= 0 && ih < H;
    const float *src = x + (((size_t)n * C + c) * H + (rin ? ih : 0)) * W;
    float *d = rows + r * W;
    for (int w0 = 0; w0 < W; w0 += 256) {
      float v[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const int w = w0 + lane + 32 * k;
        v[k] = (rin && w < W) ? __ldg(src + w) : 0.f;
      }
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        const int w = w0 + lane + 32 * k;
        if (w < W) d[w] = v[k];
      }
    }
  }
  // output: thread -> fixed channel quad q (blockDim is a multiple of Cps/4), pixels strided
  const int quads = Cps >> 2;
  const int q = threadIdx.x % quads, wstep = blockDim.x / quads;
  int roff[4], dws[4];
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    const int cc = 4 * q + u;
    roff[u] = -1;
    dws[u] = 0;
    if (cc < S * S * C) {
      const int c = cc % C, dd = cc / C, dh = dd / S, dw = dd - dh * S;
      roff[u] = (dh * C + c) * W;
      dws[u] = dw - P;
    }
  }
  __syncthreads();
  const size_t obase = ((size_t)n * Hs + hs) * Ws;
  for (int ws = threadIdx.x / quads; ws < Ws; ws += wstep) {
    float v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const int iw = S * ws + dws[u];
      v[u] = (roff[u] >= 0 && iw >= 0 && iw < W) ? rows[roff[u] + iw] : 0.f;
    }
    PackOut<ELEM>::store4(dst, (obase + ws) * Cps + 4 * q, v[0], v[1], v[2], v[3]);
  }
}

// Forward B operand in the space-to-depth geometry: Wp[co][t'*Cps + c'], t' = kh'*Ks + kw',
// c' = (dh*S + dw)*C + c, value W[co][c][S*kh'+dh][S*kw'+dw] (0 past the K x K window).
template <int ELEM>
__global__ void pack_w_fwd_s2d(const float *__restrict__ w, void *__restrict__ out, int Co, int C,
                               int K, int S, int Ks, int Cps, int Kpad) {
  pdl_launch_dependents();
  pdl_wait();
  const size_t total = (size_t)Co * Kpad;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < total;
       i += (size_t)gridDim.x * blockDim.x) {
    const int co = (int)(i / Kpad), k = (int)(i % Kpad);
    const int t = k / Cps, cc = k % Cps;
    float v = 0.f;
    if (t < Ks * Ks && cc < S * S * C) {
      const int khs = t / Ks, kws = t % Ks, c = cc % C, dd = cc / C, dh = dd / S, dw = dd % S;
      const int kh = S * khs + dh, kw = S * kws + dw;
      if (kh < K && kw < K) v = __ldg(w + (((size_t)co * C + c) * K + kh) * K + kw);
    }
    PackOut<ELEM>::store1(out, i, v);
  }
}

// W [Co][C][Kh][Kw] -> forward B operand Wp[co][tap*Cp + c] with row length Kpad (zero padded).
// grid (ceil(Kpad/256), Co): one element per thread, 32-bit index math (the old grid-stride form
// spent most of its time in 64-bit divisions).
template <int ELEM>
__global__ void __launch_bounds__(256) pack_w_fwd(const float *__restrict__ w, void *__restrict__ out,
                                                  int Co, int C, int taps, int Cp, int Kpad) {
  pdl_launch_dependents();
  pdl_wait();
  const int co = blockIdx.y, k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= Kpad) return;
  const int t = k / Cp, c = k - t * Cp;
  const float v = (t < taps && c < C) ? __ldg(w + ((size_t)co * C + c) * taps + t) : 0.f;
  PackOut<ELEM>::store1(out, (size_t)co * Kpad + k, v);
}

// W [Co][C][Kh][Kw] -> backward-data B operand Wt[ci][tap*Cop + co] (row length Kpad).
// flip = 1: tap index reversed (tap' = taps-1-tap, i.e. (Kh-1-kh, Kw-1-kw)) for the im2col-TMA
// dgrad, which walks dy from the window's top-left corner.
template <int ELEM>
__global__ void __launch_bounds__(256) pack_w_dgrad(const float *__restrict__ w, void *__restrict__ out,
                                                    int Co, int C, int taps, int Cop, int Kpad,
                                                    int flip) {
  pdl_launch_dependents();
  pdl_wait();
  const int ci = blockIdx.y, k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= Kpad) return;
  const int t = k / Cop, co = k - t * Cop;
  const float v = (t < taps && co < Co)
                      ? __ldg(w + ((size_t)co * C + ci) * taps + (flip ? taps - 1 - t : t))
                      : 0.f;
  PackOut<ELEM>::store1(out, (size_t)ci * Kpad + k, v);
}

}  // namespace glp
