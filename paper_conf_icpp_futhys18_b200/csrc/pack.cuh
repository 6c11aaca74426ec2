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

// 3xTF32 (GLP_MATH_FP32): the packs of a tf32 operand also write its lo plane, `lo` bytes past
// the hi plane (lo = 0: single plane).  Plane 0 = hi = rna(v); plane 1 = lo = rna(v - hi), the
// fp32 subtraction being exact (SURVEY §8(c) "3xTF32 hi/lo split"; oracle.split_3xtf32).
__device__ __forceinline__ uint32_t tf32_plane(float v, int pl) {
  const uint32_t hi = f32_to_tf32_rna(v);
  return pl ? f32_to_tf32_rna(v - __uint_as_float(hi)) : hi;
}

// The mixed fp32 split (plan option fp32_split = 1; DESIGN.md §7 "mixed split"): three planes,
// plane 0 = hi = rna_tf32(v) (4-byte elements), plane 1 = rne_bf16(hi), plane 2 = rne_bf16(v - hi)
// (2-byte elements; v - hi is exact in fp32).  The packs receive the planes in one argument:
// lo > 0: 3xTF32 (plane 1 = tf32 lo at +lo bytes, same element size); lo < 0: mixed, M = -lo
// holds two byte offsets from the destination pointer's element 0 -- plane 1 at M & 0xFFFFFFFF,
// plane 2 a further M >> 32 (the bf16 plane size) -- so a destination pointer already advanced
// into the hi plane (a fused-group branch's rows) still finds its bf16 elements; lo = 0: one
// plane.
__device__ __forceinline__ int plane_count(long long lo) { return lo == 0 ? 1 : (lo > 0 ? 2 : 3); }
__device__ __forceinline__ int plane_esize(long long lo, int pl) { return (lo < 0 && pl) ? 2 : 4; }
__device__ __forceinline__ long long plane_off(long long lo, int pl) {
  if (pl == 0) return 0;
  if (lo > 0) return lo;
  const unsigned long long m = (unsigned long long)(-lo);
  const long long p1 = (long long)(m & 0xFFFFFFFFull);
  return pl == 1 ? p1 : p1 + (long long)(m >> 32);
}
// bf16 bits of plane pl (1 or 2) of the mixed split
__device__ __forceinline__ uint32_t mix_bf16_bits(float v, int pl) {
  const float hi = __uint_as_float(f32_to_tf32_rna(v));
  const float t = pl == 1 ? hi : v - hi;
  __nv_bfloat16 b = __float2bfloat16_rn(t);
  return (uint32_t)*reinterpret_cast<uint16_t *>(&b);
}
__device__ __forceinline__ uint32_t mix_bf16x2(float a, float b, int pl) {
  return mix_bf16_bits(a, pl) | (mix_bf16_bits(b, pl) << 16);
}

template <int ELEM>
struct PackOut;
template <>
struct PackOut<2> {
  __device__ __forceinline__ static void store4(void *dst, size_t idx, float a, float b, float c,
                                                float d, long long = 0) {
    __nv_bfloat162 lo = __floats2bfloat162_rn(a, b), hi = __floats2bfloat162_rn(c, d);
    uint2 u;
    u.x = *reinterpret_cast<uint32_t *>(&lo);
    u.y = *reinterpret_cast<uint32_t *>(&hi);
    *reinterpret_cast<uint2 *>(static_cast<__nv_bfloat16 *>(dst) + idx) = u;
  }
  __device__ __forceinline__ static void store1(void *dst, size_t idx, float a, long long = 0) {
    static_cast<__nv_bfloat16 *>(dst)[idx] = __float2bfloat16_rn(a);
  }
};
template <>
struct PackOut<4> {
  __device__ __forceinline__ static void store4(void *dst, size_t idx, float a, float b, float c,
                                                float d, long long lo = 0) {
    uint4 u = make_uint4(f32_to_tf32_rna(a), f32_to_tf32_rna(b), f32_to_tf32_rna(c),
                         f32_to_tf32_rna(d));
    *reinterpret_cast<uint4 *>(static_cast<float *>(dst) + idx) = u;
    if (lo < 0) {   // mixed split: bf16(hi), bf16(v - hi)
#pragma unroll
      for (int pl = 1; pl <= 2; ++pl)
        *reinterpret_cast<uint2 *>(static_cast<uint8_t *>(dst) + plane_off(lo, pl) + idx * 2) =
            make_uint2(mix_bf16x2(a, b, pl), mix_bf16x2(c, d, pl));
    } else if (lo) {
      uint4 l = make_uint4(f32_to_tf32_rna(a - __uint_as_float(u.x)),
                           f32_to_tf32_rna(b - __uint_as_float(u.y)),
                           f32_to_tf32_rna(c - __uint_as_float(u.z)),
                           f32_to_tf32_rna(d - __uint_as_float(u.w)));
      *reinterpret_cast<uint4 *>(static_cast<uint8_t *>(dst) + lo + idx * 4) = l;
    }
  }
  __device__ __forceinline__ static void store1(void *dst, size_t idx, float a, long long lo = 0) {
    const uint32_t h = f32_to_tf32_rna(a);
    static_cast<uint32_t *>(dst)[idx] = h;
    if (lo < 0) {
#pragma unroll
      for (int pl = 1; pl <= 2; ++pl)
        *reinterpret_cast<uint16_t *>(static_cast<uint8_t *>(dst) + plane_off(lo, pl) + idx * 2) =
            (uint16_t)mix_bf16_bits(a, pl);
    } else if (lo) {
      *reinterpret_cast<uint32_t *>(static_cast<uint8_t *>(dst) + lo + idx * 4) =
          f32_to_tf32_rna(a - __uint_as_float(h));
    }
  }
};

// NCHW fp32 [N][C][HW] -> NHWC [N][HW][Cp] (rounded), zero for c >= C.
// Block = 32 channels x PACK_PT consecutive destination rows q of the whole batch (rows of
// consecutive images follow each other, so small images leave no ragged tile per image), 256
// threads: 16 independent coalesced loads per thread, conflict-free transposed smem reads,
// 16-byte stores.  grid (ceil(Cp/32), ceil(N*HWd/PACK_PT)): the channel blocks of a row tile are
// consecutive blocks, so the 64-byte pieces of each output row are written close in time and
// merge into whole lines in L2 (channel-block-major order wrote each row in pieces far apart).
// Padded destination (Wd != Ws): rows are positions (n, h, w) of an Hd x Wd grid per image
// (HWd = Hd*Wd), zero outside the Hs x Ws source image — the dy operand of the halo filter
// gradient (hwgrad.cuh).  Dense: Wd == Ws, HWd == HW.
// db_part (optional): [row tiles][C], each entry the sum of one channel over one row tile in a
// fixed order (lane-sequential over the 4 row quarters, then a xor-shuffle tree).
constexpr int PACK_PT = 128;

template <int ELEM>
__global__ void __launch_bounds__(256) pack_nchw_to_nhwc(const float *__restrict__ src,
                                                         void *__restrict__ dst, int N, int C,
                                                         int HW, int Cp, float *__restrict__ db_part,
                                                         unsigned int *__restrict__ tickets,
                                                         int n_tickets, int Ws, int Wd, int HWd,
                                                         int co_off, int Cw, int db_ld, int src_c,
                                                         long long lo_off) {
  // src_c: channels per image of the source tensor (> C when packing one group's channel slice).
  // (co_off, Cw, db_ld): this call writes destination channels [co_off, co_off + Cw) of rows with
  // pitch Cp (source channels 0..C-1, zeros past C) and db_part columns co_off + c of width db_ld —
  // one branch of a fused sibling group.  Single layer: co_off = 0, Cw = Cp, db_ld = C.
  __shared__ float tile[32][PACK_PT + 1];
  pdl_launch_dependents();
  pdl_wait();
  const int c0 = blockIdx.x * 32;
  const long long q0 = (long long)blockIdx.y * PACK_PT;
  const long long total = (long long)N * HWd;
  // arm the completion tickets of the deterministic db reduction that consumes db_part
  if (tickets != nullptr && (blockIdx.x | blockIdx.y) == 0)
    for (int i = threadIdx.x; i < n_tickets; i += blockDim.x) tickets[i] = 0u;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const bool padded = Wd != Ws;
  const int Hs = padded ? HW / Ws : 0;
  // source offset (n*C*HW + pixel) of this lane's 4 rows q0 + lane + 32 i: one division, then
  // increments (rows 32 apart; wraps handled by loops, any HWd / Wd)
  long long soff[4];
  bool sok[4];
  {
    const long long q = q0 + lane;
    int n = (int)(q / HWd), p = (int)(q - (long long)n * HWd);
#pragma unroll
    for (int i = 0; i < 4; ++i) {
      bool ok = (q + 32 * i) < total;
      int sp = p;
      if (padded) {
        const int h = p / Wd, w = p - h * Wd;
        ok = ok && h < Hs && w < Ws;
        sp = h * Ws + w;
      }
      sok[i] = ok;
      soff[i] = (long long)n * src_c * HW + sp;
      p += 32;
      while (p >= HWd) {
        p -= HWd;
        ++n;
      }
    }
  }
  float v[4][4];
#pragma unroll
  for (int k = 0; k < 4; ++k) {
    const int c = c0 + warp + 8 * k;
#pragma unroll
    for (int q = 0; q < 4; ++q)
      v[k][q] = (c < C && sok[q]) ? __ldg(src + soff[q] + (size_t)c * HW) : 0.f;
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
      if (lane == 0) db_part[(size_t)blockIdx.y * db_ld + co_off + c0 + cc] = t;
    }
  }
  __syncthreads();
  // 16-byte chunks: lanes cover consecutive chunks of a row's 32-channel segment (64 B bf16 /
  // 128 B fp32), so each warp store instruction writes whole contiguous row segments.
  constexpr int CPT = 16 / ELEM;            // channels per 16-byte chunk
  constexpr int CPP = 32 / CPT;             // chunks per row of the tile
  constexpr int PPP = 256 / CPP;            // rows per pass
#pragma unroll
  for (int pass = 0; pass < PACK_PT / PPP; ++pass) {
    const int pp = pass * PPP + threadIdx.x / CPP, j = threadIdx.x % CPP;
    const long long q = q0 + pp;
    const int cl = j * CPT, c = c0 + cl;
    if (q < total && c < Cw) {
      const size_t o = (size_t)q * Cp + co_off + c;
#pragma unroll
      for (int u = 0; u < CPT; u += 4)
        PackOut<ELEM>::store4(dst, o + u, tile[cl + u][pp], tile[cl + u + 1][pp],
                              tile[cl + u + 2][pp], tile[cl + u + 3][pp], lo_off);
    }
  }
}

// Warp-tiled variant (default): a warp owns 32 destination rows x 32 channels with no block-level
// barrier.  Lane = row: 32 coalesced 128-byte loads (one per channel) put one row's 32 channels in
// the lane's registers; they are rounded and packed there (16 bf16x2 / 32 tf32 words), staged in
// a per-warp smem slab with 16-byte stores, and written back as 16-byte chunks with consecutive
// lanes on consecutive chunks of a row (8 rows of 64 B bf16 per instruction).  Against the
// block-tiled kernel: 4x fewer shared-memory instructions (vector, half the bytes), no
// __syncthreads phases (measured l1tex 71 %, mio_throttle the top stall).  db partials: per
// (32-row tile, channel), the 32 rows summed by a fixed transposing butterfly (lane c ends with
// channel c's sum).  grid (ceil(Cw/32), ceil(N*HWd/256)), 256 threads.
constexpr int PACKW_ROWS = 32;
// __launch_bounds__(256, 2): two CTAs per SM (<= 128 registers).  The mixed split's third plane
// raised the unbounded allocation to 142 registers, one CTA per SM, and the fp32 packs ran at
// 2.7-3.0 TB/s (CaffeNet conv1 dy 282 us); bounded: 4.3-4.7 TB/s (180 us); 3 CTAs (80 registers,
// 150 bytes of spills) measured slower.
template <int ELEM>
__global__ void __launch_bounds__(256, 2) pack_act_warp(const float *__restrict__ src,
                                                     void *__restrict__ dst, int N, int C, int HW,
                                                     int Cp, float *__restrict__ db_part,
                                                     unsigned int *__restrict__ tickets,
                                                     int n_tickets, int Ws, int Wd, int HWd,
                                                     int co_off, int Cw, int db_ld, int src_c,
                                                     long long lo_off) {
  constexpr int RB = 32 * ELEM + 16;                    // smem bytes per staged row (+16 pad)
  __shared__ __align__(16) uint8_t slab[8][32 * RB];
  pdl_launch_dependents();
  pdl_wait();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int c0 = blockIdx.x * 32;
  const long long q0 = ((long long)blockIdx.y * 8 + warp) * PACKW_ROWS;
  const long long total = (long long)N * HWd;
  if (tickets != nullptr && (blockIdx.x | blockIdx.y) == 0)
    for (int i = threadIdx.x; i < n_tickets; i += blockDim.x) tickets[i] = 0u;
  if (q0 >= total) return;
  // this lane's row -> source (n, pixel)
  const long long q = q0 + lane;
  bool ok = q < total;
  long long soff = 0;
  if (ok) {
    const int n = (int)(q / HWd), p = (int)(q - (long long)n * HWd);
    int sp = p;
    if (Wd != Ws) {
      const int h = p / Wd, w = p - h * Wd;
      ok = h < HW / Ws && w < Ws;
      sp = h * Ws + w;
    }
    soff = (long long)n * src_c * HW + sp;
  }
  float v[32];
#pragma unroll
  for (int j = 0; j < 32; ++j)
    v[j] = (ok && c0 + j < C) ? __ldg(src + soff + (size_t)(c0 + j) * HW) : 0.f;
  if (db_part != nullptr) {
    // transposing butterfly: after step s every lane holds 32 >> s partial sums; lane c ends with
    // the sum of channel c over the 32 rows (fixed order: a function of the lane pattern only)
    float t[32];
#pragma unroll
    for (int j = 0; j < 32; ++j) t[j] = v[j];
#pragma unroll
    for (int w = 16; w >= 1; w >>= 1) {
      const bool up = (lane & w) != 0;
#pragma unroll
      for (int j = 0; j < w; ++j) {
        const float send = up ? t[j] : t[j + w];
        const float keep = up ? t[j + w] : t[j];
        t[j] = keep + __shfl_xor_sync(0xffffffffu, send, w);
      }
    }
    // step w keeps the upper half of the channels on lanes with bit w set, so t[0] of lane L is
    // channel L's sum
    if (c0 + lane < C)
      db_part[(size_t)(q0 / PACKW_ROWS) * db_ld + co_off + c0 + lane] = t[0];
  }
  // round + pack this lane's row, stage it in the warp's slab; 3xTF32 (lo_off != 0) stages and
  // writes the hi plane, then the lo plane through the same slab
  uint8_t *row = slab[warp] + lane * RB;
  const int planes = ELEM == 4 ? plane_count(lo_off) : 1;
  for (int pl = 0; pl < planes; ++pl) {
    const int es = ELEM == 4 ? plane_esize(lo_off, pl) : 2;   // element bytes of this plane
#pragma unroll
    for (int j = 0; j < 32; j += 8) {
      uint4 u0, u1;
      if (ELEM == 4 && es == 2) {   // mixed split: a bf16 plane
        u0 = make_uint4(mix_bf16x2(v[j], v[j + 1], pl), mix_bf16x2(v[j + 2], v[j + 3], pl),
                        mix_bf16x2(v[j + 4], v[j + 5], pl), mix_bf16x2(v[j + 6], v[j + 7], pl));
        *reinterpret_cast<uint4 *>(row + j * 2) = u0;
      } else if (ELEM == 2) {
        __nv_bfloat162 a = __floats2bfloat162_rn(v[j], v[j + 1]), b = __floats2bfloat162_rn(v[j + 2], v[j + 3]);
        __nv_bfloat162 c = __floats2bfloat162_rn(v[j + 4], v[j + 5]), d = __floats2bfloat162_rn(v[j + 6], v[j + 7]);
        u0 = make_uint4(*reinterpret_cast<uint32_t *>(&a), *reinterpret_cast<uint32_t *>(&b),
                        *reinterpret_cast<uint32_t *>(&c), *reinterpret_cast<uint32_t *>(&d));
        *reinterpret_cast<uint4 *>(row + j * 2) = u0;
      } else {
        u0 = make_uint4(tf32_plane(v[j], pl), tf32_plane(v[j + 1], pl), tf32_plane(v[j + 2], pl),
                        tf32_plane(v[j + 3], pl));
        u1 = make_uint4(tf32_plane(v[j + 4], pl), tf32_plane(v[j + 5], pl), tf32_plane(v[j + 6], pl),
                        tf32_plane(v[j + 7], pl));
        *reinterpret_cast<uint4 *>(row + j * 4) = u0;
        *reinterpret_cast<uint4 *>(row + j * 4 + 16) = u1;
      }
    }
    __syncwarp();
    // write back: chunk k of the 32-row slab -> row k / CPR, 16-byte chunk k % CPR
    constexpr int CPR = 32 * ELEM / 16;                   // 16-byte chunks per row (4 bf16, 8 tf32)
    uint8_t *dpl = static_cast<uint8_t *>(dst) + (ELEM == 4 ? plane_off(lo_off, pl) : 0);
    if (ELEM == 4 && es == 2) {   // a bf16 plane of the mixed split: 4 chunks per row
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int k = i * 32 + lane, r = k / 4, ch = k % 4;
        const long long qr = q0 + r;
        const int c = c0 + ch * 8;
        if (qr < total && c < Cw) {
          const uint4 val = *reinterpret_cast<const uint4 *>(slab[warp] + r * RB + ch * 16);
          *reinterpret_cast<uint4 *>(dpl + ((size_t)qr * Cp + co_off + c) * 2) = val;
        }
      }
    } else {
#pragma unroll
      for (int i = 0; i < CPR; ++i) {
        const int k = i * 32 + lane, r = k / CPR, ch = k % CPR;
        const long long qr = q0 + r;
        const int c = c0 + ch * (16 / ELEM);
        if (qr < total && c < Cw) {
          const uint4 val = *reinterpret_cast<const uint4 *>(slab[warp] + r * RB + ch * 16);
          *reinterpret_cast<uint4 *>(dpl + ((size_t)qr * Cp + co_off + c) * ELEM) = val;
        }
      }
    }
    __syncwarp();
  }
}

// Small channel counts (Cp <= 16): one thread per pixel, loads coalesced across pixels.
template <int ELEM>
__global__ void __launch_bounds__(256) pack_nchw_to_nhwc_small(const float *__restrict__ src,
                                                               void *__restrict__ dst, int N, int C,
                                                               int HW, int Cp, int src_c,
                                                               long long lo_off) {
  pdl_launch_dependents();
  pdl_wait();
  const size_t total = (size_t)N * HW;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < total;
       i += (size_t)gridDim.x * blockDim.x) {
    const size_t n = i / HW, px = i % HW;
    const float *s = src + n * src_c * HW + px;
    for (int c = 0; c < Cp; c += 4) {
      float a[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) a[u] = (c + u < C) ? __ldg(s + (size_t)(c + u) * HW) : 0.f;
      PackOut<ELEM>::store4(dst, i * Cp + c, a[0], a[1], a[2], a[3], lo_off);
    }
  }
}

// Space-to-depth pack for strided convolutions with few input channels:
//   x'[n][h'][w'][c'] = x[n][c][S*h' + dh - P][S*w' + dw - P]  (0 outside),  c' = (dh*S + dw)*C + c
// turns a stride-S, K x K conv into a stride-1, ceil(K/S) x ceil(K/S) conv over S*S*C channels
// with the same output, so the implicit GEMM runs unit-stride im2col TMA on a dense channel axis.
// Persistent: block b handles output rows (n, h') = b, b + grid, ...  The S*C source rows of an
// output row are staged in shared memory (coalesced loads; the next row's loads are issued into
// registers before the current row is written, so load latency overlaps the stores); the output
// row is written in 16-byte chunks.  Thread -> fixed chunk j of every pixel it writes, so the
// (source row, column phase) of its 16/ELEM channels is computed once (no per-element division).
// Dynamic smem = S*C*W floats.  Requires Cps*ELEM/16 chunks per pixel to divide 256.
constexpr int S2D_LD = 12;   // staged source floats per thread per row (S*C*W <= 256*S2D_LD)
template <int ELEM>
__global__ void __launch_bounds__(256) pack_s2d(const float *__restrict__ x, void *__restrict__ dst,
                                                int N, int C, int H, int W, int S, int P, int Hs,
                                                int Ws, int Cps, int src_c, long long lo_off) {
  extern __shared__ float rows[];   // [S*C][W] source rows (row r = dh*C + c)
  constexpr int CH = 16 / ELEM;     // channels per 16-byte chunk
  pdl_launch_dependents();
  pdl_wait();
  const int tid = threadIdx.x;
  const int RW = S * C * W;         // staged floats per output row
  // per-thread load slots: element e = tid + 256*i of the [S*C][W] stage
  int lsrc[S2D_LD];                 // offset in the image's x plane (c*H*W + dh*W + w), or -1
  int ldh[S2D_LD];
#pragma unroll
  for (int i = 0; i < S2D_LD; ++i) {
    const int e = tid + 256 * i;
    lsrc[i] = -1;
    ldh[i] = 0;
    if (e < RW) {
      const int r = e / W, w = e - r * W, dh = r / C, c = r - dh * C;
      lsrc[i] = c * H * W + w;
      ldh[i] = dh;
    }
  }
  // per-thread store chunk: channels j*CH .. j*CH+CH-1 of pixels pl, pl + pstep, ...
  const int cpr = Cps / CH, j = tid % cpr, pl = tid / cpr, pstep = 256 / cpr;
  int roff[CH], dws[CH];
#pragma unroll
  for (int u = 0; u < CH; ++u) {
    const int cc = j * CH + u;
    roff[u] = -1;
    dws[u] = 0;
    if (cc < S * S * C) {
      const int c = cc % C, dd = cc / C, dh = dd / S, dw = dd - dh * S;
      roff[u] = (dh * C + c) * W;
      dws[u] = dw - P;
    }
  }
  const int total = N * Hs;
  float v[S2D_LD];
  auto issue = [&](int row) {
    const int n = row / Hs, hs = row - n * Hs;
    const float *xb = x + (size_t)n * src_c * H * W;
#pragma unroll
    for (int i = 0; i < S2D_LD; ++i) {
      const int ih = S * hs + ldh[i] - P;
      v[i] = (lsrc[i] >= 0 && ih >= 0 && ih < H) ? __ldg(xb + lsrc[i] + ih * W) : 0.f;
    }
  };
  int row = blockIdx.x;
  if (row < total) issue(row);
  for (; row < total; row += gridDim.x) {
#pragma unroll
    for (int i = 0; i < S2D_LD; ++i)
      if (tid + 256 * i < RW) rows[tid + 256 * i] = v[i];
    __syncthreads();
    if (row + (int)gridDim.x < total) issue(row + gridDim.x);   // next row in flight
    const size_t obase = (size_t)row * Ws;
    for (int ws = pl; ws < Ws; ws += pstep) {
      float o[CH];
#pragma unroll
      for (int u = 0; u < CH; ++u) {
        const int iw = S * ws + dws[u];
        o[u] = (roff[u] >= 0 && iw >= 0 && iw < W) ? rows[roff[u] + iw] : 0.f;
      }
#pragma unroll
      for (int u = 0; u < CH; u += 4)
        PackOut<ELEM>::store4(dst, (obase + ws) * Cps + j * CH + u, o[u], o[u + 1], o[u + 2],
                              o[u + 3], lo_off);
    }
    __syncthreads();
  }
}

// Warp-per-32-pixels space-to-depth pack (default when S*S*C <= 64): lane = one destination pixel
// (n, h', w') of the flattened batch, its S*S*C source values gathered straight into registers
// (48 independent loads per lane for CaffeNet conv1: high memory-level parallelism, each source
// element fetched from DRAM once, the dw neighbours served by L1), rounded and packed there, staged
// in a per-warp smem slab and written back as contiguous 512-byte runs (the 32 destination rows of
// a warp are consecutive in NHWC).  No block barriers.  The block-persistent pack_s2d (row staging
// through shared memory, per-row barriers) ran at ~3.3 TB/s.  128 threads.
constexpr int S2DW_MAXC = 64;
template <int ELEM>
__global__ void __launch_bounds__(128) pack_s2d_warp(const float *__restrict__ x, void *__restrict__ dst,
                                                     int N, int C, int H, int W, int S, int P, int Hs,
                                                     int Ws, int Cps, int src_c, long long lo_off) {
  constexpr int RB = S2DW_MAXC * ELEM + 16;            // slab bytes per staged row (+16 pad)
  __shared__ __align__(16) uint8_t slab[4][32 * RB];
  pdl_launch_dependents();
  pdl_wait();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long total = (long long)N * Hs * Ws;
  const long long q0 = ((long long)blockIdx.x * 4 + warp) * 32;
  if (q0 >= total) return;
  const long long q = q0 + lane;
  const bool ok = q < total;
  int n = 0, hs = 0, ws = 0;
  if (ok) {
    n = (int)(q / ((long long)Hs * Ws));
    const int r = (int)(q - (long long)n * Hs * Ws);
    hs = r / Ws;
    ws = r - hs * Ws;
  }
  const float *xb = x + (size_t)n * src_c * H * W;
  const int nch = S * S * C;
  float v[S2DW_MAXC];
  int c = 0, dw = 0, dh = 0;   // channel cc = (dh*S + dw)*C + c, advanced incrementally
#pragma unroll
  for (int cc = 0; cc < S2DW_MAXC; ++cc) {
    const int ih = S * hs + dh - P, iw = S * ws + dw - P;
    v[cc] = (ok && cc < nch && ih >= 0 && ih < H && iw >= 0 && iw < W)
                ? __ldg(xb + ((size_t)c * H + ih) * W + iw)
                : 0.f;
    if (++c == C) {
      c = 0;
      if (++dw == S) {
        dw = 0;
        ++dh;
      }
    }
  }
  uint8_t *row = slab[warp] + lane * RB;
  const int planes = ELEM == 4 ? plane_count(lo_off) : 1;   // 3xTF32: hi, lo; mixed: hi, bf16 x2
  for (int pl = 0; pl < planes; ++pl) {
    const int es = ELEM == 4 ? plane_esize(lo_off, pl) : 2;
#pragma unroll
    for (int j = 0; j < S2DW_MAXC; j += 8) {
      if (j >= Cps) break;
      if (ELEM == 4 && es == 2) {
        *reinterpret_cast<uint4 *>(row + j * 2) =
            make_uint4(mix_bf16x2(v[j], v[j + 1], pl), mix_bf16x2(v[j + 2], v[j + 3], pl),
                       mix_bf16x2(v[j + 4], v[j + 5], pl), mix_bf16x2(v[j + 6], v[j + 7], pl));
      } else if (ELEM == 2) {
        __nv_bfloat162 a = __floats2bfloat162_rn(v[j], v[j + 1]), b = __floats2bfloat162_rn(v[j + 2], v[j + 3]);
        __nv_bfloat162 cq = __floats2bfloat162_rn(v[j + 4], v[j + 5]), d = __floats2bfloat162_rn(v[j + 6], v[j + 7]);
        *reinterpret_cast<uint4 *>(row + j * 2) =
            make_uint4(*reinterpret_cast<uint32_t *>(&a), *reinterpret_cast<uint32_t *>(&b),
                       *reinterpret_cast<uint32_t *>(&cq), *reinterpret_cast<uint32_t *>(&d));
      } else {
        *reinterpret_cast<uint4 *>(row + j * 4) =
            make_uint4(tf32_plane(v[j], pl), tf32_plane(v[j + 1], pl), tf32_plane(v[j + 2], pl),
                       tf32_plane(v[j + 3], pl));
        *reinterpret_cast<uint4 *>(row + j * 4 + 16) =
            make_uint4(tf32_plane(v[j + 4], pl), tf32_plane(v[j + 5], pl), tf32_plane(v[j + 6], pl),
                       tf32_plane(v[j + 7], pl));
      }
    }
    __syncwarp();
    // the warp's rows q0 .. q0+31 are contiguous in dst: chunk k -> row k / cpr, chunk k % cpr
    const int cpr = Cps * es / 16;
    uint8_t *out = static_cast<uint8_t *>(dst) + (ELEM == 4 ? plane_off(lo_off, pl) : 0) +
                   (size_t)q0 * Cps * es;
    const int nrows = (int)min(32LL, total - q0);
    for (int k = lane; k < nrows * cpr; k += 32) {
      const int r = k / cpr, ch = k - r * cpr;
      *reinterpret_cast<uint4 *>(out + (size_t)k * 16) =
          *reinterpret_cast<const uint4 *>(slab[warp] + r * RB + ch * 16);
    }
    __syncwarp();
  }
}

// Compile-time (S, C) form of pack_s2d_warp (CaffeNet conv1: S = 4, C = 3): the generic kernel
// was issue-bound (ncu: stall not_selected / math / wait, 69 M instructions for 264 MB) on its
// per-channel counter and bounds logic; here one row pointer per (dh, c), one column test per dw,
// and the loop fully unrolled.
template <int ELEM, int S, int C>
__global__ void __launch_bounds__(128) pack_s2d_warp_t(const float *__restrict__ x, void *__restrict__ dst,
                                                       int N, int H, int W, int P, int Hs, int Ws,
                                                       int Cps, int src_c, long long lo_off) {
  constexpr int NC = S * S * C;
  constexpr int RB = S2DW_MAXC * ELEM + 16;
  __shared__ __align__(16) uint8_t slab[4][32 * RB];
  pdl_launch_dependents();
  pdl_wait();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const long long total = (long long)N * Hs * Ws;
  const long long q0 = ((long long)blockIdx.x * 4 + warp) * 32;
  if (q0 >= total) return;
  const long long q = q0 + lane;
  const bool ok = q < total;
  int n = 0, hs = 0, ws = 0;
  if (ok) {
    n = (int)(q / ((long long)Hs * Ws));
    const int r = (int)(q - (long long)n * Hs * Ws);
    hs = r / Ws;
    ws = r - hs * Ws;
  }
  const float *xb = x + (size_t)n * src_c * H * W;
  float v[NC];
  bool cok[S];
#pragma unroll
  for (int dw = 0; dw < S; ++dw) {
    const int iw = S * ws + dw - P;
    cok[dw] = iw >= 0 && iw < W;
  }
#pragma unroll
  for (int dh = 0; dh < S; ++dh) {
    const int ih = S * hs + dh - P;
    const bool rok = ok && ih >= 0 && ih < H;
#pragma unroll
    for (int c = 0; c < C; ++c) {
      const float *row = xb + ((size_t)c * H + (rok ? ih : 0)) * W + (S * ws - P);
#pragma unroll
      for (int dw = 0; dw < S; ++dw)
        v[(dh * S + dw) * C + c] = (rok && cok[dw]) ? __ldg(row + dw) : 0.f;
    }
  }
  uint8_t *rowp = slab[warp] + lane * RB;
  const int planes = ELEM == 4 ? plane_count(lo_off) : 1;   // 3xTF32: hi, lo; mixed: hi, bf16 x2
  for (int pl = 0; pl < planes; ++pl) {
    const int es = ELEM == 4 ? plane_esize(lo_off, pl) : 2;
#pragma unroll
    for (int j = 0; j < S2DW_MAXC; j += 8) {
      if (j >= Cps) break;
      float u[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) u[k] = (j + k < NC) ? v[(j + k < NC) ? j + k : 0] : 0.f;
      if (ELEM == 4 && es == 2) {
        *reinterpret_cast<uint4 *>(rowp + j * 2) =
            make_uint4(mix_bf16x2(u[0], u[1], pl), mix_bf16x2(u[2], u[3], pl),
                       mix_bf16x2(u[4], u[5], pl), mix_bf16x2(u[6], u[7], pl));
      } else if (ELEM == 2) {
        __nv_bfloat162 a = __floats2bfloat162_rn(u[0], u[1]), b = __floats2bfloat162_rn(u[2], u[3]);
        __nv_bfloat162 cq = __floats2bfloat162_rn(u[4], u[5]), d = __floats2bfloat162_rn(u[6], u[7]);
        *reinterpret_cast<uint4 *>(rowp + j * 2) =
            make_uint4(*reinterpret_cast<uint32_t *>(&a), *reinterpret_cast<uint32_t *>(&b),
                       *reinterpret_cast<uint32_t *>(&cq), *reinterpret_cast<uint32_t *>(&d));
      } else {
        *reinterpret_cast<uint4 *>(rowp + j * 4) =
            make_uint4(tf32_plane(u[0], pl), tf32_plane(u[1], pl), tf32_plane(u[2], pl),
                       tf32_plane(u[3], pl));
        *reinterpret_cast<uint4 *>(rowp + j * 4 + 16) =
            make_uint4(tf32_plane(u[4], pl), tf32_plane(u[5], pl), tf32_plane(u[6], pl),
                       tf32_plane(u[7], pl));
      }
    }
    __syncwarp();
    const int cpr = Cps * es / 16;
    uint8_t *out = static_cast<uint8_t *>(dst) + (ELEM == 4 ? plane_off(lo_off, pl) : 0) +
                   (size_t)q0 * Cps * es;
    const int nrows = (int)min(32LL, total - q0);
    for (int k = lane; k < nrows * cpr; k += 32) {
      const int r = k / cpr, ch = k - r * cpr;
      *reinterpret_cast<uint4 *>(out + (size_t)k * 16) =
          *reinterpret_cast<const uint4 *>(slab[warp] + r * RB + ch * 16);
    }
    __syncwarp();
  }
}

// Forward B operand in the space-to-depth geometry: Wp[co][t'*Cps + c'], t' = kh'*Ks + kw',
// c' = (dh*S + dw)*C + c, value W[co][c][S*kh'+dh][S*kw'+dw] (0 past the K x K window).
template <int ELEM>
__global__ void pack_w_fwd_s2d(const float *__restrict__ w, void *__restrict__ out, int Co, int C,
                               int K, int S, int Ks, int Cps, int Kpad, long long lo_off) {
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
    PackOut<ELEM>::store1(out, i, v, lo_off);
  }
}

// W [Co][C][Kh][Kw] -> forward B operand Wp[co][tap*Cp + c] with row length Kpad (zero padded).
// grid (ceil(Kpad/256), Co): one element per thread, 32-bit index math (the old grid-stride form
// spent most of its time in 64-bit divisions).
template <int ELEM>
__global__ void __launch_bounds__(256) pack_w_fwd(const float *__restrict__ w, void *__restrict__ out,
                                                  int Co, int C, int taps, int Cp, int Kpad,
                                                  long long lo_off) {
  pdl_launch_dependents();
  pdl_wait();
  const int co = blockIdx.y, k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= Kpad) return;
  const int t = k / Cp, c = k - t * Cp;
  const float v = (t < taps && c < C) ? __ldg(w + ((size_t)co * C + c) * taps + t) : 0.f;
  PackOut<ELEM>::store1(out, (size_t)co * Kpad + k, v, lo_off);
}

// W [Co][C][Kh][Kw] -> backward-data B operand Wt[ci][tap*Cop + co] (row length Kpad).
// flip = 1: tap index reversed (tap' = taps-1-tap, i.e. (Kh-1-kh, Kw-1-kw)) for the im2col-TMA
// dgrad, which walks dy from the window's top-left corner.
// Fused sibling group: this call owns fused output channels [co_lo, co_hi) of the K index,
// holding branch channels co - co_off (< Co) and zeros past them; single layer: co_off = co_lo =
// 0, co_hi = Cop.
template <int ELEM>
__global__ void __launch_bounds__(256) pack_w_dgrad(const float *__restrict__ w, void *__restrict__ out,
                                                    int Co, int C, int taps, int Cop, int Kpad,
                                                    int flip, int co_off, int co_lo, int co_hi,
                                                    long long lo_off) {
  pdl_launch_dependents();
  pdl_wait();
  const int ci = blockIdx.y, k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= Kpad) return;
  const int t = k / Cop, co = k - t * Cop;
  if (t < taps && (co < co_lo || co >= co_hi)) return;   // another branch's channels
  const int cb = co - co_off;
  const float v = (t < taps && cb < Co)
                      ? __ldg(w + ((size_t)cb * C + ci) * taps + (flip ? taps - 1 - t : t))
                      : 0.f;
  PackOut<ELEM>::store1(out, (size_t)ci * Kpad + k, v, lo_off);
}

// Space-to-depth backward-data (strided layers, DESIGN.md §7 "strided backward-data"): the
// B operand of the stride-1 dgrad over x' -- Wt'[cs][t*Cop + co] = W'[co][tap(t)][cs] with the
// space-to-depth weights W'[co][(kh', kw')][cs = (dh*S + dw)*C + c] = W[co][c][kh'*S + dh]
// [kw'*S + dw] (zero past the K x K kernel), taps flipped when the dgrad walks them by TMA.
// grid (ceil(Kpad / 256), Cs).
template <int ELEM>
__global__ void __launch_bounds__(256) pack_w_dgrad_s2d(const float *__restrict__ w, void *__restrict__ out,
                                                        int Co, int C, int K, int S, int Ks, int Cop,
                                                        int Kpad, int flip, long long lo_off) {
  pdl_launch_dependents();
  pdl_wait();
  const int cs = blockIdx.y, k = blockIdx.x * blockDim.x + threadIdx.x;
  if (k >= Kpad) return;
  const int t = k / Cop, co = k - t * Cop, taps = Ks * Ks;
  float v = 0.f;
  if (t < taps && co < Co) {
    const int tt = flip ? taps - 1 - t : t;
    const int khs = tt / Ks, kws = tt - khs * Ks;
    const int ph = cs / C, c = cs - ph * C, dh = ph / S, dw = ph - dh * S;
    const int kh = khs * S + dh, kw = kws * S + dw;
    if (kh < K && kw < K) v = __ldg(w + (((size_t)co * C + c) * K + kh) * K + kw);
  }
  PackOut<ELEM>::store1(out, (size_t)cs * Kpad + k, v, lo_off);
}

// dx from the space-to-depth gradient dx'[n][cs][h'][w'] (NCHW, Cs = S*S*C channels, H' x W'):
// dx[n][c][h][w] = dx'[n][(dh*S + dw)*C + c][h'][w'] with h + P = S*h' + dh, w + P = S*w' + dw
// (each x element sits once in x'); elements the x' grid does not reach get 0 (they reach no
// output, Alg. 2 / DESIGN.md R2).  One thread per dx element, w fastest (coalesced
// stores).  img_c: channels per image of the dx tensor (conv groups).
__global__ void __launch_bounds__(256) unpack_s2d_dx(const float *__restrict__ dxs, float *__restrict__ dx,
                                                     int N, int C, int H, int W, int S, int P,
                                                     int Hs, int Ws, int img_c) {
  pdl_launch_dependents();
  pdl_wait();
  const long long total = (long long)N * C * H * W;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < total;
       i += (long long)gridDim.x * blockDim.x) {
    const int w = (int)(i % W);
    long long r = i / W;
    const int h = (int)(r % H);
    r /= H;
    const int c = (int)(r % C), n = (int)(r / C);
    const int hp = h + P, wp = w + P;
    const int h2 = hp / S, dh = hp - h2 * S, w2 = wp / S, dw = wp - w2 * S;
    float v = 0.f;
    if (h2 < Hs && w2 < Ws)
      v = __ldg(dxs + (((size_t)n * S * S * C + (size_t)(dh * S + dw) * C + c) * Hs + h2) * Ws + w2);
    dx[(((size_t)n * img_c + c) * H + h) * W + w] = v;
  }
}

// Row-staged weight packs (default when a staged row fits 48 KB of shared memory).  The element-
// per-thread kernels above read W with a stride of `taps` floats between neighbouring threads (one
// 32-byte sector per 4-byte load); here one block owns one destination row, reads its source
// elements once with coalesced loads into shared memory and writes the row with consecutive
// threads on consecutive destination elements (odd taps: conflict-free strided smem reads).
// Forward: block co stages W[co][0..C*taps) and writes Wp[co][t*Cp + c].
template <int ELEM>
__global__ void __launch_bounds__(256) pack_w_fwd_rows(const float *__restrict__ w, void *__restrict__ out,
                                                       int C, int taps, int Cp, int Kpad,
                                                       long long lo_off) {
  extern __shared__ float srow[];
  pdl_launch_dependents();
  pdl_wait();
  const int co = blockIdx.x, n = C * taps;
  const float *src = w + (size_t)co * n;
  for (int i = threadIdx.x; i < n; i += 256) srow[i] = __ldg(src + i);
  __syncthreads();
  for (int k = threadIdx.x; k < Kpad; k += 256) {
    const int t = k / Cp, c = k - t * Cp;
    const float v = (t < taps && c < C) ? srow[c * taps + t] : 0.f;
    PackOut<ELEM>::store1(out, (size_t)co * Kpad + k, v, lo_off);
  }
}

// Backward-data: block ci stages W[cb][ci][0..taps) for every cb < Co (runs of `taps` contiguous
// floats) and writes Wt[ci][t*Cop + co] over [co_lo, co_hi) (+ the zero tail past the taps), with
// the same flip / branch semantics as pack_w_dgrad.
template <int ELEM>
__global__ void __launch_bounds__(256) pack_w_dgrad_rows(const float *__restrict__ w, void *__restrict__ out,
                                                         int Co, int C, int taps, int Cop, int Kpad,
                                                         int flip, int co_off, int co_lo, int co_hi,
                                                         long long lo_off) {
  extern __shared__ float srow[];   // [Co][taps]
  pdl_launch_dependents();
  pdl_wait();
  const int ci = blockIdx.x, n = Co * taps;
  for (int i = threadIdx.x; i < n; i += 256) {
    const int cb = i / taps, t = i - cb * taps;
    srow[i] = __ldg(w + ((size_t)cb * C + ci) * taps + t);
  }
  __syncthreads();
  for (int k = threadIdx.x; k < Kpad; k += 256) {
    const int t = k / Cop, co = k - t * Cop;
    if (t < taps && (co < co_lo || co >= co_hi)) continue;   // another branch's channels
    const int cb = co - co_off;
    const float v = (t < taps && cb < Co) ? srow[cb * taps + (flip ? taps - 1 - t : t)] : 0.f;
    PackOut<ELEM>::store1(out, (size_t)ci * Kpad + k, v, lo_off);
  }
}

// Both weight operands in one pass over W (GLP_PACK_W_BOTH): block (ci tile of 32, co tile of 32)
// stages W[co][ci][0..taps) for its 32 x 32 (co, ci) pairs (each co contributes one contiguous run
// of 32*taps floats: coalesced), then writes the forward operand Wp[co][t*Cp + ci] (32 consecutive
// ci per (co, t)) and the backward-data operand Wt[ci][t'*Cop + co] (32 consecutive co per (ci, t),
// t' = taps-1-t when flipped).  Tiles cover ci < Cp and co < Cop, so the channel padding is written
// as zeros here; blockIdx.z == 1 zero-fills the K tails past taps*Cp / taps*Cop.  Values are the
// same rounding of the same fp32 as the separate packs (bitwise identical operands).
constexpr int PWB_MAXT = 25;   // taps (<= 5x5) that fit the stage: 32 x (32*25 + 1) floats = 100 KB
template <int ELEM>
__global__ void __launch_bounds__(256) pack_w_both(const float *__restrict__ w, void *__restrict__ wp,
                                                   void *__restrict__ wt, int Co, int C, int taps,
                                                   int Cp, int Cop, int Kpf, int Kpd, int flip,
                                                   long long lo_p, long long lo_t) {
  extern __shared__ float stg[];   // [32 co][32*taps + 1]
  pdl_launch_dependents();
  pdl_wait();
  const int ld = 32 * taps + 1;
  const int ci0 = blockIdx.x * 32, co0 = blockIdx.y * 32;
  if (blockIdx.z == 1) {   // K tails (t >= taps) of both operands
    for (int i = threadIdx.x; i < 32 * (Kpf - taps * Cp); i += 256) {
      const int r = i / (Kpf - taps * Cp), k = taps * Cp + i % (Kpf - taps * Cp);
      if (blockIdx.x == 0 && co0 + r < Co) PackOut<ELEM>::store1(wp, (size_t)(co0 + r) * Kpf + k, 0.f, lo_p);
    }
    for (int i = threadIdx.x; i < 32 * (Kpd - taps * Cop); i += 256) {
      const int r = i / (Kpd - taps * Cop), k = taps * Cop + i % (Kpd - taps * Cop);
      if (blockIdx.y == 0 && ci0 + r < C) PackOut<ELEM>::store1(wt, (size_t)(ci0 + r) * Kpd + k, 0.f, lo_t);
    }
    return;
  }
  const int run = 32 * taps;
  for (int i = threadIdx.x; i < 32 * run; i += 256) {
    const int r = i / run, e = i - r * run;   // co row r, element e = ci_l*taps + t
    const int co = co0 + r, ci = ci0 + e / taps;
    stg[r * ld + e] = (co < Co && ci < C) ? __ldg(w + ((size_t)co * C + ci) * taps + (e % taps)) : 0.f;
  }
  __syncthreads();
  const int lane = threadIdx.x & 31, wr = threadIdx.x >> 5;
  // forward: rows co (< Co), for each t: 32 consecutive ci (lane)
  for (int r = wr; r < 32; r += 8) {
    const int co = co0 + r;
    if (co >= Co || ci0 + lane >= Cp) continue;
    for (int t = 0; t < taps; ++t)
      PackOut<ELEM>::store1(wp, (size_t)co * Kpf + (size_t)t * Cp + ci0 + lane, stg[r * ld + lane * taps + t], lo_p);
  }
  // backward-data: rows ci (< C), for each t: 32 consecutive co (lane); padding co >= Co -> 0
  for (int c = wr; c < 32; c += 8) {
    const int ci = ci0 + c;
    if (ci >= C || co0 + lane >= Cop) continue;
    for (int t = 0; t < taps; ++t) {
      const int tt = flip ? taps - 1 - t : t;
      PackOut<ELEM>::store1(wt, (size_t)ci * Kpd + (size_t)tt * Cop + co0 + lane, stg[lane * ld + c * taps + t], lo_t);
    }
  }
}

}  // namespace glp
