// tiny.cuh — CUDA-core direct kernels for layers too small for the tensor-core path (VERDICT r1
// #7: LeNet conv1 is C = 1, C*Kh*Kw = 25, C_o = 20; LeNet conv2 and the CIFAR-10 layers are a few
// hundred MFMA per pass).
//
// For such a layer the implicit GEMM pads K = 25 to a 32-wide k-block and M = C_o = 20 to a
// 128-row tile, and a step is seven launches (x, W, dy packs; GEMMs; dW and db reductions) of
// which none does enough work to cover its own latency.  Here each pass is ONE launch that reads
// the NCHW fp32 tensors directly (no packs).  Stride-1 layers with square K in {3, 5}:
//   * tiny_corr<.., DG = 0> (forward, Alg. 1, P82-99): y[n,co,oh,ow] = b[co] +
//     sum_{ci,kh,kw} W[co,ci,kh,kw] * x[n,ci,oh-P+kh,ow-P+kw];
//   * tiny_corr<.., DG = 1> (backward data, Alg. 2 P119-140 with col2im folded): the same
//     correlation over dy padded by K-1-P with the flipped, transposed filter,
//     dx[n,c,h,w] = sum_{co,kh,kw} W[co,c,K-1-kh,K-1-kw] * dy[n,co,h-(K-1-P)+kh,w-(K-1-P)+kw];
//   * tiny_wgrad (P264, summed over the batch): dW[co,c,kh,kw] = sum_{n,oh,ow} dy * x and
//     db[co] = sum_{n,oh,ow} dy, one launch including the fixed-order reduction.
// Register tiling: a thread owns 4 consecutive output pixels x 4 channels (16 accumulators); each
// staged input row segment of 4 + K - 1 values feeds K * 16 FMAs.  The input of a CTA is staged
// zero-padded in shared memory, so the inner loops have no bounds checks.
// Every sum runs in an order fixed by the layer shape alone (taps in (ci, kh, kw) order; strips,
// phases and units are functions of the shape), so results are deterministic and independent of
// timing (P264).  RM: operand rounding of the math mode (0 = fp32 -- the FP32 plans, plain fp32
// FMA; 1 = TF32 rna; 2 = BF16 rne) applied to the operands as the tensor path's packs do; products
// of TF32/BF16 operands are exact in fp32, so only the summation order differs from that path.
#pragma once
#include <cuda_bf16.h>

#include <algorithm>

#include "ptx.cuh"
#include "simt.cuh"

namespace glp {

constexpr int TINY_THREADS = 256;

#ifdef TINY_PROBE_TIMING   // tools/tiny_probe.cu only: globaltimer stamps of CTA 0
__device__ unsigned long long tiny_stamp[8];
#define TINY_STAMP(i)                                                                    \
  do {                                                                                   \
    if (blockIdx.x == 0 && blockIdx.y == 0 && threadIdx.x == 0) {                        \
      unsigned long long t_;                                                             \
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));                             \
      tiny_stamp[i] = t_;                                                                \
    }                                                                                    \
  } while (0)
#else
#define TINY_STAMP(i) \
  do {                \
  } while (0)
#endif

template <int RM>
__device__ __forceinline__ float tiny_round(float v) {
  if constexpr (RM == 1) return __uint_as_float(f32_to_tf32_rna(v));
  else if constexpr (RM == 2) return __bfloat162float(__float2bfloat16_rn(v));
  else return v;
}

__host__ __device__ constexpr int tiny_rup4(int v) { return (v + 3) & ~3; }

// One stride-1 correlation pass (forward or backward data) as the kernel sees it.
struct TinyCorr {
  int Cin, Hin, Win, Cout, Hout, Wout, pad;
  int in_cs, out_cs;   // channels per image of the input / output tensors (conv-group strides)
  int Hp, Wpp;         // staged zero-padded input plane: Hout + K - 1 rows, Wpp (multiple of 4) cols
  int gpc;             // groups of 4 output channels per CTA
  int R;               // input-channel phases per output item (phase sums added in order)
};
__host__ __device__ inline int tiny_corr_smem_floats(const TinyCorr &t, int K) {
  const int items = t.Hout * (tiny_rup4(t.Wout) / 4) * t.gpc;
  return t.Cin * t.Hp * t.Wpp + t.Cin * K * K * 4 * t.gpc + (t.R > 1 ? t.R * items * 16 : 0);
}

// Operand staging.  The padded shared-memory block is zero-filled (float4 stores), then -- after a
// barrier -- the source elements are copied into its interior with 4-byte cp.async, every copy of
// the block in flight at once (a load-then-store loop waited one memory latency per iteration;
// per-row loops spent ~150 instructions per 32 floats).
//   tiny_zero:  dst[0 .. n4*4) = 0
//   tiny_copy_block: nplanes source planes (plane stride splane floats), each a contiguous block of
//     srows x scols floats starting at src + pl*splane, to dst[pl][r + rd][c + cd] of a
//     [.][prow][pcol] block.  The caller commits/waits (tiny_stage_wait) and syncs.
__device__ __forceinline__ void tiny_zero(float *dst, int n4) {
  for (int i = threadIdx.x; i < n4; i += TINY_THREADS)
    reinterpret_cast<float4 *>(dst)[i] = make_float4(0.f, 0.f, 0.f, 0.f);
}
__device__ __forceinline__ void tiny_copy_block(float *dst, int prow, int pcol, int rd, int cd,
                                                const float *__restrict__ src, size_t splane,
                                                int nplanes, int srows, int scols) {
  const int blk = srows * scols, total = nplanes * blk;
  if (total <= 0) return;
  const FastDiv fb((uint32_t)blk), fc((uint32_t)scols);
  const uint32_t d0 = smem_u32(dst);
  for (int e = threadIdx.x; e < total; e += TINY_THREADS) {
    uint32_t pl, rem, r, c;
    fb.divmod((uint32_t)e, pl, rem);
    fc.divmod(rem, r, c);
    cp_async4(d0 + 4u * (((pl * prow + r + rd) * pcol) + c + cd), src + pl * splane + rem, true);
  }
}
// Apply the math mode's operand rounding to n staged floats (after the copies landed and a
// barrier); the caller syncs again.
template <int RM>
__device__ __forceinline__ void tiny_stage_round(float *dst, int n) {
  if constexpr (RM != 0)
    for (int i = threadIdx.x; i < n; i += TINY_THREADS) dst[i] = tiny_round<RM>(dst[i]);
}
__device__ __forceinline__ void tiny_stage_wait() {
  cp_async_commit();
  cp_async_wait<0>();
}

// out[n][co0 + j][oh][ow0 + p] = acc[p][j] (+ b[co0 + j] forward)
template <int DG>
__device__ __forceinline__ void tiny_corr_store(const TinyCorr &t, const float (&acc)[4][4],
                                                const float *__restrict__ b, float *__restrict__ out,
                                                int n, int co0, int oh, int ow0) {
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const int co = co0 + j;
    if (co >= t.Cout) break;
    const float bias = DG ? 0.f : __ldg(b + co);
    float *o = out + (((size_t)n * t.out_cs + co) * t.Hout + oh) * t.Wout + ow0;
    if ((t.Wout & 3) == 0) {
      *reinterpret_cast<float4 *>(o) =
          make_float4(acc[0][j] + bias, acc[1][j] + bias, acc[2][j] + bias, acc[3][j] + bias);
    } else {
#pragma unroll
      for (int p = 0; p < 4; ++p)
        if (ow0 + p < t.Wout) o[p] = acc[p][j] + bias;
    }
  }
}

// grid (ceil(ceil(Cout/4) / gpc), N), block TINY_THREADS, dynamic smem tiny_corr_smem_floats * 4.
template <int RM, int K, int DG>
__global__ void __launch_bounds__(TINY_THREADS) tiny_corr(TinyCorr t, const float *__restrict__ in,
                                                          const float *__restrict__ w,
                                                          const float *__restrict__ b,
                                                          float *__restrict__ out) {
  extern __shared__ __align__(16) float tsm[];
  TINY_STAMP(0);
  pdl_launch_dependents();
  pdl_wait();
  constexpr int KK = K * K, NX = (4 + K - 1 + 3) & ~3;   // staged row segment per strip
  const int n = blockIdx.y, g0 = blockIdx.x * t.gpc, GC = 4 * t.gpc;
  const int plane = t.Hp * t.Wpp;
  float *sin = tsm, *sw = tsm + t.Cin * plane;   // sin [Cin][Hp][Wpp]; sw [Cin][K][K][GC]
  const float *inn = in + (size_t)n * t.in_cs * t.Hin * t.Win;
  tiny_zero(sin, t.Cin * plane / 4);
  __syncthreads();
  tiny_copy_block(sin, t.Hp, t.Wpp, t.pad, t.pad, inn, (size_t)t.Hin * t.Win, t.Cin, t.Hin, t.Win);
  // filter, sw[(ci*KK + r)*GC + j]: one warp row per (j, ci) = the KK taps of one filter slice
  // (forward: W[co][ci][r]; backward data, co = layer input channel c, ci = layer output
  // channel: W[ci][co][KK-1-r]); zero-filled copies for channels beyond Cout
  {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t s0 = smem_u32(sw);
    for (int q = warp; q < GC * t.Cin; q += TINY_THREADS / 32) {
      const int j = q / t.Cin, ci = q - j * t.Cin, co = g0 * 4 + j;
      for (int r = lane; r < KK; r += 32) {
        const bool ok = co < t.Cout;
        const float *src = !ok ? w
                           : DG ? w + ((size_t)ci * t.Cout + co) * KK + (KK - 1 - r)
                                : w + ((size_t)co * t.Cin + ci) * KK + r;
        cp_async4(s0 + 4u * (uint32_t)((ci * KK + r) * GC + j), src, ok);
      }
    }
  }
  tiny_stage_wait();
  if (RM != 0) {
    __syncthreads();
    tiny_stage_round<RM>(sin, t.Cin * plane);
    tiny_stage_round<RM>(sw, t.Cin * KK * GC);
  }
  TINY_STAMP(1);
  __syncthreads();
  const int sw4 = tiny_rup4(t.Wout) / 4, strips = t.Hout * sw4;
  const int gcta = min(t.gpc, (t.Cout + 3) / 4 - g0), items = strips * gcta;
  // thread idx = rph * items + item: input channels ci = rph, rph + R, ... of one (strip, group)
  // item; the R phase sums are added in phase order (R * items <= TINY_THREADS when R > 1)
  float *red = sw + t.Cin * KK * GC;   // [R][items][16] (R > 1)
  for (int idx = threadIdx.x; idx < items * t.R; idx += TINY_THREADS) {
    const int rph = idx / items, item = idx - rph * items;
    const int gl = item / strips, s = item - gl * strips;
    const int oh = s / sw4, ow0 = (s - oh * sw4) * 4;
    float acc[4][4];
#pragma unroll
    for (int p = 0; p < 4; ++p)
#pragma unroll
      for (int j = 0; j < 4; ++j) acc[p][j] = 0.f;
    const float *wr = sw + gl * 4;
    for (int ci = rph; ci < t.Cin; ci += t.R) {
#pragma unroll
      for (int kh = 0; kh < K; ++kh) {
        const float *xr = sin + (ci * t.Hp + oh + kh) * t.Wpp + ow0;
        float xv[NX];
#pragma unroll
        for (int q = 0; q < NX / 4; ++q) {
          const float4 v = reinterpret_cast<const float4 *>(xr)[q];
          xv[4 * q] = v.x, xv[4 * q + 1] = v.y, xv[4 * q + 2] = v.z, xv[4 * q + 3] = v.w;
        }
        const float *wk = wr + ((ci * K + kh) * K) * GC;
#pragma unroll
        for (int kw = 0; kw < K; ++kw) {
          const float4 wv = *reinterpret_cast<const float4 *>(wk + kw * GC);
#pragma unroll
          for (int p = 0; p < 4; ++p) {
            acc[p][0] = fmaf(xv[p + kw], wv.x, acc[p][0]);
            acc[p][1] = fmaf(xv[p + kw], wv.y, acc[p][1]);
            acc[p][2] = fmaf(xv[p + kw], wv.z, acc[p][2]);
            acc[p][3] = fmaf(xv[p + kw], wv.w, acc[p][3]);
          }
        }
      }
    }
    if (t.R > 1) {
      float4 *rd = reinterpret_cast<float4 *>(red + (size_t)idx * 16);
#pragma unroll
      for (int p = 0; p < 4; ++p) rd[p] = make_float4(acc[p][0], acc[p][1], acc[p][2], acc[p][3]);
    } else {
      tiny_corr_store<DG>(t, acc, b, out, n, (g0 + gl) * 4, oh, ow0);
    }
  }
  TINY_STAMP(2);
  if (t.R > 1) {
    __syncthreads();
    for (int item = threadIdx.x; item < items; item += TINY_THREADS) {
      const int gl = item / strips, s = item - gl * strips;
      const int oh = s / sw4, ow0 = (s - oh * sw4) * 4;
      float acc[4][4];
#pragma unroll
      for (int p = 0; p < 4; ++p)
#pragma unroll
        for (int j = 0; j < 4; ++j) acc[p][j] = 0.f;
      for (int rph = 0; rph < t.R; ++rph) {
        const float4 *rd = reinterpret_cast<const float4 *>(red + (size_t)(rph * items + item) * 16);
#pragma unroll
        for (int p = 0; p < 4; ++p) {
          const float4 v = rd[p];
          acc[p][0] += v.x, acc[p][1] += v.y, acc[p][2] += v.z, acc[p][3] += v.w;
        }
      }
      tiny_corr_store<DG>(t, acc, b, out, n, (g0 + gl) * 4, oh, ow0);
    }
  }
}

// Filter + bias gradient in one launch.  Items: (ci, kh, g) for the filter (the K x 4
// accumulators acc[kw][j] of channels 4g..4g+3), then G db items (g); item = (ci*K + kh)*G + g.
// The items are cut into slices of `islice`; unit u = slice * nchunks + chunk, chunk = (sample
// chunk sc, row chunk rc): samples [sc*spc, +spc), output rows [rc*rows, +rows).  Thread
// (item, phase) takes the chunk's pixel strips s = phase, phase + PH, ... sample by sample; the PH
// phase sums are added in phase order.  The chunk partials of a slice are summed in two fixed-order
// levels (groups of 8 chunks, then the groups) by the last CTA to finish at each level (tickets).
// Workspace: part[units][E], gpart[nslices][ceil(nchunks/8)][E] (E = islice * K * 4 floats),
// nslices * (ceil(nchunks/8) + 1) tickets (zero at first use; re-armed by the kernel).
struct TinyWgrad {
  int N, C, H, W, Co, Ho, Wo, P;
  int xc, yc;                 // channels per image of x and dy
  int G, items, islice, nslices;
  int spc, rowchunks, rows, nchunks;
  int PH;                     // pixel phases per item
  int Wpp, Wo4;               // staged x row length (multiple of 4), staged dy row length
  int cspan;                  // x channels a slice can touch (staged per sample)
};
struct TinyWgradSmem {
  int sx, sdy, red, total;   // float offsets and total
};
__host__ __device__ inline TinyWgradSmem tiny_wgrad_smem(const TinyWgrad &t, int K) {
  TinyWgradSmem s;
  s.sx = 0;
  s.sdy = t.cspan * (t.rows + K - 1) * t.Wpp;
  s.red = s.sdy + 4 * t.G * t.rows * t.Wo4;
  s.total = s.red + (t.PH > 1 ? t.PH * t.islice * K * 4 : 0);
  return s;
}
template <int RM, int K>
__global__ void __launch_bounds__(TINY_THREADS) tiny_wgrad(TinyWgrad t, const float *__restrict__ x,
                                                           const float *__restrict__ dy,
                                                           float *__restrict__ part,
                                                           float *__restrict__ gpart,
                                                           unsigned int *__restrict__ ticket,
                                                           float *dw, float *db, int accumulate) {
  extern __shared__ __align__(16) float tsm[];
  __shared__ bool last;
  TINY_STAMP(0);
  pdl_launch_dependents();
  pdl_wait();
  constexpr int NX = (4 + K - 1 + 3) & ~3;
  constexpr int EI = K * 4;   // floats per item
  const TinyWgradSmem L = tiny_wgrad_smem(t, K);
  float *sx = tsm + L.sx, *sdy = tsm + L.sdy, *red = tsm + L.red;
  const int u = blockIdx.x, slice = u / t.nchunks, ch = u - slice * t.nchunks;
  const int sc = ch / t.rowchunks, rc = ch - sc * t.rowchunks;
  const int n0 = sc * t.spc, n1 = min(t.N, n0 + t.spc);
  const int oh0 = rc * t.rows, nr = min(t.rows, t.Ho - oh0);
  const int it0 = slice * t.islice, nit = min(t.islice, t.items - it0);
  const int nfil = (t.items / t.G - 1) * t.G;    // filter items (C*K*G)
  const int c0 = min(it0, nfil - 1) / (K * t.G);  // first x channel of the slice
  const int xr_rows = t.rows + K - 1, xplane = xr_rows * t.Wpp, dplane = t.rows * t.Wo4;
  const int sw4 = t.Wo4 / 4, strips = nr * sw4;
  const int E = t.islice * EI;
  // this thread's (item, phase) pair: idx = ph * nit + local (islice * PH <= TINY_THREADS)
  constexpr int QN = 1;
  float acc[QN][K][4];
#pragma unroll
  for (int q = 0; q < QN; ++q)
#pragma unroll
    for (int k = 0; k < K; ++k)
#pragma unroll
      for (int j = 0; j < 4; ++j) acc[q][k][j] = 0.f;
  // zero-filled once: the copies of every sample write the same interior cells
  tiny_zero(sx, t.cspan * xplane / 4);
  tiny_zero(sdy, 4 * t.G * dplane / 4);
  // x rows oh0 - P .. oh0 - P + xr_rows - 1 clipped to the image; columns shifted by P
  const int xr_lo = max(0, oh0 - t.P), xr_hi = min(t.H, oh0 - t.P + xr_rows);
  const int ncx = min(t.cspan, t.C - c0);
  for (int n = n0; n < n1; ++n) {
    __syncthreads();   // zero fill done / previous sample consumed
    const float *xn = x + ((size_t)n * t.xc + c0) * t.H * t.W;
    tiny_copy_block(sx, xr_rows, t.Wpp, xr_lo - (oh0 - t.P), t.P, xn + (size_t)xr_lo * t.W,
                    (size_t)t.H * t.W, ncx, xr_hi - xr_lo, t.W);
    // dy rows of the chunk, [4G][rows][Wo4] (zero beyond Co, the chunk's rows and Wo);
    // unrounded (db sums the fp32 dy, the filter items round on use)
    const float *dyn = dy + ((size_t)n * t.yc * t.Ho + oh0) * t.Wo;
    tiny_copy_block(sdy, t.rows, t.Wo4, 0, 0, dyn, (size_t)t.Ho * t.Wo, t.Co, nr, t.Wo);
    tiny_stage_wait();
    if (RM != 0) {
      __syncthreads();
      tiny_stage_round<RM>(sx, t.cspan * xplane);
    }
    TINY_STAMP(1);
    __syncthreads();
#pragma unroll
    for (int q = 0; q < QN; ++q) {
      const int idx = threadIdx.x + q * TINY_THREADS;
      if (idx >= nit * t.PH) break;
      const int ph = idx / nit, item = it0 + (idx - ph * nit);
      if (item < nfil) {
        const int g = item % t.G, ck = item / t.G, c = ck / K, kh = ck - c * K;
        const float *xb = sx + ((c - c0) * xr_rows + kh) * t.Wpp;
        const float *db0 = sdy + (4 * g) * dplane;
        int r = ph / sw4, ow0 = (ph - r * sw4) * 4;   // strip s = ph, ph + PH, ... as (row, col)
        const int dr = t.PH / sw4, dc = (t.PH - dr * sw4) * 4;
        for (int s = ph; s < strips; s += t.PH) {
          float xv[NX];
#pragma unroll
          for (int v4 = 0; v4 < NX / 4; ++v4) {
            const float4 v = reinterpret_cast<const float4 *>(xb + r * t.Wpp + ow0)[v4];
            xv[4 * v4] = v.x, xv[4 * v4 + 1] = v.y, xv[4 * v4 + 2] = v.z, xv[4 * v4 + 3] = v.w;
          }
          float d[4][4];   // [j][p]
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const float4 v = *reinterpret_cast<const float4 *>(db0 + j * dplane + r * t.Wo4 + ow0);
            d[j][0] = tiny_round<RM>(v.x), d[j][1] = tiny_round<RM>(v.y);
            d[j][2] = tiny_round<RM>(v.z), d[j][3] = tiny_round<RM>(v.w);
          }
#pragma unroll
          for (int p = 0; p < 4; ++p)
#pragma unroll
            for (int kw = 0; kw < K; ++kw)
#pragma unroll
              for (int j = 0; j < 4; ++j) acc[q][kw][j] = fmaf(xv[p + kw], d[j][p], acc[q][kw][j]);
          r += dr;
          ow0 += dc;
          if (ow0 >= t.Wo4) ow0 -= t.Wo4, ++r;
        }
      } else {   // db item: dy summed per channel, pixels in strip order
        const float *db0 = sdy + (4 * (item - nfil)) * dplane;
        int r = ph / sw4, ow0 = (ph - r * sw4) * 4;
        const int dr = t.PH / sw4, dc = (t.PH - dr * sw4) * 4;
        for (int s = ph; s < strips; s += t.PH) {
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const float4 v = *reinterpret_cast<const float4 *>(db0 + j * dplane + r * t.Wo4 + ow0);
            acc[q][0][j] = (((acc[q][0][j] + v.x) + v.y) + v.z) + v.w;
          }
          r += dr;
          ow0 += dc;
          if (ow0 >= t.Wo4) ow0 -= t.Wo4, ++r;
        }
      }
    }
  }
  TINY_STAMP(2);
  float *pu = part + (size_t)u * E;
#pragma unroll
  for (int q = 0; q < QN; ++q) {
    const int idx = threadIdx.x + q * TINY_THREADS;
    if (idx >= nit * t.PH) break;
    const int ph = idx / nit, il = idx - ph * nit;
    if (t.PH > 1) {
      float *dst = red + (size_t)(ph * t.islice + il) * EI;
#pragma unroll
      for (int k = 0; k < K; ++k)
#pragma unroll
        for (int j = 0; j < 4; ++j) dst[k * 4 + j] = acc[q][k][j];
    } else {
      float *dst = pu + (size_t)il * EI;
#pragma unroll
      for (int k = 0; k < K; ++k)
#pragma unroll
        for (int j = 0; j < 4; ++j) dst[k * 4 + j] = acc[q][k][j];
    }
  }
  if (t.PH > 1) {   // phase sums in phase order
    __syncthreads();
    for (int e = threadIdx.x; e < nit * EI; e += TINY_THREADS) {
      float s = 0.f;
      for (int ph = 0; ph < t.PH; ++ph) s += red[(size_t)ph * E + e];
      pu[e] = s;
    }
  }
  __threadfence();
  __syncthreads();
  // two-level fixed-order sum of the slice's chunk partials: groups of 8 consecutive chunks
  // (the last chunk of a group to finish sums it in chunk order), then the group sums in group
  // order (the last group to finish).  Elements four at a time: 32 loads in flight per thread.
  TINY_STAMP(3);
  const int ngroups = (t.nchunks + 7) / 8, grp = ch / 8, gsize = min(8, t.nchunks - grp * 8);
  unsigned int *tk = ticket + (size_t)slice * (ngroups + 1);
  float *gp = gpart + (size_t)slice * ngroups * E;
  if (threadIdx.x == 0) last = atomicAdd(tk + grp, 1u) == (unsigned)gsize - 1;
  __syncthreads();
  if (!last) return;
  __threadfence();
  const float *pg = part + ((size_t)slice * t.nchunks + grp * 8) * E;
  const int ne = nit * EI;
  for (int e0 = threadIdx.x; e0 < ne; e0 += 4 * TINY_THREADS) {
    float v[4][8];
#pragma unroll
    for (int a = 0; a < 4; ++a) {
      const int e = min(e0 + a * TINY_THREADS, ne - 1);
#pragma unroll
      for (int k = 0; k < 8; ++k) v[a][k] = __ldcg(pg + (size_t)min(k, gsize - 1) * E + e);
    }
#pragma unroll
    for (int a = 0; a < 4; ++a) {
      float s = 0.f;
#pragma unroll
      for (int k = 0; k < 8; ++k) s += k < gsize ? v[a][k] : 0.f;
      if (e0 + a * TINY_THREADS < ne) gp[(size_t)grp * E + e0 + a * TINY_THREADS] = s;
    }
  }
  __threadfence();
  __syncthreads();
  if (threadIdx.x == 0) {
    tk[grp] = 0u;   // re-arm for the next call on this workspace
    last = atomicAdd(tk + ngroups, 1u) == (unsigned)ngroups - 1;
  }
  __syncthreads();
  if (!last) return;
  __threadfence();
  for (int e0 = threadIdx.x; e0 < ne; e0 += 2 * TINY_THREADS) {
    float s[2] = {0.f, 0.f};
    for (int g0 = 0; g0 < ngroups; g0 += 16) {
      float v[2][16];
#pragma unroll
      for (int a = 0; a < 2; ++a) {
        const int e = min(e0 + a * TINY_THREADS, ne - 1);
#pragma unroll
        for (int k = 0; k < 16; ++k) v[a][k] = __ldcg(gp + (size_t)min(g0 + k, ngroups - 1) * E + e);
      }
#pragma unroll
      for (int a = 0; a < 2; ++a)
#pragma unroll
        for (int k = 0; k < 16; ++k) s[a] += g0 + k < ngroups ? v[a][k] : 0.f;
    }
#pragma unroll
    for (int a = 0; a < 2; ++a) {
      const int e = e0 + a * TINY_THREADS;
      if (e >= ne) break;
      const int item = it0 + e / EI, r = e % EI, kw = r / 4, j = r - kw * 4;
      const bool isdb = item >= nfil;
      if (isdb && (kw != 0 || !db)) continue;
      const int g = isdb ? item - nfil : item % t.G, co = 4 * g + j;
      if (co >= t.Co) continue;
      float *d;
      if (isdb) {
        d = db + co;
      } else {
        const int ck = item / t.G, c = ck / K, kh = ck - c * K;
        d = dw + (((size_t)co * t.C + c) * K + kh) * K + kw;
      }
      *d = accumulate ? *d + s[a] : s[a];
    }
  }
  if (threadIdx.x == 0) tk[ngroups] = 0u;
}

// ---- host-side configuration (shape-only: nothing here reads the device) ----
inline TinyCorr tiny_corr_config(const ConvGeom &g, int dgrad) {
  TinyCorr t;
  const int K = g.Kh;
  if (!dgrad) {
    t.Cin = g.C, t.Hin = g.H, t.Win = g.W, t.Cout = g.Co, t.Hout = g.Ho, t.Wout = g.Wo;
    t.pad = g.Ph, t.in_cs = g.xc, t.out_cs = g.yc;
  } else {
    t.Cin = g.Co, t.Hin = g.Ho, t.Win = g.Wo, t.Cout = g.C, t.Hout = g.H, t.Wout = g.W;
    t.pad = K - 1 - g.Ph, t.in_cs = g.yc, t.out_cs = g.xc;
  }
  t.Hp = t.Hout + K - 1;
  t.Wpp = tiny_rup4(tiny_rup4(t.Wout) + K - 1);
  const int groups = (t.Cout + 3) / 4, strips = t.Hout * (tiny_rup4(t.Wout) / 4);
  // >= 64 (strip, group) items per CTA where the plane is small, then input-channel phases up to
  // TINY_THREADS threads (shape-only; the result does not depend on gpc, only on R)
  t.gpc = std::min(groups, std::max(1, (64 + strips - 1) / strips));
  t.R = std::max(1, std::min(std::min(8, t.Cin), TINY_THREADS / (strips * t.gpc)));
  return t;
}
inline TinyWgrad tiny_wgrad_config(const ConvGeom &g, int target_units = 400) {
  TinyWgrad t;
  const int K = g.Kh;
  t.N = g.N, t.C = g.C, t.H = g.H, t.W = g.W, t.Co = g.Co, t.Ho = g.Ho, t.Wo = g.Wo, t.P = g.Ph;
  t.xc = g.xc, t.yc = g.yc;
  t.G = (g.Co + 3) / 4;
  t.items = g.C * K * t.G + t.G;
  t.islice = t.items <= 256 ? t.items : 64;
  t.nslices = (t.items + t.islice - 1) / t.islice;
  t.PH = std::max(1, std::min(8, TINY_THREADS / t.islice));
  // chunks: ~400 units in all; a chunk is part of one sample's rows, or whole samples
  const int target = std::max(1, target_units / t.nslices);
  if (target >= g.N) {
    t.spc = 1;
    t.rowchunks = std::min(g.Ho, std::max(1, target / g.N));
  } else {
    t.spc = (g.N + target - 1) / target;
    t.rowchunks = 1;
  }
  t.rows = (g.Ho + t.rowchunks - 1) / t.rowchunks;
  t.rowchunks = (g.Ho + t.rows - 1) / t.rows;
  t.nchunks = ((g.N + t.spc - 1) / t.spc) * t.rowchunks;
  t.Wpp = tiny_rup4(tiny_rup4(g.Wo) + K - 1);
  t.Wo4 = tiny_rup4(g.Wo);
  // x channels a slice touches: the span of (item / (K*G)) over islice consecutive items
  t.cspan = std::min(g.C, (t.islice + K * t.G - 2) / (K * t.G) + 1);
  return t;
}
inline size_t tiny_wgrad_ws_bytes(const TinyWgrad &t, int K) {
  const size_t E = (size_t)t.islice * K * 4;
  const size_t units = (size_t)t.nslices * t.nchunks, ngroups = (t.nchunks + 7) / 8;
  return 4 * (units * E + (size_t)t.nslices * ngroups * E) + 4 * (size_t)t.nslices * (ngroups + 1) + 1024;
}

}  // namespace glp
