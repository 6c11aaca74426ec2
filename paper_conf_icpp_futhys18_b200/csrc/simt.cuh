// simt.cuh — GLP_MATH_FP32 path: fp32 CUDA-core direct convolution (the accuracy anchor,
// normwise error <= 1e-5 vs the fp64 oracle) and the deterministic split reductions shared by
// both math paths.  Every output element is produced by exactly one thread in a fixed order.
#pragma once
#include <cstdint>

#include "common.cuh"

namespace glp {

struct ConvGeom {
  int N, C, H, W, Co, Kh, Kw, Sh, Sw, Ph, Pw, Ho, Wo;
  int xc, yc;   // channels per image of the x/dx and y/dy tensors (> C, Co for a conv group)
};

// y[n,co,ho,wo] = b[co] + sum_{ci,kh,kw} W * x  (Alg. 1, P82-99).  One thread per output.
__global__ void simt_fwd(ConvGeom g, const float *__restrict__ x, const float *__restrict__ w,
                         const float *__restrict__ b, float *__restrict__ y) {
  const size_t total = (size_t)g.N * g.Co * g.Ho * g.Wo;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < total;
       i += (size_t)gridDim.x * blockDim.x) {
    const int wo = (int)(i % g.Wo);
    size_t r = i / g.Wo;
    const int ho = (int)(r % g.Ho);
    r /= g.Ho;
    const int co = (int)(r % g.Co);
    const int n = (int)(r / g.Co);
    float acc = 0.f;
    for (int ci = 0; ci < g.C; ++ci) {
      const float *xc = x + ((size_t)n * g.xc + ci) * g.H * g.W;
      const float *wc = w + ((size_t)co * g.C + ci) * g.Kh * g.Kw;
      for (int kh = 0; kh < g.Kh; ++kh) {
        const int ih = ho * g.Sh - g.Ph + kh;
        if (ih < 0 || ih >= g.H) continue;
        for (int kw = 0; kw < g.Kw; ++kw) {
          const int iw = wo * g.Sw - g.Pw + kw;
          if (iw < 0 || iw >= g.W) continue;
          acc = fmaf(__ldg(wc + kh * g.Kw + kw), __ldg(xc + (size_t)ih * g.W + iw), acc);
        }
      }
    }
    if (b) acc += __ldg(b + co);
    y[(((size_t)n * g.yc + co) * g.Ho + ho) * g.Wo + wo] = acc;
  }
}

// dx[n,ci,h,w] = sum over (co,kh,kw) with ho*S-P+kh == h, wo*S-P+kw == w of W * dy (Alg. 2):
// the col2im gather; one thread per dx element, no atomics.
__global__ void simt_dgrad(ConvGeom g, const float *__restrict__ dy, const float *__restrict__ w,
                           float *__restrict__ dx) {
  const size_t total = (size_t)g.N * g.C * g.H * g.W;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < total;
       i += (size_t)gridDim.x * blockDim.x) {
    const int iw = (int)(i % g.W);
    size_t r = i / g.W;
    const int ih = (int)(r % g.H);
    r /= g.H;
    const int ci = (int)(r % g.C);
    const int n = (int)(r / g.C);
    float acc = 0.f;
    for (int co = 0; co < g.Co; ++co) {
      const float *dyc = dy + ((size_t)n * g.yc + co) * g.Ho * g.Wo;
      const float *wc = w + ((size_t)co * g.C + ci) * g.Kh * g.Kw;
      for (int kh = 0; kh < g.Kh; ++kh) {
        const int hn = ih + g.Ph - kh;
        if (hn < 0 || hn % g.Sh) continue;
        const int ho = hn / g.Sh;
        if (ho >= g.Ho) continue;
        for (int kw = 0; kw < g.Kw; ++kw) {
          const int wn = iw + g.Pw - kw;
          if (wn < 0 || wn % g.Sw) continue;
          const int wo = wn / g.Sw;
          if (wo >= g.Wo) continue;
          acc = fmaf(__ldg(wc + kh * g.Kw + kw), __ldg(dyc + (size_t)ho * g.Wo + wo), acc);
        }
      }
    }
    dx[(((size_t)n * g.xc + ci) * g.H + ih) * g.W + iw] = acc;
  }
}

// Split partials of dW: part[s][co][ci][kh][kw] = sum over pixels q in split s (q = n*HoWo+p,
// fixed contiguous ranges of `chunk` pixels) of dy * x.  One thread per (s, dW element).
__global__ void simt_wgrad_partial(ConvGeom g, const float *__restrict__ x,
                                   const float *__restrict__ dy, float *__restrict__ part,
                                   int splits, int chunk) {
  const size_t wsz = (size_t)g.Co * g.C * g.Kh * g.Kw;
  const size_t total = wsz * splits;
  const int hw = g.Ho * g.Wo;
  const long long npix = (long long)g.N * hw;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < total;
       i += (size_t)gridDim.x * blockDim.x) {
    const int s = (int)(i / wsz);
    const size_t e = i % wsz;
    const int kw = (int)(e % g.Kw);
    size_t r = e / g.Kw;
    const int kh = (int)(r % g.Kh);
    r /= g.Kh;
    const int ci = (int)(r % g.C);
    const int co = (int)(r / g.C);
    float acc = 0.f;
    const long long q0 = (long long)s * chunk;
    const long long q1 = q0 + chunk < npix ? q0 + chunk : npix;
    for (long long q = q0; q < q1; ++q) {
      const int n = (int)(q / hw), p = (int)(q % hw);
      const int ho = p / g.Wo, wo = p % g.Wo;
      const int ih = ho * g.Sh - g.Ph + kh, iw = wo * g.Sw - g.Pw + kw;
      if (ih < 0 || ih >= g.H || iw < 0 || iw >= g.W) continue;
      acc = fmaf(__ldg(dy + ((size_t)n * g.yc + co) * hw + p),
                 __ldg(x + (((size_t)n * g.xc + ci) * g.H + ih) * g.W + iw), acc);
    }
    part[i] = acc;
  }
}

// db partials for the SIMT path: part[s][co] over the same pixel ranges.
__global__ void simt_db_partial(ConvGeom g, const float *__restrict__ dy, float *__restrict__ part,
                                int splits, int chunk) {
  const int hw = g.Ho * g.Wo;
  const long long npix = (long long)g.N * hw;
  const size_t total = (size_t)splits * g.Co;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < total;
       i += (size_t)gridDim.x * blockDim.x) {
    const int s = (int)(i / g.Co), co = (int)(i % g.Co);
    float acc = 0.f;
    const long long q0 = (long long)s * chunk;
    const long long q1 = q0 + chunk < npix ? q0 + chunk : npix;
    for (long long q = q0; q < q1; ++q) {
      const int n = (int)(q / hw), p = (int)(q % hw);
      acc += __ldg(dy + ((size_t)n * g.yc + co) * hw + p);
    }
    part[i] = acc;
  }
}

// Fixed-order sum of `cnt` partials strided by `stride`: sequential within blocks of 8, block sums
// added in block order.  The order is a function of cnt only (shape), never of the grid or S.
__device__ __forceinline__ float pairwise_sum(const float *__restrict__ p, int cnt, size_t stride) {
  float tot = 0.f;
  for (int b0 = 0; b0 < cnt; b0 += 8) {
    float a = 0.f;
    const int e = b0 + 8 < cnt ? b0 + 8 : cnt;
#pragma unroll 8
    for (int k = b0; k < e; ++k) a += __ldg(p + (size_t)k * stride);
    tot += a;
  }
  return tot;
}

// dW (Caffe layout) from SIMT partials part[s][dW element].
__global__ void reduce_simt_dw(const float *__restrict__ part, float *__restrict__ dw, size_t wsz,
                               int splits, int accumulate) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < wsz;
       i += (size_t)gridDim.x * blockDim.x) {
    const float s = pairwise_sum(part + i, splits, wsz);
    dw[i] = accumulate ? dw[i] + s : s;
  }
}

// dW (Caffe layout [co][ci][kh][kw]) from tensor-core partials part[s][tap*Cp + ci][co]
// (leading dimension ld, mpad rows per split), summed in split order.
// s2d > 1: partial rows are in the space-to-depth geometry (stride s2d, Ks = ceil(Kw/s2d)):
// row = ((kh/S)*Ks + kw/S)*Cp + ((kh%S)*S + kw%S)*C + ci.
// Block (32, 8) per tile of 32 output channels x 32 inner dW indices (i = ci*taps + t): warps read
// 32 consecutive co of one partial row per split (coalesced), the tile is transposed through
// shared memory, and dW[co][i] is written 32 consecutive i at a time.  grid (ceil(C*taps/32),
// ceil(Co/32), leaves).  Leaf plans (the deterministic exchange): blockIdx.z = leaf, `splits` are
// that leaf's splits (partials leaf*splits ...), and its dW goes leaf_stride floats further.
struct DwRed {   // arguments of the dW reductions
  const float *part;
  BrOut dw;
  int Co, C, taps, Kw, Cp, ld, mpad, splits, accumulate, s2d, Ks;
  long long leaf_stride;
};
__device__ __forceinline__ void reduce_tc_dw_body(const DwRed &r, int bx, int by, int bz) {
  __shared__ float tile[32][33];
  const float *part = r.part + (size_t)bz * r.splits * ((size_t)r.mpad * r.ld);
  const BrOut &dw = r.dw;
  const int Co = r.Co, C = r.C, taps = r.taps, Kw = r.Kw, Cp = r.Cp, ld = r.ld, mpad = r.mpad;
  const int splits = r.splits, accumulate = r.accumulate, s2d = r.s2d, Ks = r.Ks;
  const long long leaf_stride = r.leaf_stride;
  const int inner = C * taps;
  const int i0 = bx * 32, co0 = by * 32;
  const int lane = threadIdx.x & 31, ty = threadIdx.x >> 5;
  const size_t sstride = (size_t)mpad * ld;
  const float *src[4];
  bool ok[4];
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    const int i = i0 + ty + 8 * u, co = co0 + lane;
    ok[u] = i < inner && co < Co;
    int row = 0;
    if (ok[u]) {
      const int ci = i / taps, t = i - ci * taps;
      row = t * Cp + ci;
      if (s2d > 1) {
        const int kh = t / Kw, kw = t % Kw;
        row = ((kh / s2d) * Ks + kw / s2d) * Cp + ((kh % s2d) * s2d + kw % s2d) * C + ci;
      }
    }
    src[u] = part + (size_t)row * ld + (ok[u] ? co : 0);
  }
  // fixed order: splits summed sequentially in blocks of 8, block sums in block order (same for
  // every element; 32 independent loads in flight per batch)
  // all 32 loads of a batch issued before any add (the guarded load-add chain let the compiler
  // serialise them: ncu 34 % warps active, 13 % L2 throughput).  Out-of-range entries add +0.0f
  // to a batch sum that starts at +0.0f, which changes no bit, so the order is as before.
  // The loads are unconditional (split index clamped to the last split, rows outside the layer
  // read row 0) and the out-of-range values zeroed afterwards: the predicated loads of the
  // earlier form were interleaved with the adds by the compiler (3-6 loads in flight; a tiny layer
  // with 72 splits spent 42 us here).
  float tot[4] = {0.f, 0.f, 0.f, 0.f};
  for (int b0 = 0; b0 < splits; b0 += 8) {
    float v[8][4];
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const size_t off = (size_t)min(b0 + k, splits - 1) * sstride;
#pragma unroll
      for (int u = 0; u < 4; ++u) v[k][u] = __ldg(src[u] + off);
    }
#pragma unroll
    for (int k = 0; k < 8; ++k)
#pragma unroll
      for (int u = 0; u < 4; ++u)
        if (b0 + k >= splits || !ok[u]) v[k][u] = 0.f;
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      float a = 0.f;
#pragma unroll
      for (int k = 0; k < 8; ++k) a += v[k][u];
      tot[u] += a;
    }
  }
#pragma unroll
  for (int u = 0; u < 4; ++u) tile[ty + 8 * u][lane] = tot[u];
  __syncthreads();
  for (int j = ty; j < 32; j += 8) {
    const int co = co0 + j, i = i0 + lane;
    if (co < Co && i < inner) {
      float *d = dw.at(co, 0, (size_t)inner, (size_t)i) + bz * leaf_stride;
      const float v = tile[lane][j];
      *d = accumulate ? *d + v : v;
    }
  }
}

// Many-split variant (the halo filter gradient's 148 one-per-CTA partials, and small filters whose
// 32 x 32 tiles would leave most SMs idle): block = 32 channels x 8 split phases over 4 weight
// rows; thread (ty, lane) sums splits ty, ty+8, ... in ascending order, then the 8 phase sums are
// added in phase order.  Fixed order, a function of `splits` only.  Leaf plans: blockIdx.z = leaf.
__device__ __forceinline__ void reduce_tc_dw_wide_body(const DwRed &rr, int bx, int by, int bz) {
  __shared__ float red[8][4][33];
  const float *part = rr.part + (size_t)bz * rr.splits * ((size_t)rr.mpad * rr.ld);
  const BrOut &dw = rr.dw;
  const int Co = rr.Co, C = rr.C, taps = rr.taps, Kw = rr.Kw, Cp = rr.Cp, ld = rr.ld, mpad = rr.mpad;
  const int splits = rr.splits, accumulate = rr.accumulate, s2d = rr.s2d, Ks = rr.Ks;
  const long long leaf_stride = rr.leaf_stride;
  const int inner = C * taps;
  const int i0 = bx * 4, co = by * 32 + (threadIdx.x & 31), ty = threadIdx.x >> 5;
  const size_t sstride = (size_t)mpad * ld;
  const float *src[4];
  bool ok[4];
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    const int i = i0 + u;
    ok[u] = i < inner && co < Co;
    int row = 0;
    if (ok[u]) {
      const int ci = i / taps, t = i - ci * taps;
      row = t * Cp + ci;
      if (s2d > 1) {
        const int kh = t / Kw, kw = t % Kw;
        row = ((kh / s2d) * Ks + kw / s2d) * Cp + ((kh % s2d) * s2d + kw % s2d) * C + ci;
      }
    }
    src[u] = part + (size_t)row * ld + (ok[u] ? co : 0);
  }
  // splits ty, ty+8, ... added in ascending order; eight of them (32 loads) issued per batch,
  // unconditionally (clamped split index), out-of-range values zeroed after the loads
  float a[4] = {0.f, 0.f, 0.f, 0.f};
  for (int sp0 = ty; sp0 < splits; sp0 += 64) {
    float v[8][4];
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const size_t off = (size_t)min(sp0 + 8 * k, splits - 1) * sstride;
#pragma unroll
      for (int u = 0; u < 4; ++u) v[k][u] = __ldg(src[u] + off);
    }
#pragma unroll
    for (int k = 0; k < 8; ++k)
#pragma unroll
      for (int u = 0; u < 4; ++u)
        if (sp0 + 8 * k < splits && ok[u]) a[u] += v[k][u];
  }
#pragma unroll
  for (int u = 0; u < 4; ++u) red[ty][u][threadIdx.x & 31] = a[u];
  __syncthreads();
  if (ty < 4) {
    const int u = ty, lane = threadIdx.x & 31;
    float t = 0.f;
#pragma unroll
    for (int k = 0; k < 8; ++k) t += red[k][u][lane];
    const int i = i0 + u;
    if (i < inner && co < Co) {
      float *d = dw.at(co, 0, (size_t)inner, (size_t)i) + bz * leaf_stride;
      *d = accumulate ? *d + t : t;
    }
  }
}

// db[co] = sum over `rows` partial rows of part[row][co] (rows = N * pixel tiles, or SIMT splits),
// deterministic and parallel over G = db_groups(rows) row groups: block (channel block x, group g)
// sums rows g, g+G, ... (thread ty takes every 8th of those, lanes = channels, coalesced), reduces
// its 8 warps in a fixed tree, and stores part2[g][co]; the last block to finish for a channel
// block (atomic ticket) sums part2[0..G) in index order.  The order depends only on `rows` (a
// shape quantity), never on the grid size, S or timing.
constexpr int DB_GROUPS = 128;   // the largest group count (multiple of 4)
// Row groups of a db reduction over `rows` partial rows: ~32 rows per group, 4..DB_GROUPS, a
// multiple of 4 -- a function of the row count only (small layers spent ~10 us in 128 nearly
// empty groups plus the ticket pass).
__host__ __device__ constexpr int db_groups(int rows) {
  const int g = ((rows + 31) / 32 + 3) / 4 * 4;
  return g < 4 ? 4 : (g > DB_GROUPS ? DB_GROUPS : g);
}
// Leaf plans: blockIdx.z = leaf; its `rows` partial rows follow the previous leaves', its group sums
// and tickets have their own slices, and its db goes leaf_stride floats further.
struct DbRed {   // arguments of the db reduction
  const float *part;
  BrOut db;
  int Co, rows, accumulate;
  float *part2;
  unsigned int *tickets;
  long long leaf_stride;
  int G, cx;   // row groups (db_groups(rows)) and channel blocks (ceil(Co/32))
};
// block (bx = channel block, g = row group, bz = leaf)
__device__ __forceinline__ void reduce_db_body(const DbRed &r, int bx, int g, int bz) {
  __shared__ float red[8][33];
  __shared__ bool last;
  const int Co = r.Co, rows = r.rows, accumulate = r.accumulate, G = r.G;
  const BrOut &db = r.db;
  const long long leaf_stride = r.leaf_stride;
  const float *part = r.part + (size_t)bz * rows * Co;
  float *part2 = r.part2 + (size_t)bz * DB_GROUPS * Co;
  unsigned int *tickets = r.tickets + (size_t)bz * r.cx;
  const int lane = threadIdx.x & 31, ty = threadIdx.x >> 5;
  const int co = bx * 32 + lane;
  // rows g + DB_GROUPS*(ty + 8*j), j = 0, 1, ...: four interleaved accumulators (j mod 4) keep
  // four loads in flight (one dependent chain was latency-bound: ~47 L2 round trips for CaffeNet
  // conv1), the tail goes to a0, then ((a0+a1)+(a2+a3)) — an order fixed by `rows` alone
  float a = 0.f;
  if (co < Co) {
    const int STEP = G * 8;
    float a0 = 0.f, a1 = 0.f, a2 = 0.f, a3 = 0.f;
    int r = g + G * ty;
    const float *pc = part + co;
    for (; r + 3 * STEP < rows; r += 4 * STEP) {
      const float v0 = __ldg(pc + (size_t)r * Co), v1 = __ldg(pc + (size_t)(r + STEP) * Co);
      const float v2 = __ldg(pc + (size_t)(r + 2 * STEP) * Co), v3 = __ldg(pc + (size_t)(r + 3 * STEP) * Co);
      a0 += v0;
      a1 += v1;
      a2 += v2;
      a3 += v3;
    }
    for (; r < rows; r += STEP) a0 += __ldg(pc + (size_t)r * Co);
    a = (a0 + a1) + (a2 + a3);
  }
  red[ty][lane] = a;
  __syncthreads();
  if (ty == 0) {
    const float s = ((red[0][lane] + red[1][lane]) + (red[2][lane] + red[3][lane])) +
                    ((red[4][lane] + red[5][lane]) + (red[6][lane] + red[7][lane]));
    if (co < Co) part2[(size_t)g * Co + co] = s;
    __threadfence();
  }
  __syncthreads();
  if (threadIdx.x == 0) last = (atomicAdd(tickets + bx, 1u) == (unsigned)G - 1);
  __syncthreads();
  if (last && ty == 0) {
    __threadfence();
    if (co < Co) {
      // group sums in index order, four strided accumulators (k mod 4), then combined in order
      float s0 = 0.f, s1 = 0.f, s2 = 0.f, s3 = 0.f;
#pragma unroll 4
      for (int k = 0; k < G; k += 4) {
        s0 += __ldcg(part2 + (size_t)k * Co + co);
        s1 += __ldcg(part2 + (size_t)(k + 1) * Co + co);
        s2 += __ldcg(part2 + (size_t)(k + 2) * Co + co);
        s3 += __ldcg(part2 + (size_t)(k + 3) * Co + co);
      }
      const float s = (s0 + s1) + (s2 + s3);
      float *d = db.at(co, 0, 1, 0) + bz * leaf_stride;
      *d = accumulate ? *d + s : s;
    }
    if (lane == 0) tickets[bx] = 0;   // re-arm for the next call on this workspace
  }
}

// Kernels.  reduce_tc_dw: grid (ceil(C*taps/32), ceil(Co/32), leaves); reduce_tc_dw_wide: grid
// (ceil(C*taps/4), ceil(Co/32), leaves); reduce_db: grid (ceil(Co/32), G, leaves); block 256.
// reduce_wgrad<WIDE>: the dW reduction and the db reduction in ONE launch (one node fewer on the
// filter-gradient chain), grid (nA + cx * G, 1, leaves): blocks < nA = ax * ay are dW blocks
// (bx = b % ax, by = b / ax), the rest db blocks -- the same bodies, the same per-element order.
__global__ void __launch_bounds__(256) reduce_tc_dw(const DwRed r) {
  pdl_launch_dependents();
  pdl_wait();
  reduce_tc_dw_body(r, blockIdx.x, blockIdx.y, blockIdx.z);
}
__global__ void __launch_bounds__(256) reduce_tc_dw_wide(const DwRed r) {
  pdl_launch_dependents();
  pdl_wait();
  reduce_tc_dw_wide_body(r, blockIdx.x, blockIdx.y, blockIdx.z);
}
__global__ void __launch_bounds__(256) reduce_db(const DbRed r) {
  pdl_launch_dependents();
  pdl_wait();
  reduce_db_body(r, blockIdx.x, blockIdx.y, blockIdx.z);
}
template <int WIDE>
__global__ void __launch_bounds__(256) reduce_wgrad(const DwRed r, const DbRed q, int ax, int ay) {
  pdl_launch_dependents();
  pdl_wait();
  const int b = blockIdx.x, nA = ax * ay;
  if (b < nA) {
    if (WIDE) reduce_tc_dw_wide_body(r, b % ax, b / ax, blockIdx.z);
    else reduce_tc_dw_body(r, b % ax, b / ax, blockIdx.z);
  } else {
    const int bd = b - nA;
    reduce_db_body(q, bd % q.cx, bd / q.cx, blockIdx.z);
  }
}

}  // namespace glp
