// hfwd.cuh — forward pass of a unit-stride space-to-depth layer with a shared halo tile.
//
// y[n][co][h][w] = b[co] + sum_{t=(kh,kw)} sum_c x'[n][h+kh][w+kw][c] * W'[co][t][c]   (PAPER.md
// Alg. 1 P82-99, "im2col -> GEMM + bias"; north_star (3)), where x' is the packed space-to-depth
// input (an H' x W' image of one 64-channel bf16 atom per pixel, zero padded) and
// the output pixel (h, w) lives at row q = (n*H' + h)*W' + w of the flattened padded grid, so the
// A operand of tap t is the x' rows [q0 + s_t, q0 + s_t + 128) with s_t = kh*W' + kw.
//
// Why: the im2col forward re-reads x' from L2 once per tap (9x for CaffeNet conv1) on top of a
// 297 MB fp32 output; L2 traffic, not the tensor pipe, bounded it (~110 us; 77 us with the output
// stores skipped).  Here one TMA per tile stages the x' rows [q0, q0 + 128 + s_max) once; every
// tap's A operand is that smem tile read through a descriptor whose start is shifted by s_t rows
// (tcgen05 swizzles on absolute smem address bits, so any row shift is a valid SWIZZLE_128B
// K-major operand: tools/shift_probe.cu), and the whole B operand (W', <= 120 KB) is loaded once
// per CTA and stays resident.  L2 reads per tile: ~31 KB instead of ~200 KB.  Rows of the padded
// grid outside H_o x W_o are computed and dropped (CaffeNet conv1: 57^2 / 55^2 = 7 % extra MMA).
//
// CTA pairs (cluster of 2, tcgen05.mma.cta_group::2, M = 256): pair unit u covers tiles 2u and
// 2u + 1, one per CTA; each CTA keeps half of W' (bn/2 rows per tap) resident and stages its own
// tile's halo; the leader issues the MMAs for both (a single CTA ran M = 128, N = 96 MMAs at ~80
// cycles against ~56 per SM for the pair).  Persistent: unit u -> pair u mod (grid/2) (the paper's
// round-robin dispatch, P171).  CTA = 192 threads: warps 0-3 epilogue (TMEM -> bias -> NCHW fp32),
// warp 4 TMA producer, warp 5 TMEM owner + MMA issuer (leader); two TMEM accumulators so the
// epilogue of unit i overlaps unit i+1.
#pragma once
#include "common.cuh"
#include "ptx.cuh"

namespace glp {

constexpr int HF_THREADS = 320;   // + warps 6-9: a second epilogue group (alternate 32-column chunks)
constexpr int HF_MAXTAPS = 16;

struct HfwdParams {
  int taps;
  int shift[HF_MAXTAPS];   // row shift s_t = kh*W' + kw of tap t (t = kh*Ks + kw)
  int bn;                  // N = C_o rounded up to 16 (<= 256): one tile covers every channel
  int co;                  // valid output channels
  int acc_cols;            // TMEM columns per accumulator
  int tmem_cols;           // allocation (power of two >= 2 * acc_cols)
  int halo_rows;           // 128 + max shift
  int a_bytes;             // one halo stage (1024-aligned)
  int b_tap_bytes;         // one tap's B block of this CTA: bn/2 rows x 128 B (1024-aligned)
  int stages;
  int tiles;               // ceil(rows / 128)
  int units;               // ceil(tiles / 2): CTA-pair work units
  int rows;                // N * H' * W'
  FastDiv div_img, div_w;  // H' * W', W'
  int ho, wo;              // valid output region of each H' x W' image
  float *out;              // y NCHW fp32
  int out_c;               // channels per image of y (all groups' channels)
  int out_hw;              // H_o * W_o
  const float *bias;       // may be null
  int bias_floats;         // >= bn, multiple of 4
  int dbg_skip;            // diagnostics (GLP_DEBUG_SKIP): bit0 skip x' loads, bit2 MMAs, bit3 stores
};

__global__ void __launch_bounds__(HF_THREADS, 1)
    hfwd_kernel(const __grid_constant__ HfwdParams p, const __grid_constant__ CUtensorMap tmapX,
                const __grid_constant__ CUtensorMap tmapW) {
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t base = (raw + 1023u) & ~1023u;
  const uint32_t sB = base;                                        // taps x [bn rows x 128 B]
  const uint32_t sA0 = sB + (uint32_t)(p.taps * p.b_tap_bytes);    // stages x halo tiles
  const uint32_t bars = sA0 + (uint32_t)(p.stages * p.a_bytes);
  const int S_ = p.stages;
  auto full = [&](int s) { return bars + 8u * s; };
  auto empty = [&](int s) { return bars + 8u * (S_ + s); };
  auto tfull = [&](int a) { return bars + 8u * (2 * S_ + a); };
  auto tempty = [&](int a) { return bars + 8u * (2 * S_ + 2 + a); };
  const uint32_t bfull = bars + 8u * (2 * S_ + 4);
  const uint32_t tmem_slot = bars + 8u * (2 * S_ + 5);
  const uint32_t sbias = (tmem_slot + 16u + 15u) & ~15u;
  volatile uint32_t *tmem_slot_ptr =
      reinterpret_cast<volatile uint32_t *>(smem_raw + (tmem_slot - raw));
  const int warp = __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0);
  const int lane = threadIdx.x & 31;
  const uint32_t rank = blockIdx.x & 1u;   // CTA in the pair
  const bool leader = rank == 0;
  if (threadIdx.x == 0) {
    // full / bfull: armed by the leader only (both CTAs' bytes); empty / tfull: one multicast
    // commit; tempty: the 8 epilogue warps of both CTAs arrive on the leader's barrier
    for (int s = 0; s < S_; ++s) {
      mbar_init(full(s), 1);
      mbar_init(empty(s), 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(tfull(a), 1);
      mbar_init(tempty(a), 16);   // 8 epilogue warps per CTA, both CTAs
    }
    mbar_init(bfull, 1);
    fence_mbar_init();
  }
  if (warp == 5) {
    tmem_alloc_cg<2>(tmem_slot, (uint32_t)p.tmem_cols);
    tmem_relinquish_cg<2>();
  }
  if (warp == 4 && lane == 0) {
    tma_prefetch(&tmapX);
    tma_prefetch(&tmapW);
  }
  tc_fence_before();
  cluster_sync();
  tc_fence_after();
  pdl_wait();
  const uint32_t tmem_base = __shfl_sync(0xffffffffu, *tmem_slot_ptr, 0);
  const int unit0 = (int)(blockIdx.x >> 1), ustep = (int)(gridDim.x >> 1);

  if (warp == 4) {
    // ===================================== producer ========================================
    // B once: this CTA's half (rows rank*bn/2 ...) of tap t's K slice [t*64, t*64 + 64) of W'
    // (rows >= C_o zero-filled); completes on the leader's barrier
    const int half = p.bn / 2;
    if (leader) mbar_arrive_expect_tx_e(bfull, (uint32_t)(2 * p.taps * half * 128));
    for (int t = 0; t < p.taps; ++t)
      tma_load_2d_cg2_e(sB + (uint32_t)(t * p.b_tap_bytes), &tmapW, mapa_shared(bfull, 0), t * 64,
                        (int)rank * half);
    const bool la = !GLP_SKIP(p, 1);
    const uint32_t tx = la ? (uint32_t)(2 * p.halo_rows * 128) : 0u;
    int rs = 0;
    uint32_t rph = 0;
    for (int u = unit0; u < p.units; u += ustep) {
      const int tile = 2 * u + (int)rank;   // past the last tile: rows past the end -> zeros
      mbar_wait(empty(rs), rph ^ 1u);
      const uint32_t sA = sA0 + (uint32_t)(rs * p.a_bytes);
      if (leader) mbar_arrive_expect_tx_e(full(rs), tx);
      if (la) tma_load_2d_cg2_e(sA, &tmapX, mapa_shared(full(rs), 0), 0, tile * 128);
      if (++rs == S_) {
        rs = 0;
        rph ^= 1u;
      }
    }
  } else if (warp == 5 && leader) {
    // ===================================== MMA issuer ======================================
    const uint32_t idesc = make_idesc(1u, 0u, 0u, 256u, (uint32_t)p.bn);
    mbar_wait(bfull, 0);
    int rs = 0;
    uint32_t rph = 0, it = 0;
    const bool skip_mma = GLP_SKIP(p, 4);
    for (int u = unit0; u < p.units; u += ustep, ++it) {
      const uint32_t a = it & 1u, aph = (it >> 1) & 1u;
      mbar_wait(tempty(a), aph ^ 1u);
      tc_fence_after();
      mbar_wait(full(rs), rph);
      tc_fence_after();
      const uint32_t sA = sA0 + (uint32_t)(rs * p.a_bytes);
      const uint32_t d = tmem_base + a * (uint32_t)p.acc_cols;
      for (int t = 0; t < p.taps; ++t) {
        if (skip_mma && t > 0) break;
        // K-major SW128 operands: 8-row groups of 128-byte rows (SBO 1024); 4 MMAs of K = 16
        // advance the start by 32 bytes (2 descriptor units)
        const uint64_t da = make_sdesc(sA + (uint32_t)p.shift[t] * 128u, 16u, 1024u, 2u);
        const uint64_t db = make_sdesc(sB + (uint32_t)(t * p.b_tap_bytes), 16u, 1024u, 2u);
        mma_kblock_e<0, 2, 4, 2>(d, da, db, idesc, t > 0 ? 1u : 0u);
      }
      mma_commit_e<2>(empty(rs));
      mma_commit_e<2>(tfull(a));
      if (++rs == S_) {
        rs = 0;
        rph ^= 1u;
      }
    }
    __syncwarp();
  } else if (warp < 4 || warp >= 6) {
    // ===================================== epilogue ========================================
    // two groups of 4 warps (0-3 and 6-9): warp w drains TMEM lanes 32*(w % 4)..+31; group 0 takes
    // the 32-column chunks 0, 2, 4, ..., group 1 the odd ones, so twice the stores are in flight
    const int grp = warp >= 6 ? 1 : 0;
    const int quad = warp & 3;
    const int row = quad * 32 + lane;
    for (int i = row + 128 * grp; i < p.bias_floats; i += 256)
      sts_f32(sbias + 4u * (uint32_t)i, (p.bias != nullptr && i < p.co) ? __ldg(p.bias + i) : 0.f);
    named_bar_sync(1, 256);
    const size_t plane = (size_t)p.out_hw;
    uint32_t it = 0;
    for (int u = unit0; u < p.units; u += ustep, ++it) {
      const uint32_t a = it & 1u, aph = (it >> 1) & 1u;
      mbar_wait(tfull(a), aph);
      tc_fence_after();
      const int tile = 2 * u + (int)rank;
      const int q = tile * 128 + row;
      uint32_t n = 0, rem = 0, h = 0, w = 0;
      p.div_img.divmod((uint32_t)min(q, p.rows - 1), n, rem);
      p.div_w.divmod(rem, h, w);
      const bool mv = q < p.rows && (int)h < p.ho && (int)w < p.wo && !GLP_SKIP(p, 8);
      float *ob = p.out + (size_t)n * p.out_c * plane + (size_t)h * p.wo + w;
      const uint32_t taddr = tmem_base + ((uint32_t)(quad * 32) << 16) + a * (uint32_t)p.acc_cols;
      auto store_chunk = [&](int c0, uint32_t (&v)[32]) {
        if (!mv) return;
        const int lim = min(32, p.co - c0);
        float *o = ob + (size_t)c0 * plane;
        if (lim == 32) {
#pragma unroll
          for (int k = 0; k < 32; k += 4) {
            const float4 b4 = lds_f32x4(sbias + 4u * (uint32_t)(c0 + k));
            o[0] = __uint_as_float(v[k]) + b4.x;
            o += plane;
            o[0] = __uint_as_float(v[k + 1]) + b4.y;
            o += plane;
            o[0] = __uint_as_float(v[k + 2]) + b4.z;
            o += plane;
            o[0] = __uint_as_float(v[k + 3]) + b4.w;
            o += plane;
          }
        } else {
#pragma unroll
          for (int k = 0; k < 32; ++k)
            if (k < lim) o[(size_t)k * plane] = __uint_as_float(v[k]) + lds_f32(sbias + 4u * (uint32_t)(c0 + k));
        }
      };
      uint32_t va[32];
      for (int c0 = 32 * grp; c0 < p.bn; c0 += 64) {
        tmem_ld32(taddr + (uint32_t)c0, va);
        tmem_wait_ld_dep(va);
        store_chunk(c0, va);
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) mbar_arrive_cluster_relaxed(mapa_shared(tempty(a), 0));
    }
  }
  pdl_launch_dependents();
  tc_fence_before();
  cluster_sync();
  tc_fence_after();
  if (warp == 5) tmem_dealloc_cg<2>(tmem_base, (uint32_t)p.tmem_cols);
}

}  // namespace glp
