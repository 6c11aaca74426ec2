// hwgrad.cuh — filter gradient of a unit-stride (space-to-depth) layer with a shared halo tile.
//
// dW'[t][c][co] = sum_p x'[p + s_t][c] * dy[p][co]   (PAPER.md P129; north_star (3): "backward-
// filter GEMMs summed over the samples of a batch"), where p runs over the flattened padded grid
// of the packed operands (n, h, w) in [0,N) x [0,H') x [0,W') with H' x W' the space-to-depth
// image, s_t = kh*W' + kw is the row shift of tap t = (kh, kw), and dy is packed
// on the same H' x W' grid with zeros outside its H_o x W_o valid region (junk positions, so
// they contribute nothing).
//
// Why: the im2col filter gradient re-reads x once per tap from L2 (9x for CaffeNet conv1's 3x3
// s2d taps) and was L2-bandwidth bound (45 B/clk/SM measured, 373 TFLOP/s).  Here one TMA per
// k-block stages the x' rows [p0, p0 + BKP + s_max] once; the A operand of every tap is the same
// smem tile read through a descriptor whose start is shifted by s_t rows.  tcgen05 applies the
// 128-byte swizzle on absolute smem address bits, so any row shift is a valid SWIZZLE_128B
// operand (measured exactly: tools/shift_probe.cu).  One M = 128 MMA covers a pair of taps: the
// two 64-channel MN-major atoms of A are the tile at shifts s_a and s_b (LBO = (s_b - s_a) rows).
//
// Work: the N*H'*W' pixel rows are cut into `splits` contiguous ranges (shape-only count); CTA u
// accumulates all tap pairs x C_o of its range in TMEM (n_acc accumulators) and writes one fp32
// partial [u][t*64 + c][co]; reduce_tc_dw sums the partials in a fixed order (deterministic,
// independent of the grid and of S: convergence invariance, P264).
// CTA = 192 threads: warps 0-3 epilogue, warp 4 TMA producer, warp 5 TMEM owner + MMA issuer.
#pragma once
#include "common.cuh"
#include <cuda_bf16.h>

#include "ptx.cuh"

namespace glp {

constexpr int HW_THREADS = 192;
// fused-dy variant with NCG groups of 4 dy-building warps (warps 0-3, then 6-9, 10-13): group g
// builds k-blocks kb0 + g, kb0 + g + NCG, ... so NCG k-blocks' loads are in flight at once
// NCG = 1: one builder group (warps 0-3) whose loads land in shared memory by cp.async (two fp32
// landing buffers of 128 pixels x bn channels), so the loads in flight are not bounded by registers
__host__ __device__ constexpr int hw_threads(int ncg) { return ncg > 1 ? 192 + 128 * (ncg - 1) : 192; }
constexpr int HW_BKP = 128;   // pixel rows (K) per k-block

struct HwgradParams {
  int n_acc;          // accumulators = ceil(taps / 2) tap pairs
  int tap_a[8], tap_b[8];   // taps of the two 64-channel atoms of accumulator j (a < b)
  int shift_a[8], shift_b[8];
  int dup_a_mask;     // bit j: atom a of pair j duplicates an earlier pair (odd tap count)
  int bn;             // C_o tile (multiple of 16, <= 256): all output channels
  int acc_cols;       // TMEM columns per accumulator (multiple of 32)
  int tmem_cols;      // allocation (power of two >= n_acc * acc_cols)
  int halo_rows;      // rows of the x' tile per k-block (BKP + max shift)
  int a_bytes, b_bytes, stages;
  int kb_total, kb_per_split, splits;
  int cpx;            // channels of x' (64: one atom)
  int co;             // valid output channels
  float *part;        // [splits][mpad][ld] fp32
  int mpad, ld;
  int dbg_skip;       // diagnostics (GLP_DEBUG_SKIP): bit0 skip x' loads, bit1 dy loads, bit2 MMAs
  // fused-dy variant (FDY): warps 0-3 build the dy operand of every k-block from the fp32 NCHW
  // tensor themselves (round to bf16, swizzled smem stores) and emit the db partials, so the
  // separate dy pack (read 4 B + write 2 B per element, then re-read 2 B here) disappears
  const float *dy;    // NCHW fp32 (channel stride ho*wo, image stride dy_c*ho*wo)
  int dy_c, ho, wo;   // channels per image of the dy tensor; valid output region
  int rows;           // N * H' * W' (flattened padded grid)
  FastDiv div_img, div_w;   // H' * W', W'
  float *db_part;     // [splits][co]: this CTA's db partial (fixed order)
  unsigned int *db_tickets;   // reduce_db's completion tickets (armed here: no dy pack runs)
  int n_tickets;
};

template <int NCG>   // 0: dy packed in the workspace (TMA); 1: fused dy through a cp.async landing
                     // zone; 2 or 3: fused dy, NCG register-staged builder groups
__global__ void __launch_bounds__(hw_threads(NCG), 1)
    hwgrad_kernel(const __grid_constant__ HwgradParams p, const __grid_constant__ CUtensorMap tmapX,
                  const __grid_constant__ CUtensorMap tmapDy) {
  constexpr bool FDY = NCG > 0;
  constexpr int MAXG = NCG == 3 ? 3 : 4;   // 32-channel groups a builder thread holds (bn <= 32*MAXG)
  static_assert(NCG != 1 || MAXG == 4, "landing-zone builders: bn <= 128");
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t base = (raw + 1023u) & ~1023u;
  const uint32_t stage_bytes = (uint32_t)(p.a_bytes + p.b_bytes);
  const uint32_t bars = base + (uint32_t)p.stages * stage_bytes;
  const int S_ = p.stages;
  auto full = [&](int s) { return bars + 8u * s; };
  auto empty = [&](int s) { return bars + 8u * (S_ + s); };
  const uint32_t tfull = bars + 8u * (2 * S_);
  const uint32_t tmem_slot = bars + 8u * (2 * S_ + 1);
  volatile uint32_t *tmem_slot_ptr =
      reinterpret_cast<volatile uint32_t *>(smem_raw + (tmem_slot - raw));
  const int warp = __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0);
  const int lane = threadIdx.x & 31;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S_; ++s) {
      mbar_init(full(s), FDY ? 5 : 1);   // FDY: + one arrival per warp of the building group
      mbar_init(empty(s), 1);
    }
    mbar_init(tfull, 1);
    fence_mbar_init();
  }
  if (warp == 5) {
    tmem_alloc(tmem_slot, (uint32_t)p.tmem_cols);
    tmem_relinquish();
  }
  if (warp == 4 && lane == 0) {
    tma_prefetch(&tmapX);
    if (!FDY) tma_prefetch(&tmapDy);
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  pdl_wait();
  const uint32_t tmem_base = __shfl_sync(0xffffffffu, *tmem_slot_ptr, 0);
  const int u = blockIdx.x;   // one split per CTA
  const int kb0 = u * p.kb_per_split;
  const int kb1 = min(kb0 + p.kb_per_split, p.kb_total);

  if (warp == 4) {
    // ===================================== producer ========================================
    int rs = 0;
    uint32_t rph = 0;
    const bool la = !GLP_SKIP(p, 1), lb = !FDY && !GLP_SKIP(p, 2);
    const int nb = (p.bn + 63) / 64;
    const uint32_t tx = (la ? (uint32_t)(p.halo_rows * 128) : 0u) + (lb ? (uint32_t)p.b_bytes : 0u);
    for (int kb = kb0; kb < kb1; ++kb) {
      mbar_wait(empty(rs), rph ^ 1u);
      const uint32_t sA = base + (uint32_t)rs * stage_bytes, sB = sA + (uint32_t)p.a_bytes;
      mbar_arrive_expect_tx_e(full(rs), tx);
      const int row0 = kb * HW_BKP;
      if (la) tma_load_2d_e(sA, &tmapX, full(rs), 0, row0);
      if (lb)
        for (int a = 0; a < nb; ++a)
          tma_load_2d_e(sB + (uint32_t)a * (HW_BKP * 128), &tmapDy, full(rs), a * 64, row0);
      if (++rs == S_) {
        rs = 0;
        rph ^= 1u;
      }
    }
  } else if (warp == 5) {
    // ===================================== MMA issuer ======================================
    const uint32_t idesc = make_idesc(1u, 1u, 1u, 128u, (uint32_t)p.bn);
    int rs = 0;
    uint32_t rph = 0;
    uint32_t acc = 0;
    for (int kb = kb0; kb < kb1; ++kb) {
      mbar_wait(full(rs), rph);
      tc_fence_after();
      const uint32_t sA = base + (uint32_t)rs * stage_bytes, sB = sA + (uint32_t)p.a_bytes;
      // B: dy MN-major, 64-channel SW128 atoms of HW_BKP rows (LBO = one atom column)
      const uint64_t db = make_sdesc(sB, HW_BKP * 128u, 1024u, 2u);
      for (int j = 0; j < p.n_acc && !GLP_SKIP(p, 4); ++j) {
        const uint32_t sa = sA + (uint32_t)p.shift_a[j] * 128u;
        const uint64_t da =
            make_sdesc(sa, (uint32_t)(p.shift_b[j] - p.shift_a[j]) * 128u, 1024u, 2u);
        const uint32_t d = tmem_base + (uint32_t)(j * p.acc_cols);
        // 8 MMAs of K = 16 pixel rows (2048 bytes = 128 descriptor units for A and B)
        mma_kblock_e<0, 1, 4, 128>(d, da, db, idesc, acc);
        mma_kblock_e<0, 1, 4, 128>(d, da + 512u, db + 512u, idesc, 1u);
      }
      acc = 1;
      mma_commit_e<1>(empty(rs));
      if (++rs == S_) {
        rs = 0;
        rph ^= 1u;
      }
    }
    mma_commit_e<1>(tfull);
    __syncwarp();
  } else {
    if (FDY) {
      // ============================ dy operand + db partials (warps 0-3) =====================
      // thread t = pixel row t of the k-block (q = kb*128 + t on the padded grid); for each group
      // of 32 channels: 32 coalesced loads (lanes = consecutive pixels of one channel plane),
      // a transposing butterfly that leaves channel 32g+lane's sum over the warp's 32 pixels in
      // lane `lane` (added to dbacc[g] in k-block order: a fixed order), then RNE to bf16 and
      // four 16-byte swizzled stores into the MN-major SW128 atoms of the stage's B region.
      // group 0 = warps 0-3, group g >= 1 = warps 6+4(g-1) .. 9+4(g-1); group g builds k-blocks
      // kb0 + g, kb0 + g + NCG, ...
      const int grp = warp >= 6 ? (warp - 6) / 4 + 1 : 0;
      const int t = threadIdx.x - (grp ? 192 + 128 * (grp - 1) : 0);
      if (u == 0 && grp == 0)
        for (int i = t; i < p.n_tickets; i += 128) p.db_tickets[i] = 0u;
      const int ngrp = (p.bn + 31) / 32;   // <= MAXG (plan)
      const size_t hw = (size_t)p.ho * p.wo;
      float dbacc[MAXG];
#pragma unroll
      for (int g = 0; g < MAXG; ++g) dbacc[g] = 0.f;
      if constexpr (NCG == 1) {
        // landing zones after the db staging area: [2][bn][128] fp32 (thread t = pixel column t)
        const uint32_t sland = (bars + 8u * (2 * S_ + 2) + 15u) & ~15u;   // db staging reuses it
        const uint32_t lbytes = (uint32_t)p.bn * 128u * 4u;
        auto issue = [&](int kb, uint32_t buf) {
          const int q = kb * HW_BKP + t;
          uint32_t n = 0, rem = 0, h = 0, w = 0;
          p.div_img.divmod((uint32_t)min(q, p.rows - 1), n, rem);
          p.div_w.divmod(rem, h, w);
          const bool ok = q < p.rows && (int)h < p.ho && (int)w < p.wo;
          const float *src = p.dy + ((size_t)n * p.dy_c * p.ho + h) * p.wo + w;
          const uint32_t dst = sland + buf * lbytes + (uint32_t)t * 4u;
          for (int co = 0; co < p.bn; ++co)
            cp_async4(dst + (uint32_t)co * 512u, ok && co < p.co ? src + (size_t)co * hw : p.dy,
                      ok && co < p.co);
          cp_async_commit();
        };
        if (kb0 < kb1) issue(kb0, 0u);
        uint32_t cur = 0;
        for (int kb = kb0; kb < kb1; ++kb, cur ^= 1u) {
          const int rs = (kb - kb0) % S_;
          const uint32_t rph = (uint32_t)(((kb - kb0) / S_) & 1);
          if (kb + 1 < kb1) {
            issue(kb + 1, cur ^ 1u);
            cp_async_wait<1>();
          } else {
            cp_async_wait<0>();
          }
          mbar_wait(empty(rs), rph ^ 1u);
          const uint32_t sB = base + (uint32_t)rs * stage_bytes + (uint32_t)p.a_bytes;
          const float *lv = reinterpret_cast<const float *>(smem_raw + (sland + cur * lbytes - raw)) + t;
#pragma unroll
          for (int g = 0; g < MAXG; ++g) {
            if (g >= ngrp) break;
            float v[32];
#pragma unroll
            for (int j = 0; j < 32; ++j) v[j] = lv[(g * 32 + j) * 128];
            float tt[32];
#pragma unroll
            for (int j = 0; j < 32; ++j) tt[j] = v[j];
#pragma unroll
            for (int wdt = 16; wdt >= 1; wdt >>= 1) {
              const bool up = (lane & wdt) != 0;
#pragma unroll
              for (int j = 0; j < wdt; ++j) {
                const float send = up ? tt[j] : tt[j + wdt];
                const float keep = up ? tt[j + wdt] : tt[j];
                tt[j] = keep + __shfl_xor_sync(0xffffffffu, send, wdt);
              }
            }
            dbacc[g] += tt[0];
#pragma unroll
            for (int c = 0; c < 4; ++c) {
              const int co0 = g * 32 + c * 8;
              if (co0 >= p.bn) break;
              __nv_bfloat162 a = __floats2bfloat162_rn(v[c * 8], v[c * 8 + 1]);
              __nv_bfloat162 b = __floats2bfloat162_rn(v[c * 8 + 2], v[c * 8 + 3]);
              __nv_bfloat162 cc = __floats2bfloat162_rn(v[c * 8 + 4], v[c * 8 + 5]);
              __nv_bfloat162 d = __floats2bfloat162_rn(v[c * 8 + 6], v[c * 8 + 7]);
              const uint32_t atom = (uint32_t)(co0 >> 6), ch = (uint32_t)((co0 & 63) >> 3);
              const uint32_t addr = sB + atom * (uint32_t)(HW_BKP * 128) + (uint32_t)t * 128u +
                                    ((ch ^ (uint32_t)(t & 7)) << 4);
              asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(addr),
                           "r"(*reinterpret_cast<uint32_t *>(&a)), "r"(*reinterpret_cast<uint32_t *>(&b)),
                           "r"(*reinterpret_cast<uint32_t *>(&cc)), "r"(*reinterpret_cast<uint32_t *>(&d))
                           : "memory");
            }
          }
          fence_proxy_async_smem();
          __syncwarp();
          if (lane == 0) mbar_arrive(full(rs));
        }
      } else
      for (int kb = kb0 + grp; kb < kb1; kb += NCG) {
        const int rs = (kb - kb0) % S_;
        const uint32_t rph = (uint32_t)(((kb - kb0) / S_) & 1);
        const int q = kb * HW_BKP + t;
        uint32_t n = 0, rem = 0, h = 0, w = 0;
        p.div_img.divmod((uint32_t)min(q, p.rows - 1), n, rem);
        p.div_w.divmod(rem, h, w);
        const bool ok = q < p.rows && (int)h < p.ho && (int)w < p.wo;
        const float *src = p.dy + ((size_t)n * p.dy_c * p.ho + h) * p.wo + w;
        // every load of the k-block in flight before anything waits (registers, not smem: the
        // stage need not be free yet)
        float v[MAXG][32];
#pragma unroll
        for (int g = 0; g < MAXG; ++g)
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            const int co = g * 32 + j;
            v[g][j] = (ok && g < ngrp && co < p.co) ? __ldg(src + (size_t)co * hw) : 0.f;
          }
        mbar_wait(empty(rs), rph ^ 1u);
        const uint32_t sB = base + (uint32_t)rs * stage_bytes + (uint32_t)p.a_bytes;
#pragma unroll
        for (int g = 0; g < MAXG; ++g) {
          if (g >= ngrp) break;
          float tt[32];
#pragma unroll
          for (int j = 0; j < 32; ++j) tt[j] = v[g][j];
#pragma unroll
          for (int wdt = 16; wdt >= 1; wdt >>= 1) {
            const bool up = (lane & wdt) != 0;
#pragma unroll
            for (int j = 0; j < wdt; ++j) {
              const float send = up ? tt[j] : tt[j + wdt];
              const float keep = up ? tt[j + wdt] : tt[j];
              tt[j] = keep + __shfl_xor_sync(0xffffffffu, send, wdt);
            }
          }
          dbacc[g] += tt[0];
#pragma unroll
          for (int c = 0; c < 4; ++c) {
            const int co0 = g * 32 + c * 8;
            if (co0 >= p.bn) break;
            __nv_bfloat162 a = __floats2bfloat162_rn(v[g][c * 8], v[g][c * 8 + 1]);
            __nv_bfloat162 b = __floats2bfloat162_rn(v[g][c * 8 + 2], v[g][c * 8 + 3]);
            __nv_bfloat162 cc = __floats2bfloat162_rn(v[g][c * 8 + 4], v[g][c * 8 + 5]);
            __nv_bfloat162 d = __floats2bfloat162_rn(v[g][c * 8 + 6], v[g][c * 8 + 7]);
            const uint32_t atom = (uint32_t)(co0 >> 6), ch = (uint32_t)((co0 & 63) >> 3);
            const uint32_t addr = sB + atom * (uint32_t)(HW_BKP * 128) + (uint32_t)t * 128u +
                                  ((ch ^ (uint32_t)(t & 7)) << 4);
            asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(addr),
                         "r"(*reinterpret_cast<uint32_t *>(&a)), "r"(*reinterpret_cast<uint32_t *>(&b)),
                         "r"(*reinterpret_cast<uint32_t *>(&cc)), "r"(*reinterpret_cast<uint32_t *>(&d))
                         : "memory");
          }
        }
        fence_proxy_async_smem();   // generic-proxy smem writes -> visible to tcgen05.mma
        __syncwarp();
        if (lane == 0) mbar_arrive(full(rs));
      }
      // db partial of this CTA's pixel range: warps 0..3 in order (fixed), one row per CTA
      const uint32_t sred = (bars + 8u * (2 * S_ + 2) + 15u) & ~15u;   // 4*NCG x 256 floats
      float *red = reinterpret_cast<float *>(smem_raw + (sred - raw));
      if (NCG == 1) named_bar_sync(1, 128);   // the landing zone is done before it holds db
      const int slot = grp * 4 + (warp & 3);   // a fixed slot per warp (4 per group)
#pragma unroll
      for (int g = 0; g < MAXG; ++g)
        if (g < ngrp) red[slot * 256 + g * 32 + lane] = dbacc[g];
      named_bar_sync(1, 128 * NCG);
      if (grp == 0) {
        for (int co = t; co < p.co; co += 128) {
          float tot = 0.f;   // groups in order, each the sum of its 4 warps in order
#pragma unroll
          for (int gg = 0; gg < NCG; ++gg) {
            float a = 0.f;
#pragma unroll
            for (int k = 0; k < 4; ++k) a += red[(gg * 4 + k) * 256 + co];
            tot += a;
          }
          p.db_part[(size_t)u * p.co + co] = tot;
        }
      }
    }
    if (!FDY || warp < 4) {   // groups >= 1 have no epilogue role (TMEM lanes: warps 0-3)
    // ===================================== epilogue ========================================
    mbar_wait(tfull, 0);
    tc_fence_after();
    const int r = warp * 32 + lane;   // TMEM lane = M row of every accumulator
    const int atom = r >> 6, c = r & 63;
    const bool empty_range = kb1 <= kb0;
    for (int j = 0; j < p.n_acc; ++j) {
      const bool dup = atom == 0 && ((p.dup_a_mask >> j) & 1);
      const int t = atom ? p.tap_b[j] : p.tap_a[j];
      float *dst = p.part + ((size_t)u * p.mpad + (size_t)t * p.cpx + c) * p.ld;
      for (int c0 = 0; c0 < p.bn; c0 += 32) {
        uint32_t v[32];
        tmem_ld32(tmem_base + ((uint32_t)(warp * 32) << 16) + (uint32_t)(j * p.acc_cols + c0), v);
        tmem_wait_ld();
        if (dup) continue;
        const int lim = min(32, p.bn - c0);
        if (lim == 32) {
#pragma unroll
          for (int q = 0; q < 32; q += 4)
            *reinterpret_cast<float4 *>(dst + c0 + q) =
                empty_range ? make_float4(0.f, 0.f, 0.f, 0.f)
                            : make_float4(__uint_as_float(v[q]), __uint_as_float(v[q + 1]),
                                          __uint_as_float(v[q + 2]), __uint_as_float(v[q + 3]));
        } else {
#pragma unroll
          for (int q = 0; q < 32; ++q)
            if (q < lim) dst[c0 + q] = empty_range ? 0.f : __uint_as_float(v[q]);
        }
      }
    }
    }
  }
  pdl_launch_dependents();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  if (warp == 5) tmem_dealloc(tmem_base, (uint32_t)p.tmem_cols);
}

}  // namespace glp
