// igemm.cuh — persistent, warp-specialised implicit-GEMM convolution on sm_100a tensor cores.
//
// One kernel template serves the three passes of the GLP4NN hot path (Alg. 1 P82-99,
// Alg. 2 P101-121, parameter gradients P129; north_star (3)):
//   MODE_FWD  : D[pixel(n,ho,wo), co] = sum_{(kh,kw,ci)} x[n, ho*S-P+kh, wo*S-P+kw, ci] * W[co,(kh,kw,ci)]
//               (im2col never materialised: the A operand is gathered from packed NHWC x)
//   MODE_DGRAD: D[pixel(n,h,w), ci]  = sum_{(kh,kw,co)} dy[n, (h+P-kh)/S, (w+P-kw)/S, co] * Wt[ci,(kh,kw,co)]
//               (col2im folded into the gather: every dx element is owned by one CTA, no atomics)
//   MODE_WGRAD: D[(kh,kw,ci), co]    = sum_{pixels p in split} x[gather(p,kh,kw), ci] * dy[p, co]
//               (fixed, shape-only split of the N*H_o*W_o reduction; partials reduced in order)
//
// CTA = 288 threads: warps 0-3 epilogue (TMEM -> registers -> global), warps 4-7 producers,
// warp 8 TMEM allocator + single-thread tcgen05.mma issuer.
//   A operand: im2col-mode TMA issued by one thread (a_tma = 1), or, for tiny channel counts /
//              strided dgrad, a cp.async gather by 128 threads into the same SWIZZLE_128B layout.
//   B operand: dense 2-D matrix (packed weights, or packed dy for wgrad) by tiled TMA.
// smem ring of `stages` {A,B} slots (mbarrier full/empty), two TMEM accumulators (tfull/tempty)
// so the epilogue of tile i overlaps the main loop of tile i+1.  Tiles are visited by a static
// round-robin over a persistent grid (tile t -> CTA t mod grid), the device-side replacement of
// the paper's round-robin stream dispatch (P171).
//
// Shared-memory operand layouts (UMMA canonical, K-block row width KROW bytes):
//   K-major (fwd/dgrad A and B): rows of KROW bytes, 8-row atoms, SWIZZLE_128B (KROW 128) or
//     SWIZZLE_64B (KROW 64); one tcgen05.mma consumes 32 bytes of K.
//   MN-major (wgrad A and B): K-rows of one MN atom (KROW bytes = KROW/ELEM channels) stacked
//     contiguously; bf16 SWIZZLE_128B/64B (8-row groups), tf32 SWIZZLE_128B_BASE32B (4-row groups).
#pragma once
#include "common.cuh"
#include "ptx.cuh"

namespace glp {

constexpr int IGEMM_THREADS = 288;      // 4 epilogue warps, 4 producer warps, 1 MMA warp
constexpr int IGEMM_X3_THREADS = 512;   // 3xTF32: 8 epilogue warps, 4 producer, 1 MMA, 3 idle
constexpr int X3_EPI_REGS = 192, X3_OTHER_REGS = 64;   // setmaxnreg split (sum = 2 x 128 regs)
__host__ __device__ constexpr int igemm_threads(int x3) { return x3 ? IGEMM_X3_THREADS : IGEMM_THREADS; }

template <int ELEM, int KROW>
struct TileCfg {
  static constexpr int BM = 128;
  static constexpr int BK = KROW / ELEM;        // K elements per k-block (fwd/dgrad)
  static constexpr int BKP = 128 / ELEM;        // pixels per k-block (wgrad)
  static constexpr int CH = 16 / ELEM;          // elements per 16-byte chunk
  static constexpr int UMMA_K = 32 / ELEM;      // K of one tcgen05.mma (bf16 16, tf32 8)
  static constexpr int EPA = KROW / ELEM;       // MN elements per MN-major atom row
  // K-major
  static constexpr uint32_t K_LAYOUT = (KROW == 128) ? 2u : 4u;
  static constexpr uint32_t K_SBO = 8u * KROW;
  // MN-major
  static constexpr uint32_t MN_LAYOUT = (ELEM == 4) ? 1u : ((KROW == 128) ? 2u : 4u);
  static constexpr uint32_t MN_GROUP = ((ELEM == 4) ? 4u : 8u) * KROW;   // SBO
  static constexpr uint32_t MN_LBO = (uint32_t)BKP * KROW;                // one atom column
  static constexpr uint32_t MN_KSTEP = (uint32_t)UMMA_K * KROW;
  static constexpr int THREADS = 288;
  __host__ __device__ static constexpr uint32_t a_bytes(int mode) {
    return mode == MODE_WGRAD ? (uint32_t)BM * BKP * ELEM : (uint32_t)BM * KROW;
  }
  __host__ __device__ static constexpr uint32_t b_row_bytes(int mode) {
    return mode == MODE_WGRAD ? (uint32_t)BKP * ELEM : (uint32_t)KROW;
  }
};

// Advance a (slot, phase) ring position without division (the MMA issuer's loop is latency-bound:
// a runtime `gk % stages` costs more than the tcgen05.mma work of a small-N k-block).
__device__ __forceinline__ void ring_next(int &s, uint32_t &ph, int S) {
  if (++s == S) {
    s = 0;
    ph ^= 1u;
  }
}

// k-block range [kb0, kb1) of filter-gradient split `split`.  Leaf plans (p.splits_per_leaf > 0,
// the deterministic exchange): the pixel range is cut into leaves of p.kb_per_leaf k-blocks and
// each leaf into p.splits_per_leaf splits that never cross a leaf boundary, so every leaf's split
// partials are the same bits whichever rank (and local batch) computes the leaf.
__device__ __forceinline__ void wgrad_kb_range(const IgemmParams &p, int split, int &kb0, int &kb1) {
  if (p.splits_per_leaf > 0) {
    const int leaf = split / p.splits_per_leaf, j = split - leaf * p.splits_per_leaf;
    kb0 = leaf * p.kb_per_leaf + j * p.kb_per_split;
    kb1 = min(kb0 + p.kb_per_split, (leaf + 1) * p.kb_per_leaf);
  } else {
    kb0 = split * p.kb_per_split;
    kb1 = min(kb0 + p.kb_per_split, p.kb_total);
  }
}

__device__ __forceinline__ void decode_tile(int t, int n_tiles, int m_tiles, int &m_tile,
                                            int &n_tile, int &split) {
  n_tile = t % n_tiles;
  const int r = t / n_tiles;
  m_tile = r % m_tiles;
  split = r / m_tiles;
}

// Forward-gather address of one 16-byte chunk: pixel m (GEMM row) and K index k0 (tap*cp + c).
// Used by glp_debug_im2col so that the debug view uses the cp.async producer's index math.
template <int ELEM>
__device__ __forceinline__ bool fwd_gather(const Gather &g, uint32_t n, int ohS, int owS,
                                           uint32_t k0, const uint8_t *&src) {
  uint32_t t, c;
  g.div_cp.divmod(k0, t, c);
  if ((int)t >= g.taps) return false;
  uint32_t kh, kw;
  g.div_kw.divmod(t, kh, kw);
  const int ih = ohS + (int)kh, iw = owS + (int)kw;
  if (ih < 0 || ih >= g.src_h || iw < 0 || iw >= g.src_w) return false;
  src = static_cast<const uint8_t *>(g.src) +
        ((size_t)((size_t)n * g.src_h * g.src_w + (size_t)ih * g.src_w + iw) * g.src_cp + c) * ELEM;
  return true;
}

// CG = 1: one CTA per 128-row tile.  CG = 2: CTA pairs (cluster of 2) run tcgen05.mma.cta_group::2
// with M = 256: each CTA loads its own 128 A rows and half of the B tile (p.bn_smem = BN/2), the
// pair leader issues the MMAs for both SMs and multicasts its commits (A by TMA only).
//
// X3 = 1 (GLP_MATH_FP32, ELEM 4, KROW 128): 3xTF32.  Every operand has a hi and a lo plane (the
// packs write hi = rna(v) and lo = rna(v - hi)); a k-block slot holds [A_hi | A_lo] and
// [B_hi | B_lo] (each plane in the single-plane layout), the producer loads both planes (tmapA2 /
// tmapB2 = the lo planes), and the MMA issuer runs hi*hi, hi*lo, lo*hi per k-step into the same
// TMEM accumulator (mma_kblock_x3_e).
// The tensor core rounds every MMA's fp32 result toward zero (measured: the normwise error of one
// accumulator grows linearly with K, ~2^-25 of the accumulator per MMA), so a 3xTF32 tile does not
// accumulate its whole K range in TMEM: the k-blocks are cut into chunks of p.chunk_kb (a function
// of the shape only), each chunk accumulated from zero in one of two TMEM buffers, and the 8
// epilogue warps add the chunks in fp32 (round-to-nearest) in registers -- the row's running sum,
// half of the tile's columns per warp (warp w: TMEM lanes 32*(w%4), columns half w/4) -- then
// store the sum.  The buffers alternate chunk by chunk across tiles, so the MMA issuer never
// waits for the final stores.
//
// X3 = 2 (GLP_MATH_FP32 with plan option fp32_split = 1): the mixed split.  The packs write a tf32
// hi plane and two bf16 planes, bf16(hi) and bf16(v - hi) (pack.cuh); a k-block slot holds
// [A_hi | A_bhi | A_blo] and [B_hi | B_bhi | B_blo] (the bf16 tiles are 64-byte rows: K-major
// SWIZZLE_64B, or MN-major 32-element SWIZZLE_64B atoms), the same bytes as 3xTF32's two planes;
// tmapA2 / tmapB2 are the bf16(hi) planes, tmapA3 / tmapB3 the bf16(v - hi) planes.  The MMA
// issuer runs hi*hi in tf32 and the two cross terms in bf16 (mma_kblock_mix_e): 8 MMA issue slots
// per k-block instead of 12.  TMA operands, except the K-major cp.async gather of a strided
// backward-data (8-byte copies into the bf16 planes); the chunked accumulation and the epilogue
// are those of X3 = 1.
template <int MODE, int ELEM, int KROW, int CG, int X3>
__global__ void __launch_bounds__(X3 ? IGEMM_X3_THREADS : IGEMM_THREADS, 1)
    igemm_kernel(const __grid_constant__ IgemmParams p, const __grid_constant__ CUtensorMap tmapB,
                 const __grid_constant__ CUtensorMap tmapA, const __grid_constant__ CUtensorMap tmapB2,
                 const __grid_constant__ CUtensorMap tmapA2, const __grid_constant__ CUtensorMap tmapB3,
                 const __grid_constant__ CUtensorMap tmapA3) {
  using C = TileCfg<ELEM, KROW>;
  static_assert(!X3 || (ELEM == 4 && KROW == 128), "3xTF32 uses 128-byte tf32 rows");
  constexpr bool MIX = X3 == 2;
  constexpr int EW = X3 ? 8 : 4;    // epilogue warps 0 .. EW-1
  constexpr int PW = EW;            // producer warps PW .. PW+3 (TMA: warp PW alone)
  constexpr int MW = EW + 4;        // TMEM allocator + MMA issuer
  constexpr uint32_t PL = X3 ? 2u : 1u;                 // operand planes' bytes (hi, lo)
  constexpr uint32_t NPL = MIX ? 3u : PL;               // loaded planes (mixed: hi, bhi, blo)
  // byte offset of plane pl in a k-block's A or B slot of one-plane size `one`: 3xTF32 lo at
  // +one; mixed bf16(hi) at +one, bf16(v - hi) at +1.5 one (2-byte elements)
  auto plane_byte_off = [](uint32_t pl, uint32_t one) -> uint32_t {
    return pl == 0 ? 0u : (MIX && pl == 2) ? one + one / 2 : one;
  };
  constexpr uint32_t A_BYTES1 = C::a_bytes(MODE);       // one plane of one k-block's A
  constexpr uint32_t A_BYTES = PL * A_BYTES1;
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t base = (raw + 1023u) & ~1023u;
  const uint32_t b_bytes1 = (uint32_t)p.bn_smem * C::b_row_bytes(MODE);
  const uint32_t b_bytes = PL * b_bytes1;
  // a stage holds p.ksub consecutive k-blocks: [A_0 .. A_ks-1 | B_0 .. B_ks-1] (ksub = 2 halves
  // the barrier round trips per MMA; the cp.async path always uses ksub = 1)
  const uint32_t stage_bytes = (uint32_t)p.ksub * (A_BYTES + b_bytes);
  const uint32_t bars = base + (uint32_t)p.stages * stage_bytes;
  const int S_ = p.stages;
  auto full = [&](int s) { return bars + 8u * s; };
  auto empty = [&](int s) { return bars + 8u * (S_ + s); };
  auto tfull = [&](int a) { return bars + 8u * (2 * S_ + a); };
  auto tempty = [&](int a) { return bars + 8u * (2 * S_ + 2 + a); };
  const uint32_t tmem_slot = bars + 8u * (2 * S_ + 4);
  volatile uint32_t *tmem_slot_ptr =
      reinterpret_cast<volatile uint32_t *>(smem_raw + (tmem_slot - raw));

  // warp index broadcast from lane 0: the compiler then knows every role branch below is
  // warp-uniform and keeps loop state of the single-warp roles in the uniform datapath
  const int warp = __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0);
  const int lane = threadIdx.x & 31;
  const bool a_tma = (CG == 2) || p.a_tma != 0;
  // cluster of 2 CTAs along x: the rank in the pair is blockIdx.x & 1 (uniform by construction)
  const uint32_t rank = (CG == 2) ? (blockIdx.x & 1u) : 0u;
  const bool leader = rank == 0;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S_; ++s) {
      // CG1: TMA mode 1 expect_tx arrival; cp.async mode 128 cp.async arrivals (noinc) + 1.
      // CG2: only the leader arrives (expect_tx = both CTAs' bytes); the peer's TMA completes
      // bytes on the leader's barrier (as CUTLASS's 2-SM TMA pipeline).
      mbar_init(full(s), a_tma ? 1 : 129);
      mbar_init(empty(s), 1);    // tcgen05.commit (multicast to both CTAs for CG2)
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(tfull(a), 1);         // tcgen05.commit after the last k-block of a tile
      mbar_init(tempty(a), EW * CG);  // one arrival per epilogue warp (of both CTAs for CG2)
    }
    fence_mbar_init();
  }
  if (warp == MW) {
    tmem_alloc_cg<CG>(tmem_slot, (uint32_t)p.tmem_cols);
    tmem_relinquish_cg<CG>();
  }
  if (warp == PW && lane == 0) {
    tma_prefetch(&tmapB);
    if (a_tma) tma_prefetch(&tmapA);
    if (X3) {
      tma_prefetch(&tmapB2);
      if (a_tma) tma_prefetch(&tmapA2);
    }
    if (MIX) {
      tma_prefetch(&tmapB3);
      tma_prefetch(&tmapA3);
    }
  }
  tc_fence_before();
  if (CG == 2) cluster_sync();
  else __syncthreads();
  tc_fence_after();
  // prologue done (barriers, TMEM, descriptor prefetch): wait for the previous kernel's results
  // before touching global memory
  pdl_wait();
  const uint32_t tmem_base = __shfl_sync(0xffffffffu, *tmem_slot_ptr, 0);   // warp-uniform

  // work units: CG1 = one 128-row tile; CG2 = a pair of 128-row tiles (one per CTA)
  const int total_tiles = p.m_tiles * p.n_tiles * p.splits;   // p.m_tiles counts units along M
  const int unit0 = (CG == 2) ? (int)(blockIdx.x >> 1) : (int)blockIdx.x;
  const int ustep = (CG == 2) ? (int)(gridDim.x >> 1) : (int)gridDim.x;
  const Gather &g = p.g;

  // 3xTF32: the epilogue warpgroups (warps 0-7) hold the chunk sums in registers: they raise their
  // register budget, the other two warpgroups lower theirs (setmaxnreg at the top of each role
  // branch, so ptxas allocates each branch with its own budget)
  if (warp >= EW) {
  if constexpr (X3) asm volatile("setmaxnreg.dec.sync.aligned.u32 %0;" ::"n"(X3_OTHER_REGS));
  if (warp < PW + 4) {
    // ===================================== producers =======================================
    const int pt = threadIdx.x - 32 * PW;
    if (a_tma) {
      if (warp == PW) {   // one converged warp; each TMA / arrive is issued by an elected lane
        int rs = 0;          // ring slot and its phase, advanced incrementally
        uint32_t rph = 0;
        uint32_t stg_addr = base;   // shared address of ring slot rs
        const int KS = p.ksub, cbs = g.cbs, KW = g.kw;
        const bool la = !GLP_SKIP(p, 1), lb = !GLP_SKIP(p, 2);
        const uint32_t kb_tx = (la ? A_BYTES : 0u) + (lb ? b_bytes : 0u);
        const uint32_t sB_off = (uint32_t)KS * A_BYTES;
#ifdef GLP_DIAG
        long long c_empty = 0;
#endif
        for (int tile = unit0; tile < total_tiles; tile += ustep) {
          int m_tile, n_tile, split;
          decode_tile(tile, p.n_tiles, p.m_tiles, m_tile, n_tile, split);
          const int m0 = (m_tile * CG + (int)rank) * C::BM, n0 = n_tile * p.bn;
          const int nb0 = n0 + (int)rank * p.bn_smem;   // this CTA's part of the B tile
          int kb0 = 0, kb1 = p.kb_total;
          if (MODE == MODE_WGRAD) {
            wgrad_kb_range(p, split, kb0, kb1);
          }
          // per-tile geometry of the A gather
          uint32_t n_t = 0;
          int h_t = 0, w_t = 0;            // fwd/dgrad: base pixel of the tile's first row
          constexpr int NA = (MODE == MODE_WGRAD) ? 128 / C::EPA : 1;   // MN atoms (wgrad)
          int ac[NA];
          uint16_t akh[NA], akw[NA];
          if (MODE != MODE_WGRAD) {
            uint32_t rem, oh, ow;
            g.div_hw.divmod((uint32_t)m0, n_t, rem);
            g.div_w.divmod(rem, oh, ow);
            h_t = (int)oh * g.im_sh - g.im_ph;
            w_t = (int)ow * g.im_sw - g.im_pw;
          } else {
#pragma unroll
            for (int a = 0; a < NA; ++a) {
              uint32_t t, c;
              g.div_cp.divmod((uint32_t)(m0 + a * C::EPA), t, c);
              if ((int)t < g.taps) {
                uint32_t kh, kw;
                g.div_kw.divmod(t, kh, kw);
                ac[a] = (int)c;
                akh[a] = (uint16_t)kh;
                akw[a] = (uint16_t)kw;
              } else {          // rows past M: channel coordinate out of bounds -> zeros
                ac[a] = g.src_cp;
                akh[a] = 0;
                akw[a] = 0;
              }
            }
          }
          int kh = 0, kw = 0, cb = 0;       // fwd/dgrad K position (tap (kh, kw), channel block)
          for (int kbs = kb0; kbs < kb1; kbs += KS) {
            const int s = rs;
#ifdef GLP_DIAG
            long long c0 = (p.dbg_clk != nullptr) ? clock64() : 0;
#endif
            mbar_wait(empty(s), rph ^ 1u);
#ifdef GLP_DIAG
            if (p.dbg_clk != nullptr) c_empty += clock64() - c0;
#endif
            const int nsub = min(KS, kb1 - kbs);
            const uint32_t stg = stg_addr;
            const uint32_t tx = (uint32_t)nsub * kb_tx;
            uint32_t bar = full(s);
            if (CG == 1) {
              mbar_arrive_expect_tx_e(bar, tx);
            } else {
              // only the leader arrives (expect_tx = both CTAs' bytes); the peer's TMAs complete
              // bytes on the leader's barrier — a release-scoped remote arrive here would fence
              // this thread's in-flight TMA
              if (leader) mbar_arrive_expect_tx_e(bar, 2u * tx);
              bar = mapa_shared(bar, 0);
            }
            if (++rs == S_) {
              rs = 0;
              rph ^= 1u;
              stg_addr = base;
            } else {
              stg_addr += stage_bytes;
            }
#pragma unroll 1
            for (int sub = 0; sub < nsub; ++sub) {
              const int kb = kbs + sub;
              const uint32_t sA = stg + (uint32_t)sub * A_BYTES;
              const uint32_t sB = stg + sB_off + (uint32_t)sub * b_bytes;
              if (MODE != MODE_WGRAD) {
#pragma unroll
                for (uint32_t pl = 0; pl < NPL; ++pl) {
                  const CUtensorMap *mA = pl == 0 ? &tmapA : pl == 1 ? &tmapA2 : &tmapA3;
                  const CUtensorMap *mB = pl == 0 ? &tmapB : pl == 1 ? &tmapB2 : &tmapB3;
                  const uint32_t oA = plane_byte_off(pl, A_BYTES1), oB = plane_byte_off(pl, b_bytes1);
                  if (la) {
                    if (CG == 1)
                      tma_load_im2col_4d_e(sA + oA, mA, bar, cb * C::BK, w_t, h_t,
                                           (int)n_t, (uint16_t)kw, (uint16_t)kh);
                    else
                      tma_load_im2col_4d_cg2_e(sA + oA, mA, bar, cb * C::BK, w_t, h_t,
                                               (int)n_t, (uint16_t)kw, (uint16_t)kh);
                  }
                  if (lb) {
                    if (CG == 1) tma_load_2d_e(sB + oB, mB, bar, kb * C::BK, nb0);
                    else tma_load_2d_cg2_e(sB + oB, mB, bar, kb * C::BK, nb0);
                  }
                }
                if (++cb == cbs) {
                  cb = 0;
                  if (++kw == KW) {
                    kw = 0;
                    ++kh;
                  }
                }
              } else {
                uint32_t n, rem, oh, ow;
                g.div_hw.divmod((uint32_t)(kb * C::BKP), n, rem);
                g.div_w.divmod(rem, oh, ow);
                const int h0 = (int)oh * g.im_sh - g.im_ph, w0 = (int)ow * g.im_sw - g.im_pw;
#pragma unroll
                for (uint32_t pl = 0; pl < NPL; ++pl) {
                  const CUtensorMap *mA = pl == 0 ? &tmapA : pl == 1 ? &tmapA2 : &tmapA3;
                  const CUtensorMap *mB = pl == 0 ? &tmapB : pl == 1 ? &tmapB2 : &tmapB3;
                  const uint32_t pA = sA + plane_byte_off(pl, A_BYTES1), pB = sB + plane_byte_off(pl, b_bytes1);
                  // MN atom stride: the bf16 planes of the mixed split have 64-byte atom rows
                  const uint32_t lbo = (MIX && pl) ? C::MN_LBO / 2 : C::MN_LBO;
                  if (la) {
#pragma unroll
                    for (int a = 0; a < NA; ++a) {
                      if (CG == 1)
                        tma_load_im2col_4d_e(pA + (uint32_t)a * lbo, mA, bar, ac[a], w0,
                                             h0, (int)n, akw[a], akh[a]);
                      else
                        tma_load_im2col_4d_cg2_e(pA + (uint32_t)a * lbo, mA, bar, ac[a],
                                                 w0, h0, (int)n, akw[a], akh[a]);
                    }
                  }
                  if (lb) {
                    if (p.b3d) {   // all of the tile's atoms in one 3-D load
                      if (CG == 1) tma_load_3d_e(pB, mB, bar, 0, kb * C::BKP, nb0 / C::EPA);
                      else tma_load_3d_cg2_e(pB, mB, bar, 0, kb * C::BKP, nb0 / C::EPA);
                    } else {
                      for (int a = 0; a < p.bn_smem / C::EPA; ++a) {
                        if (CG == 1)
                          tma_load_2d_e(pB + (uint32_t)a * lbo, mB, bar, nb0 + a * C::EPA,
                                        kb * C::BKP);
                        else
                          tma_load_2d_cg2_e(pB + (uint32_t)a * lbo, mB, bar,
                                            nb0 + a * C::EPA, kb * C::BKP);
                      }
                    }
                  }
                }
              }
            }
          }
        }
#ifdef GLP_DIAG
        if (p.dbg_clk != nullptr && lane == 0) p.dbg_clk[blockIdx.x * 4 + 3] = c_empty;
#endif
      }
    } else if (KROW == 128 && CG == 1) {
      // -------- cp.async gather (SWIZZLE_128B layouts only) --------
      // (mixed split: the K-major gather only -- strided backward-data; the plan keeps the
      // filter gradient of a mixed layer on TMA)
      if (MIX && MODE == MODE_WGRAD) __trap();
      int rs = 0;          // ring slot and its phase, advanced incrementally
        uint32_t rph = 0;
      for (int tile = unit0; tile < total_tiles; tile += ustep) {
        int m_tile, n_tile, split;
        decode_tile(tile, p.n_tiles, p.m_tiles, m_tile, n_tile, split);
        int kb0 = 0, kb1 = p.kb_total;
        if (MODE == MODE_WGRAD) {
          wgrad_kb_range(p, split, kb0, kb1);
        }
        const int m0 = m_tile * C::BM, n0 = n_tile * p.bn;
        if (MODE != MODE_WGRAD) {
          // K-major A: thread owns 16-byte chunk j of rows rg + 16 i (i = 0..7).
          const int j = pt & 7, rg = pt >> 3;
          uint32_t pbase[8];
          int ohS[8], owS[8];
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const int m = m0 + rg + 16 * i;
            uint32_t n, rem, oh, ow;
            g.div_hw.divmod((uint32_t)(m < p.M ? m : 0), n, rem);
            g.div_w.divmod(rem, oh, ow);
            pbase[i] = n * (uint32_t)(g.src_h * g.src_w);
            if (MODE == MODE_FWD) {
              ohS[i] = (int)oh * g.stride - g.pad;
              owS[i] = (int)ow * g.stride_w - g.pad_w;
            } else {
              ohS[i] = (int)oh + g.pad;
              owS[i] = (int)ow + g.pad_w;
            }
            if (m >= p.M) ohS[i] = -(1 << 28);  // row past M: every tap fails the bounds check
          }
          const uint32_t dst0 = (uint32_t)(rg >> 3) * 1024u + (uint32_t)(rg & 7) * 128u +
                                (uint32_t)((j ^ (rg & 7)) << 4);
          // K index of this thread's chunk, advanced incrementally by BK per k-block.
          uint32_t t, c, kh, kw;
          g.div_cp.divmod((uint32_t)(kb0 * C::BK + j * C::CH), t, c);
          g.div_kw.divmod(t, kh, kw);
          const uint8_t *srcb = static_cast<const uint8_t *>(g.src);
          for (int kb = kb0; kb < kb1; ++kb, ring_next(rs, rph, S_)) {
            const int s = rs;
            const uint32_t ph = rph;
            mbar_wait(empty(s), ph ^ 1u);
            const uint32_t sA = base + (uint32_t)s * stage_bytes, sB = sA + A_BYTES;
            if (pt == 0) {
              mbar_arrive_expect_tx(full(s), b_bytes);
              tma_load_2d(sB, &tmapB, full(s), kb * C::BK, n0);
              if (X3) tma_load_2d(sB + b_bytes1, &tmapB2, full(s), kb * C::BK, n0);
              if (MIX) tma_load_2d(sB + b_bytes1 + b_bytes1 / 2, &tmapB3, full(s), kb * C::BK, n0);
            }
            const bool kv = (int)t < g.taps;
#pragma unroll
            for (int i = 0; i < 8; ++i) {
              int ih, iw;
              bool ok;
              if (MODE == MODE_FWD) {
                ih = ohS[i] + (int)kh;
                iw = owS[i] + (int)kw;
                ok = kv && (unsigned)ih < (unsigned)g.src_h && (unsigned)iw < (unsigned)g.src_w;
              } else {
                const int ihn = ohS[i] - (int)kh, iwn = owS[i] - (int)kw;
                if (g.stride == 1 && g.stride_w == 1) {
                  ih = ihn;
                  iw = iwn;
                  ok = kv && (unsigned)ih < (unsigned)g.src_h && (unsigned)iw < (unsigned)g.src_w;
                } else {
                  ok = kv && ihn >= 0 && iwn >= 0 && (ihn % g.stride == 0) &&
                       (iwn % g.stride_w == 0);
                  ih = ihn / g.stride;
                  iw = iwn / g.stride_w;
                  ok = ok && ih < g.src_h && iw < g.src_w;
                }
              }
              const uint8_t *src = srcb;
              if (ok)
                src += ((size_t)(pbase[i] + (uint32_t)(ih * g.src_w + iw)) * (uint32_t)g.src_cp + c) *
                       ELEM;
              cp_async16(sA + dst0 + (uint32_t)i * 2048u, src, ok);
              if constexpr (MIX) {
                // the chunk's 4 channels in the bf16(hi) and bf16(v - hi) planes: 8 bytes of a
                // 64-byte SWIZZLE_64B row (16-byte chunk (j/2) ^ ((r/2) & 3), half j & 1); the
                // bf16 planes start lo_off_a (the hi plane's bytes) and 1.5 x that past the hi one
                const int r = rg + 16 * i;
                const uint32_t dbf = (uint32_t)r * 64u +
                                     ((uint32_t)(((j >> 1) ^ ((r >> 1) & 3)) << 4) | ((uint32_t)(j & 1) << 3));
                const uint8_t *sb = srcb + p.lo_off_a + (src - srcb) / 2;
                cp_async8(sA + A_BYTES1 + dbf, sb, ok);
                cp_async8(sA + A_BYTES1 + A_BYTES1 / 2 + dbf, sb + p.lo_off_a / 2, ok);
              } else if (X3) {
                cp_async16(sA + A_BYTES1 + dst0 + (uint32_t)i * 2048u, src + p.lo_off_a, ok);
              }
            }
            cp_async_mbar_arrive_noinc(full(s));
            c += C::BK;
            if (c >= (uint32_t)g.cp) {
              const uint32_t q = g.div_cp.div(c);
              c -= q * (uint32_t)g.cp;
              t += q;
              g.div_kw.divmod(t, kh, kw);
            }
          }
        } else {
          // WGRAD: MN-major A (M = (tap, ci) of x, K = pixels).  CPR chunks per K-row.
          constexpr int CPR = 128 * ELEM / 16;
          constexpr int RPP = 128 / CPR;
          const int j = pt % CPR, r0 = pt / CPR;
          const uint32_t mm = (uint32_t)(m0 + j * C::CH);
          uint32_t t, c;
          g.div_cp.divmod(mm, t, c);
          const bool mvalid = (int)t < g.taps;
          uint32_t kh, kw;
          g.div_kw.divmod(mvalid ? t : 0u, kh, kw);
          const int offh = (int)kh - g.pad, offw = (int)kw - g.pad_w;
          const uint32_t dcol = (uint32_t)(j >> 3) * C::MN_LBO;
          const int jj = j & 7;
          for (int kb = kb0; kb < kb1; ++kb, ring_next(rs, rph, S_)) {
            const int s = rs;
            const uint32_t ph = rph;
            mbar_wait(empty(s), ph ^ 1u);
            const uint32_t sA = base + (uint32_t)s * stage_bytes, sB = sA + A_BYTES;
            if (pt == 0) {
              mbar_arrive_expect_tx(full(s), b_bytes);
              for (uint32_t pl = 0; pl < PL; ++pl)
                for (int a = 0; a < p.bn_smem / C::EPA; ++a)
                  tma_load_2d(sB + pl * b_bytes1 + (uint32_t)a * C::MN_LBO, pl ? &tmapB2 : &tmapB,
                              full(s), n0 + a * C::EPA, kb * C::BKP);
            }
#pragma unroll
            for (int i = 0; i < 8; ++i) {
              const int r = r0 + RPP * i;
              const int pix = kb * C::BKP + r;
              bool ok = mvalid && pix < g.n_pixels;
              uint32_t n, rem, oh, ow;
              g.div_hw.divmod((uint32_t)(ok ? pix : 0), n, rem);
              g.div_w.divmod(rem, oh, ow);
              const int ih = (int)oh * g.stride + offh, iw = (int)ow * g.stride_w + offw;
              ok = ok && ih >= 0 && ih < g.src_h && iw >= 0 && iw < g.src_w;
              const uint8_t *src = static_cast<const uint8_t *>(g.src);
              if (ok)
                src += ((size_t)((size_t)n * g.src_h * g.src_w + (size_t)ih * g.src_w + iw) *
                            g.src_cp + c) * ELEM;
              uint32_t dst;
              if (ELEM == 2)  // SWIZZLE_128B: 16-byte chunks XOR row%8, 8-row (1 KB) K-groups
                dst = sA + dcol + (uint32_t)(r >> 3) * 1024u + (uint32_t)(r & 7) * 128u +
                      (uint32_t)((jj ^ (r & 7)) << 4);
              else            // SWIZZLE_128B_BASE32B: 32-byte chunks XOR row%4, 4-row K-groups
                dst = sA + dcol + (uint32_t)(r >> 2) * 512u + (uint32_t)(r & 3) * 128u +
                      (uint32_t)((((jj >> 1) ^ (r & 3)) << 5) | ((jj & 1) << 4));
              cp_async16(dst, src, ok);
              if (X3) cp_async16(dst + A_BYTES1, src + p.lo_off_a, ok);
            }
            cp_async_mbar_arrive_noinc(full(s));
          }
        }
      }
    }
  } else if (warp == MW) {
    // ===================================== MMA issuer ======================================
    if (leader) {   // whole warp runs the loop; each tcgen05 op is issued by an elected lane
      constexpr uint32_t fmt = (ELEM == 2) ? 1u : 2u;  // BF16 : TF32
      constexpr uint32_t mn = (MODE == MODE_WGRAD) ? 1u : 0u;
      const uint32_t idesc = make_idesc(fmt, mn, mn, 128u * CG, (uint32_t)p.bn);
      constexpr int KSTEPS = (MODE == MODE_WGRAD) ? C::BKP / C::UMMA_K : C::BK / C::UMMA_K;
      constexpr int DSTEP = (int)(((MODE == MODE_WGRAD) ? C::MN_KSTEP : 32u) >> 4);
      // Descriptors of slot 0 (sub-block 0, k 0); the start-address field (bits [0,14), bytes/16)
      // of a shared address < 256 KB never carries, so later operands are plain 64-bit adds.
      uint64_t da0, db0;
      if (MODE == MODE_WGRAD) {
        da0 = make_sdesc(base, C::MN_LBO, C::MN_GROUP, C::MN_LAYOUT);
        db0 = make_sdesc(base + (uint32_t)p.ksub * A_BYTES, C::MN_LBO, C::MN_GROUP, C::MN_LAYOUT);
      } else {
        da0 = make_sdesc(base, 16u, C::K_SBO, C::K_LAYOUT);
        db0 = make_sdesc(base + (uint32_t)p.ksub * A_BYTES, 16u, C::K_SBO, C::K_LAYOUT);
      }
      const uint64_t stage16 = stage_bytes >> 4, b16 = b_bytes >> 4;
      const uint64_t alo16 = A_BYTES1 >> 4, blo16 = b_bytes1 >> 4;   // lo planes (X3)
      // mixed split: descriptors of the bf16(hi) planes as a constant difference to the tf32 hi
      // descriptor of the same slot (start address + plane offset, bf16 layout fields), and the
      // bf16(v - hi) planes half a tf32 plane further; bf16 tiles are 64-byte rows (SWIZZLE_64B)
      uint64_t dA1 = 0, dB1 = 0;
      const uint64_t ablo16 = (A_BYTES1 / 2) >> 4, bblo16 = (b_bytes1 / 2) >> 4;
      const uint32_t idesc_b = make_idesc(1u, mn, mn, 128u * CG, (uint32_t)p.bn);
      constexpr int BSTEP = (MODE == MODE_WGRAD) ? (16 * 64) >> 4 : 32 >> 4;
      if (MIX) {
        const uint32_t aB = base + A_BYTES1, bB = base + (uint32_t)p.ksub * A_BYTES + b_bytes1;
        const uint64_t a1 = (MODE == MODE_WGRAD) ? make_sdesc(aB, C::MN_LBO / 2, 512u, 4u)
                                                 : make_sdesc(aB, 16u, 512u, 4u);
        const uint64_t b1 = (MODE == MODE_WGRAD) ? make_sdesc(bB, C::MN_LBO / 2, 512u, 4u)
                                                 : make_sdesc(bB, 16u, 512u, 4u);
        dA1 = a1 - da0;
        dB1 = b1 - db0;
      }
      (void)idesc_b;
      const int KS = p.ksub, kb_total = p.kb_total;
      const bool skip_mma = GLP_SKIP(p, 4);
      int rs = 0;
      uint32_t rph = 0, it = 0;
      uint64_t da = da0, db = db0;   // descriptors of ring slot rs
#ifdef GLP_DIAG
      const bool clk = p.dbg_clk != nullptr;
#else
      constexpr bool clk = false;
#endif
      long long c_t0 = clk ? clock64() : 0, c_full = 0, c_te = 0;
      (void)c_t0;
      if constexpr (X3) {
        // 3xTF32: chunks of p.chunk_kb k-blocks, each accumulated from zero into TMEM buffer
        // (chunk count & 1); the epilogue sums the chunks of a tile in fp32 registers
        const int CK = p.chunk_kb;
        uint32_t gch = 0;   // chunks started by this CTA
        for (int tile = unit0; tile < total_tiles; tile += ustep) {
          int m_tile, n_tile, split;
          decode_tile(tile, p.n_tiles, p.m_tiles, m_tile, n_tile, split);
          int kb0 = 0, kb1 = kb_total;
          if (MODE == MODE_WGRAD) {
            wgrad_kb_range(p, split, kb0, kb1);
          }
          uint32_t acc = 0, d = tmem_base, cur = 0;
          int next_chunk = kb0;   // first k-block of the next chunk
          for (int kbs = kb0; kbs < kb1; kbs += KS) {
            mbar_wait(full(rs), rph);
            tc_fence_after();
            const int nsub = min(KS, kb1 - kbs);
#pragma unroll
            for (int sub = 0; sub < 4; ++sub) {
              if (sub >= nsub) break;
              if (kbs + sub == next_chunk) {   // chunk boundary: publish the finished chunk
                if (next_chunk != kb0) mma_commit_e<CG>(tfull(cur));
                cur = gch & 1u;
                mbar_wait(tempty(cur), ((gch >> 1) & 1u) ^ 1u);
                tc_fence_after();
                ++gch;
                d = tmem_base + cur * (uint32_t)p.acc_cols;
                acc = 0;
                next_chunk += CK;
              }
              const uint64_t a_ = da + (uint64_t)(sub * (A_BYTES >> 4)), b_ = db + (uint64_t)sub * b16;
              if constexpr (MIX)
                mma_kblock_mix_e<CG, DSTEP, BSTEP>(d, a_, b_, a_ + dA1, b_ + dB1, a_ + dA1 + ablo16,
                                                   b_ + dB1 + bblo16, idesc, idesc_b, acc);
              else
                mma_kblock_x3_e<CG, KSTEPS, DSTEP>(d, a_, b_, alo16, blo16, idesc, acc);
              acc = 1;
            }
            mma_commit_e<CG>(empty(rs));
            if (++rs == S_) {
              rs = 0;
              rph ^= 1u;
              da = da0;
              db = db0;
            } else {
              da += stage16;
              db += stage16;
            }
          }
          mma_commit_e<CG>(tfull(cur));
        }
      } else
      for (int tile = unit0; tile < total_tiles; tile += ustep, ++it) {
        int m_tile, n_tile, split;
        decode_tile(tile, p.n_tiles, p.m_tiles, m_tile, n_tile, split);
        int kb0 = 0, kb1 = kb_total;
        if (MODE == MODE_WGRAD) {
          wgrad_kb_range(p, split, kb0, kb1);
        }
        const uint32_t a = it & 1u, aph = (it >> 1) & 1u;
        long long c0 = clk ? clock64() : 0;
        mbar_wait(tempty(a), aph ^ 1u);
        if (clk) c_te += clock64() - c0;
        tc_fence_after();
        const uint32_t d = tmem_base + a * (uint32_t)p.acc_cols;
        uint32_t acc = 0;
        for (int kbs = kb0; kbs < kb1; kbs += KS) {
          if (clk) c0 = clock64();
          mbar_wait(full(rs), rph);
          if (clk) c_full += clock64() - c0;
          tc_fence_after();
          const int nsub = min(KS, kb1 - kbs);
#pragma unroll
          for (int sub = 0; sub < 4; ++sub) {
            if (sub >= nsub) break;
            if (!skip_mma || acc == 0)
              mma_kblock_e<(ELEM == 2) ? 0 : 1, CG, KSTEPS, DSTEP>(
                  d, da + (uint64_t)(sub * (A_BYTES >> 4)), db + (uint64_t)sub * b16, idesc, acc);
            acc = 1;
          }
          mma_commit_e<CG>(empty(rs));
          if (++rs == S_) {
            rs = 0;
            rph ^= 1u;
            da = da0;
            db = db0;
          } else {
            da += stage16;
            db += stage16;
          }
        }
        mma_commit_e<CG>(tfull(a));
      }
#ifdef GLP_DIAG
      if (clk && lane == 0) {
        p.dbg_clk[blockIdx.x * 4 + 0] = clock64() - c_t0;
        p.dbg_clk[blockIdx.x * 4 + 1] = c_full;
        p.dbg_clk[blockIdx.x * 4 + 2] = c_te;
      }
#endif
    }
    __syncwarp();
  }
  } else {
    if constexpr (X3) asm volatile("setmaxnreg.inc.sync.aligned.u32 %0;" ::"n"(X3_EPI_REGS));
    // ===================================== epilogue ========================================
    const int row = warp * 32 + lane;   // (X3: warps 4-7 repeat the TMEM lanes of warps 0-3)
    uint32_t it = 0;
    // the whole bias vector staged once in shared memory after the barriers (16-byte aligned,
    // p.bias_floats >= every column a tile can touch, zero past N): the per-chunk global bias
    // load had its latency exposed in every chunk of every tile (ncu: STS waiting on LDG)
    const uint32_t sbias = (tmem_slot + 16u + 15u) & ~15u;
    if (MODE == MODE_FWD) {
      for (int i = row; i < p.bias_floats; i += 32 * EW) {
        float bv = 0.f;
        if (i < p.N) {
          if (p.ybr.n > 1) {
            const int b = p.ybr.branch(i);
            if (p.bias_br[b] != nullptr) bv = __ldg(p.bias_br[b] + (i - p.ybr.off[b]));
          } else if (p.bias != nullptr) {
            bv = __ldg(p.bias + i);
          }
        }
        sts_f32(sbias + 4u * (uint32_t)i, bv);
      }
      named_bar_sync(1, 32 * EW);
    }
    if constexpr (X3) {
      // ---- 3xTF32: sum the tile's chunks in fp32 registers, then store ----
      const int q = warp & 3, hf = warp >> 2;          // TMEM lane quadrant, column half
      const int r = q * 32 + lane;                     // accumulator row of this thread
      const int H0 = min(p.bn, ((p.bn + 1) / 2 + 31) & ~31);
      const int c_lo = hf ? H0 : 0, c_hi = hf ? p.bn : H0;   // <= 128 columns, c_lo % 32 == 0
      const int CK = p.chunk_kb;
      uint32_t gch = 0;
      float S[128];
      for (int tile = unit0; tile < total_tiles; tile += ustep) {
        int m_tile, n_tile, split;
        decode_tile(tile, p.n_tiles, p.m_tiles, m_tile, n_tile, split);
        int kb0 = 0, kb1 = p.kb_total;
        if (MODE == MODE_WGRAD) {
          wgrad_kb_range(p, split, kb0, kb1);
        }
        const int nch = (kb1 - kb0 + CK - 1) / CK;
        for (int ch = 0; ch < nch; ++ch, ++gch) {
          const uint32_t b = gch & 1u;
          mbar_wait(tfull(b), (gch >> 1) & 1u);
          tc_fence_after();
          const uint32_t taddr = tmem_base + ((uint32_t)(q * 32) << 16) + b * (uint32_t)p.acc_cols;
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            if (c_lo + 32 * j < c_hi) {
              uint32_t v[32];
              tmem_ld32(taddr + (uint32_t)(c_lo + 32 * j), v);
              tmem_wait_ld_dep(v);
              if (ch == 0) {
#pragma unroll
                for (int i = 0; i < 32; ++i) S[32 * j + i] = __uint_as_float(v[i]);
              } else {
#pragma unroll
                for (int i = 0; i < 32; ++i) S[32 * j + i] += __uint_as_float(v[i]);
              }
            }
          }
          tc_fence_before();
          __syncwarp();
          if (lane == 0) {   // chunk buffer drained: one arrival per warp (on the pair leader)
            if (CG == 1) mbar_arrive_relaxed(tempty(b));
            else mbar_arrive_cluster_relaxed(mapa_shared(tempty(b), 0));
          }
        }
        const int m = (m_tile * CG + (int)rank) * C::BM + r;
        const int n0 = n_tile * p.bn;
        if (m >= p.M || GLP_SKIP(p, 8)) continue;
        if (MODE != MODE_WGRAD) {
          uint32_t n, pimg;
          g.div_hw.divmod((uint32_t)m, n, pimg);
          const size_t plane = (size_t)p.out_hw;
          // columns [c_lo, c_lo + lim) of this tile exist; lanes are 32 consecutive pixels, so
          // each store writes one channel's 128-byte pixel run; the pointer steps one plane
          const int lim = min(c_hi, p.N - n0) - c_lo;
          const uint32_t sb = sbias + 4u * (uint32_t)(n0 + c_lo);
          if (MODE == MODE_FWD && p.ybr.n > 1) {   // fused sibling group: per-branch tensors
            // one branch lookup per 32-column chunk (a chunk straddling two branches, at most one
            // per branch boundary, takes the per-element lookup)
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              if (32 * j >= lim) continue;
              const int cf = n0 + c_lo + 32 * j, lj = min(32, lim - 32 * j);
              if (p.ybr.branch(cf) == p.ybr.branch(cf + lj - 1)) {
                float *o = p.ybr.at(cf, n, plane, pimg);
#pragma unroll
                for (int i = 0; i < 32; ++i) {
                  if (i < lj) o[0] = S[32 * j + i] + lds_f32(sb + 4u * (uint32_t)(32 * j + i));
                  o += plane;
                }
              } else {
#pragma unroll
                for (int i = 0; i < 32; ++i)
                  if (i < lj)
                    *p.ybr.at(cf + i, n, plane, pimg) = S[32 * j + i] + lds_f32(sb + 4u * (uint32_t)(32 * j + i));
              }
            }
          } else {
            float *o = p.out + (size_t)n * p.out_c * plane + pimg + (size_t)(n0 + c_lo) * plane;
#pragma unroll
            for (int j = 0; j < 4; ++j) {
              if (32 * j + 32 <= lim) {
#pragma unroll
                for (int i = 0; i < 32; i += 4) {
                  float4 b4 = make_float4(0.f, 0.f, 0.f, 0.f);
                  if (MODE == MODE_FWD) b4 = lds_f32x4(sb + 4u * (uint32_t)(32 * j + i));
                  o[0] = S[32 * j + i] + b4.x;
                  o += plane;
                  o[0] = S[32 * j + i + 1] + b4.y;
                  o += plane;
                  o[0] = S[32 * j + i + 2] + b4.z;
                  o += plane;
                  o[0] = S[32 * j + i + 3] + b4.w;
                  o += plane;
                }
              } else if (32 * j < lim) {
#pragma unroll
                for (int i = 0; i < 32; ++i) {
                  if (32 * j + i < lim)
                    o[0] = S[32 * j + i] +
                           ((MODE == MODE_FWD) ? lds_f32(sb + 4u * (uint32_t)(32 * j + i)) : 0.f);
                  o += plane;
                }
              }
            }
          }
        } else {
          float *dst = p.out + ((size_t)split * p.part_mpad + (size_t)m) * p.part_ld + n0;
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const int c = c_lo + 32 * j;
            if (c + 32 <= c_hi) {
#pragma unroll
              for (int i = 0; i < 32; i += 4)
                *reinterpret_cast<float4 *>(dst + c + i) =
                    make_float4(S[32 * j + i], S[32 * j + i + 1], S[32 * j + i + 2], S[32 * j + i + 3]);
            } else {
#pragma unroll
              for (int i = 0; i < 32; ++i)
                if (c + i < c_hi) dst[c + i] = S[32 * j + i];
            }
          }
        }
      }
    } else {
#ifdef GLP_DIAG
    const bool clk = p.dbg_clk != nullptr && warp == 0;
#else
    constexpr bool clk = false;
#endif
    long long e_t0 = clk ? clock64() : 0, e_wait = 0, e_ld = 0;
    (void)e_t0;
    for (int tile = unit0; tile < total_tiles; tile += ustep, ++it) {
      int m_tile, n_tile, split;
      decode_tile(tile, p.n_tiles, p.m_tiles, m_tile, n_tile, split);
      const uint32_t a = it & 1u, aph = (it >> 1) & 1u;
      long long c0 = clk ? clock64() : 0;
      // plain try_wait (suspends in hardware); GLP_DEBUG_SKIP bit 16 selects a nanosleep back-off
      if (GLP_SKIP(p, 16)) mbar_wait_sleep(tfull(a), aph);
      else mbar_wait(tfull(a), aph);
      if (clk) e_wait += clock64() - c0;
      tc_fence_after();
      const int m = (m_tile * CG + (int)rank) * C::BM + row;
      const int n0 = n_tile * p.bn;
      const bool mv = m < p.M && !GLP_SKIP(p, 8);
      const uint32_t taddr = tmem_base + ((uint32_t)(warp * 32) << 16) + a * (uint32_t)p.acc_cols;
      if (MODE != MODE_WGRAD) {
        uint32_t n, pimg;
        g.div_hw.divmod((uint32_t)(mv ? m : 0), n, pimg);
        float *outp = p.out + (size_t)n * p.out_c * p.out_hw + pimg;
        // lanes are 32 consecutive pixels: each store writes one channel's 128-byte pixel run.
        // The chunk's 32 biases go through a per-warp smem slot (8 broadcast 16-byte loads, not
        // 32 shuffles); the output pointer advances one channel plane per store.
        const size_t plane = (size_t)p.out_hw;
        float *ob = outp + (size_t)n0 * plane;
        const uint32_t sb_tile = sbias + 4u * (uint32_t)n0;
        // one 32-column chunk: bias add + 32 coalesced 128-byte stores (one per channel)
        auto store_chunk = [&](int c0, uint32_t (&v)[32]) {
          const int lim = min(32, min(p.bn - c0, p.N - n0 - c0));
          float *o = ob + (size_t)c0 * plane;
          bool split_chunk = false;   // fused group: the chunk straddles two branch tensors
          if (MODE == MODE_FWD && p.ybr.n > 1 && lim > 0) {
            const int cf = n0 + c0;
            const int b = p.ybr.branch(cf);
            split_chunk = p.ybr.branch(cf + lim - 1) != b;
            o = p.ybr.at(cf, n, plane, pimg);
          }
          if (MODE == MODE_FWD && split_chunk) {
            if (mv) {
#pragma unroll
              for (int q = 0; q < 32; ++q)
                if (q < lim)
                  *p.ybr.at(n0 + c0 + q, n, plane, pimg) =
                      __uint_as_float(v[q]) + lds_f32(sb_tile + 4u * (uint32_t)(c0 + q));
            }
          } else if (mv && lim == 32) {
#pragma unroll
            for (int q = 0; q < 32; q += 4) {
              float4 b4 = make_float4(0.f, 0.f, 0.f, 0.f);
              if (MODE == MODE_FWD) b4 = lds_f32x4(sb_tile + 4u * (uint32_t)(c0 + q));
              o[0] = __uint_as_float(v[q]) + b4.x;
              o += plane;
              o[0] = __uint_as_float(v[q + 1]) + b4.y;
              o += plane;
              o[0] = __uint_as_float(v[q + 2]) + b4.z;
              o += plane;
              o[0] = __uint_as_float(v[q + 3]) + b4.w;
              o += plane;
            }
          } else if (mv) {
#pragma unroll
            for (int q = 0; q < 32; ++q) {
              const float b = (MODE == MODE_FWD) ? lds_f32(sb_tile + 4u * (uint32_t)(c0 + q)) : 0.f;
              if (q < lim) o[(size_t)q * plane] = __uint_as_float(v[q]) + b;
            }
          }
        };
        // software-pipelined TMEM drain: the next chunk's tcgen05.ld is in flight while the
        // current chunk is stored (the load latency was exposed once per chunk: ncu long-scoreboard
        // stalls on the first use of every chunk)
        uint32_t va[32], vb[32];
        long long c1 = clk ? clock64() : 0;
        tmem_ld32(taddr, va);
        tmem_wait_ld_dep(va);
        if (clk) e_ld += clock64() - c1;
        for (int c0 = 0; c0 < p.bn; c0 += 64) {
          const bool hb = c0 + 32 < p.bn;
          if (hb) tmem_ld32(taddr + (uint32_t)(c0 + 32), vb);
          store_chunk(c0, va);
          if (hb) {
            tmem_wait_ld_dep(vb);
            const bool ha = c0 + 64 < p.bn;
            if (ha) tmem_ld32(taddr + (uint32_t)(c0 + 64), va);
            store_chunk(c0 + 32, vb);
            if (ha) tmem_wait_ld_dep(va);
          }
        }
      } else {
        float *dst = p.out + ((size_t)split * p.part_mpad + (size_t)m) * p.part_ld + n0;
        for (int c0 = 0; c0 < p.bn; c0 += 32) {
          uint32_t v[32];
          tmem_ld32(taddr + (uint32_t)c0, v);
          tmem_wait_ld();
          if (mv) {
            const int lim = min(32, p.bn - c0);
            if (lim == 32) {
#pragma unroll
              for (int q = 0; q < 32; q += 4)
                *reinterpret_cast<float4 *>(dst + c0 + q) =
                    make_float4(__uint_as_float(v[q]), __uint_as_float(v[q + 1]),
                                __uint_as_float(v[q + 2]), __uint_as_float(v[q + 3]));
            } else {
#pragma unroll
              for (int q = 0; q < 32; ++q)
                if (q < lim) dst[c0 + q] = __uint_as_float(v[q]);
            }
          }
        }
      }
      tc_fence_before();
      __syncwarp();
      if (lane == 0) {   // one arrival per warp (on the pair leader's barrier for CG2)
        if (CG == 1) mbar_arrive_relaxed(tempty(a));
        else mbar_arrive_cluster_relaxed(mapa_shared(tempty(a), 0));
      }
    }
#ifdef GLP_DIAG
    if (clk && lane == 0) {
      p.dbg_clk[gridDim.x * 4 + blockIdx.x * 4 + 0] = clock64() - e_t0;
      p.dbg_clk[gridDim.x * 4 + blockIdx.x * 4 + 1] = e_wait;
      p.dbg_clk[gridDim.x * 4 + blockIdx.x * 4 + 2] = e_ld;
      p.dbg_clk[gridDim.x * 4 + blockIdx.x * 4 + 3] = it;
    }
#endif
    }
  }
  // all tiles done: the next kernel may start launching into the teardown
  pdl_launch_dependents();
  tc_fence_before();
  if (CG == 2) cluster_sync();
  else __syncthreads();
  tc_fence_after();
  if (warp == MW) tmem_dealloc_cg<CG>(tmem_base, (uint32_t)p.tmem_cols);
}

}  // namespace glp
