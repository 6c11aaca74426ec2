// hdgrad.cuh — backward-data pass of a unit-stride layer with a shared halo tile (CaffeNet conv2).
//
// dx[n][ci][h][w] = sum_{kh',kw',co} dy[n][co][h - Q + kh'][w - Q + kw'] * Wt[ci][(kh',kw',co)]
// with Q = K - 1 - P and the flipped taps kh' = K-1-kh of Wt (Alg. 2 P101-121: GEMM then
// col2im, here one gather with every dx element owned by one CTA; north_star (3)).
//
// Why: the im2col backward-data re-reads every dy element K_h*K_w times from L2 (25x for conv2);
// with N = C_i = 96 each A byte feeds only 96 columns, and L2 -> SM traffic, not the tensor pipe,
// bounded the kernel (192 us; 144 us with the A loads skipped).  Here a tile is R whole output rows
// of one image, each padded to a pitch of WQ pixels (WQ * R = 128 GEMM rows, m = r*WQ + w).  One
// 4-D TMA of the packed NHWC dy per 64-channel block stages the halo [h0, h0 + R + K - 1) x
// [-Q, WQ - Q) (out-of-bounds -> zeros: the padding), so in shared memory dy row (h, w) of the
// tile sits at row (h - h0)*WQ + (w + Q) and tap (kh', kw')'s A operand is the same tile read from
// row offset kh'*WQ + kw' — one K-major SWIZZLE_128B descriptor per tap (tcgen05 swizzles on
// absolute smem addresses: tools/shift_probe.cu).  Columns w >= W of each output row are computed
// and dropped (27/32 useful for conv2).  CTA pairs (cluster of 2, tcgen05.mma.cta_group::2,
// M = 256): each CTA stages its own tile's halo and half of every weight slice, the leader issues
// the MMAs for both; L2 traffic per 128 rows: 32 KB of dy halo per channel block + half of Wt,
// against 12.8 KB x 128 of im2col A + half of Wt before.  (A single-CTA two-tile form measured
// ~80 cycles per M = 128, N = 96 MMA against ~56 per SM for the pair.)
//
// Persistent: pair unit u (tiles 2u, 2u+1) -> CTA pair u mod (grid/2).  CTA = 192 threads: warps
// 0-3 epilogue, warp 4 TMA producer, warp 5 TMEM owner + MMA issuer (leader only).  Rings: A (the
// CTA's halo tile per 64-channel block) and B (b_taps (tap, block) slices of half of Wt); TMEM: two
// accumulator buffers.
#pragma once
#include "common.cuh"
#include "ptx.cuh"

namespace glp {

constexpr int HD_THREADS = 192;

struct HdgradParams {
  int K;                   // square kernel (taps = K*K)
  int Q;                   // K - 1 - P (halo offset)
  int WQ, R;               // row pitch of a tile (pixels) and output rows per tile (WQ*R = 128)
  int H, W;                // dx image (output of this pass)
  int Ho, Wo;              // dy image (the packed operand)
  int N;                   // images
  int tiles_img;           // ceil(H / R)
  int units;               // ceil(N * tiles_img / 2)
  int ncb;                 // 128-byte channel blocks of C_o (64 bf16 / 32 tf32; the K per tap)
  int cop;                 // channel pitch of the packed dy / K pitch per tap of Wt
  int bn;                  // C_i rounded up to 16 (<= 256)
  int ci;                  // valid output channels
  int acc_cols;            // TMEM columns per accumulator (multiple of 32)
  int tmem_cols;
  int a_bytes;             // one A stage: this CTA's halo tile, (R + K - 1) * WQ rows x 128 B
  int b_tap_bytes;         // one tap's B slice of this CTA: bn/2 rows x 128 B (1024-aligned)
  int b_taps;              // taps per B stage (more MMAs per barrier round trip of the issuer)
  int b_bytes;             // one B stage: b_taps slices
  int a_stages, b_stages;
  // mixed fp32 split (MIX): each A stage is [hi | bf16(hi) | bf16(v - hi)] halo tiles and each
  // tap's B slice [hi | bf16(hi) | bf16(v - hi)] (tf32 128-byte rows, bf16 64-byte rows)
  int a_hi_bytes, a_bf_bytes;   // one plane of one A stage (1024-aligned)
  int b_hi_bytes, b_bf_bytes;   // one plane of one tap's B slice (1024-aligned)
  int chunk_kb;                 // MIX: k-blocks ((channel block, tap) pairs) per TMEM chunk
  float *out;              // dx NCHW fp32
  int out_c;               // channels per image of dx
  int dbg_skip;            // diagnostics: bit0 skip A loads, bit1 skip B loads, bit2 MMAs, bit3 stores
};

// ELEM 2: bf16 operands, 64-channel blocks (kind::f16); ELEM 4: tf32 operands stored as fp32 bit
// patterns, 32-channel blocks (kind::tf32).  Either way a channel block is one 128-byte K-major row
// per pixel and four MMAs (K = 16 bf16 / 8 tf32) consume it, so the halo geometry, the rings and
// the descriptors are the same bytes.
//
// MIX = 1 (ELEM 4; GLP_MATH_FP32 by the mixed split, igemm.cuh X3 = 2): every operand is a tf32 hi
// plane and two bf16 planes, bf16(hi) and bf16(v - hi); a 32-channel block stages the three halo
// tiles (tmapDy, tmapDy2, tmapDy3: 128-byte SWIZZLE_128B rows and two 64-byte SWIZZLE_64B rows per
// pixel) and each tap's B slice the three weight planes (tmapW, tmapW2, tmapW3).  A tap's row shift
// applies to the bf16 tiles as to the tf32 one (64 B per row; the swizzle works on absolute smem
// address bits).  Per (channel block, tap) k-block: four tf32 MMAs hi*hi and four bf16 MMAs of the
// two cross terms (mma_kblock_mix_e), and -- the tensor core truncates each MMA result, igemm.cuh
// X3 -- the k-blocks, in (channel block, tap) order, are cut into chunks of p.chunk_kb, each
// accumulated from zero in one of two TMEM buffers, the 4 epilogue warps summing the chunks of a
// tile in fp32 registers (<= 128 columns per thread) before the store.
template <int ELEM, int MIX>
__global__ void __launch_bounds__(HD_THREADS, 1)
    hdgrad_kernel(const __grid_constant__ HdgradParams p, const __grid_constant__ CUtensorMap tmapDy,
                  const __grid_constant__ CUtensorMap tmapW, const __grid_constant__ CUtensorMap tmapDy2,
                  const __grid_constant__ CUtensorMap tmapW2, const __grid_constant__ CUtensorMap tmapDy3,
                  const __grid_constant__ CUtensorMap tmapW3) {
  static_assert(!MIX || ELEM == 4, "the mixed split has tf32 hi planes");
  constexpr int CB = 128 / ELEM;                   // channels per 128-byte block
  constexpr uint32_t FMT = ELEM == 2 ? 1u : 2u;    // instruction-descriptor operand format
  constexpr int KIND = ELEM == 2 ? 0 : 1;          // kind::f16 / kind::tf32
  extern __shared__ uint8_t smem_raw[];
  const uint32_t raw = smem_u32(smem_raw);
  const uint32_t base = (raw + 1023u) & ~1023u;
  const uint32_t sA0 = base;
  const uint32_t sB0 = sA0 + (uint32_t)(p.a_stages * p.a_bytes);
  const uint32_t bars = sB0 + (uint32_t)(p.b_stages * p.b_bytes);
  const int SA = p.a_stages, SB = p.b_stages;
  auto afull = [&](int s) { return bars + 8u * s; };
  auto aempty = [&](int s) { return bars + 8u * (SA + s); };
  auto bfull = [&](int s) { return bars + 8u * (2 * SA + s); };
  auto bempty = [&](int s) { return bars + 8u * (2 * SA + SB + s); };
  auto tfull = [&](int a) { return bars + 8u * (2 * SA + 2 * SB + a); };
  auto tempty = [&](int a) { return bars + 8u * (2 * SA + 2 * SB + 2 + a); };
  const uint32_t tmem_slot = bars + 8u * (2 * SA + 2 * SB + 4);
  volatile uint32_t *tmem_slot_ptr =
      reinterpret_cast<volatile uint32_t *>(smem_raw + (tmem_slot - raw));
  const int warp = __shfl_sync(0xffffffffu, (int)(threadIdx.x >> 5), 0);
  const int lane = threadIdx.x & 31;
  const uint32_t rank = blockIdx.x & 1u;   // CTA in the pair (cluster of 2 along x)
  const bool leader = rank == 0;
  if (threadIdx.x == 0) {
    // full: only the leader's are armed (expect_tx = both CTAs' bytes; the peer's TMAs complete
    // on the leader's barrier); empty / tfull: one multicast tcgen05.commit; tempty: the 8
    // epilogue warps of both CTAs arrive on the leader's barrier
    for (int s = 0; s < SA; ++s) {
      mbar_init(afull(s), 1);
      mbar_init(aempty(s), 1);
    }
    for (int s = 0; s < SB; ++s) {
      mbar_init(bfull(s), 1);
      mbar_init(bempty(s), 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(tfull(a), 1);
      mbar_init(tempty(a), 8);
    }
    fence_mbar_init();
  }
  if (warp == 5) {
    tmem_alloc_cg<2>(tmem_slot, (uint32_t)p.tmem_cols);
    tmem_relinquish_cg<2>();
  }
  if (warp == 4 && lane == 0) {
    tma_prefetch(&tmapDy);
    tma_prefetch(&tmapW);
    if (MIX) {
      tma_prefetch(&tmapDy2);
      tma_prefetch(&tmapW2);
      tma_prefetch(&tmapDy3);
      tma_prefetch(&tmapW3);
    }
  }
  tc_fence_before();
  cluster_sync();
  tc_fence_after();
  pdl_wait();
  const uint32_t tmem_base = __shfl_sync(0xffffffffu, *tmem_slot_ptr, 0);
  const int taps = p.K * p.K;
  const int halo_rows = (p.R + p.K - 1) * p.WQ;
  const int total_tiles = p.N * p.tiles_img;
  const int unit0 = (int)(blockIdx.x >> 1), ustep = (int)(gridDim.x >> 1);
  int my_tile_of_unit_offset = (int)rank;   // tile 2u + rank of pair unit u

  if (warp == 4) {
    // ===================================== producer ========================================
    const bool la = !GLP_SKIP(p, 1), lb = !GLP_SKIP(p, 2);
    const int half = p.bn / 2;
    int as = 0, bs = 0;
    uint32_t aph = 0, bph = 0;
    for (int u = unit0; u < p.units; u += ustep) {
      int tile = 2 * u + my_tile_of_unit_offset;
      if (tile >= total_tiles) tile = total_tiles - 1;   // ragged unit: recompute, dropped
      const int n = tile / p.tiles_img, r0 = (tile - n * p.tiles_img) * p.R;
      for (int cb = 0; cb < p.ncb; ++cb) {
        mbar_wait(aempty(as), aph ^ 1u);
        const uint32_t sA = sA0 + (uint32_t)(as * p.a_bytes);
        // bytes of both CTAs' halo tiles (MIX: 128 + 64 + 64 bytes per pixel)
        if (leader)
          mbar_arrive_expect_tx_e(afull(as), la ? (uint32_t)(2 * halo_rows * (MIX ? 256 : 128)) : 0u);
        if (la) {
          tma_load_4d_cg2_e(sA, &tmapDy, mapa_shared(afull(as), 0), cb * CB, -p.Q, r0 - p.Q, n);
          if (MIX) {
            tma_load_4d_cg2_e(sA + (uint32_t)p.a_hi_bytes, &tmapDy2, mapa_shared(afull(as), 0),
                              cb * CB, -p.Q, r0 - p.Q, n);
            tma_load_4d_cg2_e(sA + (uint32_t)(p.a_hi_bytes + p.a_bf_bytes), &tmapDy3,
                              mapa_shared(afull(as), 0), cb * CB, -p.Q, r0 - p.Q, n);
          }
        }
        if (++as == SA) {
          as = 0;
          aph ^= 1u;
        }
        for (int t0 = 0; t0 < taps; t0 += p.b_taps) {
          const int nsub = min(p.b_taps, taps - t0);
          mbar_wait(bempty(bs), bph ^ 1u);
          const uint32_t sB = sB0 + (uint32_t)(bs * p.b_bytes);
          if (leader)
            mbar_arrive_expect_tx_e(bfull(bs), lb ? (uint32_t)(2 * nsub * half * (MIX ? 256 : 128)) : 0u);
          if (lb)
            for (int j = 0; j < nsub; ++j) {
              const uint32_t sBj = sB + (uint32_t)(j * p.b_tap_bytes);
              const int kx = (t0 + j) * p.cop + cb * CB;
              tma_load_2d_cg2_e(sBj, &tmapW, mapa_shared(bfull(bs), 0), kx, (int)rank * half);
              if (MIX) {
                tma_load_2d_cg2_e(sBj + (uint32_t)p.b_hi_bytes, &tmapW2, mapa_shared(bfull(bs), 0),
                                  kx, (int)rank * half);
                tma_load_2d_cg2_e(sBj + (uint32_t)(p.b_hi_bytes + p.b_bf_bytes), &tmapW3,
                                  mapa_shared(bfull(bs), 0), kx, (int)rank * half);
              }
            }
          if (++bs == SB) {
            bs = 0;
            bph ^= 1u;
          }
        }
      }
    }
  } else if (MIX && warp == 5 && leader) {
    // ============================ MMA issuer (mixed split, chunked) ===========================
    const uint32_t idesc_t = make_idesc(2u, 0u, 0u, 256u, (uint32_t)p.bn);
    const uint32_t idesc_b = make_idesc(1u, 0u, 0u, 256u, (uint32_t)p.bn);
    // bf16 planes: 64-byte K-major rows (SWIZZLE_64B, 8-row groups of 512 bytes), as constant
    // descriptor differences to the tf32 hi plane's descriptor of the same slot
    const uint64_t dA1 = make_sdesc(sA0 + (uint32_t)p.a_hi_bytes, 16u, 512u, 4u) - make_sdesc(sA0, 16u, 1024u, 2u);
    const uint64_t dA2 = dA1 + (uint64_t)(p.a_bf_bytes >> 4);
    const uint64_t dB1 = make_sdesc(sB0 + (uint32_t)p.b_hi_bytes, 16u, 512u, 4u) - make_sdesc(sB0, 16u, 1024u, 2u);
    const uint64_t dB2 = dB1 + (uint64_t)(p.b_bf_bytes >> 4);
    const int CK = p.chunk_kb;
    int as = 0, bs = 0;
    uint32_t aph = 0, bph = 0, gch = 0;
    for (int u = unit0; u < p.units; u += ustep) {
      uint32_t acc = 0, d = tmem_base, cur = 0;
      int kidx = 0;   // k-block index within the tile, (channel block, tap) order
      for (int cb = 0; cb < p.ncb; ++cb) {
        mbar_wait(afull(as), aph);
        tc_fence_after();
        const uint32_t sA = sA0 + (uint32_t)(as * p.a_bytes);
        const uint64_t da0 = make_sdesc(sA, 16u, 1024u, 2u);
        int kh = 0, kw = 0;
        for (int t0 = 0; t0 < taps; t0 += p.b_taps) {
          const int nsub = min(p.b_taps, taps - t0);
          mbar_wait(bfull(bs), bph);
          tc_fence_after();
          const uint64_t db0 = make_sdesc(sB0 + (uint32_t)(bs * p.b_bytes), 16u, 1024u, 2u);
          for (int j = 0; j < nsub; ++j, ++kidx) {
            if (kidx % CK == 0) {   // chunk boundary: publish the finished chunk, take a buffer
              if (kidx) mma_commit_e<2>(tfull(cur));
              cur = gch & 1u;
              mbar_wait(tempty(cur), ((gch >> 1) & 1u) ^ 1u);
              tc_fence_after();
              ++gch;
              d = tmem_base + cur * (uint32_t)p.acc_cols;
              acc = 0;
            }
            // the tap's row shift in the halo tile (diagnostics, GLP_DEBUG_SKIP bit 5: without
            // the kw part -- 8-row-aligned operand starts only; results wrong)
            const int rows = kh * p.WQ + (GLP_SKIP(p, 32) ? 0 : kw);
            const uint64_t a_ = da0 + (uint64_t)(rows * 8);
            const uint64_t ab = da0 + (uint64_t)(rows * 4);   // bf16 rows are 64 bytes
            const uint64_t b_ = db0 + (uint64_t)(j * (p.b_tap_bytes >> 4));
            if (!GLP_SKIP(p, 4) || kidx == 0)
              mma_kblock_mix_e<2, 2, 2>(d, a_, b_, ab + dA1, b_ + dB1, ab + dA2, b_ + dB2, idesc_t,
                                        idesc_b, acc);
            acc = 1;
            if (++kw == p.K) {
              kw = 0;
              ++kh;
            }
          }
          mma_commit_e<2>(bempty(bs));
          if (++bs == SB) {
            bs = 0;
            bph ^= 1u;
          }
        }
        mma_commit_e<2>(aempty(as));
        if (++as == SA) {
          as = 0;
          aph ^= 1u;
        }
      }
      mma_commit_e<2>(tfull(cur));
    }
    __syncwarp();
  } else if (!MIX && warp == 5 && leader) {
    // ===================================== MMA issuer ======================================
    const uint32_t idesc = make_idesc(FMT, 0u, 0u, 256u, (uint32_t)p.bn);
    const bool skip_mma = GLP_SKIP(p, 4);
    int as = 0, bs = 0;
    uint32_t aph = 0, bph = 0, it = 0;
    for (int u = unit0; u < p.units; u += ustep, ++it) {
      const uint32_t a = it & 1u, tph = (it >> 1) & 1u;
      mbar_wait(tempty(a), tph ^ 1u);
      tc_fence_after();
      const uint32_t d0 = tmem_base + a * (uint32_t)p.acc_cols;
      for (int cb = 0; cb < p.ncb; ++cb) {
        mbar_wait(afull(as), aph);
        tc_fence_after();
        const uint32_t sA = sA0 + (uint32_t)(as * p.a_bytes);
        // descriptor of tap 0 (the peer's tile sits at the same offset in its smem); a tap's row
        // shift is a plain add (start field in 16-byte units, no carry below 256 KB)
        const uint64_t da0 = make_sdesc(sA, 16u, 1024u, 2u);
        int kh = 0, kw = 0;
        for (int t0 = 0; t0 < taps; t0 += p.b_taps) {
          const int nsub = min(p.b_taps, taps - t0);
          mbar_wait(bfull(bs), bph);
          tc_fence_after();
          const uint64_t db0 = make_sdesc(sB0 + (uint32_t)(bs * p.b_bytes), 16u, 1024u, 2u);
          for (int j = 0; j < nsub; ++j) {
            // (diagnostics, GLP_DEBUG_SKIP bit 5: drop the kw row shift, i.e. only 8-row-aligned
            // starts; results wrong — isolates the cost of misaligned operand starts)
            const uint64_t sh = (uint64_t)((kh * p.WQ + (GLP_SKIP(p, 32) ? 0 : kw)) * 8);
            const uint64_t db = db0 + (uint64_t)(j * (p.b_tap_bytes >> 4));
            const uint32_t acc = (cb | t0 | j) ? 1u : 0u;
            if (!skip_mma || (cb | t0 | j) == 0) mma_kblock_e<KIND, 2, 4, 2>(d0, da0 + sh, db, idesc, acc);
            if (++kw == p.K) {
              kw = 0;
              ++kh;
            }
          }
          mma_commit_e<2>(bempty(bs));
          if (++bs == SB) {
            bs = 0;
            bph ^= 1u;
          }
        }
        mma_commit_e<2>(aempty(as));
        if (++as == SA) {
          as = 0;
          aph ^= 1u;
        }
      }
      mma_commit_e<2>(tfull(a));
    }
    __syncwarp();
  } else if (MIX && warp < 4) {
    // ========================= epilogue (mixed split: chunk sums) ===========================
    const int m = warp * 32 + lane;
    const int rr = m / p.WQ, ww = m - rr * p.WQ;
    const size_t plane = (size_t)p.H * p.W;
    const int nch = (p.ncb * taps + p.chunk_kb - 1) / p.chunk_kb;
    uint32_t gch = 0;
    float S[128];
    for (int u = unit0; u < p.units; u += ustep) {
      for (int ch = 0; ch < nch; ++ch, ++gch) {
        const uint32_t b = gch & 1u;
        mbar_wait(tfull(b), (gch >> 1) & 1u);
        tc_fence_after();
        const uint32_t taddr = tmem_base + ((uint32_t)(warp * 32) << 16) + b * (uint32_t)p.acc_cols;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          if (32 * j < p.bn) {
            uint32_t v[32];
            tmem_ld32(taddr + (uint32_t)(32 * j), v);
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
        if (lane == 0) mbar_arrive_cluster_relaxed(mapa_shared(tempty(b), 0));
      }
      const int tile = 2 * u + my_tile_of_unit_offset;
      const int n = tile / p.tiles_img, r0 = (tile - n * p.tiles_img) * p.R;
      const int h = r0 + rr;
      if (!(tile < total_tiles && h < p.H && ww < p.W) || GLP_SKIP(p, 8)) continue;
      float *o = p.out + (size_t)n * p.out_c * plane + (size_t)h * p.W + ww;
#pragma unroll
      for (int q = 0; q < 128; ++q) {
        if (q < p.ci) o[0] = S[q];
        o += plane;
      }
    }
  } else if (!MIX && warp < 4) {
    // ===================================== epilogue ========================================
    // warp w holds TMEM lanes 32w..32w+31 = GEMM rows m = r*WQ + w'; lane -> (row, column)
    const int m = warp * 32 + lane;
    const int rr = m / p.WQ, ww = m - rr * p.WQ;
    const size_t plane = (size_t)p.H * p.W;
    uint32_t it = 0;
    for (int u = unit0; u < p.units; u += ustep, ++it) {
      const uint32_t a = it & 1u, tph = (it >> 1) & 1u;
      mbar_wait(tfull(a), tph);
      tc_fence_after();
      {
        const int tile = 2 * u + my_tile_of_unit_offset;
        const int n = tile / p.tiles_img, r0 = (tile - n * p.tiles_img) * p.R;
        const int h = r0 + rr;
        const bool mv = tile < total_tiles && h < p.H && ww < p.W && !GLP_SKIP(p, 8);
        float *ob = p.out + (size_t)n * p.out_c * plane + (size_t)h * p.W + ww;
        const uint32_t taddr = tmem_base + ((uint32_t)(warp * 32) << 16) + a * (uint32_t)p.acc_cols;
        for (int c0 = 0; c0 < p.bn; c0 += 32) {
          uint32_t v[32];
          tmem_ld32(taddr + (uint32_t)c0, v);
          tmem_wait_ld();
          if (!mv) continue;
          const int lim = min(32, p.ci - c0);
          float *o = ob + (size_t)c0 * plane;
#pragma unroll
          for (int q = 0; q < 32; ++q)
            if (q < lim) o[(size_t)q * plane] = __uint_as_float(v[q]);
        }
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
