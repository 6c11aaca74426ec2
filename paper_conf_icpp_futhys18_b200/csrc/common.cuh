// common.cuh — shared device/host structs of the conv hot path (not shared with the oracle).
#pragma once
#include <cstdint>

namespace glp {

// Division by a run-time constant via multiply-high (valid for 0 <= n < 2^31).
struct FastDiv {
  uint32_t d, mul, shr;
  __host__ __device__ FastDiv() : d(1), mul(0), shr(0) {}
  __host__ __device__ explicit FastDiv(uint32_t div) : d(div) {
    uint32_t l = 0;
    while ((1ull << l) < div) ++l;
    shr = l;
    mul = (uint32_t)(((1ull << 32) * ((1ull << l) - div)) / div + 1);
  }
  __device__ __forceinline__ uint32_t div(uint32_t n) const {
    return (uint32_t)(((uint64_t)__umulhi(n, mul) + n) >> shr);
  }
  __device__ __forceinline__ void divmod(uint32_t n, uint32_t &q, uint32_t &r) const {
    q = div(n);
    r = n - q * d;
  }
};

enum ConvMode : int { MODE_FWD = 0, MODE_DGRAD = 1, MODE_WGRAD = 2 };

// Diagnostic work-skipping (timing isolation of pipeline stages, wrong results) exists only in
// -DGLP_DIAG builds; the product library compiles every test to a constant false.
#ifdef GLP_DIAG
#define GLP_SKIP(p, bit) ((((p).dbg_skip) & (bit)) != 0)
#else
#define GLP_SKIP(p, bit) false
#endif

// Geometry of the activation gather (im2col never materialised).  The "pixel space" is the
// GEMM's pixel dimension: y pixels for fwd (M) and wgrad (K), dx pixels for dgrad (M).
struct Gather {
  const void *src;       // packed NHWC source: x (fwd, wgrad) or dy (dgrad)
  int src_h, src_w;      // source image dims
  int src_cp;            // channel pitch of the packed source (elements)
  int pix_hw, pix_w;     // pixel-space dims (H_o*W_o, W_o) for fwd/wgrad; (H*W, W) for dgrad
  int stride, pad;       // conv stride / pad (symmetric in h and w: stride_h == stride_w here)
  int stride_w, pad_w;
  int kw, taps;          // K_w, K_h*K_w
  int cp;                // channel pitch of the K (or M for wgrad) index: k = tap*cp + c
  int n_pixels;          // N * pix_hw
  FastDiv div_hw, div_w, div_cp, div_kw;
  // im2col-TMA view of the same gather (a_tma): base pixel of output pixel (o_h, o_w) is
  // (o_h*im_sh - im_ph, o_w*im_sw - im_pw); tap offsets are added by the TMA unit.
  int im_sh, im_sw, im_ph, im_pw;
  int cbs;               // channel blocks (of the K-block width) per tap, fwd/dgrad
};

// Output channel c of a horizontally fused sibling group (convolutions that
// read the same x with the same K/S/P, run as one GEMM over C_o = sum of the branches) -> the
// branch tensor it belongs to.  n = 1: a single layer, p[0] holds every channel.
constexpr int GLP_MAXBR = 4;
struct BrOut {
  int n;
  int off[GLP_MAXBR + 1];   // first channel of each branch; off[n] = total channels
  float *p[GLP_MAXBR];
  __host__ __device__ __forceinline__ int branch(int c) const {
    int b = 0;
    for (int k = 1; k < GLP_MAXBR; ++k) b += (k < n && c >= off[k]) ? 1 : 0;
    return b;
  }
  // element (plane q) of channel c in a [rows][C_b][plane] branch tensor, e.g. dW (rows = 1,
  // plane = C*K*K), db (plane = 1), y (rows = N, plane = H_o*W_o)
  __host__ __device__ __forceinline__ float *at(int c, size_t row, size_t plane, size_t q) const {
    const int b = branch(c);
    return p[b] + (row * (size_t)(off[b + 1] - off[b]) + (size_t)(c - off[b])) * plane + q;
  }
};

struct IgemmParams {
  Gather g;
  int M, N;              // valid GEMM extents
  int m_tiles, n_tiles, splits;
  int kb_total;          // k-blocks over the whole K extent
  int kb_per_split;
  int kb_per_leaf;       // wgrad leaf plans: k-blocks per leaf (0: no leaves)
  int splits_per_leaf;   // wgrad leaf plans: splits per leaf (0: no leaves)
  int bn;                // N tile (multiple of 16, <= 256)
  int bn_smem;           // rows/cols of B held in smem per stage
  int stages;
  int tmem_cols;         // columns allocated (power of 2 >= 2 * acc_cols)
  int acc_cols;          // columns per accumulator buffer
  // epilogue
  float *out;            // y (fwd) / dx (dgrad) NCHW, or split partials (wgrad)
  const float *bias;     // fwd only, may be null
  int bias_floats;       // fwd: floats of the smem bias stage (>= n_tiles*bn rounded to 32)
  BrOut ybr;             // fwd of a fused sibling group (ybr.n > 1): per-branch y tensors
  const float *bias_br[GLP_MAXBR];   // and per-branch biases (each may be null)
  int out_c;             // channels of out (C_o fwd, C_i dgrad)
  int out_hw;            // H_o*W_o (fwd) / H*W (dgrad)
  int part_ld;           // wgrad partial leading dimension (n_tiles * bn)
  int part_mpad;         // wgrad partial rows per split (m_tiles * 128)
  int a_tma;             // 1: A operand by im2col TMA (one thread); 0: cp.async gather
  int ksub;              // k-blocks per pipeline stage (1 or 2; cp.async path: 1)
  int b3d;               // wgrad: the MN-major B tile by one 3-D TMA load (all atoms) per plane
  long long lo_off_a;    // 3xTF32: byte offset from the packed A source's hi plane to its lo plane
  int chunk_kb;          // 3xTF32: k-blocks per TMEM accumulation chunk (summed in fp32 registers)
#ifdef GLP_DIAG
  unsigned long long *dbg_clk;  // diagnostics only (GLP_DEBUG_CLK): per-CTA cycle counters
                                //   [0] MMA loop total [1] MMA waits on full [2] MMA waits on tempty
                                //   [3] producer waits on empty
#endif
  int dbg_skip;          // diagnostics builds only (-DGLP_DIAG, GLP_DEBUG_SKIP): bit0 skip A loads,
                         // bit1 skip B loads, bit2 skip MMAs — results are garbage, timings isolate
                         // stages.  Product builds compile every GLP_SKIP test to false.
};

}  // namespace glp
