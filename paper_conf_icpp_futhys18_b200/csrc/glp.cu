// glp.cu — libglp.so: the C ABI of include/glp.h.
//
// Host side of the GLP4NN hot path re-designed for B200:
//   * descriptors (Table 5 parameters, P316),
//   * the kernel analyzer (P167, Eqs 1-9 P214-254) re-derived for sm_100a: CTAs per SM from every
//     per-SM limit, slots = #SM * beta, samples in flight S (the paper's C_out, P254),
//   * the plan ("profile once, execute many", P173): tile shapes, shape-only wgrad split count,
//     stage counts, workspace sizes, persistent grid sizes,
//   * launches of the pack / tcgen05 implicit-GEMM / reduction kernels on the caller's stream.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <string>
#include <utility>
#include <vector>

#include "../../include/glp.h"
#include "common.cuh"
#include "hwgrad.cuh"
#include "hfwd.cuh"
#include "hdgrad.cuh"
#include "igemm.cuh"
#include "pack.cuh"
#include "simt.cuh"

using namespace glp;

namespace {

thread_local std::string g_last_error;

glp_status_t fail(glp_status_t s, const std::string &msg) {
  g_last_error = msg;
  return s;
}
glp_status_t cuda_check(cudaError_t e, const char *what) {
  if (e == cudaSuccess) return GLP_OK;
  return fail(GLP_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}
#define GLP_CUDA(call)                                              \
  do {                                                              \
    glp_status_t _s = cuda_check((call), #call);                    \
    if (_s != GLP_OK) return _s;                                    \
  } while (0)
#define GLP_LAUNCH_CHECK(what)                                      \
  do {                                                              \
    glp_status_t _s = cuda_check(cudaGetLastError(), what);         \
    if (_s != GLP_OK) return _s;                                    \
  } while (0)

inline long long cdiv(long long a, long long b) { return (a + b - 1) / b; }
inline long long rup(long long a, long long b) { return cdiv(a, b) * b; }
inline size_t align1k(size_t a) { return (a + 1023) & ~size_t(1023); }

// per-branch input pointers of a fused sibling group call (n = 1: one tensor, every channel)
struct BrIn {
  int n = 1;
  const float *p[GLP_MAXBR] = {nullptr, nullptr, nullptr, nullptr};
};
inline BrIn br_in1(const float *a) {
  BrIn b;
  b.p[0] = a;
  return b;
}

}  // namespace

struct glp_conv_desc_s {
  int N, C, H, W, Co, Kh, Kw, Sh, Sw, Ph, Pw, Ho, Wo;
  // fused sibling group (glp_conv_group_desc_create): nbr branches, branch b owns output
  // channels [br_off[b], br_off[b+1]) of the C_o = sum view; single layer: nbr = 1
  int nbr = 1;
  int br_off[GLP_MAXBR + 1] = {0, 0, 0, 0, 0};
  int groups = 1;   // Caffe convolution groups (glp_conv_desc_set_groups)
};

namespace {

// ------------------------------------------------------------------ analyzer ---------------
int ctas_per_sm_closed_form(const glp_device_limits_t &L, const glp_kernel_attr_t &k) {
  const int warps = (k.threads + 31) / 32;
  int b = L.max_blocks_per_sm;
  b = std::min(b, L.max_threads_per_sm / std::max(1, warps * 32));
  if (k.regs > 0) {
    const int rpw = (int)rup((long long)k.regs * 32, 256);
    b = std::min(b, L.regs_per_sm / (rpw * warps));
  }
  const int smem_cta = (int)rup(std::max(0, k.smem_bytes), 128) + L.smem_reserved_per_cta;
  b = std::min(b, L.smem_per_sm / smem_cta);
  if (k.tmem_cols > 0 && L.tmem_cols_per_sm > 0) b = std::min(b, L.tmem_cols_per_sm / k.tmem_cols);
  return std::max(0, b);
}

// One pass of the tensor-core path, planned.
struct PassPlan {
  int M = 0, Ng = 0, Kpad = 0;      // GEMM extents (Kpad elements; wgrad: pixels)
  int bn = 0, bn_smem = 0, m_tiles = 0, n_tiles = 0, splits = 1, kb_total = 0, kb_per_split = 0;
  int stages = 0, acc_cols = 0, tmem_cols = 0, smem = 0, tiles = 0, grid = 0, ctas_per_sm = 0;
  int regs = 0, ctas_runtime = 0;
  int a_tma = 0, krow = 128;        // A operand by im2col TMA; K-block row width (bytes)
  int cg = 1, m_units = 0;          // CTAs per MMA (tcgen05 cta_group); work units along M
  int ksub = 1;                     // k-blocks per pipeline stage
  int bias_floats = 0;              // forward: floats of the epilogue's smem bias stage
  int threads = 288;                // CTA size (3xTF32: 512, eight epilogue warps)
  int kb_per_leaf = 0, splits_per_leaf = 0;   // wgrad leaf plans (deterministic exchange)
  int chunk_kb = 0;                 // 3xTF32: k-blocks per TMEM accumulation chunk
};

// Analyzer record of one shipped kernel (Table 2 "profiling input", P194-200): its attributes,
// the closed-form CTAs/SM (Eqs 4-5 re-derived + the sm_100a limits) and the CUDA occupancy API's.
struct KAttr {
  int threads = 0, regs = 0, smem = 0, tmem = 0, model = 0, rt = 0;
};

using TmapEncodeFn = CUresult (*)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                                  const cuuint64_t *, const cuuint64_t *, const cuuint32_t *,
                                  const cuuint32_t *, CUtensorMapInterleave, CUtensorMapSwizzle,
                                  CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
TmapEncodeFn g_encode = nullptr;
std::mutex g_mu;

glp_status_t get_encode() {
  std::lock_guard<std::mutex> lk(g_mu);
  if (g_encode) return GLP_OK;
  void *fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
  if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !fn)
    return fail(GLP_ERR_CUDA, "cuTensorMapEncodeTiled entry point unavailable");
  g_encode = reinterpret_cast<TmapEncodeFn>(fn);
  return GLP_OK;
}

glp_status_t encode_2d(CUtensorMap *map, int elem, const void *ptr, uint64_t inner, uint64_t outer,
                       uint64_t row_bytes, uint32_t box_inner, uint32_t box_outer,
                       CUtensorMapSwizzle swz = CU_TENSOR_MAP_SWIZZLE_128B) {
  cuuint64_t dims[2] = {inner, outer};
  cuuint64_t strides[1] = {row_bytes};
  cuuint32_t box[2] = {box_inner, box_outer};
  cuuint32_t es[2] = {1, 1};
  CUresult r = g_encode(map, elem == 2 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                        2, const_cast<void *>(ptr), dims, strides, box, es,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, swz,
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(GLP_ERR_CUDA, "cuTensorMapEncodeTiled failed (" + std::to_string((int)r) + ")");
  return GLP_OK;
}

// The filter gradient's MN-major B operand (dy packed [pixels][C_o pitch]) as a 3-D tensor
// {atom elements, pixels, atoms}: one box {EPA, BKP, atoms} lands atom-major -- the MN-major
// layout with one atom column of BKP rows per atom -- in a single TMA.
glp_status_t encode_mn3d(CUtensorMap *map, int elem, const void *ptr, uint64_t cpitch, uint64_t pixels,
                         uint32_t epa, uint32_t bkp, uint32_t natoms, CUtensorMapSwizzle swz) {
  cuuint64_t dims[3] = {(cuuint64_t)epa, (cuuint64_t)pixels, (cuuint64_t)(cpitch / epa)};
  cuuint64_t strides[2] = {(cuuint64_t)(cpitch * elem), (cuuint64_t)(epa * elem)};
  cuuint32_t box[3] = {epa, bkp, natoms};
  cuuint32_t es[3] = {1, 1, 1};
  CUresult r = g_encode(map, elem == 2 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                        3, const_cast<void *>(ptr), dims, strides, box, es,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(GLP_ERR_CUDA, "cuTensorMapEncodeTiled (3d) failed (" + std::to_string((int)r) + ")");
  return GLP_OK;
}

using TmapIm2colFn = CUresult (*)(CUtensorMap *, CUtensorMapDataType, cuuint32_t, void *,
                                  const cuuint64_t *, const cuuint64_t *, const int *, const int *,
                                  cuuint32_t, cuuint32_t, const cuuint32_t *, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion,
                                  CUtensorMapFloatOOBfill);
TmapIm2colFn g_encode_im2col = nullptr;
int g_driver_version = 0;

glp_status_t get_encode_im2col() {
  std::lock_guard<std::mutex> lk(g_mu);
  if (g_encode_im2col) return GLP_OK;
  void *fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  cudaError_t e = cudaGetDriverEntryPoint("cuTensorMapEncodeIm2col", &fn, cudaEnableDefault, &q);
  if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !fn)
    return fail(GLP_ERR_CUDA, "cuTensorMapEncodeIm2col entry point unavailable");
  cudaDriverGetVersion(&g_driver_version);
  g_encode_im2col = reinterpret_cast<TmapIm2colFn>(fn);
  return GLP_OK;
}

// im2col tensor map over a packed NHWC activation [N][H][W][cpitch]: dims {cpitch, W, H, N};
// bounding box of base pixels [lower, dim-1+upper] per spatial dim (W, H order), traversal
// strides = conv strides; each load = `pixels` pixels x `chans` channels.
// pitch_w / pitch_h: the allocated image width / height of the buffer when the tensor is the
// top-left W x H region of a larger grid (the padded dy grid of halo plans); 0 = W / H.
glp_status_t encode_im2col(CUtensorMap *map, int elem, const void *ptr, int cpitch, int W, int H,
                           int N, int lower_w, int lower_h, int upper_w, int upper_h, int chans,
                           int pixels, int stride_w, int stride_h, CUtensorMapSwizzle swz,
                           int pitch_w = 0, int pitch_h = 0) {
  if (pitch_w <= 0) pitch_w = W;
  if (pitch_h <= 0) pitch_h = H;
  if (lower_w < -128 || lower_w > 127 || lower_h < -128 || lower_h > 127 || upper_w < -128 ||
      upper_w > 127 || upper_h < -128 || upper_h > 127)
    return fail(GLP_ERR_NOT_SUPPORTED, "im2col corner out of TMA range");
  const uint64_t e = (uint64_t)elem;
  cuuint64_t dims[4] = {(cuuint64_t)cpitch, (cuuint64_t)W, (cuuint64_t)H, (cuuint64_t)N};
  cuuint64_t strides[3] = {cpitch * e, (uint64_t)pitch_w * cpitch * e,
                           (uint64_t)pitch_h * pitch_w * cpitch * e};
  int lower[2] = {lower_w, lower_h}, upper[2] = {upper_w, upper_h};
  cuuint32_t es[4] = {1, (cuuint32_t)stride_w, (cuuint32_t)stride_h, 1};
  CUresult r = g_encode_im2col(map, elem == 2 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                               4, const_cast<void *>(ptr), dims, strides, lower, upper,
                               (cuuint32_t)chans, (cuuint32_t)pixels, es,
                               CU_TENSOR_MAP_INTERLEAVE_NONE, swz,
                               CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS)
    return fail(GLP_ERR_CUDA, "cuTensorMapEncodeIm2col failed (" + std::to_string((int)r) + ")");
  // Same driver workaround CUTLASS applies to im2col descriptors of small tensors (< 128 KiB)
  // on drivers <= 13.1 (cute/atom/copy_traits_sm90_im2col.hpp).
  if (g_driver_version <= 13010 && (uint64_t)N * pitch_h * pitch_w * cpitch * e < 131072)
    reinterpret_cast<uint64_t *>(map)[1] &= ~(1ull << 21);
  return GLP_OK;
}

template <int MODE, int ELEM, int KROW, int CG, int X3>
void *kernel_ptr() {
  return reinterpret_cast<void *>(&igemm_kernel<MODE, ELEM, KROW, CG, X3>);
}
template <int MODE, int CG>
void *igemm_ptr_m(int elem, int krow, int x3) {
  if (elem == 2) return krow == 128 ? kernel_ptr<MODE, 2, 128, CG, 0>() : kernel_ptr<MODE, 2, 64, CG, 0>();
  if (x3 == 2) return kernel_ptr<MODE, 4, 128, CG, 2>();
  return x3 ? kernel_ptr<MODE, 4, 128, CG, 1>() : kernel_ptr<MODE, 4, 128, CG, 0>();
}
// x3: 1 = the 3xTF32 variant (GLP_MATH_FP32: hi/lo operand planes, three MMAs per k-step);
// 2 = the mixed split (tf32 hi*hi + two bf16 cross terms)
void *igemm_ptr(int mode, int elem, int krow, int cg, int x3) {
  if (cg == 2) {
    if (mode == MODE_FWD) return igemm_ptr_m<MODE_FWD, 2>(elem, krow, x3);
    if (mode == MODE_DGRAD) return igemm_ptr_m<MODE_DGRAD, 2>(elem, krow, x3);
    return igemm_ptr_m<MODE_WGRAD, 2>(elem, krow, x3);
  }
  if (mode == MODE_FWD) return igemm_ptr_m<MODE_FWD, 1>(elem, krow, x3);
  if (mode == MODE_DGRAD) return igemm_ptr_m<MODE_DGRAD, 1>(elem, krow, x3);
  return igemm_ptr_m<MODE_WGRAD, 1>(elem, krow, x3);
}

CUtensorMapSwizzle swz_kmajor(int krow) {
  return krow == 128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B;
}
CUtensorMapSwizzle swz_mnmajor(int elem, int krow) {
  if (elem == 4) return CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B;
  return krow == 128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B;
}

int choose_bn(int n) {
  if (n <= 256) return (int)rup(n, 16);
  const int nt = (int)cdiv(n, 256);
  return (int)rup(cdiv(n, nt), 16);
}

// Tile (N tile, CTA pairing) of the fwd / dgrad GEMMs for grids that would leave SMs idle.  No
// split of K: the per-element K order, hence every output bit, does not depend on the tile.
// The default (N tile = ceil-split of N at <= 256, CTA pairs) is kept whenever it yields at least
// two work units per slot (measured: for the large CaffeNet layers smaller tiles cost more in
// A re-reads and per-k-block overhead than the last-round quantisation they save).  Below that,
// time ~ rounds * (k-block MMA cycles ~ 2*bn, floored by the issue loop) picks the tile.
// kb_fixed: a per-k-block cost independent of the N tile, in the units of 2*bn (the MMA work).
// The mixed fp32 split streams three operand planes per k-block against 8 cheap MMAs, so smaller
// N tiles pay relatively more for operand delivery (4 pipeline stages of 48 KB cover fewer MMA
// cycles): on CaffeNet's 13x13 layers N 192 x 5 rounds beats N 128 x 7 rounds (conv3 fwd 208 ->
// 199 us, conv4 dgrad 315 -> 291 us, same box, repeated) while N 128 x 5 rounds still beats N 256
// x 3 rounds for 256 channels (conv5 fwd 217 vs 227 us); kb_fixed = 80 reproduces both.
void choose_tile_mn(int n, long long M, bool cg2_ok, int sm_count, int &bn_out, int &cg_out,
                    int min_units = 2, double kb_fixed = 0.0) {
  const int bn0 = choose_bn(n);
  const int cg0 = cg2_ok ? 2 : 1;
  bn_out = bn0;
  cg_out = cg0;
  const long long units0 = cdiv(M, 128LL * cg0) * cdiv(n, bn0);
  if (units0 >= (long long)min_units * (sm_count / cg0)) return;
  double best_c = 1e300;
  for (int cg = cg0; cg >= 1; --cg) {
    const long long m_units = cdiv(M, 128LL * cg);
    const double slots = std::max(1, sm_count / cg);
    for (int nt = (int)cdiv(n, 256); nt <= 4; ++nt) {
      const int bn = (int)rup(cdiv(n, nt), 16);
      if ((int)cdiv(n, bn) != nt || (cg == 2 && (bn / 2) % 8)) continue;
      const double rounds = std::ceil((double)m_units * nt / slots);
      const double c = rounds * (std::max(2.0 * bn, 224.0) + kb_fixed) * (1.0 + 0.03 * (nt - 1)) *
                       (cg == 1 ? 1.02 : 1.0);
      if (c < best_c) {
        best_c = c;
        bn_out = bn;
        cg_out = cg;
      }
    }
  }
}

// Shape-only split count of the wgrad reduction over N*H_o*W_o: minimises a fixed cost model
// (constants, never the queried device or S), so the fp32 summation order is a function of the
// shape alone (convergence invariance, P264).
// leaves > 1 (leaf plans): kb_total is ONE leaf's k-blocks and the model assumes `leaves` such
// leaves share the device (a constant: the global batch's 8 leaves, never the rank's count, so the
// per-leaf split count is the same on every rank).
int choose_splits(int tiles_mn, int kb_total, int bn, int mpad, int npad, int elem, int cg,
                  int x3, int leaves = 1) {
  const double sm = 148.0 / cg;   // concurrent work units (CTA pairs for cg = 2)
  // seconds per k-block (3xTF32: three MMAs per k-step)
  const double kb_s = (elem == 2 ? 2.0 : 4.0) * (x3 ? 3.0 : 1.0) * std::max(bn, 96) / 1.8e9;
  const double bw = 6.0e12;
  int best = 1;
  double best_t = 1e30;
  const int maxs = std::max(1, std::min(kb_total, 512));
  for (int s = 1; s <= maxs; ++s) {
    const int kbps = (int)cdiv(kb_total, s);
    const int real = (int)cdiv(kb_total, kbps);
    if (real != s) continue;
    const double waves = std::ceil(tiles_mn * (double)s * leaves / sm);
    // + the fixed-order reduction: each output sums its s partials in dependent batches (~1.2 us
    // per batch when the reduction grid is too small to hide the latency): batches of 8 splits
    // in reduce_tc_dw, of 64 in the 8-phase reduce_tc_dw_wide that small filters (< 64 tiles of
    // 32 x 32, ~mpad * npad < 64 Ki) use -- there the wider split grid pays (LeNet conv1: 144
    // splits 18 us vs 72 splits 28 us, GEMM alone)
    const double mn = (double)mpad * npad;
    const double red = mn < 65536.0 ? std::ceil(s / 64.0) * 1.2e-6
                       : mn < 148.0 * 1024 ? std::ceil(s / 8.0) * 1.2e-6 : 0.0;
    const double t = waves * (kbps * kb_s + 2e-6) + (double)s * leaves * mpad * npad * 8.0 / bw + red;
    if (t < best_t * 0.999) {
      best_t = t;
      best = s;
    }
  }
  return best;
}

}  // namespace

// Tensor maps of a pass depend only on the workspace address (the packed operands live there):
// cached per (pass, workspace) so repeated calls skip the driver encode (host latency that
// left the GPU idle between small launches).  Copies of a plan start with an empty cache.
struct MapCache {
  struct Entry {
    const void *ws = nullptr;
    CUtensorMap a, b, a2, b2, a3, b3;   // a2, b2: lo planes (3xTF32) / bf16(hi) (mixed); a3, b3: bf16(v - hi)
  };
  Entry e[3][8];
  int next[3] = {0, 0, 0};
  // fused-dy halo plans: the dy tensor recorded by glp_stage_pack(GLP_PACK_DY*) per workspace
  // (the filter gradient reads it in fp32 itself; nothing is packed at that point)
  struct DyRec {
    const void *ws = nullptr;
    const float *dy = nullptr;
  };
  DyRec dyrec[16];
  int dy_next = 0;
  std::mutex mu;
  MapCache() = default;
  MapCache(const MapCache &) {}
  MapCache &operator=(const MapCache &) { return *this; }
};

struct glp_plan_s {
  glp_conv_desc_s d;
  MapCache maps;
  int device = 0, math = 0, elem = 4, sm_count = 148, s_override = 0;
  int simt = 0;   // GLP_MATH_FP32_SIMT: the CUDA-core direct convolution (accuracy anchor)
  int x3 = 0;     // GLP_MATH_FP32: 3xTF32 on tcgen05 (hi/lo operand planes)
  int Cp = 0, Cop = 0, taps = 0;
  // Geometry of the x operand as the forward and filter-gradient passes see it: the layer itself,
  // or its space-to-depth form (s2d = stride S > 1: stride 1, ceil(K/S) taps, S*S*C channels).
  int s2d = 0;
  int s2d_blocks = 1;   // resident pack_s2d blocks per SM (occupancy API): its persistent grid
  // backward-data of a space-to-depth layer as the stride-1 backward-data over x' (dx' in the
  // workspace at off_dxs, then unpack_s2d_dx): 9 taps of unit stride instead of the 121-tap
  // strided gather (CaffeNet conv1)
  int s2d_dg = 0;
  size_t off_dxs = 0, sz_dxs = 0;
  glp_conv_desc_s dxg;
  int Cpx = 0, tapsx = 0;
  PassPlan fwd, dgrad, wgrad;
  // convolution groups: d above is ONE group's convolution (C/G -> C_o/G); the tensors hold
  // x_img_c / y_img_c channels per image and every workspace region exists once per group
  int groups = 1, x_img_c = 0, y_img_c = 0;
  size_t ws_group = 0;
  // halo filter gradient (hwgrad.cuh) for space-to-depth layers: dy is then packed on the padded
  // dxg.H x dxg.W grid (zeros outside H_o x W_o) and the filter gradient stages x' once per
  // k-block for all taps
  int halo = 0;
  HwgradParams hw{};
  int hw_grid = 0, hw_smem = 0, hw_regs = 0;
  KAttr hw_attr, hd_attr, hf_attr;   // analyzer records of the halo kernels the plan uses
  glp_device_limits_t lim{};         // the device's per-SM limits (analyzer input)
  long long s_slot_rows = 0, s_rows_per_sample = 0;   // the analyzer's S inputs (forward kernel)
  // halo forward (hfwd.cuh) for the same space-to-depth layers: x' staged once per tile for all
  // taps, W' resident per CTA, outputs on the padded grid (invalid rows dropped)
  int halo_fdy = 0;     // fused-dy halo filter gradient (hwgrad_kernel<NCG>): no dy pack for it
  int red_wide = 0;     // dW reduction by reduce_tc_dw_wide (small filters, many splits)
  int mix = 0;          // GLP_MATH_FP32 by the mixed split (tf32 hi*hi + bf16 cross terms)
  int wgrad_b3d = 0;    // filter-gradient B tile by one 3-D TMA per plane (all atoms)
  int hdg = 0;         // halo backward-data (hdgrad.cuh) for unit-stride layers where it pays
  HdgradParams hd{};
  int hd_grid = 0, hd_smem = 0;
  int hfwd = 0;
  HfwdParams hf{};
  int hf_grid = 0, hf_smem = 0, hf_regs = 0;
  int S = 1;
  // SIMT path
  int simt_splits = 1, simt_chunk = 1;
  // workspace layout
  size_t off_xpk = 0, off_dypk = 0, off_wpk = 0, off_wtpk = 0, off_part = 0, off_dbpart = 0;
  size_t sz_xpk = 0, sz_dypk = 0, sz_wpk = 0, sz_wtpk = 0, sz_part = 0, sz_dbpart = 0;
  // 3xTF32: byte offset from each packed operand's hi plane to its lo plane (0: one plane)
  long long lo_xpk = 0, lo_dypk = 0, lo_wpk = 0, lo_wtpk = 0;
  int db_rows = 0;
  size_t ws_fwd = 0, ws_dgrad = 0, ws_wgrad = 0, ws_bwd = 0;
  double plan_us = 0;
  int allow_cg2 = 1;   // GLP_CTA_GROUP=1 in the environment forces single-CTA MMAs (A/B runs)
  int allow_ksub2 = 1; // GLP_KSUB=1 forces one k-block per pipeline stage (A/B runs)
  int ksub_max = 4;    // GLP_KSUB=k caps the k-blocks per stage
  int wgrad_cg2 = 1;   // GLP_WGRAD_CG2=0: no CTA pairs for the filter gradient (A/B runs)
  int pdl = 0;         // GLP_PDL=1: programmatic dependent launch (measured 3% slower in the graph)
  int bn_model = 1;    // GLP_BN_MODEL=0: always the default fwd/dgrad tile (A/B runs)
  int allow_halo = 1;  // GLP_HALO=0: im2col filter gradient for space-to-depth layers (A/B runs)
  int allow_hfwd = 1;  // GLP_HFWD=0: im2col forward for space-to-depth layers (A/B runs)
  int allow_fdy = 1;   // GLP_HALO_FDY=0: halo filter gradient on the packed dy (A/B runs)
  int fdy_ncg = 0;     // GLP_FDY_NCG=1|2|3: force the fused-dy builder variant (A/B runs)
  int allow_hdg = 1;   // GLP_HDGRAD=0: im2col backward-data everywhere (A/B runs); 2 = force where legal
  int wgrad_bn = 0;    // GLP_WGRAD_BN=n: filter-gradient N tile override (A/B runs; 0 = model)
  int tile_units = 6;  // fwd/dgrad tile model applies below this many units per slot
  // Dynamic smem budget of the persistent GEMMs.  Below the 227 KB maximum it leaves room on
  // every SM for one block of the HBM-bound pack kernels (16.5 KB), so a pack issued on another
  // stream (e.g. the next layer's dy pack during a filter-gradient GEMM) runs beside the GEMM
  // instead of after it.  GLP_SMEM_CAP (bytes) overrides (A/B runs).
  int smem_cap = 232448;
  // deterministic exchange: the local batch is `leaves` equal leaves of
  // the global batch; the filter gradient's splits never cross a leaf, so each leaf's partial is
  // the same bits on any rank, and the leaves are summed by a fixed binary tree
  int leaves = 1;
  int leaf_plan = 0;   // wgrad_leaves > 0: the per-leaf split model (also with one local leaf)
  size_t off_leaf = 0, sz_leaf = 0, leaf_stride = 0;   // workspace leaf partials (composed calls)
  int pack_block = 0;  // GLP_PACK_BLOCK=1: the block-tiled activation pack (A/B runs)
  int s2d_block = 0;   // GLP_S2D_BLOCK=1: the block-persistent space-to-depth pack (A/B runs)
  unsigned long long *dbg_clk = nullptr;   // GLP_DEBUG_CLK=1: per-CTA cycle counters (diagnostics)
  int dbg_skip = 0;    // GLP_DEBUG_SKIP (diagnostics: skip A/B loads or MMAs; wrong results)
};

namespace {

// The analyzer's view of a kernel (P167: "kernel analyzer"): attributes from the runtime, CTAs per
// SM from the closed form over every per-SM limit, cross-checked against the occupancy API.  TMEM:
// the runtime admits one tcgen05 (TMEM-allocating) CTA per SM whatever its column count (R16), so
// such a kernel is charged the whole per-SM TMEM.
glp_status_t analyze_kernel(const glp_plan_s &P, const void *fn, int threads, int dyn_smem,
                            int tmem_cols, KAttr &k) {
  cudaFuncAttributes fa;
  GLP_CUDA(cudaFuncGetAttributes(&fa, fn));
  k.threads = threads;
  k.regs = fa.numRegs;
  k.smem = dyn_smem + (int)fa.sharedSizeBytes;
  k.tmem = tmem_cols;
  glp_kernel_attr_t ka{threads, fa.numRegs, k.smem,
                       (tmem_cols > 0 && P.lim.tmem_cols_per_sm > 0) ? P.lim.tmem_cols_per_sm : tmem_cols};
  k.model = ctas_per_sm_closed_form(P.lim, ka);
  GLP_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&k.rt, fn, threads, dyn_smem));
  if (k.model < 1) return fail(GLP_ERR_INTERNAL, "kernel does not fit on an SM");
  return GLP_OK;
}

// Halo filter gradient (hwgrad.cuh) for space-to-depth layers whose x' rows are one 64-channel
// bf16 atom and whose tap pairs' accumulators fit TMEM.  Split count: shape-only (a fixed
// constant of 148 ranges, never the queried device), so the reduction order is fixed.
glp_status_t plan_halo(glp_plan_s &P) {
  P.halo = 0;
  P.halo_fdy = 0;
  const glp_conv_desc_s &x = P.dxg;
  if (!P.allow_halo || !P.s2d || P.elem != 2 || P.Cpx != 64 || P.tapsx < 2) return GLP_OK;
  const int Ks = x.Kh, T = P.tapsx;
  const int n_acc = (T + 1) / 2;
  const int bn = (int)rup(x.Co, 16), acc_cols = (int)rup(bn, 32);
  const int shift_max = (Ks - 1) * x.W + (Ks - 1);
  const int halo_rows = HW_BKP + shift_max;
  if (n_acc > 8 || bn > 256 || n_acc * acc_cols > 512 || halo_rows > 256) return GLP_OK;
  HwgradParams &h = P.hw;
  memset(&h, 0, sizeof(h));
  h.n_acc = n_acc;
  for (int j = 0; j < n_acc; ++j) {
    int a = 2 * j, b = 2 * j + 1;
    if (b >= T) {   // odd tap count: the last pair repeats tap T-2 (its rows are discarded)
      a = T - 2;
      b = T - 1;
      h.dup_a_mask |= 1 << j;
    }
    h.tap_a[j] = a;
    h.tap_b[j] = b;
    h.shift_a[j] = (a / Ks) * x.W + a % Ks;
    h.shift_b[j] = (b / Ks) * x.W + b % Ks;
  }
  h.bn = bn;
  h.acc_cols = acc_cols;
  int tc = 32;
  while (tc < n_acc * acc_cols) tc *= 2;
  h.tmem_cols = tc;
  h.halo_rows = halo_rows;
  h.a_bytes = (int)rup((long long)halo_rows * 128, 1024);
  h.b_bytes = (int)cdiv(bn, 64) * HW_BKP * 128;
  const int stage = h.a_bytes + h.b_bytes;
  h.stages = std::min(8, (P.smem_cap - 2048) / stage);
  if (h.stages < 2) return GLP_OK;
  const long long rows = (long long)x.N * x.H * x.W;
  h.kb_total = (int)cdiv(rows, HW_BKP);
  h.splits = (int)std::min<long long>(h.kb_total, 148);
  h.kb_per_split = (int)cdiv(h.kb_total, h.splits);
  h.splits = (int)cdiv(h.kb_total, h.kb_per_split);
  h.cpx = P.Cpx;
  h.co = x.Co;
  h.mpad = T * P.Cpx;
  h.ld = bn;
  // fused dy (single layers): the filter gradient builds its dy operand from the fp32 tensor
  const int fdy = (P.allow_fdy && P.d.nbr <= 1 && bn <= 128 && rows < (1LL << 31) - 256) ? 1 : 0;
  // builders: register-staged groups, 3 when a thread's channels fit 3 x 32 registers (C_o <= 96),
  // else 2.  GLP_FDY_NCG=1 selects one group with a cp.async landing zone (2 x 128 pixels x bn
  // fp32, which also holds the db staging afterwards; only 2 pipeline stages fit beside it):
  // measured 171 us against 128 us for CaffeNet conv1.  GLP_FDY_NCG=2|3 forces the group count.
  int ncg = 0;
  int red_bytes = 0;
  if (fdy) {
    const int land = 2 * bn * 128 * 4 + 16;
    if (P.fdy_ncg == 1 && (P.smem_cap - 2048 - land) / stage >= 2) {   // measured slower: opt-in
      ncg = 1;
      red_bytes = land;
    } else {
      ncg = P.fdy_ncg == 2 ? 2 : (P.fdy_ncg == 3 ? 3 : (bn <= 96 ? 3 : 2));
      red_bytes = 4 * ncg * 256 * 4 + 16;
    }
  }
  h.stages = std::min(8, (P.smem_cap - 2048 - red_bytes) / stage);
  if (h.stages < 2) return GLP_OK;
  h.ho = P.d.Ho;
  h.wo = P.d.Wo;
  h.rows = (int)rows;
  h.div_img = FastDiv((uint32_t)(x.H * x.W));
  h.div_w = FastDiv((uint32_t)x.W);
  P.hw_grid = h.splits;
  P.hw_smem = 1024 + h.stages * stage + 8 * (2 * h.stages + 2) + 16 + red_bytes;
  const void *fn = ncg == 3 ? reinterpret_cast<const void *>(hwgrad_kernel<3>)
                 : ncg == 2 ? reinterpret_cast<const void *>(hwgrad_kernel<2>)
                 : ncg == 1 ? reinterpret_cast<const void *>(hwgrad_kernel<1>)
                            : reinterpret_cast<const void *>(hwgrad_kernel<0>);
  GLP_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, 232448));
  glp_status_t s = analyze_kernel(P, fn, hw_threads(ncg), P.hw_smem, h.tmem_cols, P.hw_attr);
  if (s) return s;
  P.hw_regs = P.hw_attr.regs;
  // grid = the shape-only split count (148 ranges, never the queried device: the reduction order
  // is fixed); the analyzer's slots (#SM x CTAs/SM) bound how many run at once
  P.halo = 1;
  P.halo_fdy = ncg;
  return GLP_OK;
}

// Halo backward-data (hdgrad.cuh): unit stride, square kernel, bf16, tf32 or the mixed fp32 split
// (not 3xTF32; the mixed split with C_i <= 128: the epilogue's chunk sums in registers), the
// flipped-tap Wt of the im2col-TMA dgrad, 128-byte channel blocks of C_o (64 bf16 / 32 tf32), and a
// tile geometry (R output rows padded to a pitch of WQ >= W + K - 1 pixels, R*WQ = 128) that
// wastes at most 30 % of the rows.  Used when the im2col A traffic dominates: >= 9 taps and
// C_i <= 128 (each A byte feeds few columns).
const void *hdgrad_fn(int elem, int mix) {
  return elem == 2 ? reinterpret_cast<const void *>(hdgrad_kernel<2, 0>)
         : mix     ? reinterpret_cast<const void *>(hdgrad_kernel<4, 1>)
                   : reinterpret_cast<const void *>(hdgrad_kernel<4, 0>);
}
glp_status_t plan_hdgrad(glp_plan_s &P) {
  P.hdg = 0;
  const glp_conv_desc_s &d = P.d;
  const int cb = 128 / P.elem;   // channels per 128-byte block
  if (!P.allow_hdg || (P.x3 && !P.mix) || P.simt || d.nbr > 1 || d.Sh != 1 || d.Sw != 1 || d.Kh != d.Kw ||
      d.Ph != d.Pw || d.Ph > d.Kh - 1 || !P.dgrad.a_tma || P.dgrad.krow != 128 || P.Cop % cb != 0)
    return GLP_OK;
  const int K = d.Kh, taps = K * K;
  int WQ = 8;
  while (WQ < d.W + K - 1) WQ *= 2;
  if (WQ > 128) return GLP_OK;
  const int R = 128 / WQ;
  const int tiles_img = (int)cdiv(d.H, R);
  const double junk = (double)tiles_img * R * WQ / ((double)d.H * d.W);
  const int bn = (int)rup(d.C, 16);
  if (P.allow_hdg != 2 && (junk > 1.3 || taps < 9 || bn > 128)) return GLP_OK;
  if (bn > 256 || (bn / 2) % 16 != 0) return GLP_OK;   // CTA pairs: half of B per CTA, N % 32
  if (P.mix && bn > 128) return GLP_OK;   // chunk sums: <= 128 fp32 registers per epilogue thread
  // mixed split: opt-in only (halo_dgrad = 2).  Measured on CaffeNet conv2 (b256): 740 us against
  // the im2col kernel's 723 us -- the 27-of-32 useful columns of a WQ = 32 row and the ragged last
  // wave (13 rounds for 12.1 units per pair) cost more than the halo saves on the L2
  if (P.mix && P.allow_hdg != 2) return GLP_OK;
  HdgradParams &h = P.hd;
  memset(&h, 0, sizeof(h));
  h.K = K;
  h.Q = K - 1 - d.Ph;
  h.WQ = WQ;
  h.R = R;
  h.H = d.H;
  h.W = d.W;
  h.Ho = d.Ho;
  h.Wo = d.Wo;
  h.N = d.N;
  h.tiles_img = tiles_img;
  h.units = (int)cdiv((long long)d.N * tiles_img, 2);
  h.ncb = P.Cop / cb;
  h.cop = P.Cop;
  h.bn = bn;
  h.ci = d.C;
  h.acc_cols = (int)rup(bn, 32);
  int tc = 32;
  while (tc < 2 * h.acc_cols) tc *= 2;
  h.tmem_cols = tc;
  h.a_hi_bytes = (int)rup((long long)(R + K - 1) * WQ * 128, 1024);
  h.b_hi_bytes = (int)rup((long long)(bn / 2) * 128, 1024);
  if (P.mix) {   // + the two bf16 planes (64-byte rows)
    h.a_bf_bytes = (int)rup((long long)(R + K - 1) * WQ * 64, 1024);
    h.b_bf_bytes = (int)rup((long long)(bn / 2) * 64, 1024);
    h.chunk_kb = P.dgrad.chunk_kb;   // the igemm passes' shape-only chunk (K = 32 per k-block)
    if (h.chunk_kb <= 0) return GLP_OK;
  }
  h.a_bytes = h.a_hi_bytes + 2 * h.a_bf_bytes;
  h.b_tap_bytes = h.b_hi_bytes + 2 * h.b_bf_bytes;
  h.a_stages = P.mix ? 2 : 3;   // a mixed halo stage is twice the bytes (and 25 taps of MMAs)
#ifdef GLP_DIAG
  if (const char *e = getenv("GLP_HD_ASTAGES")) h.a_stages = std::max(2, atoi(e));   // A/B runs
#endif
  const int fixed = 1024 + h.a_stages * h.a_bytes + 8 * 64 + 16;
  // as many taps per B stage as keep >= 4 stages (the issuer's barrier round trip costs more than
  // the 8 MMAs of one tap)
  int min_bst = 4;
#ifdef GLP_DIAG
  if (const char *e = getenv("GLP_HD_BSTAGES")) min_bst = std::max(2, atoi(e));   // A/B runs
#endif
  h.b_taps = 1;
  while (h.b_taps < taps && (P.smem_cap - fixed) / ((h.b_taps + 1) * h.b_tap_bytes) >= min_bst) ++h.b_taps;
  h.b_bytes = h.b_taps * h.b_tap_bytes;
  h.b_stages = std::min(8, (P.smem_cap - fixed) / h.b_bytes);
  if (h.b_stages < 3) return GLP_OK;
  P.hd_smem = 1024 + h.a_stages * h.a_bytes + h.b_stages * h.b_bytes +
              8 * (2 * h.a_stages + 2 * h.b_stages + 4) + 16;
  GLP_CUDA(cudaFuncSetAttribute(hdgrad_fn(P.elem, P.mix), cudaFuncAttributeMaxDynamicSharedMemorySize,
                                232448));
  glp_status_t s = analyze_kernel(P, hdgrad_fn(P.elem, P.mix), HD_THREADS, P.hd_smem, h.tmem_cols,
                                  P.hd_attr);
  if (s) return s;
  // persistent grid: the analyzer's resident CTA-pair slots (#SM x CTAs/SM / 2), at most the units
  long long pairs = std::min<long long>(h.units, (long long)P.sm_count * P.hd_attr.model / 2);
  if (P.s_override > 0)
    pairs = std::max(1LL, std::min(pairs, cdiv((long long)P.s_override * tiles_img, 2)));
  P.hd_grid = (int)(2 * pairs);
  P.hdg = 1;
  return GLP_OK;
}

// Halo forward (hfwd.cuh) for space-to-depth layers whose x' rows are one 64-channel bf16 atom,
// whose taps x C_o weight block fits shared memory next to >= 2 halo stages, and that are not a
// fused sibling group.  Tiles of 128 rows over the flattened padded grid; no K split, so the
// output never depends on the grid (convergence invariance, P264).
glp_status_t plan_hfwd(glp_plan_s &P) {
  P.hfwd = 0;
  const glp_conv_desc_s &x = P.dxg;
  if (!P.allow_hfwd || !P.s2d || P.elem != 2 || P.Cpx != 64 || P.d.nbr > 1) return GLP_OK;
  const int Ks = x.Kh, T = P.tapsx;
  if (T > HF_MAXTAPS || P.fwd.Kpad < T * 64) return GLP_OK;
  const int bn = (int)rup(x.Co, 16);
  const int shift_max = (Ks - 1) * x.W + (Ks - 1);
  const int halo_rows = 128 + shift_max;
  if (bn > 256 || (bn / 2) % 8 != 0 || halo_rows > 256) return GLP_OK;   // pairs: bn/2 per CTA
  HfwdParams &h = P.hf;
  memset(&h, 0, sizeof(h));
  h.taps = T;
  for (int t = 0; t < T; ++t) h.shift[t] = (t / Ks) * x.W + t % Ks;
  h.bn = bn;
  h.co = x.Co;
  h.acc_cols = (int)rup(bn, 32);
  int tc = 32;
  while (tc < 2 * h.acc_cols) tc *= 2;
  h.tmem_cols = tc;
  h.halo_rows = halo_rows;
  h.a_bytes = (int)rup((long long)halo_rows * 128, 1024);
  h.b_tap_bytes = (int)rup((long long)(bn / 2) * 128, 1024);
  h.bias_floats = (int)rup(bn, 4);
  const int fixed = 1024 + T * h.b_tap_bytes + 16 + 16 + 4 * h.bias_floats + 8 * 8;
  h.stages = std::min(6, (P.smem_cap - fixed - 8 * 2 * 6) / h.a_bytes);
  if (h.stages < 2) return GLP_OK;
  const long long rows = (long long)x.N * x.H * x.W;
  if (rows >= (1LL << 31) - 256) return GLP_OK;
  h.rows = (int)rows;
  h.tiles = (int)cdiv(rows, 128);
  h.units = (int)cdiv(h.tiles, 2);
  h.div_img = FastDiv((uint32_t)(x.H * x.W));
  h.div_w = FastDiv((uint32_t)x.W);
  h.ho = P.d.Ho;
  h.wo = P.d.Wo;
  P.hf_smem = fixed + 8 * (2 * h.stages + 6) + h.stages * h.a_bytes;
  GLP_CUDA(cudaFuncSetAttribute(reinterpret_cast<const void *>(hfwd_kernel),
                                cudaFuncAttributeMaxDynamicSharedMemorySize, 232448));
  glp_status_t s = analyze_kernel(P, reinterpret_cast<const void *>(hfwd_kernel), HF_THREADS,
                                  P.hf_smem, h.tmem_cols, P.hf_attr);
  if (s) return s;
  P.hf_regs = P.hf_attr.regs;
  // persistent grid: the analyzer's resident CTA-pair slots, at most the units
  long long pairs = std::min<long long>(h.units, (long long)P.sm_count * P.hf_attr.model / 2);
  if (P.s_override > 0)   // test override: only the tiles of S samples in flight at once
    pairs = std::max(1LL, std::min(pairs, cdiv((long long)P.s_override * x.H * x.W, 256)));
  P.hf_grid = (int)(2 * pairs);
  P.hfwd = 1;
  return GLP_OK;
}

glp_status_t plan_pass(glp_plan_s &P, PassPlan &pp, int mode, const glp_device_limits_t &L) {
  const int elem = P.elem;
  // backward-data: the layer's own geometry, or (s2d_dg) the stride-1 space-to-depth one
  const glp_conv_desc_s &d = (mode == MODE_DGRAD && !P.s2d_dg) ? P.d : P.dxg;
  const int Cpx = P.Cpx, tapsx = P.tapsx;
  const int taps_dg = P.s2d_dg ? P.tapsx : P.taps;
  // A by im2col TMA when the channel pitch is a multiple of a 64-byte row; K-block rows of 128
  // bytes when the pitch allows, else 64 (bf16).  Otherwise the cp.async gather (128-byte rows).
  const int u64 = 64 / elem, u128 = 128 / elem;
  if (mode == MODE_FWD) {
    pp.a_tma = (Cpx % u64 == 0 && (elem == 2 || Cpx % u128 == 0)) ? 1 : 0;
    pp.krow = (!pp.a_tma || Cpx % u128 == 0) ? 128 : 64;
  } else if (mode == MODE_DGRAD) {
    pp.a_tma = (P.Cop % u64 == 0 && (elem == 2 || P.Cop % u128 == 0) && d.Sh == 1 && d.Sw == 1) ? 1 : 0;
    pp.krow = (!pp.a_tma || P.Cop % u128 == 0) ? 128 : 64;
  } else {
    pp.a_tma = (Cpx % u64 == 0 && P.Cop % u64 == 0 &&
                (elem == 2 || (Cpx % u128 == 0 && P.Cop % u128 == 0))) ? 1 : 0;
    pp.krow = (!pp.a_tma || (Cpx % u128 == 0 && P.Cop % u128 == 0)) ? 128 : 64;
    // CTA pairs split the MN-major B tile into halves of whole swizzle atoms: when the 128-byte
    // atom (64 bf16) does not divide bn/2 but the 64-byte one does (C_o = 384 -> bn 192), use
    // 64-byte rows so the pair still forms
    const int bnw = P.wgrad_bn > 0 ? P.wgrad_bn : choose_bn(d.Co);
    if (pp.a_tma && elem == 2 && P.wgrad_cg2 && pp.krow == 128 && (bnw / 2) % 64 != 0 &&
        (bnw / 2) % 32 == 0 && (long long)tapsx * Cpx > 128)
      pp.krow = 64;
  }
  const int BK = pp.krow / elem;     // K elements per k-block (fwd/dgrad)
  const int BKP = 128 / elem;        // pixels per k-block (wgrad)
  const int EPA = pp.krow / elem;    // MN elements per MN-major atom (wgrad)
  if (mode == MODE_FWD) {
    pp.M = d.N * d.Ho * d.Wo;
    pp.Ng = d.Co;
    pp.Kpad = (int)rup((long long)tapsx * Cpx, BK);
    pp.kb_total = pp.Kpad / BK;
    pp.bn = choose_bn(d.Co);
    pp.bn_smem = pp.bn;
  } else if (mode == MODE_DGRAD) {
    pp.M = d.N * d.H * d.W;
    pp.Ng = d.C;
    pp.Kpad = (int)rup((long long)taps_dg * P.Cop, BK);
    pp.kb_total = pp.Kpad / BK;
    pp.bn = choose_bn(d.C);
    pp.bn_smem = pp.bn;
  } else {
    pp.M = tapsx * Cpx;
    pp.Ng = d.Co;
    pp.Kpad = d.N * d.Ho * d.Wo;
    pp.kb_total = (int)cdiv(pp.Kpad, BKP);
    pp.bn = P.wgrad_bn > 0 ? P.wgrad_bn : choose_bn(d.Co);
    pp.bn_smem = (int)rup(pp.bn, EPA);
  }
  pp.m_tiles = (int)cdiv(pp.M, 128);
  // CTA pairs (tcgen05 cta_group::2, M = 256): each SM loads half of B.  Needs the TMA A path,
  // at least two row tiles, and (MN-major B of the filter gradient) half tiles that are whole
  // swizzle atoms.
  pp.cg = 1;
  const bool wg_cg2 = P.wgrad_cg2 && (pp.bn / 2) % EPA == 0;   // MN-major B halves: whole atoms
  if (pp.a_tma && pp.m_tiles >= 2 && P.allow_cg2 && (mode != MODE_WGRAD || wg_cg2)) pp.cg = 2;
  if (mode != MODE_WGRAD && P.bn_model) {
    choose_tile_mn(pp.Ng, pp.M, pp.cg == 2, P.sm_count, pp.bn, pp.cg, P.tile_units,
                   P.mix ? 80.0 : 0.0);
    pp.bn_smem = pp.bn;
  }
  if (pp.cg == 2) pp.bn_smem = pp.bn / 2;
  pp.n_tiles = (int)cdiv(pp.Ng, pp.bn);
  pp.m_units = (int)cdiv(pp.m_tiles, pp.cg);
  if (mode == MODE_WGRAD && P.leaf_plan) {
    // leaf plan: the split count of ONE leaf (its shape only: the same for every rank count)
    const long long pleaf = (long long)(d.N / P.leaves) * d.Ho * d.Wo;
    if (d.N % P.leaves || pleaf % BKP)
      return fail(GLP_ERR_NOT_SUPPORTED, "wgrad leaves: the batch must split into leaves whose "
                                         "pixel count is a multiple of the k-block");
    pp.kb_per_leaf = (int)(pleaf / BKP);
    pp.splits_per_leaf = choose_splits(pp.m_units * pp.n_tiles, pp.kb_per_leaf, pp.bn,
                                       pp.m_units * pp.cg * 128, pp.n_tiles * pp.bn, elem, pp.cg,
                                       P.x3, /*leaves of the global batch*/ 8);
    pp.kb_per_split = (int)cdiv(pp.kb_per_leaf, pp.splits_per_leaf);
    pp.splits_per_leaf = (int)cdiv(pp.kb_per_leaf, pp.kb_per_split);
    pp.splits = P.leaves * pp.splits_per_leaf;
  } else if (mode == MODE_WGRAD) {
    pp.splits = choose_splits(pp.m_units * pp.n_tiles, pp.kb_total, pp.bn,
                              pp.m_units * pp.cg * 128, pp.n_tiles * pp.bn, elem, pp.cg, P.x3);
#ifdef GLP_DIAG
    if (const char *e = getenv("GLP_DEBUG_SPLITS"))   // diagnostics: forced split count
      pp.splits = std::max(1, std::min((int)pp.kb_total, atoi(e)));
#endif
    pp.kb_per_split = (int)cdiv(pp.kb_total, pp.splits);
    pp.splits = (int)cdiv(pp.kb_total, pp.kb_per_split);
  } else {
    pp.splits = 1;
    pp.kb_per_split = pp.kb_total;
  }
  const int planes = P.x3 ? 2 : 1;   // 3xTF32: hi and lo plane of every operand in the stage
  // 3xTF32 accumulation chunk (shape-only constant: 16 k-blocks = K 512): bounds the error of the
  // tensor core's round-toward-zero accumulation to ~1e-6 normwise
  pp.chunk_kb = P.x3 ? 16 : 0;
#ifdef GLP_DIAG
  if (const char *e = getenv("GLP_DEBUG_CHUNK"))   // diagnostics: chunk length A/B
    if (P.x3) pp.chunk_kb = std::max(1, atoi(e));
#endif
  const int a_bytes = planes * (mode == MODE_WGRAD ? 128 * BKP * elem : 128 * pp.krow);
  const int b_row = planes * (mode == MODE_WGRAD ? BKP * elem : pp.krow);
  // forward: the bias vector is staged once per CTA in smem (every column a tile can touch)
  pp.bias_floats = (mode == MODE_FWD) ? (int)rup((long long)pp.n_tiles * pp.bn, 32) + 32 : 0;
  // ring budget: the cap minus the 1 KB alignment slack, the 4 extra barriers + TMEM slot + bias
  // alignment (64 bytes) and the bias stage; each stage also takes its two 8-byte barriers (the
  // exact layout of pp.smem below: a 1 KB reserve for the barriers cost the N = 192 mixed forward
  // tiles their fourth stage by 512 bytes)
  const int budget = P.smem_cap - 1024 - 64 - 4 * pp.bias_floats;
  // k-blocks per pipeline stage: as many (<= 4) as keep >= 3 stages in the ring.  One
  // full/empty round trip of the single MMA-issuing warp costs ~250-700 cycles whatever the stage
  // size (tools/sync_probe*.cu, GLP_DEBUG_SKIP=15 runs), more than the tensor work of one small-N
  // k-block, so a stage must carry several k-blocks (TMA path only; cp.async fills one).
  pp.ksub = 1;
  const int kb_bytes = a_bytes + pp.bn_smem * b_row;
  if (pp.a_tma && P.allow_ksub2)
    while (pp.ksub < P.ksub_max && budget / ((pp.ksub + 1) * kb_bytes) >= 3 &&
           pp.kb_per_split >= 2 * (pp.ksub + 1))
      ++pp.ksub;
  const int stage_bytes = pp.ksub * kb_bytes;
  pp.stages = std::min(8, budget / (stage_bytes + 16));
#ifdef GLP_DIAG
  if (const char *e = getenv("GLP_DEBUG_STAGES"))   // diagnostics: fewer ring stages
    pp.stages = std::max(2, std::min(pp.stages, atoi(e)));
#endif
  if (pp.stages < 2) return fail(GLP_ERR_INTERNAL, "tile does not fit in smem");
  pp.acc_cols = (int)rup(pp.bn, 32);
  int tc = 32;
  while (tc < 2 * pp.acc_cols) tc *= 2;
  pp.tmem_cols = tc;
  // ring + barriers + TMEM slot + the epilogue's bias stage (16-byte aligned)
  pp.smem = 1024 + pp.stages * stage_bytes + 8 * (2 * pp.stages + 4) + 16 + 16 + 4 * pp.bias_floats;
  pp.tiles = pp.m_units * pp.n_tiles * pp.splits;   // work units (tile pairs for cg = 2)

  void *fn = igemm_ptr(mode, elem, pp.krow, pp.cg, P.mix ? 2 : P.x3);
  // The attribute is per function (not per plan): always allow the largest tile of any plan.
  GLP_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, 232448));
  cudaFuncAttributes fa;
  GLP_CUDA(cudaFuncGetAttributes(&fa, fn));
  pp.regs = fa.numRegs;
  // TMEM term: the CUDA runtime admits one TMEM-allocating (tcgen05) CTA per SM regardless of
  // the columns it asks for (measured with tools/occ_probe2.cu; R16), so the record
  // charges the whole per-SM TMEM to each CTA.
  pp.threads = igemm_threads(P.x3);
  glp_kernel_attr_t ka{pp.threads, fa.numRegs, pp.smem + (int)fa.sharedSizeBytes,
                       L.tmem_cols_per_sm > 0 ? L.tmem_cols_per_sm : pp.tmem_cols};
  pp.ctas_per_sm = ctas_per_sm_closed_form(L, ka);
  int rt = 0;
  GLP_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&rt, fn, pp.threads, pp.smem));
  pp.ctas_runtime = rt;
  if (pp.ctas_per_sm < 1) return fail(GLP_ERR_INTERNAL, "kernel does not fit on an SM");
  const int slots = P.sm_count * pp.ctas_per_sm / pp.cg;   // resident work-unit slots
  int grid = std::min(pp.tiles, slots);
  if (P.s_override > 0 && mode != MODE_WGRAD) {
    // S samples in flight: the grid covers the tiles of S samples (P262 batch-level parallelism).
    const int hw = (mode == MODE_FWD) ? d.Ho * d.Wo : d.H * d.W;
    const long long tiles_s = cdiv(cdiv((long long)P.s_override * hw, 128), pp.cg) * pp.n_tiles;
    grid = (int)std::max(1LL, std::min<long long>(grid, tiles_s));
  } else if (P.s_override > 0) {
    const long long tiles_s = cdiv((long long)pp.tiles * P.s_override, d.N);
    grid = (int)std::max(1LL, std::min<long long>(grid, tiles_s));
  }
  pp.grid = std::max(1, grid) * pp.cg;   // CTAs (pairs are clusters of 2)
  return GLP_OK;
}

// The tensor maps of one pass: A (activation gather), B (dense operand) and, for 3xTF32 plans,
// the same two over the lo planes.
struct Maps {
  CUtensorMap a, b, a2, b2, a3, b3;
};

glp_status_t validate_ptrs(std::initializer_list<const void *> ps) {
  for (const void *p : ps) {
    if (!p) return fail(GLP_ERR_INVALID_VALUE, "null pointer argument");
    if (reinterpret_cast<uintptr_t>(p) % 16) return fail(GLP_ERR_INVALID_VALUE, "pointer not 16-byte aligned");
  }
  return GLP_OK;
}

IgemmParams make_params(const glp_plan_s &P, const PassPlan &pp, int mode, const void *src) {
  const glp_conv_desc_s &d = (mode == MODE_DGRAD && !P.s2d_dg) ? P.d : P.dxg;
  IgemmParams p;
  memset(&p, 0, sizeof(p));
  Gather &g = p.g;
  g.src = src;
  g.stride = d.Sh;
  g.stride_w = d.Sw;
  g.pad = d.Ph;
  g.pad_w = d.Pw;
  g.kw = d.Kw;
  g.taps = (mode == MODE_DGRAD && !P.s2d_dg) ? P.taps : P.tapsx;
  if (mode == MODE_DGRAD) {
    // halo plans pack dy on the padded dxg grid (zeros outside H_o x W_o): same values
    g.src_h = P.halo ? P.dxg.H : d.Ho;
    g.src_w = P.halo ? P.dxg.W : d.Wo;
    g.src_cp = P.Cop;
    g.cp = P.Cop;
    g.pix_hw = d.H * d.W;
    g.pix_w = d.W;
  } else {
    g.src_h = d.H;
    g.src_w = d.W;
    g.src_cp = P.Cpx;
    g.cp = P.Cpx;
    g.pix_hw = d.Ho * d.Wo;
    g.pix_w = d.Wo;
  }
  g.n_pixels = d.N * g.pix_hw;
  if (mode == MODE_DGRAD) {   // im2col over dy with flipped taps (stride 1 only)
    g.im_sh = 1;
    g.im_sw = 1;
    g.im_ph = d.Kh - 1 - d.Ph;
    g.im_pw = d.Kw - 1 - d.Pw;
  } else {
    g.im_sh = d.Sh;
    g.im_sw = d.Sw;
    g.im_ph = d.Ph;
    g.im_pw = d.Pw;
  }
  g.cbs = g.cp / (pp.krow / P.elem);
  p.a_tma = pp.a_tma;
  p.lo_off_a = (mode == MODE_DGRAD) ? P.lo_dypk : P.lo_xpk;
  p.chunk_kb = pp.chunk_kb;
#ifdef GLP_DIAG
  p.dbg_skip = P.dbg_skip;
  p.dbg_clk = P.dbg_clk;
#endif
  g.div_hw = FastDiv((uint32_t)g.pix_hw);
  g.div_w = FastDiv((uint32_t)g.pix_w);
  g.div_cp = FastDiv((uint32_t)g.cp);
  g.div_kw = FastDiv((uint32_t)g.kw);
  p.M = pp.M;
  p.N = pp.Ng;
  p.m_tiles = pp.m_units;   // the kernel iterates work units along M
  p.n_tiles = pp.n_tiles;
  p.splits = pp.splits;
  p.kb_total = pp.kb_total;
  p.kb_per_split = pp.kb_per_split;
  p.kb_per_leaf = pp.kb_per_leaf;
  p.splits_per_leaf = pp.splits_per_leaf;
  p.bn = pp.bn;
  p.bn_smem = pp.bn_smem;
  p.stages = pp.stages;
  p.ksub = pp.ksub;
  p.b3d = (mode == MODE_WGRAD && P.wgrad_b3d) ? 1 : 0;
  p.tmem_cols = pp.tmem_cols;
  p.acc_cols = pp.acc_cols;
  p.part_ld = pp.n_tiles * pp.bn;
  p.part_mpad = pp.m_units * pp.cg * 128;
  return p;
}

template <int MODE>
glp_status_t launch_igemm(const glp_plan_s &P, const PassPlan &pp, const IgemmParams &p,
                          const Maps &m, cudaStream_t st) {
  void *fn = igemm_ptr(MODE, P.elem, pp.krow, pp.cg, P.mix ? 2 : P.x3);
  cudaLaunchConfig_t cfg;
  memset(&cfg, 0, sizeof(cfg));
  cfg.gridDim = dim3((unsigned)pp.grid);
  cfg.blockDim = dim3((unsigned)pp.threads);
  cfg.dynamicSmemBytes = (size_t)pp.smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = (unsigned)pp.cg;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = P.pdl ? 2 : 1;
  // plans with fewer planes pass their hi maps again in the unused slots (never read)
  const CUtensorMap &b2 = P.x3 ? m.b2 : m.b, &a2 = P.x3 ? m.a2 : m.a;
  const CUtensorMap &b3 = P.mix ? m.b3 : m.b, &a3 = P.mix ? m.a3 : m.a;
  void *args[] = {const_cast<IgemmParams *>(&p), const_cast<CUtensorMap *>(&m.b),
                  const_cast<CUtensorMap *>(&m.a), const_cast<CUtensorMap *>(&b2),
                  const_cast<CUtensorMap *>(&a2), const_cast<CUtensorMap *>(&b3),
                  const_cast<CUtensorMap *>(&a3)};
  GLP_CUDA(cudaLaunchKernelExC(&cfg, fn, args));
  GLP_LAUNCH_CHECK("igemm_kernel");
  return GLP_OK;
}

// db reduction scratch: [rows x Co partials | DB_GROUPS x Co group sums | ceil(Co/32) tickets]
// Launch with programmatic stream serialization (PDL) when the plan allows it: the kernel may
// begin while its predecessor drains; it calls pdl_wait() before touching global memory.
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(bool pdl, void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem,
                       cudaStream_t st, Args &&...args) {
  cudaLaunchConfig_t cfg;
  memset(&cfg, 0, sizeof(cfg));
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...);
}

struct DbAux {
  float *part, *part2;
  unsigned int *tickets;
};
// (leaves: one group-sum slice and one ticket slice per leaf of a leaf plan)
size_t db_aux_bytes(int rows, int Co, int leaves = 1) {
  return align1k((size_t)rows * Co * 4) + align1k((size_t)leaves * DB_GROUPS * Co * 4) +
         align1k((size_t)leaves * cdiv(Co, 32) * 4);
}
DbAux db_aux(const glp_plan_s &P, uint8_t *base, int rows) {
  DbAux a;
  a.part = reinterpret_cast<float *>(base);
  a.part2 = reinterpret_cast<float *>(base + align1k((size_t)rows * P.d.Co * 4));
  a.tickets = reinterpret_cast<unsigned int *>(base + align1k((size_t)rows * P.d.Co * 4) +
                                               align1k((size_t)P.leaves * DB_GROUPS * P.d.Co * 4));
  return a;
}

// lo: byte offset of dst's lo plane (3xTF32 plans: the region's lo_* offset; 0 otherwise)
// Operand planes of a plan (1; 3xTF32: hi, lo; mixed: hi, bf16(hi), bf16(v - hi)), the byte
// offset of plane pl from the hi plane (L = the hi plane's bytes), its element size and the TMA
// swizzle of its 128-row k-block tiles (the bf16 planes of the mixed split are 64-byte rows).
int nplanes(const glp_plan_s &P) { return P.mix ? 3 : (P.x3 ? 2 : 1); }
long long plane_offset(const glp_plan_s &P, int pl, long long L) {
  return pl == 0 ? 0 : (P.mix && pl == 2 ? L + L / 2 : L);
}
int plane_elem(const glp_plan_s &P, int pl) { return (P.mix && pl) ? 2 : P.elem; }
CUtensorMap *plane_map(CUtensorMap *m1, CUtensorMap *m2, CUtensorMap *m3, int pl) {
  return pl == 0 ? m1 : pl == 1 ? m2 : m3;
}
// The packs' plane argument (pack.cuh plane_off): 3xTF32, the lo plane's byte offset L (the hi
// plane's bytes); the mixed split, -((L/2) << 32 | (L - delta/2)) -- the bf16(hi) plane's byte
// offset from a destination pointer `delta` bytes into the hi plane, and the bf16 plane size.
long long plo(const glp_plan_s &P, long long L, long long delta = 0) {
  if (!P.mix) return L;
  return -(long long)(((unsigned long long)(L / 2) << 32) | (unsigned long long)(L - delta / 2));
}
glp_status_t launch_pack_act(const glp_plan_s &P, const float *src, void *dst, long long lo, int C,
                             int HW, int Cp, float *db_part, cudaStream_t st, int Ws = 1,
                             int Wd = 1, int HWd = -1, int co_off = 0, int Cw = -1, int db_ld = -1,
                             int img_c = -1) {
  if (HWd < 0) HWd = HW;   // default: dense destination (Ws == Wd)
  if (img_c < 0) img_c = C;   // default: the source holds exactly C channels per image
  if (Cw < 0) Cw = Cp;     // default: the whole row (single layer)
  if (db_ld < 0) db_ld = C;
  if (db_part == nullptr && Cp * P.elem <= 32 && Ws == Wd && co_off == 0 && Cw == Cp) {
    const size_t n = (size_t)P.d.N * HW;
    const int g = (int)std::min<size_t>(cdiv((long long)n, 256), 148 * 32);
    if (P.elem == 2) GLP_CUDA(launch_pdl(P.pdl, pack_nchw_to_nhwc_small<2>, dim3(g), dim3(256), 0, st, src, dst, P.d.N, C, HW, Cp, img_c, 0LL));
    else GLP_CUDA(launch_pdl(P.pdl, pack_nchw_to_nhwc_small<4>, dim3(g), dim3(256), 0, st, src, dst, P.d.N, C, HW, Cp, img_c, lo));
    GLP_LAUNCH_CHECK("pack_nchw_to_nhwc_small");
    return GLP_OK;
  }
  unsigned int *tickets = nullptr;
  if (db_part) tickets = db_aux(P, reinterpret_cast<uint8_t *>(db_part), P.db_rows).tickets;
  const int nt = (int)cdiv(P.d.Co, 32) * P.leaves;   // every leaf's tickets are armed
  if (!P.pack_block) {   // warp-tiled pack (default)
    dim3 gw((unsigned)cdiv(Cw, 32), (unsigned)cdiv((long long)P.d.N * HWd, 8 * PACKW_ROWS));
    if (P.elem == 2) GLP_CUDA(launch_pdl(P.pdl, pack_act_warp<2>, gw, dim3(256), 0, st, src, dst, P.d.N, C, HW, Cp, db_part, tickets, nt, Ws, Wd, HWd, co_off, Cw, db_ld, img_c, 0LL));
    else GLP_CUDA(launch_pdl(P.pdl, pack_act_warp<4>, gw, dim3(256), 0, st, src, dst, P.d.N, C, HW, Cp, db_part, tickets, nt, Ws, Wd, HWd, co_off, Cw, db_ld, img_c, lo));
    GLP_LAUNCH_CHECK("pack_act_warp");
    return GLP_OK;
  }
  dim3 grid((unsigned)cdiv(Cw, 32), (unsigned)cdiv((long long)P.d.N * HWd, PACK_PT));
  if (P.elem == 2) GLP_CUDA(launch_pdl(P.pdl, pack_nchw_to_nhwc<2>, dim3(grid), dim3(256), 0, st, src, dst, P.d.N, C, HW, Cp, db_part, tickets, nt, Ws, Wd, HWd, co_off, Cw, db_ld, img_c, 0LL));
  else GLP_CUDA(launch_pdl(P.pdl, pack_nchw_to_nhwc<4>, dim3(grid), dim3(256), 0, st, src, dst, P.d.N, C, HW, Cp, db_part, tickets, nt, Ws, Wd, HWd, co_off, Cw, db_ld, img_c, lo));
  GLP_LAUNCH_CHECK("pack_nchw_to_nhwc");
  return GLP_OK;
}

// dy -> its packed operand (dense NHWC, or on the padded dxg grid for halo plans) + db partials
// A fused sibling group (dy.n > 1) packs branch b into channels [off_b, off_b+1) of the rows
// (the last branch also zero-fills the pitch padding) with its db partials in columns off_b + c.
glp_status_t launch_pack_dy(const glp_plan_s &P, const BrIn &dy, uint8_t *ws, bool with_db,
                            cudaStream_t st) {
  const glp_conv_desc_s &d = P.d;
  // fused-dy plans: db partials come from the filter-gradient kernel (this pack only feeds dgrad)
  float *dbp = (with_db && !P.halo_fdy) ? reinterpret_cast<float *>(ws + P.off_dbpart) : nullptr;
  const int Ws = P.halo ? d.Wo : 1, Wd = P.halo ? P.dxg.W : 1;
  const int HWd = P.halo ? P.dxg.H * P.dxg.W : -1;
  if (dy.n <= 1)
    return launch_pack_act(P, dy.p[0], ws + P.off_dypk, plo(P, P.lo_dypk), d.Co, d.Ho * d.Wo, P.Cop, dbp, st, Ws, Wd,
                           HWd, 0, -1, -1, P.y_img_c);
  for (int b = 0; b < dy.n; ++b) {
    const int off = d.br_off[b], cb = d.br_off[b + 1] - off;
    const int cw = (b == dy.n - 1) ? P.Cop - off : cb;
    glp_status_t s = launch_pack_act(P, dy.p[b], ws + P.off_dypk, plo(P, P.lo_dypk), cb, d.Ho * d.Wo, P.Cop, dbp, st,
                                     Ws, Wd, HWd, off, cw, d.Co);
    if (s) return s;
  }
  return GLP_OK;
}

int ew_grid(size_t n) { return (int)std::min<size_t>(cdiv((long long)n, 256), 148 * 16); }

glp_status_t run_pack_w_fwd_one(glp_plan_s &P, const float *w, int co_off, int Co, uint8_t *ws,
                                cudaStream_t st) {
  const glp_conv_desc_s &d0 = P.d;
  glp_conv_desc_s d = d0;
  d.Co = Co;   // rows [co_off, co_off + Co) of the forward B operand
  void *wpk = ws + P.off_wpk + (size_t)co_off * P.fwd.Kpad * P.elem;
  const size_t wn = (size_t)d.Co * P.fwd.Kpad;
  const long long lo = plo(P, P.lo_wpk, (long long)co_off * P.fwd.Kpad * P.elem);
  if (P.s2d) {
    if (P.elem == 2)
      GLP_CUDA(launch_pdl(P.pdl, pack_w_fwd_s2d<2>, dim3(ew_grid(wn)), dim3(256), 0, st, w, wpk, d.Co, d.C, d.Kh, P.s2d, P.dxg.Kh, P.Cpx, P.fwd.Kpad, 0LL));
    else
      GLP_CUDA(launch_pdl(P.pdl, pack_w_fwd_s2d<4>, dim3(ew_grid(wn)), dim3(256), 0, st, w, wpk, d.Co, d.C, d.Kh, P.s2d, P.dxg.Kh, P.Cpx, P.fwd.Kpad, lo));
  } else if ((size_t)d.C * P.taps * 4 <= 48 * 1024) {
    const size_t sm = (size_t)d.C * P.taps * 4;
    if (P.elem == 2)
      GLP_CUDA(launch_pdl(P.pdl, pack_w_fwd_rows<2>, dim3((unsigned)d.Co), dim3(256), sm, st, w, wpk, d.C, P.taps, P.Cpx, P.fwd.Kpad, 0LL));
    else
      GLP_CUDA(launch_pdl(P.pdl, pack_w_fwd_rows<4>, dim3((unsigned)d.Co), dim3(256), sm, st, w, wpk, d.C, P.taps, P.Cpx, P.fwd.Kpad, lo));
  } else if (P.elem == 2) {
    GLP_CUDA(launch_pdl(P.pdl, pack_w_fwd<2>, dim3(dim3((unsigned)cdiv(P.fwd.Kpad, 256), (unsigned)d.Co)), dim3(256), 0, st, w, wpk, d.Co, d.C, P.taps, P.Cpx, P.fwd.Kpad, 0LL));
  } else {
    GLP_CUDA(launch_pdl(P.pdl, pack_w_fwd<4>, dim3(dim3((unsigned)cdiv(P.fwd.Kpad, 256), (unsigned)d.Co)), dim3(256), 0, st, w, wpk, d.Co, d.C, P.taps, P.Cpx, P.fwd.Kpad, lo));
  }
  GLP_LAUNCH_CHECK("pack_w_fwd");
  return GLP_OK;
}

glp_status_t run_pack_w_fwd(glp_plan_s &P, const BrIn &w, uint8_t *ws, cudaStream_t st) {
  const glp_conv_desc_s &d = P.d;
  if (w.n <= 1) return run_pack_w_fwd_one(P, w.p[0], 0, d.Co, ws, st);
  for (int b = 0; b < w.n; ++b) {
    glp_status_t s = run_pack_w_fwd_one(P, w.p[b], d.br_off[b], d.br_off[b + 1] - d.br_off[b], ws, st);
    if (s) return s;
  }
  return GLP_OK;
}

// x -> the packed operand of the forward / filter-gradient passes (direct NHWC or space-to-depth).
glp_status_t launch_pack_x(const glp_plan_s &P, const float *x, void *dst, cudaStream_t st) {
  const glp_conv_desc_s &d = P.d;
  if (P.s2d && P.s2d * P.s2d * d.C <= S2DW_MAXC && P.Cpx <= S2DW_MAXC && !P.s2d_block) {
    const long long px = (long long)d.N * P.dxg.H * P.dxg.W;
    const dim3 grid((unsigned)cdiv(px, 128));
    if (P.s2d == 4 && d.C == 3) {   // CaffeNet conv1: compile-time geometry
      if (P.elem == 2)
        GLP_CUDA(launch_pdl(P.pdl, pack_s2d_warp_t<2, 4, 3>, grid, dim3(128), 0, st, x, dst, d.N, d.H, d.W, d.Ph, P.dxg.H, P.dxg.W, P.Cpx, P.x_img_c, 0LL));
      else
        GLP_CUDA(launch_pdl(P.pdl, pack_s2d_warp_t<4, 4, 3>, grid, dim3(128), 0, st, x, dst, d.N, d.H, d.W, d.Ph, P.dxg.H, P.dxg.W, P.Cpx, P.x_img_c, plo(P, P.lo_xpk)));
      GLP_LAUNCH_CHECK("pack_s2d_warp_t");
      return GLP_OK;
    }
    if (P.elem == 2)
      GLP_CUDA(launch_pdl(P.pdl, pack_s2d_warp<2>, grid, dim3(128), 0, st, x, dst, d.N, d.C, d.H, d.W, P.s2d, d.Ph, P.dxg.H, P.dxg.W, P.Cpx, P.x_img_c, 0LL));
    else
      GLP_CUDA(launch_pdl(P.pdl, pack_s2d_warp<4>, grid, dim3(128), 0, st, x, dst, d.N, d.C, d.H, d.W, P.s2d, d.Ph, P.dxg.H, P.dxg.W, P.Cpx, P.x_img_c, plo(P, P.lo_xpk)));
    GLP_LAUNCH_CHECK("pack_s2d_warp");
    return GLP_OK;
  }
  if (P.s2d) {
    const int S = P.s2d;
    const size_t smem = (size_t)S * d.C * d.W * sizeof(float);
    const int cpr = P.Cpx * P.elem / 16;
    if (256 % cpr || (long long)S * d.C * d.W > 256LL * S2D_LD)
      return fail(GLP_ERR_NOT_SUPPORTED, "space-to-depth geometry too large for the pack kernel");
    const int rows = d.N * P.dxg.H;
    dim3 grid((unsigned)std::min(rows, P.sm_count * std::max(1, P.s2d_blocks)));
    if (P.elem == 2)
      GLP_CUDA(launch_pdl(P.pdl, pack_s2d<2>, dim3(grid), dim3(256), smem, st, x, dst, d.N, d.C, d.H, d.W, S, d.Ph, P.dxg.H, P.dxg.W, P.Cpx, P.x_img_c, 0LL));
    else
      GLP_CUDA(launch_pdl(P.pdl, pack_s2d<4>, dim3(grid), dim3(256), smem, st, x, dst, d.N, d.C, d.H, d.W, S, d.Ph, P.dxg.H, P.dxg.W, P.Cpx, P.x_img_c, plo(P, P.lo_xpk)));
    GLP_LAUNCH_CHECK("pack_s2d");
    return GLP_OK;
  }
  return launch_pack_act(P, x, dst, plo(P, P.lo_xpk), d.C, d.H * d.W, P.Cpx, nullptr, st, 1, 1, -1, 0, -1,
                         -1, P.x_img_c);
}

glp_status_t run_pack_w_dgrad(glp_plan_s &P, const BrIn &w, uint8_t *ws, cudaStream_t st) {
  const glp_conv_desc_s &d = P.d;
  void *wtpk = ws + P.off_wtpk;
  const int flip = P.dgrad.a_tma;  // the im2col-TMA dgrad walks taps flipped
  if (P.s2d_dg) {   // Wt' of the space-to-depth weights, rows = the S*S*C x' channels
    const dim3 g2((unsigned)cdiv(P.dgrad.Kpad, 256), (unsigned)P.dxg.C);
    if (P.elem == 2)
      GLP_CUDA(launch_pdl(P.pdl, pack_w_dgrad_s2d<2>, g2, dim3(256), 0, st, w.p[0], wtpk, d.Co, d.C, d.Kh, P.s2d, P.dxg.Kh, P.Cop, P.dgrad.Kpad, flip, 0LL));
    else
      GLP_CUDA(launch_pdl(P.pdl, pack_w_dgrad_s2d<4>, g2, dim3(256), 0, st, w.p[0], wtpk, d.Co, d.C, d.Kh, P.s2d, P.dxg.Kh, P.Cop, P.dgrad.Kpad, flip, plo(P, P.lo_wtpk)));
    GLP_LAUNCH_CHECK("pack_w_dgrad_s2d");
    return GLP_OK;
  }
  const dim3 grid((unsigned)cdiv(P.dgrad.Kpad, 256), (unsigned)d.C);
  const int n = std::max(1, w.n);
  for (int b = 0; b < n; ++b) {
    const int off = n > 1 ? d.br_off[b] : 0;
    const int co = n > 1 ? d.br_off[b + 1] - off : d.Co;
    const int hi = (b == n - 1) ? P.Cop : off + co;
    const size_t sm = (size_t)co * P.taps * 4;
    if (sm <= 48 * 1024) {
      if (P.elem == 2)
        GLP_CUDA(launch_pdl(P.pdl, pack_w_dgrad_rows<2>, dim3((unsigned)d.C), dim3(256), sm, st, w.p[b], wtpk, co, d.C, P.taps, P.Cop, P.dgrad.Kpad, flip, off, off, hi, 0LL));
      else
        GLP_CUDA(launch_pdl(P.pdl, pack_w_dgrad_rows<4>, dim3((unsigned)d.C), dim3(256), sm, st, w.p[b], wtpk, co, d.C, P.taps, P.Cop, P.dgrad.Kpad, flip, off, off, hi, plo(P, P.lo_wtpk)));
    } else if (P.elem == 2)
      GLP_CUDA(launch_pdl(P.pdl, pack_w_dgrad<2>, grid, dim3(256), 0, st, w.p[b], wtpk, co, d.C, P.taps, P.Cop, P.dgrad.Kpad, flip, off, off, hi, 0LL));
    else
      GLP_CUDA(launch_pdl(P.pdl, pack_w_dgrad<4>, grid, dim3(256), 0, st, w.p[b], wtpk, co, d.C, P.taps, P.Cop, P.dgrad.Kpad, flip, off, off, hi, plo(P, P.lo_wtpk)));
    GLP_LAUNCH_CHECK("pack_w_dgrad");
  }
  return GLP_OK;
}

// Both weight operands in one kernel (single layers without space-to-depth, taps <= 25); the
// separate packs otherwise.  Same operand bits either way.
glp_status_t run_pack_w_both(glp_plan_s &P, const BrIn &w, uint8_t *ws, cudaStream_t st) {
  const glp_conv_desc_s &d = P.d;
  if (P.s2d || w.n > 1 || P.taps > PWB_MAXT) {
    glp_status_t s = run_pack_w_fwd(P, w, ws, st);
    return s ? s : run_pack_w_dgrad(P, w, ws, st);
  }
  const size_t smem = (size_t)32 * (32 * P.taps + 1) * 4;
  // the attribute is per device: set on every call (a host-side driver call, no launch)
  void *fn = P.elem == 2 ? reinterpret_cast<void *>(pack_w_both<2>) : reinterpret_cast<void *>(pack_w_both<4>);
  GLP_CUDA(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, 32 * (32 * PWB_MAXT + 1) * 4));
  const dim3 grid((unsigned)cdiv(std::max(P.Cpx, d.C), 32), (unsigned)cdiv(P.Cop, 32), 2);
  void *wp = ws + P.off_wpk, *wt = ws + P.off_wtpk;
  const int flip = P.dgrad.a_tma;
  if (P.elem == 2)
    GLP_CUDA(launch_pdl(P.pdl, pack_w_both<2>, grid, dim3(256), smem, st, w.p[0], wp, wt, d.Co, d.C, P.taps, P.Cpx, P.Cop, P.fwd.Kpad, P.dgrad.Kpad, flip, 0LL, 0LL));
  else
    GLP_CUDA(launch_pdl(P.pdl, pack_w_both<4>, grid, dim3(256), smem, st, w.p[0], wp, wt, d.Co, d.C, P.taps, P.Cpx, P.Cop, P.fwd.Kpad, P.dgrad.Kpad, flip, plo(P, P.lo_wpk), plo(P, P.lo_wtpk)));
  GLP_LAUNCH_CHECK("pack_w_both");
  return GLP_OK;
}

// output table of a call: n = 1 -> every channel in p[0]; fused group -> the plan's branches
BrOut br_out(const glp_plan_s &P, int n, float *const *ptrs) {
  BrOut t;
  memset(&t, 0, sizeof(t));
  if (n <= 1) {
    t.n = 1;
    t.off[1] = P.d.Co;
    t.p[0] = ptrs[0];
    return t;
  }
  t.n = n;
  for (int b = 0; b <= n; ++b) t.off[b] = P.d.br_off[b];
  for (int b = 0; b < n; ++b) t.p[b] = ptrs[b];
  return t;
}

template <typename F>
glp_status_t cached_maps(glp_plan_s &P, int pass, const void *ws, Maps &m, F encode) {
  std::lock_guard<std::mutex> lk(P.maps.mu);
  for (auto &e : P.maps.e[pass])
    if (e.ws == ws) {
      m.a = e.a;
      m.b = e.b;
      m.a2 = e.a2;
      m.b2 = e.b2;
      m.a3 = e.a3;
      m.b3 = e.b3;
      return GLP_OK;
    }
  memset(&m, 0, sizeof(m));
  glp_status_t s = encode(m);
  if (s) return s;
  auto &e = P.maps.e[pass][P.maps.next[pass]];
  P.maps.next[pass] = (P.maps.next[pass] + 1) % 8;
  e.ws = ws;
  e.a = m.a;
  e.b = m.b;
  e.a2 = m.a2;
  e.b2 = m.b2;
  e.a3 = m.a3;
  e.b3 = m.b3;
  return GLP_OK;
}

void record_dy(glp_plan_s &P, const void *ws, const float *dy) {
  std::lock_guard<std::mutex> lk(P.maps.mu);
  for (auto &r : P.maps.dyrec)
    if (r.ws == ws) {
      r.dy = dy;
      return;
    }
  auto &r = P.maps.dyrec[P.maps.dy_next];
  P.maps.dy_next = (P.maps.dy_next + 1) % 16;
  r.ws = ws;
  r.dy = dy;
}
const float *recorded_dy(glp_plan_s &P, const void *ws) {
  std::lock_guard<std::mutex> lk(P.maps.mu);
  for (auto &r : P.maps.dyrec)
    if (r.ws == ws) return r.dy;
  return nullptr;
}

glp_status_t run_fwd_halo(glp_plan_s &P, const BrIn &b, const BrOut &y, uint8_t *ws,
                          cudaStream_t st) {
  const glp_conv_desc_s &d = P.dxg;
  const uint64_t rows = (uint64_t)d.N * d.H * d.W;   // flat padded grid of x'
  Maps m;
  glp_status_t s = cached_maps(P, 0, ws, m, [&](Maps &q) {
    glp_status_t r = encode_2d(&q.a, 2, ws + P.off_xpk, (uint64_t)P.Cpx, rows, (uint64_t)P.Cpx * 2,
                               64u, (uint32_t)P.hf.halo_rows, CU_TENSOR_MAP_SWIZZLE_128B);
    if (r) return r;
    return encode_2d(&q.b, 2, ws + P.off_wpk, (uint64_t)P.fwd.Kpad, (uint64_t)d.Co,
                     (uint64_t)P.fwd.Kpad * 2, 64u, (uint32_t)(P.hf.bn / 2), CU_TENSOR_MAP_SWIZZLE_128B);
  });
  if (s) return s;
  CUtensorMap &mapX = m.a, &mapW = m.b;
  HfwdParams p = P.hf;
  p.out = y.p[0];
  p.bias = b.p[0];
  p.out_c = P.y_img_c;
  p.out_hw = P.d.Ho * P.d.Wo;
  p.dbg_skip = P.dbg_skip;
  cudaLaunchConfig_t cfg;
  memset(&cfg, 0, sizeof(cfg));
  cfg.gridDim = dim3((unsigned)P.hf_grid);
  cfg.blockDim = dim3(HF_THREADS);
  cfg.dynamicSmemBytes = (size_t)P.hf_smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = 2;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = P.pdl ? 2 : 1;
  void *args[] = {&p, &mapX, &mapW};
  GLP_CUDA(cudaLaunchKernelExC(&cfg, reinterpret_cast<void *>(hfwd_kernel), args));
  GLP_LAUNCH_CHECK("hfwd_kernel");
  return GLP_OK;
}

glp_status_t run_fwd_gemm(glp_plan_s &P, const BrIn &b, const BrOut &y, uint8_t *ws,
                          cudaStream_t st) {
  if (P.hfwd) return run_fwd_halo(P, b, y, ws, st);
  const glp_conv_desc_s &d = P.dxg;
  const PassPlan &pp = P.fwd;
  void *xpk = ws + P.off_xpk, *wpk = ws + P.off_wpk;
  const int BK = pp.krow / P.elem;
  Maps m;
  glp_status_t s = cached_maps(P, 0, ws, m, [&](Maps &q) {
    for (int pl = 0; pl < nplanes(P); ++pl) {   // hi plane, then the lo / bf16 planes
      const long long lw = plane_offset(P, pl, P.lo_wpk), lx = plane_offset(P, pl, P.lo_xpk);
      const int e = plane_elem(P, pl);
      const CUtensorMapSwizzle sw = swz_kmajor(e * BK);   // 128- or 64-byte rows
      glp_status_t r = encode_2d(plane_map(&q.b, &q.b2, &q.b3, pl), e, static_cast<uint8_t *>(wpk) + lw,
                                 (uint64_t)pp.Kpad, (uint64_t)d.Co, (uint64_t)pp.Kpad * e,
                                 (uint32_t)BK, (uint32_t)pp.bn_smem, sw);
      if (r) return r;
      if (!pp.a_tma) continue;
      if ((r = get_encode_im2col())) return r;
      r = encode_im2col(plane_map(&q.a, &q.a2, &q.a3, pl), e, static_cast<uint8_t *>(xpk) + lx, P.Cpx, d.W,
                        d.H, d.N, -d.Pw, -d.Ph, d.Pw - (d.Kw - 1), d.Ph - (d.Kh - 1), BK, 128,
                        d.Sw, d.Sh, sw);
      if (r) return r;
    }
    return GLP_OK;
  });
  if (s) return s;
  IgemmParams p = make_params(P, pp, MODE_FWD, xpk);
  p.out = y.p[0];
  p.bias = b.p[0];
  p.ybr = y;
  for (int i = 0; i < GLP_MAXBR; ++i) p.bias_br[i] = b.p[i];
  p.bias_floats = pp.bias_floats;
  p.out_c = P.y_img_c;   // channels per image of y (the whole tensor for a conv group)
  p.out_hw = d.Ho * d.Wo;
  return launch_igemm<MODE_FWD>(P, pp, p, m, st);
}

glp_status_t encode_4d_nhwc(CUtensorMap *map, int elem, const void *ptr, int cpitch, int W, int H,
                            int N, uint32_t box_w, uint32_t box_h, uint32_t box_c = 0,
                            CUtensorMapSwizzle swz = CU_TENSOR_MAP_SWIZZLE_128B) {
  cuuint64_t dims[4] = {(cuuint64_t)cpitch, (cuuint64_t)W, (cuuint64_t)H, (cuuint64_t)N};
  cuuint64_t strides[3] = {(cuuint64_t)cpitch * elem, (cuuint64_t)W * cpitch * elem,
                           (cuuint64_t)H * W * cpitch * elem};
  // one 128-byte channel block (or box_c channels: the 64-byte bf16 rows of the mixed split)
  cuuint32_t box[4] = {box_c ? box_c : (cuuint32_t)(128 / elem), box_w, box_h, 1u};
  cuuint32_t es[4] = {1, 1, 1, 1};
  CUresult r = g_encode(map, elem == 2 ? CU_TENSOR_MAP_DATA_TYPE_BFLOAT16 : CU_TENSOR_MAP_DATA_TYPE_FLOAT32,
                        4, const_cast<void *>(ptr), dims,
                        strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, swz,
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return fail(GLP_ERR_CUDA, "cuTensorMapEncodeTiled (4d) failed (" + std::to_string((int)r) + ")");
  return GLP_OK;
}

glp_status_t run_dgrad_halo(glp_plan_s &P, float *dx, uint8_t *ws, cudaStream_t st) {
  const glp_conv_desc_s &d = P.d;
  Maps m;
  glp_status_t s = cached_maps(P, 1, ws, m, [&](Maps &q) {
    // one plane (bf16 / tf32), or the mixed split's tf32 hi plane and two bf16 planes (32
    // channels per 64-byte row, SWIZZLE_64B)
    const int CB = 128 / P.elem;
    for (int pl = 0; pl < (P.mix ? 3 : 1); ++pl) {
      const int e = plane_elem(P, pl);
      const CUtensorMapSwizzle sw = e * CB == 128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_64B;
      glp_status_t r = encode_4d_nhwc(plane_map(&q.a, &q.a2, &q.a3, pl), e,
                                      ws + P.off_dypk + plane_offset(P, pl, P.lo_dypk), P.Cop, d.Wo,
                                      d.Ho, d.N, (uint32_t)P.hd.WQ, (uint32_t)(P.hd.R + P.hd.K - 1),
                                      (uint32_t)CB, sw);
      if (r) return r;
      r = encode_2d(plane_map(&q.b, &q.b2, &q.b3, pl), e, ws + P.off_wtpk + plane_offset(P, pl, P.lo_wtpk),
                    (uint64_t)P.dgrad.Kpad, (uint64_t)d.C, (uint64_t)P.dgrad.Kpad * e, (uint32_t)CB,
                    (uint32_t)(P.hd.bn / 2), sw);
      if (r) return r;
    }
    return GLP_OK;
  });
  if (s) return s;
  CUtensorMap &mapDy = m.a, &mapW = m.b;
  HdgradParams p = P.hd;
  p.out = dx;
  p.out_c = P.x_img_c;
  p.dbg_skip = P.dbg_skip;
  cudaLaunchConfig_t cfg;
  memset(&cfg, 0, sizeof(cfg));
  cfg.gridDim = dim3((unsigned)P.hd_grid);
  cfg.blockDim = dim3(HD_THREADS);
  cfg.dynamicSmemBytes = (size_t)P.hd_smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = 2;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = P.pdl ? 2 : 1;
  void *args[] = {&p, &mapDy, &mapW, &m.a2, &m.b2, &m.a3, &m.b3};
  GLP_CUDA(cudaLaunchKernelExC(&cfg, hdgrad_fn(P.elem, P.mix), args));
  GLP_LAUNCH_CHECK("hdgrad_kernel");
  return GLP_OK;
}

glp_status_t run_dgrad_gemm(glp_plan_s &P, float *dx, uint8_t *ws, cudaStream_t st) {
  if (P.hdg) return run_dgrad_halo(P, dx, ws, st);
  // space-to-depth layers: the stride-1 backward-data of the x' convolution into dx' (workspace),
  // then dx' -> dx
  const glp_conv_desc_s &d = P.s2d_dg ? P.dxg : P.d;
  // halo plans pack dy on the padded x' grid: the dgrad's dy tensor is its top-left H_o x W_o
  const int dy_pw = P.halo ? P.dxg.W : 0, dy_ph = P.halo ? P.dxg.H : 0;
  const PassPlan &pp = P.dgrad;
  void *wtpk = ws + P.off_wtpk;
  const void *dypk = ws + P.off_dypk;
  const int BK = pp.krow / P.elem;
  Maps m;
  glp_status_t s = cached_maps(P, 1, ws, m, [&](Maps &q) {
    for (int pl = 0; pl < nplanes(P); ++pl) {   // hi plane, then the lo / bf16 planes
      const long long lw = plane_offset(P, pl, P.lo_wtpk), ld = plane_offset(P, pl, P.lo_dypk);
      const int e = plane_elem(P, pl);
      const CUtensorMapSwizzle sw = swz_kmajor(e * BK);   // 128- or 64-byte rows
      glp_status_t r = encode_2d(plane_map(&q.b, &q.b2, &q.b3, pl), e, static_cast<uint8_t *>(wtpk) + lw,
                                 (uint64_t)pp.Kpad, (uint64_t)d.C, (uint64_t)pp.Kpad * e,
                                 (uint32_t)BK, (uint32_t)pp.bn_smem, sw);
      if (r) return r;
      if (!pp.a_tma) continue;
      // dx pixel (h, w) reads dy at (h - (Kh-1-Ph) + kh', w - (Kw-1-Pw) + kw') with kh' = Kh-1-kh
      if ((r = get_encode_im2col())) return r;
      r = encode_im2col(plane_map(&q.a, &q.a2, &q.a3, pl), e, static_cast<const uint8_t *>(dypk) + ld, P.Cop,
                        d.Wo, d.Ho, d.N, -(d.Kw - 1 - d.Pw), -(d.Kh - 1 - d.Ph), -d.Pw, -d.Ph, BK,
                        128, 1, 1, sw, dy_pw, dy_ph);
      if (r) return r;
    }
    return GLP_OK;
  });
  if (s) return s;
  IgemmParams p = make_params(P, pp, MODE_DGRAD, dypk);
  if (!P.s2d_dg) {
    p.out = dx;
    p.out_c = P.x_img_c;   // channels per image of dx (the whole tensor for a conv group)
    p.out_hw = d.H * d.W;
    return launch_igemm<MODE_DGRAD>(P, pp, p, m, st);
  }
  float *dxs = reinterpret_cast<float *>(ws + P.off_dxs);
  p.out = dxs;
  p.out_c = d.C;
  p.out_hw = d.H * d.W;
  if ((s = launch_igemm<MODE_DGRAD>(P, pp, p, m, st))) return s;
  const glp_conv_desc_s &o = P.d;
  const long long total = (long long)o.N * o.C * o.H * o.W;
  GLP_CUDA(launch_pdl(P.pdl, unpack_s2d_dx, dim3((unsigned)std::min<long long>(cdiv(total, 256), 148 * 16)),
                      dim3(256), 0, st, (const float *)dxs, dx, o.N, o.C, o.H, o.W, P.s2d, o.Ph,
                      P.dxg.H, P.dxg.W, P.x_img_c));
  GLP_LAUNCH_CHECK("unpack_s2d_dx");
  return GLP_OK;
}

glp_status_t run_wgrad_halo(glp_plan_s &P, uint8_t *ws, cudaStream_t st, const float *dy) {
  const glp_conv_desc_s &d = P.dxg;
  if (P.halo_fdy && !dy)
    return fail(GLP_ERR_INVALID_VALUE, "filter gradient: no dy recorded for this workspace "
                                       "(glp_stage_pack(GLP_PACK_DY*) first)");
  const uint64_t rows = (uint64_t)d.N * d.H * d.W;   // flat padded grid of x' and dy
  Maps m;
  glp_status_t s = cached_maps(P, 2, ws, m, [&](Maps &q) {
    glp_status_t r = encode_2d(&q.a, 2, ws + P.off_xpk, (uint64_t)P.Cpx, rows, (uint64_t)P.Cpx * 2,
                               64u, (uint32_t)P.hw.halo_rows, CU_TENSOR_MAP_SWIZZLE_128B);
    if (r) return r;
    return encode_2d(&q.b, 2, ws + P.off_dypk, (uint64_t)P.Cop, rows, (uint64_t)P.Cop * 2, 64u,
                     (uint32_t)HW_BKP, CU_TENSOR_MAP_SWIZZLE_128B);
  });
  if (s) return s;
  CUtensorMap &mapX = m.a, &mapDy = m.b;
  HwgradParams p = P.hw;
  p.part = reinterpret_cast<float *>(ws + P.off_part);
  p.dbg_skip = P.dbg_skip;
  if (P.halo_fdy) {
    p.dy = dy;
    p.dy_c = P.y_img_c;
    const DbAux a = db_aux(P, ws + P.off_dbpart, P.db_rows);
    p.db_part = a.part;
    p.db_tickets = a.tickets;
    p.n_tickets = (int)cdiv(P.d.Co, 32);
  }
  cudaLaunchConfig_t cfg;
  memset(&cfg, 0, sizeof(cfg));
  cfg.gridDim = dim3((unsigned)P.hw_grid);
  cfg.blockDim = dim3(hw_threads(P.halo_fdy));
  cfg.dynamicSmemBytes = (size_t)P.hw_smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = P.pdl ? 1 : 0;
  void *args[] = {&p, &mapX, &mapDy};
  GLP_CUDA(cudaLaunchKernelExC(&cfg, P.halo_fdy == 3 ? reinterpret_cast<void *>(hwgrad_kernel<3>)
                                : P.halo_fdy == 2 ? reinterpret_cast<void *>(hwgrad_kernel<2>)
                                : P.halo_fdy == 1 ? reinterpret_cast<void *>(hwgrad_kernel<1>)
                                                  : reinterpret_cast<void *>(hwgrad_kernel<0>),
                                args));
  GLP_LAUNCH_CHECK("hwgrad_kernel");
  return GLP_OK;
}

// dy: the fp32 dy tensor, used only by fused-dy halo plans (which pack nothing for the filter
// gradient); every other plan reads the packed dy in the workspace.
glp_status_t run_wgrad_gemm(glp_plan_s &P, uint8_t *ws, cudaStream_t st, const float *dy = nullptr) {
  if (P.halo) return run_wgrad_halo(P, ws, st, dy);
  const glp_conv_desc_s &d = P.dxg;
  const PassPlan &pp = P.wgrad;
  const void *xpk = ws + P.off_xpk, *dypk = ws + P.off_dypk;
  float *part = reinterpret_cast<float *>(ws + P.off_part);
  const int BKP = 128 / P.elem, EPA = pp.krow / P.elem;
  Maps m;
  glp_status_t s = cached_maps(P, 2, ws, m, [&](Maps &q) {
    for (int pl = 0; pl < nplanes(P); ++pl) {   // hi plane, then the lo / bf16 planes
      const long long ld = plane_offset(P, pl, P.lo_dypk), lx = plane_offset(P, pl, P.lo_xpk);
      const int e = plane_elem(P, pl);
      // MN-major atoms of EPA elements: 32 tf32 (128-byte rows, 32-byte swizzle base) or, for the
      // bf16 planes of the mixed split, 32 bf16 (64-byte rows, SWIZZLE_64B)
      const CUtensorMapSwizzle sw = e == P.elem ? swz_mnmajor(P.elem, pp.krow) : CU_TENSOR_MAP_SWIZZLE_64B;
      glp_status_t r = P.wgrad_b3d
          ? encode_mn3d(plane_map(&q.b, &q.b2, &q.b3, pl), e, static_cast<const uint8_t *>(dypk) + ld,
                        (uint64_t)P.Cop, (uint64_t)d.N * d.Ho * d.Wo, (uint32_t)EPA, (uint32_t)BKP,
                        (uint32_t)(pp.bn_smem / EPA), sw)
          : encode_2d(plane_map(&q.b, &q.b2, &q.b3, pl), e, static_cast<const uint8_t *>(dypk) + ld,
                      (uint64_t)P.Cop, (uint64_t)d.N * d.Ho * d.Wo,
                      (uint64_t)P.Cop * e, (uint32_t)EPA, (uint32_t)BKP, sw);
      if (r) return r;
      if (!pp.a_tma) continue;
      if ((r = get_encode_im2col())) return r;
      r = encode_im2col(plane_map(&q.a, &q.a2, &q.a3, pl), e, static_cast<const uint8_t *>(xpk) + lx, P.Cpx,
                        d.W, d.H, d.N, -d.Pw, -d.Ph, d.Pw - (d.Kw - 1), d.Ph - (d.Kh - 1), EPA,
                        BKP, d.Sw, d.Sh, sw);
      if (r) return r;
    }
    return GLP_OK;
  });
  if (s) return s;
  IgemmParams p = make_params(P, pp, MODE_WGRAD, xpk);
  p.out = part;
  return launch_igemm<MODE_WGRAD>(P, pp, p, m, st);
}

// leaf_stride > 0 (leaf plans): leaf l's dW / db go to dw / db + l * leaf_stride floats (one
// reduction per leaf, grid z = leaf); leaf plans called with leaf_stride = 0 reduce into the
// workspace leaf region and sum the leaves with the fixed tree into dw / db.
glp_status_t run_tree(const float *const *parts, int n, float *out, size_t count, int accumulate,
                      cudaStream_t st);
glp_status_t run_wgrad_reduce(glp_plan_s &P, const BrOut &dw_in, const BrOut *db_in, int accumulate,
                              uint8_t *ws, cudaStream_t st, long long leaf_stride = 0) {
  const glp_conv_desc_s &d = P.d;
  float *part = reinterpret_cast<float *>(ws + P.off_part);
  const int L = P.leaves;
  BrOut dw = dw_in, dbl;
  const BrOut *db = db_in;
  const size_t wsz = (size_t)d.Co * d.C * d.Kh * d.Kw;
  const bool via_ws = L > 1 && leaf_stride == 0;   // composed call on a leaf plan
  float *leaf = reinterpret_cast<float *>(ws + P.off_leaf);
  if (via_ws) {   // leaf l at leaf + l * P.leaf_stride: [dW | db]
    if (dw_in.n > 1) return fail(GLP_ERR_NOT_SUPPORTED, "leaf plans run single layers");
    dw = br_out(P, 1, &leaf);
    float *lb = leaf + wsz;
    dbl = br_out(P, 1, &lb);
    if (db_in) db = &dbl;
    leaf_stride = (long long)P.leaf_stride;
  }
  const int acc_red = via_ws ? 0 : accumulate;
  if (P.halo) {
    const DwRed r{part, dw, d.Co, d.C, P.taps, d.Kw, P.Cpx, P.hw.ld, P.hw.mpad, P.hw.splits,
                  accumulate, P.s2d, P.dxg.Kw, 0LL};
    GLP_CUDA(launch_pdl(P.pdl, reduce_tc_dw_wide,
                        dim3((unsigned)cdiv((long long)d.C * P.taps, 4), (unsigned)cdiv(d.Co, 32)),
                        dim3(256), 0, st, r));
    GLP_LAUNCH_CHECK("reduce_tc_dw_wide");
    if (db) {
      DbAux a = db_aux(P, ws + P.off_dbpart, P.db_rows);
      const DbRed q{a.part, *db, d.Co, P.db_rows, accumulate, a.part2, a.tickets, 0LL,
                    db_groups(P.db_rows), (int)cdiv(d.Co, 32)};
      GLP_CUDA(launch_pdl(P.pdl, reduce_db, dim3((unsigned)q.cx, (unsigned)q.G), dim3(256), 0, st, q));
      GLP_LAUNCH_CHECK("reduce_db");
    }
  } else {
    const DwRed r{part, dw, d.Co, d.C, P.taps, d.Kw, P.Cpx, P.wgrad.n_tiles * P.wgrad.bn,
                  P.wgrad.m_units * P.wgrad.cg * 128, P.wgrad.splits / L, acc_red, P.s2d,
                  P.dxg.Kw, leaf_stride};
    // dW blocks: 32 x 32 tiles, or 4 weight rows x 32 channels for small filters (red_wide)
    const int ax = (int)cdiv((long long)d.C * P.taps, P.red_wide ? 4 : 32), ay = (int)cdiv(d.Co, 32);
    if (db) {   // dW and db reductions in one launch
      DbAux a = db_aux(P, ws + P.off_dbpart, P.db_rows);
      const DbRed q{a.part, *db, d.Co, P.db_rows / L, acc_red, a.part2, a.tickets, leaf_stride,
                    db_groups(P.db_rows / L), (int)cdiv(d.Co, 32)};
      const dim3 grid((unsigned)(ax * ay + q.cx * q.G), 1, (unsigned)L);
      if (P.red_wide) GLP_CUDA(launch_pdl(P.pdl, reduce_wgrad<1>, grid, dim3(256), 0, st, r, q, ax, ay));
      else GLP_CUDA(launch_pdl(P.pdl, reduce_wgrad<0>, grid, dim3(256), 0, st, r, q, ax, ay));
      GLP_LAUNCH_CHECK("reduce_wgrad");
    } else {
      const dim3 grid((unsigned)ax, (unsigned)ay, (unsigned)L);
      if (P.red_wide) GLP_CUDA(launch_pdl(P.pdl, reduce_tc_dw_wide, grid, dim3(256), 0, st, r));
      else GLP_CUDA(launch_pdl(P.pdl, reduce_tc_dw, grid, dim3(256), 0, st, r));
      GLP_LAUNCH_CHECK("reduce_tc_dw");
    }
  }
  if (via_ws) {   // dW || db = the fixed tree over the leaves (glp_tree_sum order)
    const float *parts[8];
    for (int l = 0; l < L; ++l) parts[l] = leaf + (size_t)l * P.leaf_stride;
    float *out = dw_in.p[0];
    glp_status_t s = run_tree(parts, L, out, wsz, accumulate, st);
    if (s) return s;
    if (db_in) {
      const float *pb[8];
      for (int l = 0; l < L; ++l) pb[l] = parts[l] + wsz;
      if ((s = run_tree(pb, L, db_in->p[0], (size_t)d.Co, accumulate, st))) return s;
    }
  }
  return GLP_OK;
}

// Composed tensor-core passes (single layer: one-entry tables; fused group: one per branch).
glp_status_t tc_fwd(glp_plan_s &P, const float *x, const BrIn &w, const BrIn &b, const BrOut &y,
                    uint8_t *ws, cudaStream_t st) {
  glp_status_t s = launch_pack_x(P, x, ws + P.off_xpk, st);
  if (s) return s;
  if ((s = run_pack_w_fwd(P, w, ws, st))) return s;
  return run_fwd_gemm(P, b, y, ws, st);
}
glp_status_t tc_bwd(glp_plan_s &P, const float *x, const BrIn &dy, const BrIn &w, float *dx,
                    const BrOut &dw, const BrOut &db, bool with_db, int accumulate, uint8_t *ws,
                    cudaStream_t st) {
  glp_status_t s = GLP_OK;
  if (!P.halo_fdy || dx)   // fused-dy plans pack dy only for the backward-data pass
    if ((s = launch_pack_dy(P, dy, ws, with_db, st))) return s;
  if (dx) {
    if ((s = run_pack_w_dgrad(P, w, ws, st))) return s;
    if ((s = run_dgrad_gemm(P, dx, ws, st))) return s;
  }
  if ((s = launch_pack_x(P, x, ws + P.off_xpk, st))) return s;
  if ((s = run_wgrad_gemm(P, ws, st, dy.p[0]))) return s;
  return run_wgrad_reduce(P, dw, with_db ? &db : nullptr, accumulate, ws, st);
}

// out = a + b elementwise (one IEEE fp32 add per element: commutative, so a tree of these is
// bitwise independent of which rank holds which operand).  out may alias a or b (the tree adds
// in place), so no pointer is __restrict__.
__global__ void __launch_bounds__(256) sum2_kernel(const float *a, const float *b, float *out,
                                                   size_t n) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n;
       i += (size_t)gridDim.x * blockDim.x)
    out[i] = a[i] + b[i];
}

// Stream-pool comparator: dst[i] (+)= sum over the pool's S per-stream accumulators, s = 0..S-1
// in order (fixed, so the pool's result is deterministic for a given S).
__global__ void __launch_bounds__(256) pool_sum_slots(const float *__restrict__ src, size_t stride,
                                                      int S, float *__restrict__ dst, size_t n,
                                                      int accumulate) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n;
       i += (size_t)gridDim.x * blockDim.x) {
    float a = 0.f;
    for (int s = 0; s < S; ++s) a += src[(size_t)s * stride + i];
    dst[i] = accumulate ? dst[i] + a : a;
  }
}

// ---- deterministic exchange: the fixed binary tree ----
// Pointer tables by value (kernel parameters): up to 8 leaves / ranks.
struct Ptr8 {
  const float *p[8];
};
struct MPtr8 {
  float *p[8];
};

// out[i] (+)= T(parts[0..n))[i], T = the balanced binary tree over n (a power of two <= 8)
// operands in index order: level by level, v[k] = v[k] + v[k + w] for k = 0, 2w, ... -- the same
// fp32 adds, in the same order, as dist.tree_sum over glp_sum2.
__global__ void __launch_bounds__(256) tree_sum_kernel(const Ptr8 parts, int n, float *out,
                                                       size_t count, int accumulate) {
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < count;
       i += (size_t)gridDim.x * blockDim.x) {
    float v[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) v[k] = k < n ? __ldg(parts.p[k] + i) : 0.f;
#pragma unroll
    for (int w = 1; w < 8; w <<= 1)
#pragma unroll
      for (int k = 0; k + w < 8; k += 2 * w)
        if (k + w < n) v[k] = v[k] + v[k + w];
    out[i] = accumulate ? out[i] + v[0] : v[0];
  }
}

// The top of the tree across ranks over NVLink peer memory (torch symmetric memory): element slice
// [rank*count/world, (rank+1)*count/world) of T(subtrees[0..world)) -- the rank-ordered subtree
// sums of every rank, read by peer loads -- is computed by this rank and stored into every rank's
// output buffer (peer stores), so after a barrier every rank holds the same bits, those of the
// tree over all leaves.  Plain volatile-free global loads/stores on mapped peer pointers.
__global__ void __launch_bounds__(256) tree_exchange_kernel(const Ptr8 subtrees, const MPtr8 outs,
                                                            int world, int rank, size_t count) {
  const size_t lo = count * (size_t)rank / world, hi = count * (size_t)(rank + 1) / world;
  for (size_t i = lo + blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < hi;
       i += (size_t)gridDim.x * blockDim.x) {
    float v[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) v[k] = k < world ? subtrees.p[k][i] : 0.f;
#pragma unroll
    for (int w = 1; w < 8; w <<= 1)
#pragma unroll
      for (int k = 0; k + w < 8; k += 2 * w)
        if (k + w < world) v[k] = v[k] + v[k + w];
#pragma unroll
    for (int k = 0; k < 8; ++k)
      if (k < world) outs.p[k][i] = v[0];
  }
}

glp_status_t run_tree(const float *const *parts, int n, float *out, size_t count, int accumulate,
                      cudaStream_t st) {
  if (n < 1 || n > 8 || (n & (n - 1))) return fail(GLP_ERR_INVALID_VALUE, "tree: n must be 1, 2, 4 or 8");
  if (count == 0) return GLP_OK;
  Ptr8 t{};
  for (int k = 0; k < n; ++k) t.p[k] = parts[k];
  tree_sum_kernel<<<ew_grid(count), 256, 0, st>>>(t, n, out, count, accumulate);
  GLP_LAUNCH_CHECK("tree_sum_kernel");
  return GLP_OK;
}

ConvGeom geomP(const glp_plan_s &P) {
  const glp_conv_desc_s &d = P.d;
  return ConvGeom{d.N, d.C, d.H, d.W, d.Co, d.Kh, d.Kw, d.Sh, d.Sw, d.Ph, d.Pw, d.Ho, d.Wo,
                  P.x_img_c, P.y_img_c};
}

glp_status_t run_wgrad_simt(glp_plan_s &P, const float *x, const float *dy, float *dw, float *db,
                            int accumulate, uint8_t *ws, cudaStream_t st) {
  const glp_conv_desc_s &d = P.d;
  const size_t wsz = (size_t)d.Co * d.C * d.Kh * d.Kw;
  float *part = reinterpret_cast<float *>(ws);
  float *dbp = reinterpret_cast<float *>(ws + align1k(wsz * P.simt_splits * 4));
  simt_wgrad_partial<<<ew_grid(wsz * P.simt_splits), 256, 0, st>>>(geomP(P), x, dy, part, P.simt_splits, P.simt_chunk);
  GLP_LAUNCH_CHECK("simt_wgrad_partial");
  reduce_simt_dw<<<ew_grid(wsz), 256, 0, st>>>(part, dw, wsz, P.simt_splits, accumulate);
  GLP_LAUNCH_CHECK("reduce_simt_dw");
  if (db) {
    simt_db_partial<<<ew_grid((size_t)P.simt_splits * d.Co), 256, 0, st>>>(geomP(P), dy, dbp, P.simt_splits, P.simt_chunk);
    GLP_LAUNCH_CHECK("simt_db_partial");
    DbAux a = db_aux(P, reinterpret_cast<uint8_t *>(dbp), P.simt_splits);
    GLP_CUDA(cudaMemsetAsync(a.tickets, 0, (size_t)cdiv(d.Co, 32) * 4, st));
    float *dbs[1] = {db};
    const DbRed q{a.part, br_out(P, 1, dbs), d.Co, P.simt_splits, accumulate, a.part2, a.tickets,
                  0LL, db_groups(P.simt_splits), (int)cdiv(d.Co, 32)};
    reduce_db<<<dim3((unsigned)q.cx, (unsigned)q.G), 256, 0, st>>>(q);
    GLP_LAUNCH_CHECK("reduce_db");
  }
  return GLP_OK;
}

// Debug im2col through the forward producer's gather (fwd_gather) on the packed operand.
template <int ELEM>
__global__ void debug_im2col_kernel(Gather g, int n, int C, int Kh, int Kw, int Ho, int Wo,
                                    float *col) {
  const size_t rows = (size_t)C * Kh * Kw, hw = (size_t)Ho * Wo;
  for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < rows * hw;
       i += (size_t)gridDim.x * blockDim.x) {
    const int pix = (int)(i % hw);
    const int r = (int)(i / hw);
    const int kw = r % Kw, kh = (r / Kw) % Kh, ci = r / (Kw * Kh);
    const int ho = pix / Wo, wo = pix % Wo;
    const uint32_t k = (uint32_t)((kh * Kw + kw) * g.cp + ci);
    const uint32_t kc = k - k % (16 / ELEM);
    const uint8_t *src = nullptr;
    float v = 0.f;
    if (fwd_gather<ELEM>(g, (uint32_t)n, ho * g.stride - g.pad, wo * g.stride_w - g.pad_w, kc, src)) {
      const int e = (int)(k - kc);
      if (ELEM == 2) v = __bfloat162float(reinterpret_cast<const __nv_bfloat16 *>(src)[e]);
      else v = reinterpret_cast<const float *>(src)[e];
    }
    col[i] = v;
  }
}

}  // namespace

// ====================================================================== C ABI =================
extern "C" {

int glp_version(void) { return 1; }

const char *glp_status_string(glp_status_t s) {
  switch (s) {
    case GLP_OK: return "GLP_OK";
    case GLP_ERR_INVALID_VALUE: return "GLP_ERR_INVALID_VALUE";
    case GLP_ERR_NOT_SUPPORTED: return "GLP_ERR_NOT_SUPPORTED";
    case GLP_ERR_CUDA: return "GLP_ERR_CUDA";
    case GLP_ERR_WORKSPACE_TOO_SMALL: return "GLP_ERR_WORKSPACE_TOO_SMALL";
    case GLP_ERR_INTERNAL: return "GLP_ERR_INTERNAL";
  }
  return "GLP_ERR_UNKNOWN";
}

const char *glp_last_error_string(void) { return g_last_error.c_str(); }

glp_status_t glp_conv_desc_create(glp_conv_desc_t *out, int N, int C, int H, int W, int Co, int Kh,
                                  int Kw, int Sh, int Sw, int Ph, int Pw) {
  if (!out) return fail(GLP_ERR_INVALID_VALUE, "out is NULL");
  *out = nullptr;
  if (N <= 0 || C <= 0 || H <= 0 || W <= 0 || Co <= 0 || Kh <= 0 || Kw <= 0 || Sh <= 0 || Sw <= 0 ||
      Ph < 0 || Pw < 0)
    return fail(GLP_ERR_INVALID_VALUE, "non-positive dimension / negative pad");
  if (H + 2 * Ph < Kh || W + 2 * Pw < Kw) return fail(GLP_ERR_INVALID_VALUE, "H_out < 1");
  const long long Ho = (H + 2LL * Ph - Kh) / Sh + 1, Wo = (W + 2LL * Pw - Kw) / Sw + 1;
  // 32-bit index math on the device (FastDiv): every flattened extent must stay < 2^31.
  if ((long long)N * C * H * W >= (1LL << 31) || (long long)N * Co * Ho * Wo >= (1LL << 31) ||
      (long long)Co * C * Kh * Kw >= (1LL << 31))
    return fail(GLP_ERR_NOT_SUPPORTED, "tensor too large for 32-bit indexing");
  auto *d = new glp_conv_desc_s{N, C, H, W, Co, Kh, Kw, Sh, Sw, Ph, Pw, (int)Ho, (int)Wo};
  *out = d;
  return GLP_OK;
}

glp_status_t glp_conv_group_desc_create(glp_conv_desc_t *out, int N, int C, int H, int W,
                                        int n_branches, const int *C_out, int Kh, int Kw, int Sh,
                                        int Sw, int Ph, int Pw) {
  if (!out || !C_out) return fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  *out = nullptr;
  if (n_branches < 1 || n_branches > GLP_MAXBR)
    return fail(GLP_ERR_INVALID_VALUE, "n_branches must be 1.." + std::to_string(GLP_MAXBR));
  long long tot = 0;
  for (int b = 0; b < n_branches; ++b) {
    if (C_out[b] <= 0) return fail(GLP_ERR_INVALID_VALUE, "non-positive branch C_out");
    tot += C_out[b];
  }
  if (tot >= (1LL << 30)) return fail(GLP_ERR_INVALID_VALUE, "C_out too large");
  glp_status_t s = glp_conv_desc_create(out, N, C, H, W, (int)tot, Kh, Kw, Sh, Sw, Ph, Pw);
  if (s) return s;
  glp_conv_desc_s *d = *out;
  d->nbr = n_branches;
  d->br_off[0] = 0;
  for (int b = 0; b < n_branches; ++b) d->br_off[b + 1] = d->br_off[b] + C_out[b];
  return GLP_OK;
}

glp_status_t glp_conv_desc_set_groups(glp_conv_desc_t d, int groups) {
  if (!d) return fail(GLP_ERR_INVALID_VALUE, "desc is NULL");
  if (groups < 1 || d->C % groups || d->Co % groups)
    return fail(GLP_ERR_INVALID_VALUE, "groups must divide C_in and C_out");
  if (groups > 1 && d->nbr > 1)
    return fail(GLP_ERR_NOT_SUPPORTED, "a desc is either a conv group or a fused sibling group");
  d->groups = groups;
  return GLP_OK;
}

glp_status_t glp_conv_desc_get_output(glp_conv_desc_t d, int *Ho, int *Wo) {
  if (!d || !Ho || !Wo) return fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  *Ho = d->Ho;
  *Wo = d->Wo;
  return GLP_OK;
}

glp_status_t glp_conv_desc_destroy(glp_conv_desc_t d) {
  delete d;
  return GLP_OK;
}

glp_status_t glp_device_limits_b200(glp_device_limits_t *L) {
  if (!L) return fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  *L = glp_device_limits_t{148, 2048, 32, 65536, 228 * 1024, 1024, 512, 128};
  return GLP_OK;
}

glp_status_t glp_analyze_ctas_per_sm(const glp_device_limits_t *L, const glp_kernel_attr_t *k, int *b) {
  if (!L || !k || !b) return fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  if (k->threads <= 0 || k->regs < 0 || k->smem_bytes < 0 || k->tmem_cols < 0)
    return fail(GLP_ERR_INVALID_VALUE, "bad kernel attributes");
  *b = ctas_per_sm_closed_form(*L, *k);
  return GLP_OK;
}

glp_status_t glp_analyze_samples_in_flight(int slots, int tiles_per_sample, int n_local, int *S) {
  if (!S || slots <= 0 || tiles_per_sample <= 0 || n_local <= 0)
    return fail(GLP_ERR_INVALID_VALUE, "bad analyzer input");
  *S = std::max(1, std::min(n_local, slots / tiles_per_sample));
  return GLP_OK;
}

glp_status_t glp_analyze_eq7(const glp_device_limits_t *L, const glp_kernel_attr_t *k, int blocks,
                             double t_kernel, double t_launch, int *bound) {
  if (!L || !k || !bound || blocks <= 0 || k->threads <= 0)
    return fail(GLP_ERR_INVALID_VALUE, "bad analyzer input");
  double m = (double)L->max_threads_per_sm * L->sm_count / ((double)k->threads * blocks);
  if (k->smem_bytes > 0) m = std::min(m, (double)L->smem_per_sm * L->sm_count / ((double)k->smem_bytes * blocks));
  if (t_kernel > 0 && t_launch > 0) m = std::min(m, std::ceil(t_kernel / t_launch));
  *bound = (int)std::floor(m);
  return GLP_OK;
}

glp_status_t glp_plan_options_default(glp_plan_options_t *o) {
  if (!o) return fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  *o = glp_plan_options_t{1, 1, 1, 1, 1, 1, 0, 4, 0, 6, 1, 2, 0, 232448, 0, 0, 2};
  return GLP_OK;
}

glp_status_t glp_plan(glp_plan_t *out, glp_conv_desc_t d, int device, glp_math_t math, int S) {
  return glp_plan_ex(out, d, device, math, S, nullptr);
}

glp_status_t glp_plan_ex(glp_plan_t *out, glp_conv_desc_t d, int device, glp_math_t math, int S,
                         const glp_plan_options_t *opts) {
  if (!out || !d) return fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  glp_plan_options_t o;
  glp_plan_options_default(&o);
  if (opts) o = *opts;
  if (o.halo_dgrad < 0 || o.halo_dgrad > 2 || o.fused_dy_builders < 0 || o.fused_dy_builders > 3 ||
      o.max_kblocks_per_stage < 1 || o.max_kblocks_per_stage > 4 || o.wgrad_tile_n < 0 ||
      o.wgrad_tile_n > 256 || o.wgrad_tile_n % 16 || o.tile_units < 0 || o.smem_cap < 65536 ||
      o.smem_cap > 232448 || (o.wgrad_leaves != 0 && o.wgrad_leaves != 1 && o.wgrad_leaves != 2 &&
                              o.wgrad_leaves != 4 && o.wgrad_leaves != 8))
    return fail(GLP_ERR_INVALID_VALUE, "plan option out of range");
  if (o.fp32_split < 0 || o.fp32_split > 2 || o.pack_block < 0 || o.pack_block > 2)
    return fail(GLP_ERR_INVALID_VALUE, "plan option out of range");
  if (o.wgrad_leaves > 0 && (math == GLP_MATH_FP32_SIMT || d->nbr > 1))
    return fail(GLP_ERR_NOT_SUPPORTED, "wgrad leaves: tensor-core single-layer plans only");
  *out = nullptr;
  if (math != GLP_MATH_FP32 && math != GLP_MATH_TF32 && math != GLP_MATH_BF16 &&
      math != GLP_MATH_FP32_SIMT)
    return fail(GLP_ERR_INVALID_VALUE, "unknown math mode");
  if (S < 0) return fail(GLP_ERR_INVALID_VALUE, "samples_in_flight < 0");
  const auto t0 = std::chrono::steady_clock::now();
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev == 0) {
    cudaGetLastError();
    return fail(GLP_ERR_NOT_SUPPORTED, "no CUDA device (there is no CPU fallback)");
  }
  if (device < 0 || device >= ndev) return fail(GLP_ERR_INVALID_VALUE, "bad device ordinal");
  cudaDeviceProp prop;
  GLP_CUDA(cudaGetDeviceProperties(&prop, device));
  if (prop.major != 10) return fail(GLP_ERR_NOT_SUPPORTED, "libglp.so is built for sm_100a (B200) only");
  int cur = 0;
  GLP_CUDA(cudaGetDevice(&cur));
  if (cur != device) GLP_CUDA(cudaSetDevice(device));

  if (d->groups > 1 && d->nbr > 1)
    return fail(GLP_ERR_NOT_SUPPORTED, "a desc is either a conv group or a fused sibling group");
  auto *P = new glp_plan_s();
  P->d = *d;
  P->groups = std::max(1, d->groups);
  P->x_img_c = d->C;
  P->y_img_c = d->Co;
  if (P->groups > 1) {   // plan ONE group's convolution; the calls loop over the groups
    P->d.C = d->C / P->groups;
    P->d.Co = d->Co / P->groups;
    P->d.groups = 1;
    P->d.br_off[1] = P->d.Co;
  }
  d = &P->d;   // everything below plans the (per-group) convolution
  P->device = device;
  P->math = (int)math;
  P->elem = (math == GLP_MATH_BF16) ? 2 : 4;
  P->simt = (math == GLP_MATH_FP32_SIMT) ? 1 : 0;
  P->x3 = (math == GLP_MATH_FP32) ? 1 : 0;
  P->sm_count = prop.multiProcessorCount;
  P->s_override = S;
  // plan options (include/glp.h glp_plan_options_t): alternative kernels / tilings of the same
  // computation, bitwise-equal outputs
  P->allow_cg2 = o.cta_pairs != 0;
  P->ksub_max = o.max_kblocks_per_stage;
  P->allow_ksub2 = P->ksub_max > 1;
  P->wgrad_cg2 = o.wgrad_cta_pairs != 0;
  P->pdl = o.pdl != 0;
  P->bn_model = o.bn_model != 0;
  P->allow_halo = o.halo_wgrad != 0;
  P->allow_hfwd = o.halo_fwd != 0;
  P->allow_fdy = o.fused_dy != 0;
  P->fdy_ncg = o.fused_dy_builders;
  P->allow_hdg = o.halo_dgrad;
  P->wgrad_bn = o.wgrad_tile_n;
  P->tile_units = o.tile_units;
  // activation pack: 2 (default) = block-tiled for 4-byte operands (tf32 and the fp32 splits:
  // measured 4.4-6.1 TB/s against the warp-tiled kernel's 3.3-4.7 on CaffeNet's packs, fp32 step
  // +2.8 %, tf32 +5 %), warp-tiled for bf16 (equal within noise)
  P->pack_block = o.pack_block == 2 ? (P->elem == 4 ? 1 : 0) : (o.pack_block != 0);
  P->s2d_block = o.s2d_block != 0;
  P->smem_cap = o.smem_cap;
  P->leaves = std::max(1, o.wgrad_leaves);
  P->leaf_plan = o.wgrad_leaves > 0 ? 1 : 0;
  if (P->leaf_plan) {   // leaf plans use the im2col filter gradient and the warp-tiled dy pack
    P->allow_halo = 0;
    P->pack_block = 0;
  }
#ifdef GLP_DIAG
  // diagnostic builds only (never the shipped library): GLP_DEBUG_CLK = device address of
  // >= 4 * grid uint64 counters (tools/clk_probe.py); GLP_DEBUG_SKIP = work-skipping bits
  if (const char *e = getenv("GLP_DEBUG_CLK")) P->dbg_clk = reinterpret_cast<unsigned long long *>(strtoull(e, nullptr, 10));
  if (const char *e = getenv("GLP_DEBUG_SKIP")) P->dbg_skip = atoi(e) & 63;
#endif
  // Channel pitch of the packed NHWC operands: a multiple of 32 channels (64-byte bf16 / 128-byte
  // tf32 rows, what the im2col TMA path needs) unless the channel count is tiny, where padding to
  // 32 would multiply the MMA work; those use the 16-byte-chunk cp.async gather.
  const int CH = 16 / P->elem;
  P->Cp = (int)(d->C >= 16 ? rup(d->C, 32) : rup(d->C, CH));
  P->Cop = (int)(d->Co >= 16 ? rup(d->Co, 32) : rup(d->Co, CH));
  P->taps = d->Kh * d->Kw;
  // Space-to-depth for strided layers when it shrinks the padded K of the GEMM (CaffeNet conv1:
  // 121 taps x 8 channels -> 9 taps x 64 channels).  Square kernels/strides/pads only.
  P->dxg = *d;
  P->Cpx = P->Cp;
  P->tapsx = P->taps;
  if (!P->simt && d->Sh == d->Sw && d->Sh > 1 && d->Kh == d->Kw && d->Ph == d->Pw &&
      d->Kh >= d->Sh) {
    const int S2 = d->Sh, Ks = (int)cdiv(d->Kh, S2), cs = S2 * S2 * d->C;
    const int cps = (int)rup(cs, 32);
    if ((long long)Ks * Ks * cps < (long long)P->taps * rup(P->Cp, 128 / P->elem) &&
        (long long)S2 * d->C * d->W <= 256LL * S2D_LD && 256 % (cps * P->elem / 16) == 0) {
      P->s2d = S2;
      P->dxg = glp_conv_desc_s{d->N, cs, d->Ho + Ks - 1, d->Wo + Ks - 1, d->Co, Ks, Ks, 1, 1,
                               0, 0, d->Ho, d->Wo};
      P->Cpx = cps;
      P->tapsx = Ks * Ks;
      const size_t ssm = (size_t)S2 * d->C * d->W * sizeof(float);
      void *fn = P->elem == 2 ? reinterpret_cast<void *>(pack_s2d<2>) : reinterpret_cast<void *>(pack_s2d<4>);
      if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&P->s2d_blocks, fn, 256, ssm) != cudaSuccess) {
        cudaGetLastError();
        P->s2d_blocks = 1;
      }
    }
  }
  P->s2d_dg = (P->s2d && d->nbr <= 1) ? 1 : 0;
  glp_device_limits_t L;
  glp_device_limits_b200(&L);
  L.sm_count = prop.multiProcessorCount;
  L.smem_per_sm = (int)prop.sharedMemPerMultiprocessor;
  L.regs_per_sm = prop.regsPerMultiprocessor;
  L.max_threads_per_sm = prop.maxThreadsPerMultiProcessor;
  L.max_blocks_per_sm = prop.maxBlocksPerMultiProcessor;
  L.smem_reserved_per_cta = (int)prop.reservedSharedMemPerBlock;

  P->lim = L;
  glp_status_t s = GLP_OK;
  if (d->nbr > 1 && !P->simt) {
    // a branch's packed channels start on a 16-byte chunk of the pitch (8 bf16 / 4 tf32)
    const int ch = 16 / P->elem;
    for (int b = 1; b < d->nbr; ++b)
      if (d->br_off[b] % ch) {
        delete P;
        if (cur != device) cudaSetDevice(cur);
        return fail(GLP_ERR_NOT_SUPPORTED, "fused group: every branch but the last needs C_out % " +
                                               std::to_string(ch) + " == 0");
      }
  }
  // the mixed fp32 split (option fp32_split): every pass must take its operands with 128-byte
  // tf32 rows (the packs write one representation for all three passes): channel pitches
  // (space-to-depth: of x') multiples of 32; forward and filter gradient by TMA, the backward-data
  // by TMA or -- strided layers -- by the K-major cp.async gather;
  // and enough work per pass: below ~2 GFLOP (CIFAR-10 conv2/conv3) the third operand plane's TMA
  // loads cost more than the MMA issue slots saved (measured: CIFAR-10 -2.3 %, GoogLeNet +3 %).
  // Strided layers only when forced (fp32_split = 1): CaffeNet conv1 measured forward 334 -> 316
  // us but filter gradient 418 -> 442 us (its MN-major operands are shared-memory bound, and the
  // 64-byte bf16 atoms read no cheaper), so the default keeps them on 3xTF32
  const double pass_flop = 2.0 * P->d.N * P->d.Ho * P->d.Wo * P->d.Co * P->d.C * P->d.Kh * P->d.Kw;
  P->mix = (P->x3 && o.fp32_split && P->Cpx % 32 == 0 && P->Cop % 32 == 0 &&
            (P->d.Sh == P->d.Sw) && (P->d.Sh == 1 || o.fp32_split == 1) &&
            (o.fp32_split == 1 || pass_flop >= 2e9)) ? 1 : 0;
  if (!P->simt) {
    if ((s = plan_pass(*P, P->fwd, MODE_FWD, L)) || (s = plan_pass(*P, P->dgrad, MODE_DGRAD, L)) ||
        (s = plan_pass(*P, P->wgrad, MODE_WGRAD, L))) {
      delete P;
      if (cur != device) cudaSetDevice(cur);
      return s;
    }
    // filter-gradient B (dy) tile: one 3-D TMA per plane instead of one per atom (same smem bytes);
    // the channel pitch must be whole atoms (the 3-D view's atom dimension; a partial last atom
    // would read the next pixel's channels instead of the 2-D map's zero fill)
    // and every tile must start on an atom (N tile and its per-CTA half multiples of the atom)
    const int epa = P->wgrad.krow / P->elem;
    P->wgrad_b3d = (P->wgrad.a_tma && P->wgrad.bn_smem / epa >= 2 && P->Cop % epa == 0 &&
                    P->wgrad.bn % epa == 0 && P->wgrad.bn_smem % epa == 0) ? 1 : 0;
#ifdef GLP_DIAG
    if (const char *e = getenv("GLP_DEBUG_B3D")) P->wgrad_b3d = P->wgrad_b3d && atoi(e);
#endif
    if (P->mix && !(P->fwd.a_tma && P->wgrad.a_tma && P->fwd.krow == 128 &&
                    P->dgrad.krow == 128 && P->wgrad.krow == 128 &&
                    (P->dgrad.a_tma || P->dgrad.cg == 1))) {
      delete P;
      if (cur != device) cudaSetDevice(cur);
      return fail(GLP_ERR_INTERNAL, "mixed fp32 split planned for a non-TMA pass");
    }
    if ((s = plan_halo(*P)) || (s = plan_hfwd(*P)) || (s = plan_hdgrad(*P))) {
      delete P;
      if (cur != device) cudaSetDevice(cur);
      return s;
    }
    const glp_conv_desc_s &c = *d;
    // x region: the forward/filter-gradient operand, or the direct packing of glp_debug_im2col
    // every packed operand region holds one plane, or (3xTF32) its hi plane then its lo plane
    const size_t pl_x = align1k(std::max((size_t)c.N * c.H * c.W * P->Cp,
                                         (size_t)c.N * P->dxg.H * P->dxg.W * P->Cpx) * P->elem);
    const size_t dy_hw = P->halo ? (size_t)P->dxg.H * P->dxg.W : (size_t)c.Ho * c.Wo;
    const size_t pl_dy = align1k((size_t)c.N * dy_hw * P->Cop * P->elem);
    const size_t pl_w = align1k((size_t)c.Co * P->fwd.Kpad * P->elem);
    const size_t pl_wt = align1k((size_t)(P->s2d_dg ? P->dxg.C : c.C) * P->dgrad.Kpad * P->elem);
    const size_t planes = P->x3 ? 2 : 1;
    P->sz_xpk = planes * pl_x;
    P->sz_dypk = planes * pl_dy;
    P->sz_wpk = planes * pl_w;
    P->sz_wtpk = planes * pl_wt;
    if (P->x3) {
      P->lo_xpk = (long long)pl_x;
      P->lo_dypk = (long long)pl_dy;
      P->lo_wpk = (long long)pl_w;
      P->lo_wtpk = (long long)pl_wt;
    }
    P->sz_part = P->halo ? align1k((size_t)P->hw.splits * P->hw.mpad * P->hw.ld * 4)
                         : align1k((size_t)P->wgrad.splits * P->wgrad.m_units * P->wgrad.cg * 128 *
                                   P->wgrad.n_tiles * P->wgrad.bn * 4);
    P->db_rows = (int)cdiv((long long)c.N * dy_hw, P->pack_block ? PACK_PT : PACKW_ROWS);
    if (P->halo_fdy) P->db_rows = P->hw.splits;   // one db partial per filter-gradient CTA
    // dW reduction kernel (shape-only): filters whose 32 x 32 reduction tiles number < 64 take
    // the 4-row x 8-phase variant (8x the blocks; LeNet conv1: 1 block -> 7)
    if (!P->halo) {
      const long long tiles32 = cdiv((long long)c.C * P->taps, 32) * cdiv(c.Co, 32);
      P->red_wide = tiles32 < 64 && P->wgrad.splits / std::max(1, P->leaves) >= 16 ? 1 : 0;
    }
    P->sz_dbpart = db_aux_bytes(P->db_rows, c.Co, P->leaves);
    // one layout serves every call: [xpk | dypk | wpk | wtpk | part | dbpart]
    P->off_xpk = 0;
    P->off_dypk = P->sz_xpk;
    P->off_wpk = P->off_dypk + P->sz_dypk;
    P->off_wtpk = P->off_wpk + P->sz_wpk;   // own region: both weight packs can live at once
    P->off_part = P->off_wtpk + P->sz_wtpk;
    P->off_dbpart = P->off_part + P->sz_part;
    P->ws_fwd = P->off_wpk + P->sz_wpk;
    P->ws_dgrad = P->off_wtpk + P->sz_wtpk;
    if (P->leaves > 1) {   // leaf partials [dW | db] of the composed calls (summed by the tree)
      P->leaf_stride = (size_t)rup((long long)c.Co * c.C * c.Kh * c.Kw + c.Co, 4);
      P->sz_leaf = align1k((size_t)P->leaves * P->leaf_stride * 4);
    }
    P->off_leaf = P->off_dbpart + P->sz_dbpart;
    P->ws_wgrad = P->off_leaf + P->sz_leaf;
    P->ws_bwd = P->ws_wgrad;
    if (P->s2d_dg) {   // dx' of the space-to-depth backward-data, after every other region
      P->off_dxs = P->ws_wgrad;
      P->sz_dxs = align1k((size_t)c.N * P->dxg.C * P->dxg.H * P->dxg.W * 4);
      P->ws_dgrad = P->off_dxs + P->sz_dxs;
      P->ws_bwd = P->ws_dgrad;
    }
    // Samples in flight (the paper's C_out, Eq. 9 re-derived, R18) through the analyzer: the
    // forward kernel's resident rows (#SM x CTAs/SM x 128 GEMM rows) over the rows a sample
    // occupies (H_o*W_o pixels -- the padded x' grid for the halo forward -- times the N tiles)
    const bool hf = P->hfwd != 0;
    const int beta = hf ? P->hf_attr.model : P->fwd.ctas_per_sm;
    P->s_slot_rows = (long long)P->sm_count * beta * 128;
    P->s_rows_per_sample = hf ? (long long)P->dxg.H * P->dxg.W
                              : (long long)d->Ho * d->Wo * P->fwd.n_tiles;
    if (P->s_slot_rows >= (1LL << 31) || P->s_rows_per_sample >= (1LL << 31)) {
      delete P;
      if (cur != device) cudaSetDevice(cur);
      return fail(GLP_ERR_NOT_SUPPORTED, "analyzer inputs exceed 32 bits");
    }
    if ((s = glp_analyze_samples_in_flight((int)P->s_slot_rows, (int)P->s_rows_per_sample, d->N,
                                           &P->S))) {
      delete P;
      if (cur != device) cudaSetDevice(cur);
      return s;
    }
    if (S > 0) P->S = std::min(S, d->N);
  } else {
    const long long npix = (long long)d->N * d->Ho * d->Wo;
    P->simt_chunk = (int)std::max(256LL, cdiv(npix, 256));
    P->simt_splits = (int)cdiv(npix, P->simt_chunk);
    const size_t wsz = (size_t)d->Co * d->C * d->Kh * d->Kw;
    P->ws_fwd = 0;
    P->ws_dgrad = 0;
    P->ws_wgrad = align1k(wsz * P->simt_splits * 4) + db_aux_bytes(P->simt_splits, d->Co);
    P->ws_bwd = P->ws_wgrad;
    P->S = S > 0 ? std::min(S, d->N) : d->N;
  }
  // one workspace slice per convolution group (staged calls keep every group's packs alive)
  P->ws_group = align1k(std::max({P->ws_fwd, P->ws_dgrad, P->ws_wgrad, P->ws_bwd}));
  if (P->groups > 1) {
    P->ws_fwd = P->ws_dgrad = P->ws_wgrad = P->ws_bwd = (size_t)P->groups * P->ws_group;
  }
  if (cur != device) cudaSetDevice(cur);
  P->plan_us = std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - t0).count();
  *out = P;
  return GLP_OK;
}

glp_status_t glp_plan_get_info(glp_plan_t P, glp_plan_info_t *I) {
  if (!P || !I) return fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  memset(I, 0, sizeof(*I));
  I->samples_in_flight = P->S;
  I->ctas_per_sm = P->fwd.ctas_per_sm;
  I->grid_fwd = P->fwd.grid;
  I->grid_bwd_data = P->dgrad.grid;
  I->grid_bwd_filter = P->halo ? P->hw_grid : P->wgrad.grid;
  I->tile_m = 128;
  I->tile_n_fwd = P->fwd.bn;
  I->tile_n_bwd_data = P->dgrad.bn;
  I->tile_n_bwd_filter = P->halo ? P->hw.bn : P->wgrad.bn;
  I->stages_fwd = P->fwd.stages;
  I->stages_bwd_data = P->dgrad.stages;
  I->stages_bwd_filter = P->halo ? P->hw.stages : P->wgrad.stages;
  I->splits_wgrad = P->simt ? P->simt_splits : P->halo ? P->hw.splits : P->wgrad.splits;
  I->tiles_fwd = P->fwd.tiles;
  I->tiles_bwd_data = P->dgrad.tiles;
  I->tiles_bwd_filter = P->halo ? P->hw.splits : P->wgrad.tiles;
  I->ws_fwd = P->ws_fwd;
  I->ws_bwd_data = P->ws_dgrad;
  I->ws_bwd_filter = P->ws_wgrad;
  I->ws_bwd = P->ws_bwd;
  I->plan_us = P->plan_us;
  I->math = P->math;
  I->wgrad_halo = P->halo;
  I->fwd_halo = P->hfwd;
  I->wgrad_fused_dy = P->halo_fdy ? 1 : 0;
  I->dgrad_halo = P->hdg;
  I->s_slot_rows = P->s_slot_rows;
  I->s_rows_per_sample = P->s_rows_per_sample;
  I->wgrad_reduce_wide = P->red_wide;
  I->fp32_split = P->mix;
  I->dgrad_s2d = P->s2d_dg;
  if (P->hdg) {
    I->grid_bwd_data = P->hd_grid;
    I->tile_n_bwd_data = P->hd.bn;
    I->stages_bwd_data = P->hd.b_stages;
    I->tiles_bwd_data = P->hd.units;
  }
  if (P->hfwd) {
    I->grid_fwd = P->hf_grid;
    I->tile_n_fwd = P->hf.bn;
    I->stages_fwd = P->hf.stages;
    I->tiles_fwd = P->hf.units;
  }
  return GLP_OK;
}

glp_status_t glp_plan_kernel_attr(glp_plan_t P, int which, glp_kernel_attr_t *a, int *model, int *rt) {
  if (!P || !a || !model || !rt || which < 0 || which > 2) return fail(GLP_ERR_INVALID_VALUE, "bad argument");
  if (P->simt) return fail(GLP_ERR_NOT_SUPPORTED, "SIMT path has no persistent kernel");
  // the kernel the plan actually launches for the pass: a halo kernel where the plan chose one
  const KAttr *h = (which == 0 && P->hfwd) ? &P->hf_attr
                 : (which == 1 && P->hdg) ? &P->hd_attr
                 : (which == 2 && P->halo) ? &P->hw_attr : nullptr;
  if (h) {
    *a = glp_kernel_attr_t{h->threads, h->regs, h->smem, h->tmem};
    *model = h->model;
    *rt = h->rt;
    return GLP_OK;
  }
  const PassPlan &pp = which == 0 ? P->fwd : which == 1 ? P->dgrad : P->wgrad;
  *a = glp_kernel_attr_t{pp.threads, pp.regs, pp.smem, pp.tmem_cols};
  *model = pp.ctas_per_sm;
  *rt = pp.ctas_runtime;
  return GLP_OK;
}

glp_status_t glp_plan_destroy(glp_plan_t P) {
  delete P;
  return GLP_OK;
}

static glp_status_t check_ws(const glp_plan_s *P, const void *ws, size_t have, size_t need) {
  if (need == 0) return GLP_OK;
  if (!ws) return fail(GLP_ERR_INVALID_VALUE, "workspace is NULL");
  if (reinterpret_cast<uintptr_t>(ws) % 1024)
    return fail(GLP_ERR_INVALID_VALUE, "workspace must be 1024-byte aligned");
  if (have < need) return fail(GLP_ERR_WORKSPACE_TOO_SMALL, "workspace too small");
  (void)P;
  return GLP_OK;
}

// Pointer offsets of convolution group g (Caffe "group": x/dx channels [g*C_g, (g+1)*C_g),
// y/dy channels [g*C_o,g, ...), W rows [g*C_o,g, ...) of [C_o][C_g][K_h][K_w], one workspace
// slice per group).  groups = 1: all zero.
struct GOff {
  size_t x, y, w, b, ws;
};
static GOff goff(const glp_plan_s *P, int g) {
  const glp_conv_desc_s &d = P->d;   // the per-group convolution
  return GOff{(size_t)g * d.C * d.H * d.W, (size_t)g * d.Co * d.Ho * d.Wo,
              (size_t)g * d.Co * d.C * d.Kh * d.Kw, (size_t)g * d.Co, (size_t)g * P->ws_group};
}
static const float *offc(const float *p, size_t o) { return p ? p + o : p; }
static float *offm(float *p, size_t o) { return p ? p + o : p; }

glp_status_t glp_conv_fwd(glp_plan_t P, const float *x, const float *w, const float *b, float *y,
                          void *ws, size_t ws_bytes, glp_stream_t stream) {
  if (!P) return fail(GLP_ERR_INVALID_VALUE, "plan is NULL");
  glp_status_t s = validate_ptrs({x, w, y});
  if (s) return s;
  if (b && (reinterpret_cast<uintptr_t>(b) % 4)) return fail(GLP_ERR_INVALID_VALUE, "bias misaligned");
  if ((s = check_ws(P, ws, ws_bytes, P->ws_fwd))) return s;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (!P->simt && (s = get_encode())) return s;
  for (int g = 0; g < P->groups; ++g) {
    const GOff o = goff(P, g);
    float *yg = y + o.y;
    if (P->simt) {
      const size_t n = (size_t)P->d.N * P->d.Co * P->d.Ho * P->d.Wo;
      simt_fwd<<<ew_grid(n), 256, 0, st>>>(geomP(*P), x + o.x, w + o.w, offc(b, o.b), yg);
      GLP_LAUNCH_CHECK("simt_fwd");
    } else if ((s = tc_fwd(*P, x + o.x, br_in1(w + o.w), br_in1(offc(b, o.b)), br_out(*P, 1, &yg),
                           static_cast<uint8_t *>(ws) + o.ws, st))) {
      return s;
    }
  }
  return GLP_OK;
}

glp_status_t glp_conv_bwd_data(glp_plan_t P, const float *dy, const float *w, float *dx, void *ws,
                               size_t ws_bytes, glp_stream_t stream) {
  if (!P) return fail(GLP_ERR_INVALID_VALUE, "plan is NULL");
  glp_status_t s = validate_ptrs({dy, w, dx});
  if (s) return s;
  if ((s = check_ws(P, ws, ws_bytes, P->ws_dgrad))) return s;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (!P->simt && (s = get_encode())) return s;
  for (int g = 0; g < P->groups; ++g) {
    const GOff o = goff(P, g);
    if (P->simt) {
      const size_t n = (size_t)P->d.N * P->d.C * P->d.H * P->d.W;
      simt_dgrad<<<ew_grid(n), 256, 0, st>>>(geomP(*P), dy + o.y, w + o.w, dx + o.x);
      GLP_LAUNCH_CHECK("simt_dgrad");
      continue;
    }
    uint8_t *wsb = static_cast<uint8_t *>(ws) + o.ws;
    if ((s = launch_pack_dy(*P, br_in1(dy + o.y), wsb, false, st)) ||
        (s = run_pack_w_dgrad(*P, br_in1(w + o.w), wsb, st)) ||
        (s = run_dgrad_gemm(*P, dx + o.x, wsb, st)))
      return s;
  }
  return GLP_OK;
}

glp_status_t glp_conv_bwd_filter(glp_plan_t P, const float *x, const float *dy, float *dw, float *db,
                                 int accumulate, void *ws, size_t ws_bytes, glp_stream_t stream) {
  if (!P) return fail(GLP_ERR_INVALID_VALUE, "plan is NULL");
  glp_status_t s = validate_ptrs({x, dy, dw});
  if (s) return s;
  if (db && (reinterpret_cast<uintptr_t>(db) % 4)) return fail(GLP_ERR_INVALID_VALUE, "db misaligned");
  if ((s = check_ws(P, ws, ws_bytes, P->ws_wgrad))) return s;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (!P->simt && (s = get_encode())) return s;
  for (int g = 0; g < P->groups; ++g) {
    const GOff o = goff(P, g);
    uint8_t *wsb = static_cast<uint8_t *>(ws) + o.ws;
    float *dwg = dw + o.w, *dbg = offm(db, o.b);
    if (P->simt) {
      if ((s = run_wgrad_simt(*P, x + o.x, dy + o.y, dwg, dbg, accumulate ? 1 : 0, wsb, st))) return s;
      continue;
    }
    const BrOut dbt = br_out(*P, 1, &dbg);
    if ((s = launch_pack_x(*P, x + o.x, wsb + P->off_xpk, st)) ||
        (!P->halo_fdy && (s = launch_pack_dy(*P, br_in1(dy + o.y), wsb, db != nullptr, st))) ||
        (s = run_wgrad_gemm(*P, wsb, st, dy + o.y)) ||
        (s = run_wgrad_reduce(*P, br_out(*P, 1, &dwg), db ? &dbt : nullptr, accumulate ? 1 : 0, wsb, st)))
      return s;
  }
  return GLP_OK;
}

glp_status_t glp_conv_bwd(glp_plan_t P, const float *x, const float *dy, const float *w, float *dx,
                          float *dw, float *db, int accumulate, void *ws, size_t ws_bytes,
                          glp_stream_t stream) {
  if (!P) return fail(GLP_ERR_INVALID_VALUE, "plan is NULL");
  glp_status_t s = validate_ptrs({x, dy, w, dw});
  if (s) return s;
  if (dx && (reinterpret_cast<uintptr_t>(dx) % 16)) return fail(GLP_ERR_INVALID_VALUE, "dx misaligned");
  if (db && (reinterpret_cast<uintptr_t>(db) % 4)) return fail(GLP_ERR_INVALID_VALUE, "db misaligned");
  if ((s = check_ws(P, ws, ws_bytes, P->ws_bwd))) return s;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (!P->simt && (s = get_encode())) return s;
  for (int g = 0; g < P->groups; ++g) {
    const GOff o = goff(P, g);
    uint8_t *wsb = static_cast<uint8_t *>(ws) + o.ws;
    float *dwg = dw + o.w, *dbg = offm(db, o.b);
    if (P->simt) {
      if (dx) {
        const size_t n = (size_t)P->d.N * P->d.C * P->d.H * P->d.W;
        simt_dgrad<<<ew_grid(n), 256, 0, st>>>(geomP(*P), dy + o.y, w + o.w, dx + o.x);
        GLP_LAUNCH_CHECK("simt_dgrad");
      }
      if ((s = run_wgrad_simt(*P, x + o.x, dy + o.y, dwg, dbg, accumulate ? 1 : 0, wsb, st))) return s;
      continue;
    }
    if ((s = tc_bwd(*P, x + o.x, br_in1(dy + o.y), br_in1(w + o.w), offm(dx, o.x),
                    br_out(*P, 1, &dwg), db ? br_out(*P, 1, &dbg) : BrOut{}, db != nullptr,
                    accumulate ? 1 : 0, wsb, st)))
      return s;
  }
  return GLP_OK;
}

static glp_status_t stage_check(glp_plan_t P, void *ws, size_t ws_bytes) {
  if (!P) return fail(GLP_ERR_INVALID_VALUE, "plan is NULL");
  if (P->simt) return fail(GLP_ERR_NOT_SUPPORTED, "staged API needs a tensor-core plan");
  glp_status_t s = check_ws(P, ws, ws_bytes, P->ws_bwd);
  if (s) return s;
  return get_encode();
}

glp_status_t glp_stage_pack(glp_plan_t P, glp_pack_t what, const float *src, void *ws,
                            size_t ws_bytes, glp_stream_t stream) {
  glp_status_t s = stage_check(P, ws, ws_bytes);
  if (s) return s;
  if ((s = validate_ptrs({src}))) return s;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (what < GLP_PACK_X || what > GLP_PACK_W_BOTH) return fail(GLP_ERR_INVALID_VALUE, "unknown pack kind");
  for (int g = 0; g < P->groups; ++g) {
    const GOff o = goff(P, g);
    uint8_t *wsb = static_cast<uint8_t *>(ws) + o.ws;
    switch (what) {
      case GLP_PACK_X: s = launch_pack_x(*P, src + o.x, wsb + P->off_xpk, st); break;
      case GLP_PACK_DY:
      case GLP_PACK_DY_DB:
        if (P->halo_fdy)   // recorded only: the filter gradient reads it, bwd_data packs it
          record_dy(*P, wsb, src + o.y);
        else
          s = launch_pack_dy(*P, br_in1(src + o.y), wsb, what == GLP_PACK_DY_DB, st);
        break;
      case GLP_PACK_W_FWD: s = run_pack_w_fwd(*P, br_in1(src + o.w), wsb, st); break;
      case GLP_PACK_W_BWD_DATA: s = run_pack_w_dgrad(*P, br_in1(src + o.w), wsb, st); break;
      case GLP_PACK_W_BOTH: s = run_pack_w_both(*P, br_in1(src + o.w), wsb, st); break;
    }
    if (s) return s;
  }
  return GLP_OK;
}

glp_status_t glp_stage_fwd(glp_plan_t P, const float *b, float *y, void *ws, size_t ws_bytes,
                           glp_stream_t stream) {
  glp_status_t s = stage_check(P, ws, ws_bytes);
  if (s) return s;
  if ((s = validate_ptrs({y}))) return s;
  for (int g = 0; g < P->groups; ++g) {
    const GOff o = goff(P, g);
    float *yg = y + o.y;
    if ((s = run_fwd_gemm(*P, br_in1(offc(b, o.b)), br_out(*P, 1, &yg), static_cast<uint8_t *>(ws) + o.ws,
                          static_cast<cudaStream_t>(stream))))
      return s;
  }
  return GLP_OK;
}

glp_status_t glp_stage_bwd_data(glp_plan_t P, float *dx, void *ws, size_t ws_bytes,
                                glp_stream_t stream) {
  glp_status_t s = stage_check(P, ws, ws_bytes);
  if (s) return s;
  if ((s = validate_ptrs({dx}))) return s;
  for (int g = 0; g < P->groups; ++g) {
    const GOff o = goff(P, g);
    uint8_t *wsb = static_cast<uint8_t *>(ws) + o.ws;
    if (P->halo_fdy) {   // dy was only recorded by glp_stage_pack: pack it now for dgrad
      const float *dy = recorded_dy(*P, wsb);
      if (!dy) return fail(GLP_ERR_INVALID_VALUE, "bwd_data: glp_stage_pack(GLP_PACK_DY*) first");
      if ((s = launch_pack_dy(*P, br_in1(dy), wsb, false, static_cast<cudaStream_t>(stream))))
        return s;
    }
    if ((s = run_dgrad_gemm(*P, dx + o.x, wsb, static_cast<cudaStream_t>(stream))))
      return s;
  }
  return GLP_OK;
}

glp_status_t glp_stage_bwd_filter(glp_plan_t P, void *ws, size_t ws_bytes, glp_stream_t stream) {
  glp_status_t s = stage_check(P, ws, ws_bytes);
  if (s) return s;
  for (int g = 0; g < P->groups; ++g) {
    uint8_t *wsb = static_cast<uint8_t *>(ws) + goff(P, g).ws;
    if ((s = run_wgrad_gemm(*P, wsb, static_cast<cudaStream_t>(stream),
                            P->halo_fdy ? recorded_dy(*P, wsb) : nullptr)))
      return s;
  }
  return GLP_OK;
}

glp_status_t glp_stage_reduce(glp_plan_t P, float *dw, float *db, int accumulate, void *ws,
                              size_t ws_bytes, glp_stream_t stream) {
  glp_status_t s = stage_check(P, ws, ws_bytes);
  if (s) return s;
  if ((s = validate_ptrs({dw}))) return s;
  for (int g = 0; g < P->groups; ++g) {
    const GOff o = goff(P, g);
    float *dwg = dw + o.w, *dbg = offm(db, o.b);
    const BrOut dbt = br_out(*P, 1, &dbg);
    if ((s = run_wgrad_reduce(*P, br_out(*P, 1, &dwg), db ? &dbt : nullptr, accumulate ? 1 : 0,
                              static_cast<uint8_t *>(ws) + o.ws, static_cast<cudaStream_t>(stream))))
      return s;
  }
  return GLP_OK;
}

// ---- fused sibling groups ----
static glp_status_t group_tables(glp_plan_t P, const float *const *in, BrIn &t, bool allow_null_entries) {
  t.n = P->d.nbr;
  for (int b = 0; b < t.n; ++b) {
    t.p[b] = in ? in[b] : nullptr;
    if (!allow_null_entries && !t.p[b]) return fail(GLP_ERR_INVALID_VALUE, "NULL branch tensor");
    if (t.p[b] && reinterpret_cast<uintptr_t>(t.p[b]) % 4) return fail(GLP_ERR_INVALID_VALUE, "misaligned branch tensor");
  }
  return GLP_OK;
}
static glp_status_t group_check(glp_plan_t P, void *ws, size_t ws_bytes, size_t need) {
  if (!P) return fail(GLP_ERR_INVALID_VALUE, "plan is NULL");
  if (P->simt) return fail(GLP_ERR_NOT_SUPPORTED, "fused groups need a tensor-core plan");
  glp_status_t s = check_ws(P, ws, ws_bytes, need);
  if (s) return s;
  return get_encode();
}
static BrOut group_out(glp_plan_t P, float *const *p) {
  float *q[GLP_MAXBR] = {nullptr, nullptr, nullptr, nullptr};
  for (int b = 0; b < P->d.nbr; ++b) q[b] = p[b];
  return br_out(*P, P->d.nbr, q);
}

glp_status_t glp_conv_group_fwd(glp_plan_t P, const float *x, const float *const *w,
                                const float *const *b, float *const *y, void *ws, size_t ws_bytes,
                                glp_stream_t stream) {
  glp_status_t s = group_check(P, ws, ws_bytes, P ? P->ws_fwd : 0);
  if (s) return s;
  if (!w || !y || (s = validate_ptrs({x}))) return s ? s : fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  BrIn wt, bt, yt;
  if ((s = group_tables(P, w, wt, false)) || (s = group_tables(P, b, bt, true)) ||
      (s = group_tables(P, y, yt, false)))
    return s;
  return tc_fwd(*P, x, wt, bt, group_out(P, y), static_cast<uint8_t *>(ws),
                static_cast<cudaStream_t>(stream));
}

glp_status_t glp_conv_group_bwd(glp_plan_t P, const float *x, const float *const *dy,
                                const float *const *w, float *dx, float *const *dw,
                                float *const *db, int accumulate, void *ws, size_t ws_bytes,
                                glp_stream_t stream) {
  glp_status_t s = group_check(P, ws, ws_bytes, P ? P->ws_bwd : 0);
  if (s) return s;
  if (!dy || !w || !dw || (s = validate_ptrs({x}))) return s ? s : fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  if (dx && (reinterpret_cast<uintptr_t>(dx) % 16)) return fail(GLP_ERR_INVALID_VALUE, "dx misaligned");
  BrIn dyt, wt, dwt, dbt;
  if ((s = group_tables(P, dy, dyt, false)) || (s = group_tables(P, w, wt, false)) ||
      (s = group_tables(P, reinterpret_cast<const float *const *>(dw), dwt, false)) ||
      (db && (s = group_tables(P, reinterpret_cast<const float *const *>(db), dbt, false))))
    return s;
  return tc_bwd(*P, x, dyt, wt, dx, group_out(P, dw), db ? group_out(P, db) : BrOut{}, db != nullptr,
                accumulate ? 1 : 0, static_cast<uint8_t *>(ws), static_cast<cudaStream_t>(stream));
}

glp_status_t glp_stage_pack_group(glp_plan_t P, glp_pack_t what, const float *const *src, void *ws,
                                  size_t ws_bytes, glp_stream_t stream) {
  glp_status_t s = stage_check(P, ws, ws_bytes);
  if (s) return s;
  if (!src) return fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  uint8_t *wsb = static_cast<uint8_t *>(ws);
  if (what == GLP_PACK_X) {
    if ((s = validate_ptrs({src[0]}))) return s;
    return launch_pack_x(*P, src[0], wsb + P->off_xpk, st);
  }
  BrIn t;
  if ((s = group_tables(P, src, t, false))) return s;
  switch (what) {
    case GLP_PACK_DY: return launch_pack_dy(*P, t, wsb, false, st);
    case GLP_PACK_DY_DB: return launch_pack_dy(*P, t, wsb, true, st);
    case GLP_PACK_W_FWD: return run_pack_w_fwd(*P, t, wsb, st);
    case GLP_PACK_W_BWD_DATA: return run_pack_w_dgrad(*P, t, wsb, st);
    case GLP_PACK_W_BOTH: return run_pack_w_both(*P, t, wsb, st);
    default: break;
  }
  return fail(GLP_ERR_INVALID_VALUE, "unknown pack kind");
}

glp_status_t glp_stage_fwd_group(glp_plan_t P, const float *const *b, float *const *y, void *ws,
                                 size_t ws_bytes, glp_stream_t stream) {
  glp_status_t s = stage_check(P, ws, ws_bytes);
  if (s) return s;
  if (!y) return fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  BrIn bt, yt;
  if ((s = group_tables(P, b, bt, true)) || (s = group_tables(P, y, yt, false))) return s;
  return run_fwd_gemm(*P, bt, group_out(P, y), static_cast<uint8_t *>(ws),
                      static_cast<cudaStream_t>(stream));
}

glp_status_t glp_stage_reduce_group(glp_plan_t P, float *const *dw, float *const *db, int accumulate,
                                    void *ws, size_t ws_bytes, glp_stream_t stream) {
  glp_status_t s = stage_check(P, ws, ws_bytes);
  if (s) return s;
  if (!dw) return fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  BrIn dwt, dbt;
  if ((s = group_tables(P, reinterpret_cast<const float *const *>(dw), dwt, false)) ||
      (db && (s = group_tables(P, reinterpret_cast<const float *const *>(db), dbt, false))))
    return s;
  const BrOut dbo = db ? group_out(P, db) : BrOut{};
  return run_wgrad_reduce(*P, group_out(P, dw), db ? &dbo : nullptr, accumulate ? 1 : 0,
                          static_cast<uint8_t *>(ws), static_cast<cudaStream_t>(stream));
}

glp_status_t glp_debug_im2col(glp_plan_t P, const float *x, int n, float *col, void *ws,
                              size_t ws_bytes, glp_stream_t stream) {
  if (!P) return fail(GLP_ERR_INVALID_VALUE, "plan is NULL");
  glp_status_t s = validate_ptrs({x, col});
  if (s) return s;
  if (n < 0 || n >= P->d.N) return fail(GLP_ERR_INVALID_VALUE, "sample index out of range");
  if (P->groups > 1) return fail(GLP_ERR_NOT_SUPPORTED, "debug im2col of a grouped layer");
  if (P->simt) return fail(GLP_ERR_NOT_SUPPORTED, "SIMT path has no packed operand");
  if ((s = check_ws(P, ws, ws_bytes, P->ws_fwd))) return s;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  uint8_t *wsb = static_cast<uint8_t *>(ws);
  void *xpk = wsb + P->off_xpk;
  if ((s = launch_pack_act(*P, x, xpk, plo(*P, P->lo_xpk), P->d.C, P->d.H * P->d.W, P->Cp, nullptr, st)))
    return s;
  // the direct (non space-to-depth) gather geometry of the layer
  glp_plan_s Q = *P;
  Q.s2d = 0;
  Q.dxg = Q.d;
  Q.Cpx = Q.Cp;
  Q.tapsx = Q.taps;
  IgemmParams p = make_params(Q, Q.fwd, MODE_FWD, xpk);
  const size_t total = (size_t)P->d.C * P->taps * P->d.Ho * P->d.Wo;
  if (P->elem == 2)
    debug_im2col_kernel<2><<<ew_grid(total), 256, 0, st>>>(p.g, n, P->d.C, P->d.Kh, P->d.Kw, P->d.Ho, P->d.Wo, col);
  else
    debug_im2col_kernel<4><<<ew_grid(total), 256, 0, st>>>(p.g, n, P->d.C, P->d.Kh, P->d.Kw, P->d.Ho, P->d.Wo, col);
  GLP_LAUNCH_CHECK("debug_im2col_kernel");
  return GLP_OK;
}

// ---- deterministic gradient exchange: the tree's add step ----
glp_status_t glp_sum2(const float *a, const float *b, float *out, size_t n, glp_stream_t stream) {
  if (n == 0) return GLP_OK;
  if (!a || !b || !out) return fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  sum2_kernel<<<ew_grid(n), 256, 0, st>>>(a, b, out, n);
  GLP_LAUNCH_CHECK("sum2_kernel");
  return GLP_OK;
}

glp_status_t glp_tree_sum(const float *const *parts, int n, float *out, size_t count,
                          int accumulate, glp_stream_t stream) {
  if (!parts || !out) return fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  for (int k = 0; k < n && k < 8; ++k)
    if (!parts[k]) return fail(GLP_ERR_INVALID_VALUE, "NULL tree operand");
  return run_tree(parts, n, out, count, accumulate ? 1 : 0, static_cast<cudaStream_t>(stream));
}

glp_status_t glp_tree_exchange(const float *const *subtrees, float *const *outs, int world, int rank,
                               size_t count, glp_stream_t stream) {
  if (!subtrees || !outs) return fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  if (world < 1 || world > 8 || (world & (world - 1)) || rank < 0 || rank >= world)
    return fail(GLP_ERR_INVALID_VALUE, "world must be 1, 2, 4 or 8 and 0 <= rank < world");
  Ptr8 a{};
  MPtr8 b{};
  for (int k = 0; k < world; ++k) {
    if (!subtrees[k] || !outs[k]) return fail(GLP_ERR_INVALID_VALUE, "NULL peer pointer");
    a.p[k] = subtrees[k];
    b.p[k] = outs[k];
  }
  if (count == 0) return GLP_OK;
  const size_t mine = count / world + 1;
  tree_exchange_kernel<<<ew_grid(mine), 256, 0, static_cast<cudaStream_t>(stream)>>>(a, b, world, rank, count);
  GLP_LAUNCH_CHECK("tree_exchange_kernel");
  return GLP_OK;
}

glp_status_t glp_stage_reduce_leaves(glp_plan_t P, float *dw, float *db, size_t leaf_stride,
                                     void *ws, size_t ws_bytes, glp_stream_t stream) {
  glp_status_t s = stage_check(P, ws, ws_bytes);
  if (s) return s;
  if ((s = validate_ptrs({dw}))) return s;
  if (P->leaves < 2 && leaf_stride == 0) leaf_stride = 1;   // one leaf: the stride is unused
  if (leaf_stride == 0 || leaf_stride % 4)
    return fail(GLP_ERR_INVALID_VALUE, "leaf_stride must be a positive multiple of 4 floats");
  if (P->groups > 1) return fail(GLP_ERR_NOT_SUPPORTED, "leaf reduction of a grouped layer");
  float *dwp = dw;
  const BrOut dbt = br_out(*P, 1, &db);
  return run_wgrad_reduce(*P, br_out(*P, 1, &dwp), db ? &dbt : nullptr, 0, static_cast<uint8_t *>(ws),
                          static_cast<cudaStream_t>(stream), (long long)leaf_stride);
}

// ---- prior-art comparator: the paper's per-sample stream pool ----
}  // extern "C"

struct glp_pool_s {
  glp_conv_desc_s d1;            // the per-sample (N = 1) layer
  glp_plan_t plan1 = nullptr;    // its plan (shared by every stream: plans are immutable)
  int N = 0, device = 0, math = 0, S = 1, eq7 = 1;
  int eq7_launch = 0;           // Eq. 7 bound with the measured T_K / T_launch term (0: not set)
  int n_streams_req = 0, cap = 1;  // caller's pool size (0 = the Eq. 7 bound); streams created
  glp_kernel_attr_t ka{};       // the per-sample forward kernel's record (Eq. 7 input)
  int blocks = 1;
  double t_kernel = 0, t_launch = 0;
  size_t slot_ws = 0, acc_floats = 0, ws_bytes = 0;
  std::vector<cudaStream_t> streams;
  std::vector<cudaEvent_t> joins;
  cudaEvent_t fork = nullptr;
};

namespace {
glp_status_t pool_fork(glp_pool_s *Q, cudaStream_t st) {
  GLP_CUDA(cudaEventRecord(Q->fork, st));
  for (int s = 0; s < Q->S; ++s) GLP_CUDA(cudaStreamWaitEvent(Q->streams[s], Q->fork, 0));
  return GLP_OK;
}
glp_status_t pool_join(glp_pool_s *Q, cudaStream_t st) {
  for (int s = 0; s < Q->S; ++s) {
    GLP_CUDA(cudaEventRecord(Q->joins[s], Q->streams[s]));
    GLP_CUDA(cudaStreamWaitEvent(st, Q->joins[s], 0));
  }
  return GLP_OK;
}
}  // namespace

extern "C" {

glp_status_t glp_pool_create(glp_pool_t *out, glp_conv_desc_t d, int device, glp_math_t math,
                             int n_streams) {
  if (!out || !d) return fail(GLP_ERR_INVALID_VALUE, "NULL argument");
  *out = nullptr;
  if (n_streams < 0) return fail(GLP_ERR_INVALID_VALUE, "n_streams < 0");
  if (d->nbr > 1 || d->groups > 1)
    return fail(GLP_ERR_NOT_SUPPORTED, "the stream pool runs single ungrouped layers");
  auto *Q = new glp_pool_s();
  Q->d1 = *d;
  Q->d1.N = 1;
  Q->N = d->N;
  Q->device = device;
  Q->math = (int)math;
  glp_status_t s = glp_plan(&Q->plan1, &Q->d1, device, math, 0);
  if (s) {
    delete Q;
    return s;
  }
  // Eq. 7 (P245): how many instances of the per-sample forward kernel fit the device at once
  // (thread and shared-memory terms; no launch term, R17), capped by the concurrent-kernel
  // limit C (Eq. 6).  FP32 plans: their per-sample kernel is the SIMT forward (256 threads).
  glp_device_limits_t L;
  glp_device_limits_b200(&L);
  glp_kernel_attr_t ka{256, 0, 0, 0};
  int blocks = (int)std::max<long long>(1, cdiv((long long)Q->d1.Co * Q->d1.Ho * Q->d1.Wo, 256));
  if (math != GLP_MATH_FP32_SIMT) {
    int m = 0, r = 0;
    glp_plan_kernel_attr(Q->plan1, 0, &ka, &m, &r);
    blocks = Q->plan1->hfwd ? Q->plan1->hf_grid : Q->plan1->fwd.grid;
  }
  Q->ka = ka;
  Q->blocks = blocks;
  int bound = 1;
  glp_analyze_eq7(&L, &ka, blocks, 0.0, 0.0, &bound);
  Q->eq7 = std::max(1, std::min(bound, L.max_concurrent_kernels));
  Q->n_streams_req = n_streams;
  Q->cap = std::max(1, std::min(Q->N, 64));
  Q->S = std::max(1, std::min(n_streams > 0 ? n_streams : Q->eq7, Q->cap));
  Q->slot_ws = align1k(std::max<size_t>(Q->plan1->ws_bwd, 1));
  Q->acc_floats = (size_t)rup((long long)d->Co * d->C * d->Kh * d->Kw + d->Co, 64);
  Q->ws_bytes = (size_t)Q->S * Q->slot_ws + align1k((size_t)Q->S * Q->acc_floats * 4);
  int cur = 0;
  cudaGetDevice(&cur);
  if (cur != device) cudaSetDevice(device);
  for (int i = 0; i < Q->cap; ++i) {   // every stream the pool may use after a recalibration
    cudaStream_t st;
    cudaEvent_t ev;
    if (cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess) {
      glp_pool_destroy(Q);
      if (cur != device) cudaSetDevice(cur);
      return fail(GLP_ERR_CUDA, "stream pool creation failed");
    }
    Q->streams.push_back(st);
    Q->joins.push_back(ev);
  }
  cudaEventCreateWithFlags(&Q->fork, cudaEventDisableTiming);
  if (cur != device) cudaSetDevice(cur);
  *out = Q;
  return GLP_OK;
}

glp_status_t glp_pool_set_launch_term(glp_pool_t Q, double t_kernel_us, double t_launch_us) {
  if (!Q || !(t_kernel_us > 0) || !(t_launch_us > 0))
    return fail(GLP_ERR_INVALID_VALUE, "T_K and T_launch must be positive");
  glp_device_limits_t L;
  glp_device_limits_b200(&L);
  int bound = 1;
  glp_status_t s = glp_analyze_eq7(&L, &Q->ka, Q->blocks, t_kernel_us, t_launch_us, &bound);
  if (s) return s;
  Q->t_kernel = t_kernel_us;
  Q->t_launch = t_launch_us;
  Q->eq7_launch = std::max(1, std::min(bound, L.max_concurrent_kernels));
  Q->S = std::max(1, std::min(Q->n_streams_req > 0 ? Q->n_streams_req : Q->eq7_launch, Q->cap));
  Q->ws_bytes = (size_t)Q->S * Q->slot_ws + align1k((size_t)Q->S * Q->acc_floats * 4);
  return GLP_OK;
}

glp_status_t glp_pool_get_eq7(glp_pool_t Q, int *without_launch_term, int *with_launch_term) {
  if (!Q) return fail(GLP_ERR_INVALID_VALUE, "pool is NULL");
  if (without_launch_term) *without_launch_term = Q->eq7;
  if (with_launch_term) *with_launch_term = Q->eq7_launch;
  return GLP_OK;
}

glp_status_t glp_pool_get_info(glp_pool_t Q, int *n_streams, int *eq7_bound, size_t *ws_bytes) {
  if (!Q) return fail(GLP_ERR_INVALID_VALUE, "pool is NULL");
  if (n_streams) *n_streams = Q->S;
  if (eq7_bound) *eq7_bound = Q->eq7;
  if (ws_bytes) *ws_bytes = Q->ws_bytes;
  return GLP_OK;
}

glp_status_t glp_pool_destroy(glp_pool_t Q) {
  if (!Q) return GLP_OK;
  for (auto st : Q->streams) cudaStreamDestroy(st);
  for (auto ev : Q->joins) cudaEventDestroy(ev);
  if (Q->fork) cudaEventDestroy(Q->fork);
  if (Q->plan1) glp_plan_destroy(Q->plan1);
  delete Q;
  return GLP_OK;
}

glp_status_t glp_pool_conv_fwd(glp_pool_t Q, const float *x, const float *w, const float *b,
                               float *y, void *ws, size_t ws_bytes, glp_stream_t stream) {
  if (!Q) return fail(GLP_ERR_INVALID_VALUE, "pool is NULL");
  glp_status_t s = validate_ptrs({x, w, y});
  if (s) return s;
  if ((s = check_ws(Q->plan1, ws, ws_bytes, Q->ws_bytes))) return s;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  uint8_t *wsb = static_cast<uint8_t *>(ws);
  const glp_conv_desc_s &d = Q->d1;
  const size_t xs = (size_t)d.C * d.H * d.W, ys = (size_t)d.Co * d.Ho * d.Wo;
  const bool tc = Q->math != GLP_MATH_FP32_SIMT;
  if ((s = pool_fork(Q, st))) return s;
  // internal calls: per-sample slices are only 4-byte aligned (e.g. 3 x 227 x 227 floats)
  glp_plan_s &P1 = *Q->plan1;
  if (tc) {
    if ((s = get_encode())) return s;
    for (int i = 0; i < Q->S; ++i)   // each stream's workspace holds its own packed weights
      if ((s = run_pack_w_fwd(P1, br_in1(w), wsb + i * Q->slot_ws, Q->streams[i]))) return s;
  }
  for (int n = 0; n < Q->N; ++n) {   // round-robin dispatch of per-sample kernels (P171)
    const int i = n % Q->S;
    uint8_t *wsi = wsb + i * Q->slot_ws;
    cudaStream_t si = Q->streams[i];
    float *yn = y + n * ys;
    if (tc) {
      if ((s = launch_pack_x(P1, x + n * xs, wsi + P1.off_xpk, si)) ||
          (s = run_fwd_gemm(P1, br_in1(b), br_out(P1, 1, &yn), wsi, si)))
        return s;
    } else {
      simt_fwd<<<ew_grid(ys), 256, 0, si>>>(geomP(P1), x + n * xs, w, b, yn);
      GLP_LAUNCH_CHECK("simt_fwd");
    }
  }
  return pool_join(Q, st);
}

glp_status_t glp_pool_conv_bwd(glp_pool_t Q, const float *x, const float *dy, const float *w,
                               float *dx, float *dw, float *db, void *ws, size_t ws_bytes,
                               glp_stream_t stream) {
  if (!Q) return fail(GLP_ERR_INVALID_VALUE, "pool is NULL");
  glp_status_t s = validate_ptrs({x, dy, w, dw});
  if (s) return s;
  if ((s = check_ws(Q->plan1, ws, ws_bytes, Q->ws_bytes))) return s;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  uint8_t *wsb = static_cast<uint8_t *>(ws);
  const glp_conv_desc_s &d = Q->d1;
  const size_t xs = (size_t)d.C * d.H * d.W, ys = (size_t)d.Co * d.Ho * d.Wo;
  const size_t wsz = (size_t)d.Co * d.C * d.Kh * d.Kw;
  float *acc = reinterpret_cast<float *>(wsb + (size_t)Q->S * Q->slot_ws);
  const bool tc = Q->math != GLP_MATH_FP32_SIMT;
  if ((s = pool_fork(Q, st))) return s;
  // The paper's concurrent streams would all accumulate (beta = 1) into one dW and race
  // (P262-264); each stream here owns an accumulator, summed in stream order at the join.
  glp_plan_s &P1 = *Q->plan1;
  if (tc && (s = get_encode())) return s;
  for (int i = 0; i < Q->S; ++i) {
    GLP_CUDA(cudaMemsetAsync(acc + i * Q->acc_floats, 0, Q->acc_floats * 4, Q->streams[i]));
    if (tc && dx && (s = run_pack_w_dgrad(P1, br_in1(w), wsb + i * Q->slot_ws, Q->streams[i])))
      return s;
  }
  for (int n = 0; n < Q->N; ++n) {
    const int i = n % Q->S;
    uint8_t *wsi = wsb + i * Q->slot_ws;
    float *dwi = acc + i * Q->acc_floats, *dbi = db ? dwi + wsz : nullptr;
    cudaStream_t si = Q->streams[i];
    const float *xn = x + n * xs, *dyn = dy + n * ys;
    if (tc) {
      if ((!P1.halo_fdy || dx) && (s = launch_pack_dy(P1, br_in1(dyn), wsi, db != nullptr, si)))
        return s;
      if (dx && (s = run_dgrad_gemm(P1, dx + n * xs, wsi, si))) return s;
      const BrOut dbo = br_out(P1, 1, &dbi);
      if ((s = launch_pack_x(P1, xn, wsi + P1.off_xpk, si)) || (s = run_wgrad_gemm(P1, wsi, si, dyn)) ||
          (s = run_wgrad_reduce(P1, br_out(P1, 1, &dwi), db ? &dbo : nullptr, 1, wsi, si)))
        return s;
    } else {
      if (dx) {
        simt_dgrad<<<ew_grid(xs), 256, 0, si>>>(geomP(P1), dyn, w, dx + n * xs);
        GLP_LAUNCH_CHECK("simt_dgrad");
      }
      if ((s = run_wgrad_simt(P1, xn, dyn, dwi, dbi, 1, wsi, si))) return s;
    }
  }
  if ((s = pool_join(Q, st))) return s;
  pool_sum_slots<<<ew_grid(wsz), 256, 0, st>>>(acc, Q->acc_floats, Q->S, dw, wsz, 0);
  GLP_LAUNCH_CHECK("pool_sum_slots");
  if (db) {
    pool_sum_slots<<<ew_grid(d.Co), 256, 0, st>>>(acc + wsz, Q->acc_floats, Q->S, db, (size_t)d.Co, 0);
    GLP_LAUNCH_CHECK("pool_sum_slots");
  }
  return GLP_OK;
}

}  // extern "C"
