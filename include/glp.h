/*
 * glp.h — C ABI of the B200-native GLP4NN conv-layer training hot path (libglp.so).
 *
 * The calls follow the paper's problem statement (PAPER.md, "P<n>" = line n):
 *   - Alg. 1 forward propagation (P82-99): top = BLAS(weight, bias, bottom), for a conv layer
 *     im2col -> sgemm -> bias gemm (P173)                          -> glp_conv_fwd
 *   - Alg. 2 backward propagation (P101-121): bottom_gradient = BLAS(top_gradient, weight),
 *     i.e. GEMM W^T dy -> col2im                                  -> glp_conv_bwd_data
 *   - parameter gradients "for parameter update" (P129), summed over the samples of the batch
 *     (BASELINE.json north_star)                                   -> glp_conv_bwd_filter
 *   - layer parameters N, C_i, H, W, C_o, F_h, F_w, S, P (Table 5 definitions, P316)
 *                                                                  -> glp_conv_desc_create
 *   - the kernel analyzer (§3.1 P167, §3.2 Eqs 1-9 P214-254) re-derived for sm_100a; its output
 *     (the paper's C_out, P254) is the number of samples in flight S that sizes the persistent
 *     tile scheduler replacing the stream pool (P169-173)          -> glp_plan, glp_analyze_*
 *
 * Conventions (readings R1-R13):
 *   - x, y, dx, dy: NCHW fp32; W: [C_o][C_i][K_h][K_w] fp32; b, db: [C_o] fp32 (Caffe blobs, P87).
 *   - cross-correlation (no flip), zero padding, H_o = floor((H + 2P - K_h)/S) + 1, group = 1,
 *     dilation = 1.
 *   - N in the descriptor is the per-rank batch (multi-GPU sharding is the caller's, BJ.ns (4)).
 *
 * Ownership: the caller owns every tensor and the workspace (device pointers, e.g. from the
 * PyTorch caching allocator; 16-byte aligned).  The library owns only the opaque desc/plan
 * objects (create/destroy pairs).  A plan is bound to one device (P159: a private analyzer and
 * scheduler per GPU) and immutable after glp_plan; it may be used concurrently on different
 * streams with distinct workspaces.
 *
 * Errors: every call returns a status code; no exception or abort crosses the ABI.  Arguments
 * are validated before any launch (NULL, misalignment, non-positive dims, H_o < 1, workspace too
 * small).  GLP_ERR_CUDA reports a launch error; glp_last_error_string() gives its text.
 * Execution: all compute calls are asynchronous on the given stream; no host synchronisation
 * and no hidden device allocation.  There is no CPU fallback: without a usable sm_100 device
 * glp_plan fails with GLP_ERR_NOT_SUPPORTED.
 */
#ifndef GLP_H_
#define GLP_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  GLP_OK = 0,
  GLP_ERR_INVALID_VALUE = 1,
  GLP_ERR_NOT_SUPPORTED = 2,
  GLP_ERR_CUDA = 3,
  GLP_ERR_WORKSPACE_TOO_SMALL = 4,
  GLP_ERR_INTERNAL = 5
} glp_status_t;

typedef enum {
  /* fp32-accurate (normwise error <= 1e-5, the paper's FP32 sgemm arithmetic, P173/P314): 3xTF32
   * on tcgen05.  The packs split every operand v into hi = rna_tf32(v) and lo = rna_tf32(v - hi)
   * (two planes); each k-step issues hi*hi, hi*lo, lo*hi kind::tf32 MMAs, in that fixed order,
   * into one fp32 TMEM accumulator (SURVEY §8(c) "3xTF32 hi/lo split", §7.1 phase 9). */
  GLP_MATH_FP32 = 0,
  GLP_MATH_TF32 = 1, /* tcgen05 kind::tf32 (operands RNA-rounded in the pack), fp32 accumulate */
  GLP_MATH_BF16 = 2, /* tcgen05 kind::f16 with bf16 operands (RNE), fp32 accumulate           */
  /* fp32 CUDA-core direct convolution (one thread per output, fixed K order): the accuracy
   * anchor the tests compare the tensor-core modes with; no staged API, no fused groups. */
  GLP_MATH_FP32_SIMT = 3
} glp_math_t;

typedef struct glp_conv_desc_s *glp_conv_desc_t;
typedef struct glp_plan_s *glp_plan_t;
typedef void *glp_stream_t; /* a cudaStream_t (e.g. torch.cuda.Stream.cuda_stream); NULL = legacy */

/* Plan summary = the analyzer's inputs and outputs (Fig. 8 analog: S per layer). */
typedef struct {
  int samples_in_flight; /* S: the paper's C_out re-derived (P254) for the forward kernel      */
  int ctas_per_sm;       /* beta per SM of the forward kernel (Eq. 8 re-derived)                */
  int grid_fwd, grid_bwd_data, grid_bwd_filter; /* persistent grid sizes                        */
  int tile_m, tile_n_fwd, tile_n_bwd_data, tile_n_bwd_filter;
  int stages_fwd, stages_bwd_data, stages_bwd_filter;
  int splits_wgrad;      /* shape-only split count of the N*H_o*W_o reduction                   */
  int tiles_fwd, tiles_bwd_data, tiles_bwd_filter;
  size_t ws_fwd, ws_bwd_data, ws_bwd_filter, ws_bwd; /* workspace bytes per call               */
  double plan_us;        /* host time spent in glp_plan (Table 6 T_a analog)                   */
  int math;
  int wgrad_halo;        /* 1: filter gradient by the shared-halo kernel (space-to-depth layers;
                            dy packed on the padded grid), 0: im2col implicit GEMM             */
  int fwd_halo;          /* 1: forward by the shared-halo kernel (space-to-depth layers: x' staged
                            once per tile for all taps, outputs on the padded grid), 0: im2col   */
  int wgrad_fused_dy;    /* 1: the halo filter gradient builds its dy operand (and db) from the fp32
                            dy itself: glp_stage_pack(GLP_PACK_DY*) then only records the dy
                            pointer for this workspace (it must stay valid until the filter-gradient
                            and backward-data stages have run; the backward-data stage packs it) */
  int dgrad_halo;        /* 1: backward-data by the shared-halo kernel (unit stride: a 4-D TMA halo
                            of the packed dy per 64-channel block, tap operands by row shift)     */
  /* The analyzer's inputs for samples_in_flight, S = glp_analyze_samples_in_flight(s_slot_rows,
   * s_rows_per_sample, N): the forward kernel's resident GEMM rows (#SM x CTAs/SM of the kernel
   * glp_plan_kernel_attr(0) describes x 128) and the rows one sample occupies (H_o*W_o, or the
   * padded grid of the halo forward, x the N tiles). */
  long long s_slot_rows, s_rows_per_sample;
  int wgrad_reduce_wide; /* 1: the dW split reduction runs 4 weight rows x 8 split phases per block
                            (small filters: < 64 tiles of 32 x 32); 0: 32 x 32 tiles             */
  int fp32_split;        /* 1: this GLP_MATH_FP32 plan runs the mixed split (glp_plan_options_t)  */
  int dgrad_s2d;         /* 1: strided layer whose backward-data runs as the stride-1 backward-data
                            of its space-to-depth form (dx' over x', then scattered into dx);
                            ws_bwd_data then includes the dx' buffer (N*S*S*C_in*H'*W' floats)    */
} glp_plan_info_t;

/* Per-SM limits (Table 2 "device property", P183-193) plus the sm_100a-only ones. */
typedef struct {
  int sm_count;            /* #SM                                   */
  int max_threads_per_sm;  /* tau_max                               */
  int max_blocks_per_sm;   /* rho_max                               */
  int regs_per_sm;         /* hard limit on sm_100a (R16)           */
  int smem_per_sm;         /* sm_max (bytes)                        */
  int smem_reserved_per_cta;
  int tmem_cols_per_sm;    /* 512 on sm_100a                        */
  int max_concurrent_kernels; /* C (Eq. 6)                          */
} glp_device_limits_t;

/* Per-kernel record (Table 2 "profiling input", P194-200; D5). */
typedef struct {
  int threads;    /* tau_Ki              */
  int regs;       /* registers / thread  */
  int smem_bytes; /* sm_Ki (static + dynamic) */
  int tmem_cols;  /* TMEM columns / CTA  */
} glp_kernel_attr_t;

/* ---- descriptors (Table 5 parameters, P316) ------------------------------------------------ */
glp_status_t glp_conv_desc_create(glp_conv_desc_t *out, int N, int C_in, int H, int W, int C_out,
                                  int K_h, int K_w, int stride_h, int stride_w, int pad_h,
                                  int pad_w);
/* Caffe convolution groups (e.g. CaffeNet conv2/conv4/conv5 use 2, which
 * Table 5 does not list, R4): group g convolves x channels [g*C_in/G, (g+1)*C_in/G) with W rows
 * [g*C_out/G, (g+1)*C_out/G) of W [C_out][C_in/G][K_h][K_w] into the same y channels; dx, dW, db
 * likewise.  groups must divide C_in and C_out (GLP_ERR_INVALID_VALUE).  Set before glp_plan;
 * the plan covers one group's convolution and every call runs the groups in order, each with
 * its own workspace slice (info.ws_* include all groups).  Not combinable with fused sibling
 * groups, the stream pool or glp_debug_im2col (GLP_ERR_NOT_SUPPORTED). */
glp_status_t glp_conv_desc_set_groups(glp_conv_desc_t desc, int groups);
glp_status_t glp_conv_desc_get_output(glp_conv_desc_t desc, int *H_out, int *W_out);
glp_status_t glp_conv_desc_destroy(glp_conv_desc_t desc);

/* ---- plan: analyzer + scheduler setup, once per (shape, device, math) ("profile once", P173) -
 * samples_in_flight: 0 = analyzer's choice; > 0 = override (tests of convergence invariance,
 * P264: outputs must be bitwise identical for every S). */
glp_status_t glp_plan(glp_plan_t *out, glp_conv_desc_t desc, int device, glp_math_t math,
                      int samples_in_flight);
/* Plan options: choices between alternative kernels / tilings of the SAME computation.  Every
 * option value gives bitwise the same outputs as the default for a given (shape, math mode)
 * (the GEMMs have no K split but the wgrad one, whose split count and order are shape-only; each
 * alternative is tested for bitwise equality), so the options only move time.  They exist for
 * tests and A/B measurements; the library reads no environment variables (diagnostic builds,
 * -DGLP_DIAG, add work-skipping timing hooks and never ship).  glp_plan == glp_plan_ex with the
 * defaults of glp_plan_options_default. */
typedef struct {
  int cta_pairs;          /* 1: tcgen05 cta_group::2 CTA pairs where they apply; 0: single-CTA MMAs */
  int wgrad_cta_pairs;    /* 1: CTA pairs for the filter gradient too; 0: not                      */
  int halo_wgrad;         /* 1: shared-halo filter gradient for space-to-depth layers; 0: im2col   */
  int halo_fwd;           /* 1: shared-halo forward for space-to-depth layers; 0: im2col           */
  int halo_dgrad;         /* 1: shared-halo backward-data where the cost model picks it (bf16,
                             tf32); 0: never; 2: wherever legal (also the mixed fp32 split's
                             three-plane halo kernel, measured slower than im2col: opt-in only)    */
  int fused_dy;           /* 1: the halo filter gradient builds its dy operand from fp32 dy; 0: it
                             reads the packed dy                                                   */
  int fused_dy_builders;  /* 0: model; 1: cp.async landing zone; 2 or 3: register builder groups   */
  int max_kblocks_per_stage; /* 1..4 (k-blocks per pipeline stage cap; 4 = default)                */
  int wgrad_tile_n;       /* 0: model; else the filter-gradient N tile (multiple of 16, <= 256)    */
  int tile_units;         /* fwd/dgrad tile model applies below this many work units per slot (6)  */
  int bn_model;           /* 1: fwd/dgrad N-tile model for small grids; 0: always the default tile */
  int pack_block;         /* 0: warp-tiled activation pack; 1: block-tiled; 2 (default): block-
                             tiled for 4-byte operands (tf32, fp32 splits), warp-tiled for bf16  */
  int s2d_block;          /* 0: warp-per-32-pixel space-to-depth pack; 1: block-persistent          */
  int smem_cap;           /* dynamic shared memory budget of the persistent GEMMs, bytes (232448)  */
  int pdl;                /* 1: programmatic dependent launch between the plan's kernels; 0: not   */
  int wgrad_leaves;       /* 0 (default): no leaves.  1, 2, 4 or 8: a leaf plan -- the local batch
                             is this many equal leaves of the global batch's 8 (the deterministic
                             exchange, NEXT-2).  The filter gradient's splits are chosen for ONE
                             leaf (as if the 8 leaves shared the device) and never cross a leaf
                             boundary, so a leaf's partial is the same bits on any rank; the
                             composed calls and
                             glp_stage_reduce return the fixed tree (glp_tree_sum) over the leaves,
                             glp_stage_reduce_leaves the leaves themselves.  Needs N divisible by the
                             leaves and a leaf's N*H_o*W_o a multiple of the k-block (32 pixels
                             tf32 / fp32, 64 bf16); tensor-core single-layer plans (no fused
                             sibling groups).  Changes the split order, hence low bits, vs 1.      */
  int fp32_split;         /* GLP_MATH_FP32 on tensor cores: the mixed split -- hi*hi in tf32 plus
                             bf16(hi)*bf16(lo) and bf16(lo)*bf16(hi) in bf16 (8 instead of 12 MMA
                             issue slots per k-block; representation error ~6e-7 normwise, that of
                             an fp32 sgemm) -- or 3xTF32 (hi*hi + hi*lo + lo*hi, three kind::tf32
                             MMAs per k-step).  0: 3xTF32 everywhere; 1: the mixed split wherever
                             the passes take 128-byte tf32 rows (channel pitches % 32; forward
                             and filter gradient by TMA, backward-data by TMA or, strided, by the
                             K-major cp.async gather); 2 (default): as 1 for unit-stride layers
                             with passes of >= 2 GFLOP (smaller and strided layers measured
                             faster in 3xTF32).  A shape-only choice: results stay deterministic. */
} glp_plan_options_t;
glp_status_t glp_plan_options_default(glp_plan_options_t *opts);
/* opts may be NULL (defaults).  GLP_ERR_INVALID_VALUE for an out-of-range option. */
glp_status_t glp_plan_ex(glp_plan_t *out, glp_conv_desc_t desc, int device, glp_math_t math,
                         int samples_in_flight, const glp_plan_options_t *opts);
glp_status_t glp_plan_get_info(glp_plan_t plan, glp_plan_info_t *info);
glp_status_t glp_plan_destroy(glp_plan_t plan);

/* ---- compute (asynchronous on `stream`) --------------------------------------------------- */
/* y = b + W (*) x.  b may be NULL (no bias).  ws >= info.ws_fwd bytes. */
glp_status_t glp_conv_fwd(glp_plan_t plan, const float *x, const float *w, const float *b,
                          float *y, void *ws, size_t ws_bytes, glp_stream_t stream);
/* dx = col2im(W^T dy) (overwrite).  ws >= info.ws_bwd_data bytes. */
glp_status_t glp_conv_bwd_data(glp_plan_t plan, const float *dy, const float *w, float *dx,
                               void *ws, size_t ws_bytes, glp_stream_t stream);
/* dW = sum_n dy_n col_n^T, db = sum dy (db may be NULL).  accumulate = 0: overwrite;
 * 1: dW += .., db += .. (Caffe beta = 1 diff accumulation).  The reduction over N*H_o*W_o uses
 * a split count fixed by the shape and a fixed summation order: bitwise independent of S, the
 * grid and the run (convergence-invariant, P264).  ws >= info.ws_bwd_filter bytes. */
glp_status_t glp_conv_bwd_filter(glp_plan_t plan, const float *x, const float *dy, float *dw,
                                 float *db, int accumulate, void *ws, size_t ws_bytes,
                                 glp_stream_t stream);
/* Both backward passes of one layer with dy packed once: dx may be NULL (data-fed layer,
 * DESIGN.md R9).  Results are bitwise identical to the two separate calls.
 * ws >= info.ws_bwd bytes. */
glp_status_t glp_conv_bwd(glp_plan_t plan, const float *x, const float *dy, const float *w,
                          float *dx, float *dw, float *db, int accumulate, void *ws,
                          size_t ws_bytes, glp_stream_t stream);

/* ---- staged execution (tensor-core plans only) ------------------------------------------- *
 * The compute calls above are compositions of these stages; a training step that keeps the
 * layer's workspace between forward and backward packs x once (forward) and reuses it in the
 * filter gradient, and packs dy once for both backward GEMMs.  Every stage works on the plan's
 * single workspace layout: ws must hold info.ws_bwd bytes (1024-byte aligned).  Results are
 * bitwise identical to the composed calls.  Stages are asynchronous on `stream`; a stage reads
 * what earlier stages on the same stream wrote.  Each pack has its own workspace region (x, dy,
 * forward W, backward-data W, partials), so stages that touch disjoint regions may run on
 * different streams when the caller orders them with events (e.g. both weight packs up front,
 * the filter-gradient GEMM + reduce beside the next layer's backward-data work).
 * GLP_MATH_FP32_SIMT plans return GLP_ERR_NOT_SUPPORTED. */
typedef enum {
  GLP_PACK_X = 0,          /* x  NCHW fp32 -> packed NHWC operand (rounded to the math mode)  */
  GLP_PACK_DY = 1,         /* dy NCHW fp32 -> packed NHWC operand                              */
  GLP_PACK_DY_DB = 2,      /* as GLP_PACK_DY, plus the fixed-order partial sums of db          */
  GLP_PACK_W_FWD = 3,      /* W -> forward B operand [C_o][(kh,kw,ci)]                         */
  GLP_PACK_W_BWD_DATA = 4, /* W -> backward-data B operand [C_i][(kh,kw,co)]                   */
  GLP_PACK_W_BOTH = 5      /* both weight operands in one pass over W (same bits as 3 + 4)       */
} glp_pack_t;
glp_status_t glp_stage_pack(glp_plan_t plan, glp_pack_t what, const float *src, void *ws,
                            size_t ws_bytes, glp_stream_t stream);
/* tcgen05 implicit GEMM of Alg. 1 with the fused bias epilogue: needs GLP_PACK_X, GLP_PACK_W_FWD. */
glp_status_t glp_stage_fwd(glp_plan_t plan, const float *b, float *y, void *ws, size_t ws_bytes,
                           glp_stream_t stream);
/* tcgen05 implicit GEMM of Alg. 2 (col2im folded): needs GLP_PACK_DY(_DB), GLP_PACK_W_BWD_DATA. */
glp_status_t glp_stage_bwd_data(glp_plan_t plan, float *dx, void *ws, size_t ws_bytes,
                                glp_stream_t stream);
/* tcgen05 implicit GEMM of the filter gradient into the split partials: needs GLP_PACK_X and
 * GLP_PACK_DY(_DB). */
glp_status_t glp_stage_bwd_filter(glp_plan_t plan, void *ws, size_t ws_bytes, glp_stream_t stream);
/* Fixed-order reduction of the split partials into dW (Caffe layout) and of the db partials
 * (requires GLP_PACK_DY_DB when db != NULL). */
glp_status_t glp_stage_reduce(glp_plan_t plan, float *dw, float *db, int accumulate, void *ws,
                              size_t ws_bytes, glp_stream_t stream);

/* ---- fused sibling groups (horizontal fusion) --------------------------- *
 * The paper runs different kernels concurrently (Eq. 9 sums over kernel kinds, P252-254) and
 * names kernel fusion for small kernels as future work (P401).  Sibling convolutions that read
 * the same input x with the same K, stride and pad -- e.g. GoogLeNet inception 5b's 1x1, 3x3-reduce
 * and 5x5-reduce branches (Table 5 conv_3, conv_5, conv_6, P350-355) -- run here as ONE implicit
 * GEMM per pass over C_out = sum C_out[b]: x is packed and read once per pass, the branches share
 * one persistent grid.  Branch b owns output channels [sum_{a<b} C_out[a], sum_{a<=b} C_out[a]).
 *   forward:   y_b = b_b + W_b (*) x                       (one tensor per branch)
 *   backward:  dx  = sum_b W_b^T dy_b (col2im)              (one tensor: the branches' sum)
 *              dW_b, db_b per branch.
 * A group desc is an ordinary desc with C_out = sum: glp_plan / glp_plan_get_info / the single-
 * tensor calls above apply and then read the CONCATENATED tensors (W [sum C_out][C_in][K_h][K_w],
 * y/dy [N][sum C_out][H_o][W_o]); the *_group calls below take one pointer per branch instead.
 * 1 <= n_branches <= 4.  Tensor-core plans require every branch but the last to have C_out a
 * multiple of 8 (BF16) / 4 (TF32) (GLP_ERR_NOT_SUPPORTED from glp_plan otherwise); the *_group
 * calls return GLP_ERR_NOT_SUPPORTED for GLP_MATH_FP32_SIMT plans.  Same ownership, workspace sizes
 * (info.ws_*) and error behaviour as the single-tensor calls; results are bitwise identical to the
 * single-tensor calls on the concatenated tensors. */
glp_status_t glp_conv_group_desc_create(glp_conv_desc_t *out, int N, int C_in, int H, int W,
                                        int n_branches, const int *C_out, int K_h, int K_w,
                                        int stride_h, int stride_w, int pad_h, int pad_w);
/* w[b], y[b] per branch; b may be NULL (no bias) or hold NULL entries. */
glp_status_t glp_conv_group_fwd(glp_plan_t plan, const float *x, const float *const *w,
                                const float *const *b, float *const *y, void *ws, size_t ws_bytes,
                                glp_stream_t stream);
/* dy[b], w[b], dw[b] per branch; dx (may be NULL) receives the sum over branches; db NULL or one
 * pointer per branch. */
glp_status_t glp_conv_group_bwd(glp_plan_t plan, const float *x, const float *const *dy,
                                const float *const *w, float *dx, float *const *dw,
                                float *const *db, int accumulate, void *ws, size_t ws_bytes,
                                glp_stream_t stream);
/* Staged forms: GLP_PACK_X takes src[0]; the other packs one pointer per branch.  bwd_data and
 * bwd_filter stages are the single-tensor glp_stage_bwd_data / glp_stage_bwd_filter. */
glp_status_t glp_stage_pack_group(glp_plan_t plan, glp_pack_t what, const float *const *src,
                                  void *ws, size_t ws_bytes, glp_stream_t stream);
glp_status_t glp_stage_fwd_group(glp_plan_t plan, const float *const *b, float *const *y, void *ws,
                                 size_t ws_bytes, glp_stream_t stream);
glp_status_t glp_stage_reduce_group(glp_plan_t plan, float *const *dw, float *const *db,
                                    int accumulate, void *ws, size_t ws_bytes, glp_stream_t stream);

/* ---- deterministic gradient exchange ----------------------------------- *
 * "Convergence-invariant" (P264) extended across GPU counts: the global batch is cut into a
 * fixed number of leaves (8); each leaf's dW||db is computed by the same plan (shape-only split
 * order) whichever rank holds it, and the leaves are summed by a fixed binary tree — the rank's
 * local subtree, then recursive doubling over ranks (paper_conf_icpp_futhys18_b200.dist.
 * TreeAllreduce; the transfers are torch.distributed point-to-point, NCCL over NVLink).  Every
 * tree node is this call: out = a + b elementwise in fp32 (a, b, out device pointers of n floats;
 * out may alias a or b; asynchronous on `stream`).  Since a + b == b + a bitwise, dW is bitwise
 * identical for 1, 2, 4 and 8 ranks. */
glp_status_t glp_sum2(const float *a, const float *b, float *out, size_t n, glp_stream_t stream);
/* out (+)= T(parts[0..n)): the balanced binary tree over n = 1, 2, 4 or 8 device arrays of count
 * floats in index order (level by level, adjacent pairs: ((p0+p1)+(p2+p3))+((p4+p5)+(p6+p7))) --
 * bitwise the glp_sum2 tree -- in one launch.  accumulate = 1 adds the tree to out.  A rank sums
 * its contiguous block of leaves with it (a complete subtree of the 8-leaf tree). */
glp_status_t glp_tree_sum(const float *const *parts, int n, float *out, size_t count,
                          int accumulate, glp_stream_t stream);
/* The tree's top levels across ranks over NVLink peer memory: subtrees[r] / outs[r] are rank r's
 * subtree sum and output buffers as mapped on this device (torch symmetric memory), world = 1, 2,
 * 4 or 8.  This rank computes the element slice [rank*count/world, (rank+1)*count/world) of
 * T(subtrees[0..world)) with peer loads and stores it into every rank's output (peer stores).
 * The caller brackets the call with barriers (every subtree complete before; every slice written
 * after); then every rank holds bitwise the tree over all leaves, for any world. */
glp_status_t glp_tree_exchange(const float *const *subtrees, float *const *outs, int world, int rank,
                               size_t count, glp_stream_t stream);
/* Leaf plans (wgrad_leaves > 1): the fixed-order reduction of each leaf's split partials, leaf l's
 * dW (Caffe layout) at dw + l*leaf_stride and db at db + l*leaf_stride (db may be NULL; leaf_stride
 * in floats, a multiple of 4).  Needs GLP_PACK_DY_DB when db != NULL.  Overwrites. */
glp_status_t glp_stage_reduce_leaves(glp_plan_t plan, float *dw, float *db, size_t leaf_stride,
                                     void *ws, size_t ws_bytes, glp_stream_t stream);

/* ---- prior-art comparator: the paper's stream pool --------------------- *
 * GLP4NN's own scheme (P165-173, Figs 4/6): every layer pass runs as per-sample kernels (batch 1,
 * the sample's im2col+GEMM chain) dispatched round-robin (P171) over a pool of CUDA streams whose
 * size is the paper's Eq. 7 bound for the per-sample forward kernel (P245: thread and shared-
 * memory terms, plus the launch term once glp_pool_set_launch_term has supplied the measured
 * T_K / T_launch; capped by the concurrent-kernel limit C of Eq. 6) or the caller's n_streams
 * (> 0; both capped by N and 64).  Kept to measure what the persistent tile scheduler
 * of the glp_conv_* calls buys on B200 (bench.py --scheme pool); not the product path.
 * A pool owns its streams and a per-sample plan; desc must be a single layer (no groups).
 * Calls fork from `stream` (event), run on the pool's streams and join back to `stream`.
 * ws >= the ws_bytes of glp_pool_get_info (1024-byte aligned): one per-sample workspace per
 * stream plus one dW||db accumulator per stream.  Forward and backward-data results are bitwise
 * those of glp_conv_fwd / glp_conv_bwd_data (no K split; the per-element order is the same).
 * The filter gradient: each stream accumulates its samples in order (beta = 1, Caffe style; one
 * accumulator per stream instead of the race the paper leaves open, P262-264), and the
 * accumulators are summed in stream order at the join: deterministic for a given n_streams,
 * equal to glp_conv_bwd_filter within rounding (bit-exact on integer data). */
typedef struct glp_pool_s *glp_pool_t;
glp_status_t glp_pool_create(glp_pool_t *out, glp_conv_desc_t desc, int device, glp_math_t math,
                             int n_streams);
glp_status_t glp_pool_get_info(glp_pool_t pool, int *n_streams, int *eq7_bound, size_t *ws_bytes);
/* Eq. 7's launch term (P243-245, reading R17): #K_i <= ceil(T_K / T_launch), with T_K the
 * per-sample forward kernel's duration and T_launch the host launch cost, both measured (us) by
 * the CUPTI resource tracker (include/glp_tracker.h) in a profiling run of the pool ("profile once",
 * P173).  Recomputes the Eq. 7 bound with the term and, unless the caller fixed n_streams, resizes
 * the pool to it (re-query ws_bytes with glp_pool_get_info).  GLP_ERR_INVALID_VALUE unless both
 * times are positive. */
glp_status_t glp_pool_set_launch_term(glp_pool_t pool, double t_kernel_us, double t_launch_us);
/* The pool's Eq. 7 bound without and with the launch term (0 until glp_pool_set_launch_term). */
glp_status_t glp_pool_get_eq7(glp_pool_t pool, int *without_launch_term, int *with_launch_term);
glp_status_t glp_pool_conv_fwd(glp_pool_t pool, const float *x, const float *w, const float *b,
                               float *y, void *ws, size_t ws_bytes, glp_stream_t stream);
/* dx may be NULL (data-fed layer), db may be NULL.  dW, db are overwritten. */
glp_status_t glp_pool_conv_bwd(glp_pool_t pool, const float *x, const float *dy, const float *w,
                               float *dx, float *dw, float *db, void *ws, size_t ws_bytes,
                               glp_stream_t stream);
glp_status_t glp_pool_destroy(glp_pool_t pool);

/* ---- analyzer (host only, no device needed) ----------------------------------------------- */
/* The north_star's sm_100a limits: 148 SMs, 64K regs, 228 KB smem, 2048 threads, 32 blocks,
 * + 512 TMEM columns, 1 KB smem reserved per CTA, C = 128. */
glp_status_t glp_device_limits_b200(glp_device_limits_t *lim);
/* CTAs per SM (beta) from every per-SM limit (Eqs 4-5 + registers/blocks/TMEM, R16). */
glp_status_t glp_analyze_ctas_per_sm(const glp_device_limits_t *lim, const glp_kernel_attr_t *k,
                                     int *ctas_per_sm);
/* S = clamp(floor(slots / tiles_per_sample), 1, n_local)  (Eq. 9 re-derived, R18). */
glp_status_t glp_analyze_samples_in_flight(int slots, int tiles_per_sample, int n_local, int *S);
/* Paper Eq. 7 bound (P245) for a kernel with #beta blocks; t_kernel/t_launch <= 0 = no launch
 * term (R17).  Output floor(min(...)). */
glp_status_t glp_analyze_eq7(const glp_device_limits_t *lim, const glp_kernel_attr_t *k,
                             int blocks, double t_kernel, double t_launch, int *bound);
/* Attributes of the kernel the plan launches for a pass (the halo kernel where the plan chose
 * one; the occupancy-API cross-check and the samples-in-flight inputs). which:
 * 0 = forward, 1 = backward-data, 2 = backward-filter. */
glp_status_t glp_plan_kernel_attr(glp_plan_t plan, int which, glp_kernel_attr_t *attr,
                                  int *ctas_per_sm_model, int *ctas_per_sm_runtime);

/* ---- diagnostics ---------------------------------------------------------------------------- */
const char *glp_status_string(glp_status_t s);
const char *glp_last_error_string(void);
int glp_version(void);
/* Test-only, off the hot path: materialise the im2col matrix of sample n,
 * col[(ci*K_h+kh)*K_w+kw][ho*W_o+wo], using the tensor-core producer's own index math
 * (the packed NHWC operand and its gather).  Values are the packed (rounded) operands. */
glp_status_t glp_debug_im2col(glp_plan_t plan, const float *x, int n, float *col, void *ws,
                              size_t ws_bytes, glp_stream_t stream);

#ifdef __cplusplus
}
#endif
#endif /* GLP_H_ */
