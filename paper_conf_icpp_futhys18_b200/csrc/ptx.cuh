// ptx.cuh — thin inline-PTX wrappers for the sm_100a primitives the kernels use:
// mbarrier, cp.async (zero-fill), TMA tiled loads, tcgen05 (alloc / mma / commit / ld / fences).
// Encodings follow the PTX ISA; descriptor bitfields cross-checked against the CUTLASS/CuTe
// headers vendored in the venv (cute/arch/mma_sm100_desc.hpp, used as an encoding reference only).
#pragma once
#include <cstdint>
#include <cuda.h>

namespace glp {

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

// ------------------------------------------------------- programmatic dependent launch ---
// Launched with cudaLaunchAttributeProgrammaticStreamSerialization, a kernel may start while its
// predecessor in the stream drains: pdl_launch_dependents() lets the next kernel begin launching
// once every CTA of this one has issued it; pdl_wait() blocks until the predecessor grid has
// completed and its memory is visible (a no-op without the attribute).  Every kernel of the
// tensor-core path calls pdl_wait() before its first global-memory access.
__device__ __forceinline__ void pdl_launch_dependents() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

// ------------------------------------------------------------------ shared memory --------
__device__ __forceinline__ void sts_f32(uint32_t addr, float v) {
  asm volatile("st.shared.f32 [%0], %1;" ::"r"(addr), "f"(v) : "memory");
}
__device__ __forceinline__ float lds_f32(uint32_t addr) {
  float v;
  asm volatile("ld.shared.f32 %0, [%1];" : "=f"(v) : "r"(addr) : "memory");
  return v;
}
__device__ __forceinline__ float4 lds_f32x4(uint32_t addr) {
  float4 v;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(addr) : "memory");
  return v;
}

// ------------------------------------------------------------------ mbarrier -------------
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint32_t bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred P1;\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, P1;\n\t}"
      : "=r"(ok)
      : "r"(bar), "r"(parity)
      : "memory");
  return ok != 0;
}
// Blocking wait with a watchdog: a pipeline deadlock becomes a device trap (an error the host
// sees) instead of a hung GPU.  The bound (~2^26 suspended polls) is far beyond any real wait.
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  uint32_t polls = 0;
  while (!mbar_try_wait(bar, parity)) {
    if (++polls == (1u << 26)) __trap();
  }
}
// Wait for a long-latency event (a whole tile) with back-off, so idle warps do not steal issue
// slots from the producer warps sharing their SM sub-partition.
__device__ __forceinline__ void mbar_wait_sleep(uint32_t bar, uint32_t parity) {
  uint32_t polls = 0;
  while (!mbar_try_wait(bar, parity)) {
    __nanosleep(128);
    if (++polls == (1u << 26)) __trap();
  }
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// ------------------------------------------------------------------ cp.async -------------
// 16-byte global->shared copy; src_bytes = 0 zero-fills the destination (padding, ragged tails).
__device__ __forceinline__ void cp_async16(uint32_t dst, const void *src, bool valid) {
  const uint32_t n = valid ? 16u : 0u;
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(dst), "l"(src), "r"(n)
               : "memory");
}
// 8-byte cp.async (.ca); zero-fills when !valid (the bf16 planes of the mixed split's gather)
__device__ __forceinline__ void cp_async8(uint32_t dst, const void *src, bool valid) {
  const uint32_t n = valid ? 8u : 0u;
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" ::"r"(dst), "l"(src), "r"(n)
               : "memory");
}
// 4-byte cp.async (L1-allocating .ca: the only form for sizes < 16); zero-fills when !valid
__device__ __forceinline__ void cp_async4(uint32_t dst, const void *src, bool valid) {
  const uint32_t n = valid ? 4u : 0u;
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4, %2;" ::"r"(dst), "l"(src), "r"(n)
               : "memory");
}
// Arrive on `bar` when every cp.async previously issued by this thread has completed; noinc:
// the arrival counts against the barrier's expected count (no pending-count increment).
// Same completion mechanism as CUTLASS's sm100 cp.async mainloop (cpasync_barrier_arrive).
__device__ __forceinline__ void cp_async_mbar_arrive_noinc(uint32_t bar) {
  asm volatile("cp.async.mbarrier.arrive.noinc.shared::cta.b64 [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void cp_async_commit() {
  asm volatile("cp.async.commit_group;" ::: "memory");
}
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

// ------------------------------------------------------------------ TMA ------------------
__device__ __forceinline__ void tma_prefetch(const CUtensorMap *map) {
  asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(map)) : "memory");
}
__device__ __forceinline__ void tma_load_2d(uint32_t dst, const CUtensorMap *map, uint32_t bar,
                                            int c0, int c1) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
      " [%0], [%1, {%3, %4}], [%2];" ::"r"(dst),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(bar), "r"(c0), "r"(c1)
      : "memory");
}

// ------------------------------------------------------------------ warp-converged issue ---
// Single-lane async ops issued by a converged warp: `elect.sync` inside the instruction block
// picks one lane, so the operands stay warp-uniform (uniform datapath) and the compiler does not
// wrap each op in a per-lane ELECT/BRA.U.ANY loop.  Call with all 32 lanes active.
#define GLP_ELECT "{\n\t.reg .pred P_e;\n\telect.sync _|P_e, 0xffffffff;\n\t"
__device__ __forceinline__ void mbar_arrive_expect_tx_e(uint32_t bar, uint32_t bytes) {
  asm volatile(GLP_ELECT "@P_e mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n\t}" ::"r"(bar),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void tma_load_2d_e(uint32_t dst, const CUtensorMap *map, uint32_t bar,
                                              int c0, int c1) {
  asm volatile(GLP_ELECT
               "@P_e cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes"
               " [%0], [%1, {%3, %4}], [%2];\n\t}" ::"r"(dst),
               "l"(reinterpret_cast<uint64_t>(map)), "r"(bar), "r"(c0), "r"(c1)
               : "memory");
}
__device__ __forceinline__ void tma_load_4d_cg2_e(uint32_t dst, const CUtensorMap *map, uint32_t bar,
                                                  int c0, int c1, int c2, int c3) {
  asm volatile(GLP_ELECT
               "@P_e cp.async.bulk.tensor.4d.cta_group::2.shared::cluster.global.tile.mbarrier::complete_tx::bytes"
               " [%0], [%1, {%3, %4, %5, %6}], [%2];\n\t}" ::"r"(dst),
               "l"(reinterpret_cast<uint64_t>(map)), "r"(bar), "r"(c0), "r"(c1), "r"(c2), "r"(c3)
               : "memory");
}
__device__ __forceinline__ void tma_load_im2col_4d_e(uint32_t dst, const CUtensorMap *map,
                                                     uint32_t bar, int c, int w, int h, int n,
                                                     uint16_t off_w, uint16_t off_h) {
  asm volatile(GLP_ELECT
               "@P_e cp.async.bulk.tensor.4d.shared::cluster.global.im2col.mbarrier::complete_tx::bytes"
               " [%0], [%1, {%3, %4, %5, %6}], [%2], {%7, %8};\n\t}" ::"r"(dst),
               "l"(reinterpret_cast<uint64_t>(map)), "r"(bar), "r"(c), "r"(w), "r"(h), "r"(n),
               "h"(off_w), "h"(off_h)
               : "memory");
}
// 3-D tiled loads: the filter gradient's MN-major B (dy) tile as ONE load of all its atoms
// (tensor dims {atom elements, pixels, atoms}: the box lands atom-major, i.e. the MN-major layout)
__device__ __forceinline__ void tma_load_3d_e(uint32_t dst, const CUtensorMap *map, uint32_t bar,
                                              int c0, int c1, int c2) {
  asm volatile(GLP_ELECT
               "@P_e cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes"
               " [%0], [%1, {%3, %4, %5}], [%2];\n\t}" ::"r"(dst),
               "l"(reinterpret_cast<uint64_t>(map)), "r"(bar), "r"(c0), "r"(c1), "r"(c2)
               : "memory");
}
__device__ __forceinline__ void tma_load_3d_cg2_e(uint32_t dst, const CUtensorMap *map, uint32_t bar,
                                                  int c0, int c1, int c2) {
  asm volatile(GLP_ELECT
               "@P_e cp.async.bulk.tensor.3d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes"
               " [%0], [%1, {%3, %4, %5}], [%2];\n\t}" ::"r"(dst),
               "l"(reinterpret_cast<uint64_t>(map)), "r"(bar), "r"(c0), "r"(c1), "r"(c2)
               : "memory");
}
__device__ __forceinline__ void tma_load_2d_cg2_e(uint32_t dst, const CUtensorMap *map,
                                                  uint32_t bar, int c0, int c1) {
  asm volatile(GLP_ELECT
               "@P_e cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes"
               " [%0], [%1, {%3, %4}], [%2];\n\t}" ::"r"(dst),
               "l"(reinterpret_cast<uint64_t>(map)), "r"(bar), "r"(c0), "r"(c1)
               : "memory");
}
__device__ __forceinline__ void tma_load_im2col_4d_cg2_e(uint32_t dst, const CUtensorMap *map,
                                                         uint32_t bar, int c, int w, int h, int n,
                                                         uint16_t off_w, uint16_t off_h) {
  asm volatile(GLP_ELECT
               "@P_e cp.async.bulk.tensor.4d.im2col.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes"
               " [%0], [%1, {%3, %4, %5, %6}], [%2], {%7, %8};\n\t}" ::"r"(dst),
               "l"(reinterpret_cast<uint64_t>(map)), "r"(bar), "r"(c), "r"(w), "r"(h), "r"(n),
               "h"(off_w), "h"(off_h)
               : "memory");
}
// All NSTEP tcgen05.mma of one k-block in one instruction block (one elect, descriptors advanced
// by STEP 16-byte units per MMA inside the block): the MMA-issuing warp's loop is latency-bound,
// so the per-MMA overhead of separate blocks (re-elect, uniform-register broadcasts) counts.
// `accumulate` applies to the first MMA only; the rest always accumulate.
template <int KIND, int CG, int NSTEP, int STEP>
__device__ __forceinline__ void mma_kblock_e(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc,
                                             uint32_t idesc, uint32_t accumulate) {
  static_assert(NSTEP == 2 || NSTEP == 4, "k-block = 2 or 4 MMAs");
#define GLP_MMA_HEAD                                                                    \
  "{\n\t.reg .pred P_e, p, q;\n\t.reg .b64 a1, b1;\n\t"                                 \
  "elect.sync _|P_e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\tsetp.eq.b32 q, %3, %3;\n\t"
#define GLP_MMA_I(CGS, KINDS, A, B, P)                                                  \
  "@P_e tcgen05.mma.cta_group::" CGS ".kind::" KINDS " [%0], " A ", " B ", %3, " P ";\n\t"
#define GLP_MMA_ADV(A0, B0) "add.s64 a1, " A0 ", %5;\n\tadd.s64 b1, " B0 ", %5;\n\t"
#define GLP_MMA_K2(CGS, KINDS)                                                          \
  asm volatile(GLP_MMA_HEAD GLP_MMA_I(CGS, KINDS, "%1", "%2", "p") GLP_MMA_ADV("%1", "%2") \
               GLP_MMA_I(CGS, KINDS, "a1", "b1", "q") "}"                               \
               ::"r"(d_tmem), "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate),      \
               "n"(STEP) : "memory")
#define GLP_MMA_K4(CGS, KINDS)                                                          \
  asm volatile(GLP_MMA_HEAD GLP_MMA_I(CGS, KINDS, "%1", "%2", "p") GLP_MMA_ADV("%1", "%2") \
               GLP_MMA_I(CGS, KINDS, "a1", "b1", "q") GLP_MMA_ADV("a1", "b1")           \
               GLP_MMA_I(CGS, KINDS, "a1", "b1", "q") GLP_MMA_ADV("a1", "b1")           \
               GLP_MMA_I(CGS, KINDS, "a1", "b1", "q") "}"                               \
               ::"r"(d_tmem), "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate),      \
               "n"(STEP) : "memory")
  if (NSTEP == 2) {
    if (KIND == 0 && CG == 1) GLP_MMA_K2("1", "f16");
    else if (KIND == 0) GLP_MMA_K2("2", "f16");
    else if (CG == 1) GLP_MMA_K2("1", "tf32");
    else GLP_MMA_K2("2", "tf32");
  } else {
    if (KIND == 0 && CG == 1) GLP_MMA_K4("1", "f16");
    else if (KIND == 0) GLP_MMA_K4("2", "f16");
    else if (CG == 1) GLP_MMA_K4("1", "tf32");
    else GLP_MMA_K4("2", "tf32");
  }
#undef GLP_MMA_K4
#undef GLP_MMA_K2
#undef GLP_MMA_ADV
#undef GLP_MMA_I
#undef GLP_MMA_HEAD
}
// 3xTF32 k-block (GLP_MATH_FP32): every operand is a hi plane and a lo plane (hi = rna(v),
// lo = rna(v - hi)) at byte offsets 16*alo16 (A) / 16*blo16 (B) from the hi plane.  Per k-step
// three kind::tf32 MMAs accumulate, in this fixed order, hi*hi, hi*lo and lo*hi into the same
// TMEM accumulator (lo*lo, below 2^-22 of a product, is dropped).  NSTEP k-steps advanced by STEP
// 16-byte units, all in one instruction block; `accumulate` applies to the first MMA only.
template <int CG, int NSTEP, int STEP>
__device__ __forceinline__ void mma_kblock_x3_e(uint32_t d_tmem, uint64_t adesc, uint64_t bdesc,
                                                uint64_t alo16, uint64_t blo16, uint32_t idesc,
                                                uint32_t accumulate) {
  static_assert(NSTEP == 4, "3xTF32 k-block = 4 k-steps of K = 8");
#define GLP_X3_HEAD                                                                     \
  "{\n\t.reg .pred P_e, p, q;\n\t.reg .b64 a, b, al, bl;\n\t"                           \
  "elect.sync _|P_e, 0xffffffff;\n\tsetp.ne.b32 p, %4, 0;\n\tsetp.eq.b32 q, %3, %3;\n\t" \
  "mov.b64 a, %1;\n\tmov.b64 b, %2;\n\t"
#define GLP_X3_STEP(CGS, P)                                                             \
  "add.s64 al, a, %5;\n\tadd.s64 bl, b, %6;\n\t"                                        \
  "@P_e tcgen05.mma.cta_group::" CGS ".kind::tf32 [%0], a, b, %3, " P ";\n\t"           \
  "@P_e tcgen05.mma.cta_group::" CGS ".kind::tf32 [%0], a, bl, %3, q;\n\t"              \
  "@P_e tcgen05.mma.cta_group::" CGS ".kind::tf32 [%0], al, b, %3, q;\n\t"
#define GLP_X3_ADV "add.s64 a, a, %7;\n\tadd.s64 b, b, %7;\n\t"
#define GLP_X3_K4(CGS)                                                                  \
  asm volatile(GLP_X3_HEAD GLP_X3_STEP(CGS, "p") GLP_X3_ADV GLP_X3_STEP(CGS, "q")      \
               GLP_X3_ADV GLP_X3_STEP(CGS, "q") GLP_X3_ADV GLP_X3_STEP(CGS, "q") "}"   \
               ::"r"(d_tmem), "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate),      \
               "l"(alo16), "l"(blo16), "n"(STEP) : "memory")
  if (CG == 1) GLP_X3_K4("1");
  else GLP_X3_K4("2");
#undef GLP_X3_K4
#undef GLP_X3_ADV
#undef GLP_X3_STEP
#undef GLP_X3_HEAD
}

// Mixed fp32 split k-block (GLP_MATH_FP32 with plan option fp32_split = 1): A and B each have a
// tf32 hi plane (descriptors a, b) and two bf16 planes, bf16(hi) (a1, b1) and bf16(v - hi)
// (a2, b2).  In this fixed order: four kind::tf32 MMAs hi*hi (K = 8 each, descriptors advanced by
// TSTEP 16-byte units), two kind::f16 MMAs bf16(hi_A)*bf16(lo_B) and two bf16(lo_A)*bf16(hi_B)
// (K = 16 each, advanced by BSTEP), all into one TMEM accumulator; `accumulate` applies to the
// first MMA only.  Eight MMA issue slots per 32-deep k-block instead of 3xTF32's twelve.
template <int CG, int TSTEP, int BSTEP>
__device__ __forceinline__ void mma_kblock_mix_e(uint32_t d_tmem, uint64_t a, uint64_t b,
                                                 uint64_t a1, uint64_t b1, uint64_t a2, uint64_t b2,
                                                 uint32_t idesc_t, uint32_t idesc_b,
                                                 uint32_t accumulate) {
#define GLP_MX_T(CGS, X, Y, P) "@P_e tcgen05.mma.cta_group::" CGS ".kind::tf32 [%0], " X ", " Y ", %7, " P ";\n\t"
#define GLP_MX_B(CGS, X, Y) "@P_e tcgen05.mma.cta_group::" CGS ".kind::f16 [%0], " X ", " Y ", %8, q;\n\t"
#define GLP_MX(CGS)                                                                          \
  asm volatile("{\n\t.reg .pred P_e, p, q;\n\t.reg .b64 x, y;\n\t"                         \
               "elect.sync _|P_e, 0xffffffff;\n\tsetp.ne.b32 p, %9, 0;\n\tsetp.eq.b32 q, %7, %7;\n\t" \
               GLP_MX_T(CGS, "%1", "%2", "p")                                                \
               "add.s64 x, %1, %10;\n\tadd.s64 y, %2, %10;\n\t" GLP_MX_T(CGS, "x", "y", "q")   \
               "add.s64 x, x, %10;\n\tadd.s64 y, y, %10;\n\t" GLP_MX_T(CGS, "x", "y", "q")     \
               "add.s64 x, x, %10;\n\tadd.s64 y, y, %10;\n\t" GLP_MX_T(CGS, "x", "y", "q")     \
               GLP_MX_B(CGS, "%3", "%6")                                                      \
               "add.s64 x, %3, %11;\n\tadd.s64 y, %6, %11;\n\t" GLP_MX_B(CGS, "x", "y")        \
               GLP_MX_B(CGS, "%5", "%4")                                                      \
               "add.s64 x, %5, %11;\n\tadd.s64 y, %4, %11;\n\t" GLP_MX_B(CGS, "x", "y") "}"    \
               ::"r"(d_tmem), "l"(a), "l"(b), "l"(a1), "l"(b1), "l"(a2), "l"(b2), "r"(idesc_t),  \
               "r"(idesc_b), "r"(accumulate), "n"(TSTEP), "n"(BSTEP) : "memory")
  if (CG == 1) GLP_MX("1");
  else GLP_MX("2");
#undef GLP_MX
#undef GLP_MX_B
#undef GLP_MX_T
}

template <int CG>
__device__ __forceinline__ void mma_commit_e(uint32_t bar) {
  if (CG == 1)
    asm volatile(GLP_ELECT
                 "@P_e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n\t}" ::"r"(bar)
                 : "memory");
  else
    asm volatile(GLP_ELECT
                 "@P_e tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64"
                 " [%0], %1;\n\t}" ::"r"(bar), "h"((uint16_t)3)
                 : "memory");
}

__device__ __forceinline__ void cluster_sync() {
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::
                   : "memory");
}
// shared::cluster address of the same smem variable in CTA `rank` of the cluster
__device__ __forceinline__ uint32_t mapa_shared(uint32_t addr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(rank));
  return r;
}
// Relaxed arrivals (no release fence): the epilogue's "accumulator drained" signal.  Its TMEM
// reads are complete (tcgen05.wait::ld) and ordered by tcgen05.fence::before_thread_sync; a
// release-scoped arrive would also wait for every global store the warp has issued (MEMBAR +
// ERRBAR in SASS), capping the epilogue's store stream at one tile in flight (ncu, conv1 fwd).
__device__ __forceinline__ void mbar_arrive_relaxed(uint32_t bar) {
  asm volatile("mbarrier.arrive.relaxed.cta.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}
__device__ __forceinline__ void mbar_arrive_cluster_relaxed(uint32_t cluster_bar) {
  asm volatile("mbarrier.arrive.relaxed.cluster.shared::cluster.b64 _, [%0];" ::"r"(cluster_bar)
               : "memory");
}

// ------------------------------------------------------------------ tcgen05 --------------
template <int CG>
__device__ __forceinline__ void tmem_alloc_cg(uint32_t dst_smem, uint32_t ncols) {
  if (CG == 1)
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(dst_smem),
                 "r"(ncols) : "memory");
  else
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(dst_smem),
                 "r"(ncols) : "memory");
}
template <int CG>
__device__ __forceinline__ void tmem_relinquish_cg() {
  if (CG == 1) asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
  else asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
}
template <int CG>
__device__ __forceinline__ void tmem_dealloc_cg(uint32_t taddr, uint32_t ncols) {
  if (CG == 1)
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
  else
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}
__device__ __forceinline__ void tmem_alloc(uint32_t dst_smem, uint32_t ncols) {
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(dst_smem),
               "r"(ncols)
               : "memory");
}
__device__ __forceinline__ void tmem_relinquish() {
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
}
__device__ __forceinline__ void tmem_dealloc(uint32_t taddr, uint32_t ncols) {
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols)
               : "memory");
}
// named barrier `id` over `n` threads (a subset of the CTA, e.g. the four epilogue warps)
__device__ __forceinline__ void named_bar_sync(int id, int n) {
  asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(n) : "memory");
}
__device__ __forceinline__ void tc_fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tmem_wait_ld() {
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
}
// wait::ld that also pins the destination registers of an earlier asynchronous tcgen05.ld: the
// "+r" operands keep the compiler from moving any use of r above the wait (software-pipelined
// epilogue: the next chunk's load is in flight while the current chunk is stored).
__device__ __forceinline__ void tmem_wait_ld_dep(uint32_t (&r)[32]) {
  asm volatile("tcgen05.wait::ld.sync.aligned;"
               : "+r"(r[0]), "+r"(r[1]), "+r"(r[2]), "+r"(r[3]), "+r"(r[4]), "+r"(r[5]),
                 "+r"(r[6]), "+r"(r[7]), "+r"(r[8]), "+r"(r[9]), "+r"(r[10]), "+r"(r[11]),
                 "+r"(r[12]), "+r"(r[13]), "+r"(r[14]), "+r"(r[15]), "+r"(r[16]), "+r"(r[17]),
                 "+r"(r[18]), "+r"(r[19]), "+r"(r[20]), "+r"(r[21]), "+r"(r[22]), "+r"(r[23]),
                 "+r"(r[24]), "+r"(r[25]), "+r"(r[26]), "+r"(r[27]), "+r"(r[28]), "+r"(r[29]),
                 "+r"(r[30]), "+r"(r[31])
               :
               : "memory");
}
// 32 lanes x 32 bit, 32 consecutive columns -> 32 registers per thread (thread i = lane i).
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 "
      "{%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,"
      "%16,%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
        "=r"(r[7]), "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]),
        "=r"(r[14]), "=r"(r[15]), "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]),
        "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]), "=r"(r[24]), "=r"(r[25]),
        "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr)
      : "memory");
}

// Shared-memory matrix descriptor (tcgen05 "matrix descriptor"): start>>4 [0,14), LBO>>4 [16,30),
// SBO>>4 [32,46), version = 1 [46,48), base offset 0, LBO mode 0, layout type [61,64).
// layout 2 = SWIZZLE_128B (1024-byte atoms, 16-byte chunk index XOR row-in-atom);
// layout 1 = SWIZZLE_128B_BASE32B (512-byte atoms, 32-byte chunk index XOR row%4) — the only
// MN-major layout for 32-bit (tf32) operands.
__device__ __forceinline__ uint64_t make_sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo,
                                               uint32_t layout = 2) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3FFF) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)layout << 61;
  return d;
}

// Instruction descriptor (kind::f16 / kind::tf32): c_format F32 = 1 [4,6), a_format [7,10),
// b_format [10,13) (BF16 = 1, TF32 = 2), a_major [15], b_major [16] (0 = K, 1 = MN),
// N>>3 [17,23), M>>4 [24,29).
__host__ __device__ constexpr uint32_t make_idesc(uint32_t fmt, uint32_t a_mn, uint32_t b_mn,
                                                  uint32_t M, uint32_t N) {
  return (1u << 4) | (fmt << 7) | (fmt << 10) | (a_mn << 15) | (b_mn << 16) | ((N >> 3) << 17) |
         ((M >> 4) << 24);
}

__device__ __forceinline__ uint32_t f32_to_tf32_rna(float f) {
  uint32_t r;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(f));
  return r;
}

}  // namespace glp
