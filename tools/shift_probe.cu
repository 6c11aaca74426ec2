// Probe: can a tcgen05 smem descriptor start at an arbitrary 128-byte row of a SWIZZLE_128B
// buffer (the "halo" implicit-GEMM trick: the A operand of tap (kh, kw) is the staged input tile
// shifted by kh*Wp + kw pixel rows)?  Data is written with the 128B swizzle keyed on absolute
// smem address bits [7,10) (what TMA produces into a 1024-byte-aligned buffer); the MMA reads
// it through descriptors whose start address is shifted by s rows, with the base-offset field
// [49,52) either 0 or (start >> 7) & 7.  Checked exactly on small integers.
//   K-major  (fwd/dgrad A): M = 128 pixel rows starting at row s, K = 64 channels (one 128-B row)
//   MN-major (wgrad A)    : M = 2 atoms of 64 channels at row shifts s0, s1 (LBO = (s1-s0)*128),
//                           K = 64 pixel rows
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda_bf16.h>
#include "../paper_conf_icpp_futhys18_b200/csrc/ptx.cuh"
using namespace glp;

constexpr int R = 320;   // staged rows (128 B each)

__device__ __forceinline__ uint32_t swz(uint32_t addr) {   // absolute-address SW128
  return addr ^ (((addr >> 7) & 7u) << 4);
}

// mode 0: K-major A (rows s..s+127), B K-major 64 x 64.  mode 1: MN-major A (atoms at s0, s1),
// B MN-major (64 pixel rows x 64 channels at row 0 of its own buffer).
__global__ void __launch_bounds__(128, 1) probe(const float *X, const float *Bm, int mode, int s0,
                                                int s1, int bo_mode, float *out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  const uint32_t raw = smem_u32(sm);
  const uint32_t base = (raw + 1023) & ~1023u;
  const uint32_t bbase = base + R * 128;   // 1024-aligned (R multiple of 8)
  uint8_t *gen = sm + (base - raw);
  // stage X (R x 64 bf16) and B (64 x 64 bf16) with the absolute-address swizzle
  for (int i = threadIdx.x; i < R * 64; i += blockDim.x) {
    const int r = i / 64, c = i % 64;
    const uint32_t a = swz(base + r * 128 + c * 2);
    *reinterpret_cast<__nv_bfloat16 *>(gen + (a - base)) = __float2bfloat16(X[i]);
  }
  for (int i = threadIdx.x; i < 64 * 64; i += blockDim.x) {
    const int r = i / 64, c = i % 64;
    const uint32_t a = swz(bbase + r * 128 + c * 2);
    *reinterpret_cast<__nv_bfloat16 *>(gen + (a - base)) = __float2bfloat16(Bm[i]);
  }
  if (threadIdx.x == 0) { mbar_init(smem_u32(&bar), 1); fence_mbar_init(); }
  if (threadIdx.x < 32) { tmem_alloc(smem_u32(&slot), 64); tmem_relinquish(); }
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tm = slot;
  if (threadIdx.x == 0) {
    if (mode == 0) {
      const uint32_t idesc = make_idesc(1, 0, 0, 128, 64);
      const uint32_t astart = base + s0 * 128;
      uint64_t ad = make_sdesc(astart, 16, 1024, 2), bd = make_sdesc(bbase, 16, 1024, 2);
      if (bo_mode) ad |= (uint64_t)((astart >> 7) & 7) << 49;
      for (int kk = 0; kk < 4; ++kk) mma_f16(tm, ad + 2 * kk, bd + 2 * kk, idesc, kk > 0);
    } else {
      const uint32_t idesc = make_idesc(1, 1, 1, 128, 64);
      const uint32_t astart = base + s0 * 128;
      uint64_t ad = make_sdesc(astart, (uint32_t)(s1 - s0) * 128u, 1024, 2);
      uint64_t bd = make_sdesc(bbase, 8192, 1024, 2);
      if (bo_mode) ad |= (uint64_t)((astart >> 7) & 7) << 49;
      // K = 64 pixel rows = 4 MMAs of 16 rows (2 groups of 8 rows = 2 KB each)
      for (int kk = 0; kk < 4; ++kk) mma_f16(tm, ad + 128 * kk, bd + 128 * kk, idesc, kk > 0);
    }
    mma_commit(smem_u32(&bar));
  }
  mbar_wait(smem_u32(&bar), 0);
  tc_fence_after();
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (int c0 = 0; c0 < 64; c0 += 32) {
    uint32_t v[32];
    tmem_ld32(tm + ((uint32_t)(w * 32) << 16) + c0, v);
    tmem_wait_ld();
    for (int q = 0; q < 32; ++q) out[(w * 32 + lane) * 64 + c0 + q] = __uint_as_float(v[q]);
  }
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x < 32) tmem_dealloc(tm, 64);
}

int main() {
  std::vector<float> X(R * 64), B(64 * 64), out(128 * 64);
  srand(1);
  for (auto &x : X) x = (float)(rand() % 5 - 2);
  for (auto &x : B) x = (float)(rand() % 5 - 2);
  float *dX, *dB, *dO;
  cudaMalloc(&dX, X.size() * 4); cudaMalloc(&dB, B.size() * 4); cudaMalloc(&dO, out.size() * 4);
  cudaMemcpy(dX, X.data(), X.size() * 4, cudaMemcpyHostToDevice);
  cudaMemcpy(dB, B.data(), B.size() * 4, cudaMemcpyHostToDevice);
  cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  const int shifts[][2] = {{0, 64}, {1, 2}, {3, 58}, {5, 6}, {7, 62}, {8, 9}, {13, 70}, {57, 58}, {2, 57}};
  for (int mode = 0; mode < 2; ++mode)
    for (int bo = 0; bo < 2; ++bo)
      for (auto &sh : shifts) {
        const int s0 = sh[0], s1 = sh[1];
        cudaMemset(dO, 0, out.size() * 4);
        probe<<<1, 128, 100 * 1024>>>(dX, dB, mode, s0, s1, bo, dO);
        cudaError_t e = cudaDeviceSynchronize();
        cudaMemcpy(out.data(), dO, out.size() * 4, cudaMemcpyDeviceToHost);
        double maxerr = 0;
        for (int m = 0; m < 128; ++m)
          for (int n = 0; n < 64; ++n) {
            double ref = 0;
            if (mode == 0) {
              for (int k = 0; k < 64; ++k) ref += X[(s0 + m) * 64 + k] * B[n * 64 + k];
            } else {
              const int s = (m < 64) ? s0 : s1, c = m % 64;
              for (int k = 0; k < 64; ++k) ref += X[(s + k) * 64 + c] * B[k * 64 + n];
            }
            maxerr = std::max(maxerr, std::abs(ref - out[m * 64 + n]));
          }
        printf("mode=%s base_offset=%s s0=%3d s1=%3d : max|err| = %g  (%s)\n",
               mode ? "MN-major" : "K-major ", bo ? "(start>>7)&7" : "0           ", s0, s1,
               maxerr, cudaGetErrorString(e));
        if (e != cudaSuccess) return 1;
      }
  return 0;
}
