// Microbenchmark: raw tcgen05.mma issue rate, cta_group::1 (M=128) vs cta_group::2 (M=256),
// operands resident in smem (no loads).  Diagnostic tool for the CTA-pair design.
#include <cstdio>
#include "../paper_conf_icpp_futhys18_b200/csrc/ptx.cuh"
using namespace glp;
template <int CG, int N>
__global__ void __launch_bounds__(128, 1) k(int iters, unsigned long long *cyc) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  const uint32_t base = (smem_u32(sm) + 1023) & ~1023u;
  const uint32_t rank = CG == 2 ? cluster_ctarank() : 0;
  for (int i = threadIdx.x; i < 64 * 1024 / 4; i += blockDim.x) ((uint32_t *)(sm + (base - smem_u32(sm))))[i] = 0;
  if (threadIdx.x == 0) { mbar_init(smem_u32(&bar), 1); fence_mbar_init(); }
  if (threadIdx.x < 32) { tmem_alloc_cg<CG>(smem_u32(&slot), 256); tmem_relinquish_cg<CG>(); }
  asm volatile("fence.proxy.async.shared::cta;");
  tc_fence_before();
  if (CG == 2) cluster_sync(); else __syncthreads();
  tc_fence_after();
  const uint32_t tm = slot;
  if (threadIdx.x == 0 && rank == 0) {
    const uint32_t idesc = make_idesc(1, 0, 0, 128 * CG, N);
    const uint64_t ad = make_sdesc(base, 16, 1024, 2), bd = make_sdesc(base + 16384, 16, 1024, 2);
    unsigned long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        if (CG == 1) mma_f16(tm, ad + 2 * kk, bd + 2 * kk, idesc, 1);
        else mma_f16_cg2(tm, ad + 2 * kk, bd + 2 * kk, idesc, 1);
      }
    }
    if (CG == 1) mma_commit(smem_u32(&bar)); else mma_commit_cg2_mc(smem_u32(&bar), 3);
    mbar_wait(smem_u32(&bar), 0);
    cyc[blockIdx.x] = clock64() - t0;
  } else if (threadIdx.x == 0 && CG == 2) {
    mbar_wait(smem_u32(&bar), 0);
  }
  tc_fence_before();
  if (CG == 2) cluster_sync(); else __syncthreads();
  if (threadIdx.x < 32) tmem_dealloc_cg<CG>(tm, 256);
}
template <int CG, int N> void run(int grid) {
  unsigned long long *d; cudaMalloc(&d, grid * 8);
  auto fn = k<CG, N>;
  cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, 100 * 1024);
  cudaLaunchConfig_t cfg = {}; cfg.gridDim = grid; cfg.blockDim = 128; cfg.dynamicSmemBytes = 100 * 1024;
  cudaLaunchAttribute at[1]; at[0].id = cudaLaunchAttributeClusterDimension; at[0].val.clusterDim.x = CG;
  at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1; cfg.attrs = at; cfg.numAttrs = 1;
  int iters = 20000;
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaLaunchKernelEx(&cfg, fn, iters, d);
  cudaEventRecord(e0);
  cudaLaunchKernelEx(&cfg, fn, iters, d);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  unsigned long long c; cudaMemcpy(&c, d, 8, cudaMemcpyDeviceToHost);
  double flops = 2.0 * 128 * CG * N * 64 * (double)iters * (grid / CG);
  printf("CG=%d N=%d grid=%d: %.3f ms, %.1f TFLOP/s, %.1f cyc per 4-MMA group (err=%s)\n", CG, N, grid, ms,
         flops / ms / 1e9, (double)c / iters, cudaGetErrorString(cudaGetLastError()));
}
int main() {
  run<1, 256>(148); run<2, 256>(148); run<1, 128>(148); run<2, 128>(148); run<1, 96>(148); run<2, 96>(148);
  return 0;
}
