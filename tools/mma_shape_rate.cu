// Microbenchmark: tcgen05.mma kind::f16 (bf16) issue rate per operand layout / N / LBO, one CTA
// per SM, operands resident in smem (no loads).  Diagnostic for the halo filter gradient: does an
// MN-major A whose two atoms overlap (LBO = 128 B, row-shifted taps) run at the same rate as
// disjoint atoms, and how does the rate depend on N?
#include <cstdio>
#include "../paper_conf_icpp_futhys18_b200/csrc/ptx.cuh"
using namespace glp;

__global__ void __launch_bounds__(128, 1) k(int iters, int n, int a_mn, int b_mn, int a_lbo,
                                            int b_lbo, unsigned long long *cyc) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint64_t bar;
  __shared__ uint32_t slot;
  const uint32_t base = (smem_u32(sm) + 1023) & ~1023u;
  for (int i = threadIdx.x; i < 160 * 1024 / 4; i += blockDim.x)
    ((uint32_t *)(sm + (base - smem_u32(sm))))[i] = 0x3c003c00u;
  if (threadIdx.x == 0) { mbar_init(smem_u32(&bar), 1); fence_mbar_init(); }
  if (threadIdx.x < 32) { tmem_alloc(smem_u32(&slot), 256); tmem_relinquish(); }
  asm volatile("fence.proxy.async.shared::cta;");
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tm = slot;
  if (threadIdx.x == 0) {
    const uint32_t idesc = make_idesc(1, a_mn, b_mn, 128, n);
    // K-major: rows of 128 B, SBO 1024, K step +32 B (2 units).  MN-major: K rows of 128 B,
    // SBO 1024 (8 K rows), LBO = atom stride, K step 16 rows = 2048 B (128 units).
    const uint64_t ad = a_mn ? make_sdesc(base, a_lbo, 1024, 2) : make_sdesc(base, 16, 1024, 2);
    const uint64_t bd = b_mn ? make_sdesc(base + 65536, b_lbo, 1024, 2)
                             : make_sdesc(base + 65536, 16, 1024, 2);
    const uint64_t ast = a_mn ? 128 : 2, bst = b_mn ? 128 : 2;
    unsigned long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) mma_f16(tm, ad + ast * kk, bd + bst * kk, idesc, 1);
    }
    mma_commit(smem_u32(&bar));
    mbar_wait(smem_u32(&bar), 0);
    cyc[blockIdx.x] = clock64() - t0;
  }
  tc_fence_before();
  __syncthreads();
  if (threadIdx.x < 32) tmem_dealloc(tm, 256);
}

void run(const char *name, int n, int a_mn, int b_mn, int a_lbo, int b_lbo) {
  const int grid = 148, iters = 20000;
  unsigned long long *d;
  cudaMalloc(&d, grid * 8);
  cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, 170 * 1024);
  k<<<grid, 128, 170 * 1024>>>(100, n, a_mn, b_mn, a_lbo, b_lbo, d);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  cudaEventRecord(e0);
  k<<<grid, 128, 170 * 1024>>>(iters, n, a_mn, b_mn, a_lbo, b_lbo, d);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms;
  cudaEventElapsedTime(&ms, e0, e1);
  unsigned long long c;
  cudaMemcpy(&c, d, 8, cudaMemcpyDeviceToHost);
  const double flops = 2.0 * 128 * n * 16 * 4.0 * iters * grid;
  const double cyc_per = (double)c / (iters * 4.0);
  printf("%-44s N=%3d: %7.1f TFLOP/s  %6.1f cyc/MMA (ideal %5.1f)  %s\n", name, n, flops / ms / 1e9,
         cyc_per, 128.0 * n * 16 * 2 / 8192.0, cudaGetErrorString(cudaGetLastError()));
  cudaFree(d);
}

int main() {
  for (int n : {64, 96, 128, 192, 256}) {
    run("K-major A, K-major B", n, 0, 0, 0, 0);
    run("MN-major A (disjoint atoms), MN-major B", n, 1, 1, 8192, 8192);
    run("MN-major A (LBO 128: shifted taps), MN B", n, 1, 1, 128, 8192);
    run("MN-major A (disjoint), MN B (LBO 128 taps)", n, 1, 1, 8192, 128);
    run("K-major A, MN-major B", n, 0, 1, 0, 8192);
  }
  return 0;
}
