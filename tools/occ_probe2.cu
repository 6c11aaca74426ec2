// Probe: what limits CTAs/SM for tcgen05 kernels in the CUDA occupancy API (diagnostic tool).
#include <cstdio>
#include <cstdint>
__global__ void __launch_bounds__(288, 1) plain(float *x) { if (x) x[threadIdx.x] = 1.f; }
__global__ void __launch_bounds__(288) plain_nolb(float *x) { if (x) x[threadIdx.x] = 1.f; }
__global__ void __launch_bounds__(288, 1) with_tmem(float *x) {
  __shared__ uint32_t slot;
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 32;" ::"r"((uint32_t)__cvta_generic_to_shared(&slot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  __syncthreads();
  if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 32;" ::"r"(slot));
  if (x) x[threadIdx.x] = 1.f;
}
template <typename F> void q(const char *n, F f, int smem) {
  cudaFuncSetAttribute((void *)f, cudaFuncAttributeMaxDynamicSharedMemorySize, 232448);
  int rt = -1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&rt, (void *)f, 288, smem);
  cudaFuncAttributes fa; cudaFuncGetAttributes(&fa, (void *)f);
  printf("%-12s smem %6d -> %d  (regs %d)\n", n, smem, rt, fa.numRegs);
}
int main() {
  for (int s : {0, 60000, 99504}) { q("plain", plain, s); q("plain_nolb", plain_nolb, s); q("with_tmem", with_tmem, s); }
  return 0;
}
