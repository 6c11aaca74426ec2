// Probe: CUDA occupancy API vs dynamic-smem attribute for the igemm kernel (diagnostic tool).
#include <cstdio>
#include "../paper_conf_icpp_futhys18_b200/csrc/igemm.cuh"
using namespace glp;
int main() {
  void *fn = (void *)&igemm_kernel<MODE_FWD, 2, 64>;
  int sizes[] = {60000, 99504, 110000, 116000};
  int attrs[] = {232448, 99504 + 1024, 120000};
  for (int a : attrs) {
    cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, a);
    for (int s : sizes) {
      if (s > a) continue;
      int rt = -1;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&rt, fn, 288, s);
      printf("attr %6d smem %6d -> %d (%s)\n", a, s, rt, cudaGetErrorString(e));
    }
  }
  for (int c : {-1, 0, 50, 100}) {
    cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, 232448);
    cudaFuncSetAttribute(fn, cudaFuncAttributePreferredSharedMemoryCarveout, c);
    int rt = -1;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&rt, fn, 288, 99504);
    printf("carveout %d -> %d\n", c, rt);
  }
  cudaFuncAttributes fa;
  cudaFuncGetAttributes(&fa, fn);
  printf("regs %d static smem %zu maxThreads %d\n", fa.numRegs, fa.sharedSizeBytes, fa.maxThreadsPerBlock);
  cudaDeviceProp p;
  cudaGetDeviceProperties(&p, 0);
  printf("smem/SM %zu reserved/block %zu smem/block optin %zu regs/SM %d\n", p.sharedMemPerMultiprocessor,
         p.reservedSharedMemPerBlock, p.sharedMemPerBlockOptin, p.regsPerMultiprocessor);
  return 0;
}
