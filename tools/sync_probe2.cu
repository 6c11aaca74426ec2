// Microbenchmark: per-stage cost of a single-thread consumer loop (wait full -> [MMAs] -> commit)
// with incremental stage/phase counters (no div/mod), vs try_wait / test_wait variants.
#include <cstdio>
#include "../paper_conf_icpp_futhys18_b200/csrc/ptx.cuh"
using namespace glp;
__device__ __forceinline__ bool test_wait(uint32_t bar, uint32_t parity) {
  uint32_t ok;
  asm volatile("{\n\t.reg .pred P1;\n\tmbarrier.test_wait.parity.shared::cta.b64 P1, [%1], %2;\n\tselp.u32 %0, 1, 0, P1;\n\t}"
               : "=r"(ok) : "r"(bar), "r"(parity) : "memory");
  return ok != 0;
}
template <int MODE>
__global__ void __launch_bounds__(128, 1) probe(int iters, long long *out) {
  constexpr int S = 6;
  __shared__ uint64_t bars[2 * S];
  __shared__ uint32_t slot;
  const int warp = threadIdx.x / 32;
  if (threadIdx.x == 0) { for (int i = 0; i < 2 * S; ++i) mbar_init(smem_u32(&bars[i]), 1); fence_mbar_init(); }
  if (warp == 0) { tmem_alloc(smem_u32(&slot), 32); tmem_relinquish(); }
  tc_fence_before(); __syncthreads(); tc_fence_after();
  const uint32_t fb = smem_u32(&bars[0]), eb = smem_u32(&bars[S]);
  long long t0 = clock64();
  if (threadIdx.x == 32) {
    int s = 0; uint32_t ph = 0;
    for (int g = 0; g < iters; ++g) {
      while (!mbar_try_wait(eb + 8 * s, ph ^ 1)) {}
      mbar_arrive(fb + 8 * s);
      if (++s == S) { s = 0; ph ^= 1; }
    }
  } else if (threadIdx.x == 64) {
    int s = 0; uint32_t ph = 0;
    for (int g = 0; g < iters; ++g) {
      if (MODE == 1) { while (!test_wait(fb + 8 * s, ph)) {} }
      else { while (!mbar_try_wait(fb + 8 * s, ph)) {} }
      tc_fence_after();
      if (MODE == 2) mbar_arrive(eb + 8 * s); else mma_commit(eb + 8 * s);
      if (++s == S) { s = 0; ph ^= 1; }
    }
    out[MODE] = (clock64() - t0) / iters;
  }
  __syncthreads();
  if (warp == 0) tmem_dealloc(slot, 32);
}
int main() {
  long long *d; cudaMalloc(&d, 64);
  probe<0><<<1, 128>>>(4000, d); probe<1><<<1, 128>>>(4000, d); probe<2><<<1, 128>>>(4000, d);
  long long h[3]; cudaMemcpy(h, d, 24, cudaMemcpyDeviceToHost);
  printf("try_wait+commit %lld cyc/stage; test_wait+commit %lld; try_wait+arrive %lld (%s)\n", h[0], h[1], h[2],
         cudaGetErrorString(cudaGetLastError()));
  return 0;
}
