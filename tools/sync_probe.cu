// Microbenchmark: latency of the pipeline handshakes used by igemm (diagnostic tool).
//  (1) tcgen05.commit -> mbarrier -> wait (no MMA pending)
//  (2) mbarrier.arrive -> wait by another warp (ping-pong round trip)
//  (3) ring of S stages: producer thread (arrive full / wait empty) vs consumer thread
//      (wait full / tcgen05.commit empty) -- cycles per stage
#include <cstdio>
#include "../paper_conf_icpp_futhys18_b200/csrc/ptx.cuh"
using namespace glp;
__global__ void __launch_bounds__(128, 1) probe(int iters, int S, long long *out) {
  __shared__ uint64_t bars[40];
  __shared__ uint32_t slot;
  const int warp = threadIdx.x / 32, lane = threadIdx.x % 32;
  if (threadIdx.x == 0) { for (int i = 0; i < 40; ++i) mbar_init(smem_u32(&bars[i]), 1); fence_mbar_init(); }
  if (warp == 0) { tmem_alloc(smem_u32(&slot), 32); tmem_relinquish(); }
  tc_fence_before(); __syncthreads(); tc_fence_after();
  // (1) commit latency
  if (threadIdx.x == 0) {
    long long t0 = clock64();
    for (int i = 0; i < iters; ++i) { mma_commit(smem_u32(&bars[39])); mbar_wait(smem_u32(&bars[39]), i & 1); }
    out[0] = (clock64() - t0) / iters;
  }
  __syncthreads();
  // (3) ring
  auto full = [&](int s) { return smem_u32(&bars[s]); };
  auto empty = [&](int s) { return smem_u32(&bars[16 + s]); };
  long long t0 = clock64();
  if (threadIdx.x == 32) {        // producer
    for (int g = 0; g < iters; ++g) { int s = g % S; mbar_wait(empty(s), ((g / S) & 1) ^ 1); mbar_arrive(full(s)); }
  } else if (threadIdx.x == 64) { // consumer with commit release
    for (int g = 0; g < iters; ++g) { int s = g % S; mbar_wait(full(s), (g / S) & 1); tc_fence_after(); mma_commit(empty(s)); }
    out[1] = (clock64() - t0) / iters;
  }
  __syncthreads();
  if (threadIdx.x == 0) { for (int i = 0; i < 40; ++i) mbar_init(smem_u32(&bars[i]), 1); fence_mbar_init(); }
  __syncthreads();
  t0 = clock64();
  if (threadIdx.x == 32) {
    for (int g = 0; g < iters; ++g) { int s = g % S; mbar_wait(empty(s), ((g / S) & 1) ^ 1); mbar_arrive(full(s)); }
  } else if (threadIdx.x == 64) { // consumer with plain arrive release
    for (int g = 0; g < iters; ++g) { int s = g % S; mbar_wait(full(s), (g / S) & 1); mbar_arrive(empty(s)); }
    out[2] = (clock64() - t0) / iters;
  }
  __syncthreads();
  if (warp == 0) tmem_dealloc(slot, 32);
}
int main() {
  long long *d; cudaMalloc(&d, 64);
  for (int S : {1, 2, 4, 8}) {
    probe<<<1, 128>>>(2000, S, d);
    long long h[3]; cudaMemcpy(h, d, 24, cudaMemcpyDeviceToHost);
    printf("S=%d: commit->wait %lld cyc; ring(commit release) %lld cyc/stage; ring(arrive release) %lld cyc/stage (%s)\n",
           S, h[0], h[1], h[2], cudaGetErrorString(cudaGetLastError()));
  }
  return 0;
}
