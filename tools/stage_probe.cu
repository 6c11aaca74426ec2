// Global -> shared staging throughput of small CTAs (the tiny-layer kernels' operand staging):
// plain loads, 4-byte cp.async and 16-byte cp.async, 64 CTAs x 20k floats, timed in a graph.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_icpp_futhys18_b200/csrc tools/stage_probe.cu -o tools/stage_probe
#include <cstdio>
#include "../tools/tiny_kernels.cuh"
using namespace glp;
#define CK(x) do { cudaError_t e = (x); if (e) { printf("%d %s\n", __LINE__, cudaGetErrorString(e)); return 1; } } while (0)
__device__ unsigned long long stamp[4];
__device__ float sink;
template <int MODE>
__global__ void __launch_bounds__(256) stage(const float *src, int n) {
  extern __shared__ __align__(16) float sm[];
  unsigned long long t0, t1;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
  const float *s = src + (size_t)blockIdx.x * n;
  if (MODE == 0) {
    for (int i0 = threadIdx.x; i0 < n; i0 += 8 * 256) {
      float v[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) v[k] = i0 + k * 256 < n ? __ldg(s + i0 + k * 256) : 0.f;
#pragma unroll
      for (int k = 0; k < 8; ++k) if (i0 + k * 256 < n) sm[i0 + k * 256] = v[k];
    }
  } else if (MODE == 1) {
    const uint32_t d = smem_u32(sm);
    for (int i = threadIdx.x; i < n; i += 256) cp_async4(d + 4 * i, s + i, true);
    cp_async_commit(); cp_async_wait<0>();
  } else if (MODE == 2) {
    const uint32_t d = smem_u32(sm);
    for (int i = threadIdx.x; i < n / 4; i += 256) cp_async16(d + 16 * i, s + 4 * i, true);
    cp_async_commit(); cp_async_wait<0>();
  } else {   // tiny_stage_planes: 20 planes x 28 rows x 32 cols from 20 x 24 x 24, pad 4 (LeNet conv1 dgrad)
    tiny_stage_planes(sm, 20, 28, 32, s, 24 * 24, 20, 24, 24, -4, -4);
    tiny_stage_wait();
  }
  __syncthreads();
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t1));
  if (threadIdx.x == 0 && blockIdx.x == 0) { stamp[0] = t1 - t0; }
  if (sm[threadIdx.x * 7 % n] == 12345.f) sink = 1.f;
}
int main() {
  const int n = 20000, ctas = 64;
  float *src;
  CK(cudaMalloc(&src, (size_t)n * ctas * 4 * 4)); CK(cudaMemset(src, 0, (size_t)n * ctas * 16));
  cudaStream_t s; CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  cudaEvent_t e0, e1; CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  for (int mode = 0; mode < 4; ++mode) {
    auto fn = mode == 0 ? stage<0> : mode == 1 ? stage<1> : mode == 2 ? stage<2> : stage<3>;
    CK(cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, 100000));
    cudaGraph_t g; cudaGraphExec_t ge;
    CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal));
    for (int i = 0; i < 20; ++i) fn<<<ctas, 256, 100000, s>>>(src, n);
    CK(cudaStreamEndCapture(s, &g)); CK(cudaGraphInstantiate(&ge, g, 0));
    for (int i = 0; i < 10; ++i) CK(cudaGraphLaunch(ge, s));
    CK(cudaEventRecord(e0, s));
    for (int i = 0; i < 50; ++i) CK(cudaGraphLaunch(ge, s));
    CK(cudaEventRecord(e1, s)); CK(cudaEventSynchronize(e1));
    float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
    unsigned long long st[4]; CK(cudaMemcpyFromSymbol(st, stamp, sizeof(st)));
    printf("mode %d: %.2f us per kernel, CTA0 staging %.2f us\n", mode, ms * 1e3 / 1000, st[0] * 1e-3);
  }
  return 0;
}
