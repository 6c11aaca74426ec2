// Back-to-back launch cadence of trivial kernels (stream launches and a captured graph):
// does a kernel's wall time quantise, and what does griddepcontrol.wait cost without PDL?
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 tools/launch_probe.cu -o tools/launch_probe
#include <cstdio>
#define CK(x) do { cudaError_t e = (x); if (e) { printf("%d %s\n", __LINE__, cudaGetErrorString(e)); return 1; } } while (0)
__global__ void k_empty() {}
__global__ void k_pdl() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__global__ void k_spin(int ns) { long long t0 = clock64(); while (clock64() - t0 < ns) {} }
__global__ void k_ldst(const float *a, float *b) { b[threadIdx.x + blockIdx.x * blockDim.x] = a[threadIdx.x + blockIdx.x * blockDim.x] + 1.f; }
int main() {
  float *a, *b;
  CK(cudaMalloc(&a, 1 << 24)); CK(cudaMalloc(&b, 1 << 24));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
  cudaStream_t s; CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  auto T = [&](const char *nm, auto L) {
    for (int i = 0; i < 500; ++i) L();
    cudaEventRecord(e0, s);
    for (int i = 0; i < 4000; ++i) L();
    cudaEventRecord(e1, s); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    printf("%-40s %.3f us per launch\n", nm, ms * 1e3 / 4000);
  };
  T("empty <<<1,32>>>", [&] { k_empty<<<1, 32, 0, s>>>(); });
  T("empty <<<148,256>>>", [&] { k_empty<<<148, 256, 0, s>>>(); });
  T("pdl wait <<<148,256>>>", [&] { k_pdl<<<148, 256, 0, s>>>(); });
  T("ldst 4MB <<<4096,256>>>", [&] { k_ldst<<<4096, 256, 0, s>>>(a, b); });
  for (int c : {1000, 2000, 4000, 6000, 8000})
    { char nm[64]; snprintf(nm, 64, "spin %d cycles <<<148,32>>>", c); T(nm, [&] { k_spin<<<148, 32, 0, s>>>(c); }); }
  T("empty smem 100KB <<<148,256>>>", [&] { k_empty<<<148, 256, 100000, s>>>(); });
  // graph of 20 empty kernels
  cudaGraph_t g; cudaGraphExec_t ge;
  CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal));
  for (int i = 0; i < 20; ++i) k_empty<<<148, 256, 0, s>>>();
  CK(cudaStreamEndCapture(s, &g)); CK(cudaGraphInstantiate(&ge, g, 0));
  T("graph of 20 empty (per replay)", [&] { cudaGraphLaunch(ge, s); });
  CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal));
  for (int i = 0; i < 20; ++i) k_spin<<<148, 32, 0, s>>>(3000);
  CK(cudaStreamEndCapture(s, &g)); CK(cudaGraphInstantiate(&ge, g, 0));
  T("graph of 20 spin3000 (per replay)", [&] { cudaGraphLaunch(ge, s); });
  return 0;
}
