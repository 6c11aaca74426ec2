// Standalone correctness/timing probe of the tiny-layer kernels (csrc/tiny.cuh): forward,
// backward-data and filter-gradient passes on LeNet / CIFAR-10 shapes against a double CPU
// reference.  Kernel durations: run under `ncu --metrics gpu__time_duration.sum`.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I paper_conf_icpp_futhys18_b200/csrc tools/tiny_probe.cu -o tools/tiny_probe
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <vector>

#define TINY_PROBE_TIMING
#include "../tools/tiny_kernels.cuh"
using namespace glp;
#define CK(x) do { cudaError_t e = (x); if (e) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1);} } while (0)

template <int K>
void run(const char *name, int N, int C, int H, int W, int Co, int Pd, int reps, int target = 400) {
  ConvGeom g{N, C, H, W, Co, K, K, 1, 1, Pd, Pd, H + 2 * Pd - K + 1, W + 2 * Pd - K + 1, C, Co};
  const int P = g.Ho * g.Wo, CKK = C * K * K;
  std::vector<float> x((size_t)N * C * H * W), w((size_t)Co * CKK), b(Co), dy((size_t)N * Co * P);
  srand(1);
  for (auto &v : x) v = rand() / (float)RAND_MAX - 0.5f;
  for (auto &v : w) v = rand() / (float)RAND_MAX - 0.5f;
  for (auto &v : b) v = rand() / (float)RAND_MAX - 0.5f;
  for (auto &v : dy) v = rand() / (float)RAND_MAX - 0.5f;
  float *d_x, *d_w, *d_b, *d_dy, *d_y, *d_dx, *d_dw, *d_db;
  CK(cudaMalloc(&d_x, x.size() * 4)); CK(cudaMalloc(&d_w, w.size() * 4)); CK(cudaMalloc(&d_b, 4 * Co));
  CK(cudaMalloc(&d_dy, dy.size() * 4)); CK(cudaMalloc(&d_y, dy.size() * 4)); CK(cudaMalloc(&d_dx, x.size() * 4));
  CK(cudaMalloc(&d_dw, w.size() * 4)); CK(cudaMalloc(&d_db, 4 * Co));
  CK(cudaMemcpy(d_x, x.data(), x.size() * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(d_w, w.data(), w.size() * 4, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(d_b, b.data(), 4 * Co, cudaMemcpyHostToDevice));
  CK(cudaMemcpy(d_dy, dy.data(), dy.size() * 4, cudaMemcpyHostToDevice));
  const TinyCorr tf = tiny_corr_config(g, 0), td = tiny_corr_config(g, 1);
  const TinyWgrad tw = tiny_wgrad_config(g, target);
  const size_t wsb = tiny_wgrad_ws_bytes(tw, K);
  char *ws;
  CK(cudaMalloc(&ws, wsb)); CK(cudaMemset(ws, 0, wsb));
  const size_t E = (size_t)tw.islice * K * 4, units = (size_t)tw.nslices * tw.nchunks, ngr = (tw.nchunks + 7) / 8;
  float *part = (float *)ws, *gpart = part + units * E;
  unsigned *tk = (unsigned *)(gpart + tw.nslices * ngr * E);
  CK(cudaMemset(tk, 0, 4 * tw.nslices * (ngr + 1)));
  const int fsm = 4 * tiny_corr_smem_floats(tf, K), dsm = 4 * tiny_corr_smem_floats(td, K);
  const int wsm = 4 * tiny_wgrad_smem(tw, K).total;
  CK(cudaFuncSetAttribute(tiny_corr<0, K, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, fsm));
  CK(cudaFuncSetAttribute(tiny_corr<0, K, 1>, cudaFuncAttributeMaxDynamicSharedMemorySize, dsm));
  CK(cudaFuncSetAttribute(tiny_wgrad<0, K>, cudaFuncAttributeMaxDynamicSharedMemorySize, wsm));
  printf("%s: fwd grid %dx%d gpc %d R %d smem %d | dgrad grid %dx%d gpc %d R %d smem %d | wgrad slices %d x chunks %d (spc %d rows %d PH %d islice %d) smem %d ws %zu\n",
         name, ((Co + 3) / 4 + tf.gpc - 1) / tf.gpc, N, tf.gpc, tf.R, fsm, ((C + 3) / 4 + td.gpc - 1) / td.gpc, N, td.gpc, td.R, dsm,
         tw.nslices, tw.nchunks, tw.spc, tw.rows, tw.PH, tw.islice, wsm, wsb);
  for (int r = 0; r < reps; ++r) {
    tiny_corr<0, K, 0><<<dim3(((Co + 3) / 4 + tf.gpc - 1) / tf.gpc, N), TINY_THREADS, fsm>>>(tf, d_x, d_w, d_b, d_y);
    tiny_corr<0, K, 1><<<dim3(((C + 3) / 4 + td.gpc - 1) / td.gpc, N), TINY_THREADS, dsm>>>(td, d_dy, d_w, nullptr, d_dx);
    tiny_wgrad<0, K><<<(unsigned)units, TINY_THREADS, wsm>>>(tw, d_x, d_dy, part, gpart, tk, d_dw, d_db, 0);
  }
  CK(cudaDeviceSynchronize()); CK(cudaGetLastError());
  {  // back-to-back launches (warm caches): average time per launch
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1));
    for (int which = 0; which < 3; ++which) {
      auto L = [&](cudaStream_t st) {
        if (which == 0) tiny_corr<0, K, 0><<<dim3(((Co + 3) / 4 + tf.gpc - 1) / tf.gpc, N), TINY_THREADS, fsm, st>>>(tf, d_x, d_w, d_b, d_y);
        else if (which == 1) tiny_corr<0, K, 1><<<dim3(((C + 3) / 4 + td.gpc - 1) / td.gpc, N), TINY_THREADS, dsm, st>>>(td, d_dy, d_w, nullptr, d_dx);
        else tiny_wgrad<0, K><<<(unsigned)units, TINY_THREADS, wsm, st>>>(tw, d_x, d_dy, part, gpart, tk, d_dw, d_db, 0);
      };
      // a graph of 20 launches replayed 100 times (stream launches are host-bound at ~2 us)
      cudaStream_t cs;
      CK(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
      cudaGraph_t gr;
      cudaGraphExec_t ge;
      CK(cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal));
      cudaStream_t save = 0;
      (void)save;
      for (int i = 0; i < 20; ++i) L(cs);
      CK(cudaStreamEndCapture(cs, &gr));
      CK(cudaGraphInstantiate(&ge, gr, 0));
      for (int i = 0; i < 20; ++i) CK(cudaGraphLaunch(ge, cs));
      CK(cudaEventRecord(e0, cs));
      for (int i = 0; i < 100; ++i) CK(cudaGraphLaunch(ge, cs));
      CK(cudaEventRecord(e1, cs)); CK(cudaEventSynchronize(e1));
      float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
      unsigned long long st[8];
      CK(cudaMemcpyFromSymbol(st, tiny_stamp, sizeof(st)));
      if (which < 2) printf("    CTA0 (last launch): staged %.2f us, computed %.2f us after start\n", (st[1] - st[0]) * 1e-3, (st[2] - st[0]) * 1e-3);
      else printf("    CTA0 (last launch): staged %.2f us, computed %.2f, partial %.2f us after start\n", (st[1] - st[0]) * 1e-3, (st[2] - st[0]) * 1e-3, (st[3] - st[0]) * 1e-3);
      printf("  %s: %.2f us per kernel (graph of 20)\n", which == 0 ? "fwd" : which == 1 ? "dgrad" : "wgrad", ms * 1e3 / 2000);
      CK(cudaGraphExecDestroy(ge)); CK(cudaGraphDestroy(gr)); CK(cudaStreamDestroy(cs));
    }
  }
  std::vector<float> y(dy.size()), gx(x.size()), gw(w.size()), gb(Co);
  CK(cudaMemcpy(y.data(), d_y, y.size() * 4, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(gx.data(), d_dx, gx.size() * 4, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(gw.data(), d_dw, gw.size() * 4, cudaMemcpyDeviceToHost));
  CK(cudaMemcpy(gb.data(), d_db, 4 * Co, cudaMemcpyDeviceToHost));
  std::vector<double> ry(y.size()), rx(x.size(), 0.0), rw(w.size(), 0.0), rb(Co, 0.0);
  for (int n = 0; n < N; ++n)
    for (int co = 0; co < Co; ++co)
      for (int p = 0; p < P; ++p) {
        const int oh = p / g.Wo, ow = p % g.Wo;
        double a = b[co];
        const double d = dy[((size_t)n * Co + co) * P + p];
        rb[co] += d;
        for (int c = 0; c < C; ++c)
          for (int kh = 0; kh < K; ++kh)
            for (int kw = 0; kw < K; ++kw) {
              const int ih = oh - Pd + kh, iw = ow - Pd + kw;
              if (ih < 0 || ih >= H || iw < 0 || iw >= W) continue;
              const size_t xi = (((size_t)n * C + c) * H + ih) * W + iw, wi = (size_t)co * CKK + (c * K + kh) * K + kw;
              a += w[wi] * (double)x[xi];
              rw[wi] += d * x[xi];
              rx[xi] += d * w[wi];
            }
        ry[((size_t)n * Co + co) * P + p] = a;
      }
  auto err = [](const std::vector<float> &a, const std::vector<double> &r) {
    double e = 0, nn = 0;
    for (size_t i = 0; i < a.size(); ++i) { e += (a[i] - r[i]) * (a[i] - r[i]); nn += r[i] * r[i]; }
    return sqrt(e / nn);
  };
  printf("  err y %.2e dx %.2e dW %.2e db %.2e\n", err(y, ry), err(gx, rx), err(gw, rw), err(gb, rb));
  CK(cudaFree(d_x)); CK(cudaFree(d_w)); CK(cudaFree(d_b)); CK(cudaFree(d_dy)); CK(cudaFree(d_y));
  CK(cudaFree(d_dx)); CK(cudaFree(d_dw)); CK(cudaFree(d_db)); CK(cudaFree(ws));
}

int main(int argc, char **argv) {
  const int reps = argc > 1 ? atoi(argv[1]) : 3;
  for (int tg : {64, 128, 192, 256, 400}) run<5>("lenet conv1", 64, 1, 28, 28, 20, 0, reps, tg);
  for (int tg : {64, 128, 256}) run<5>("lenet conv2", 64, 20, 12, 12, 50, 0, reps, tg);
  if (reps > 0) return 0;
  run<5>("lenet conv2", 64, 20, 12, 12, 50, 0, reps);
  run<5>("cifar conv1", 100, 3, 32, 32, 32, 2, reps);
  run<5>("cifar conv2", 100, 32, 16, 16, 32, 2, reps);
  run<5>("cifar conv3", 100, 32, 8, 8, 64, 2, reps);
  run<3>("k3 ragged", 5, 7, 13, 11, 9, 1, reps);
  return 0;
}
