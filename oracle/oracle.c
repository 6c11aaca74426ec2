/*
 * ORACLE — TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, obviously-correct CPU definition of what the GLP4NN hot path
 * computes: Caffe-style convolution-layer training (forward, backward-data,
 * backward-filter + bias gradient), written as direct nested loops with fp64
 * accumulation.  Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load this library.  It shares no
 * code, header, table or helper with the CUDA path (paper_conf_icpp_futhys18_b200/csrc).
 *
 * Passages followed (PAPER.md line numbers, "P<n>"):
 *   - Alg. 1 forward propagation, P82-99: top[f(n,.)] = BLAS(weight, bias, bottom[g(n,.)]).
 *     For a conv layer this is im2col -> GEMM + bias (P173: kernels im2col, sgemm, gemmk).
 *     Its plain definition (what im2col+GEMM reaches exactly up to rounding order) is
 *         y[n,co,ho,wo] = b[co] + sum_{ci,kh,kw} W[co,ci,kh,kw] * x[n,ci,ho*S-P+kh, wo*S-P+kw]
 *     with x = 0 outside the image (zero padding, P316 "P is the number of pixels to add to
 *     each side of the input").  Cross-correlation, no filter flip (reading R1).
 *   - Alg. 2 backward propagation, P101-121: bottom_gradient = BLAS(top_gradient, weight),
 *     i.e. GEMM W^T * dy -> col2im.  Plain definition = the adjoint of the forward map:
 *         dx[n,ci,h,w] = sum over every (co,ho,wo,kh,kw) with ho*S-P+kh == h, wo*S-P+kw == w
 *                        of W[co,ci,kh,kw] * dy[n,co,ho,wo].
 *     Implemented here as a SCATTER-ADD (col2im order), deliberately a different loop order
 *     from the GPU gather.
 *   - Parameter gradients, P129 ("a gradient value is computed ... for parameter update") and
 *     BASELINE.json north_star ("backward-filter GEMMs summed over the samples of a batch"):
 *         dW[co,ci,kh,kw] = sum_{n,ho,wo} dy[n,co,ho,wo] * x[n,ci,ho*S-P+kh, wo*S-P+kw]
 *         db[co]          = sum_{n,ho,wo} dy[n,co,ho,wo]
 *   - Output size, Table 5 parameter definitions P316: H_o = floor((H + 2P - F_h)/S) + 1
 *     (reading R2: floor, as Caffe's conv layer).
 *   - im2col layout (P173 names the im2col kernel): col[(ci*K_h+kh)*K_w+kw][ho*W_o+wo]
 *     (reading R6, Caffe's layout).
 *
 * Layouts: x, y, dx, dy NCHW; W [C_o][C_i][K_h][K_w]; b [C_o].  Inputs are the fp32 arrays
 * handed to the GPU; outputs are fp64.  When `absmode` is non-zero every product uses |a|*|b|
 * (the condition-number denominator sum|a||b| used for condition-aware error reports).
 *
 * Parallelism: OpenMP over OUTPUT elements only (never over a reduction), so the result is
 * bitwise independent of the thread count (pinned by tests/test_oracle_pins.py).
 */
#include <math.h>
#include <stddef.h>
#include <stdint.h>
#ifdef _OPENMP
#include <omp.h>
#endif

static int out_dim(int in, int k, int s, int p) { return (in + 2 * p - k) / s + 1; }

static double mulp(double a, double b, int absmode) { return absmode ? fabs(a) * fabs(b) : a * b; }

int oracle_version(void) { return 1; }

void oracle_set_threads(int n) {
#ifdef _OPENMP
  if (n > 0) omp_set_num_threads(n);
#else
  (void)n;
#endif
}

int oracle_max_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

/* Alg. 1 (P82-99) for a conv layer: direct definition, fp64 accumulate. */
void oracle_conv_fwd(int N, int C, int H, int W, int Co, int Kh, int Kw, int Sh, int Sw, int Ph,
                     int Pw, const float *x, const float *w, const float *b, double *y,
                     int absmode) {
  const int Ho = out_dim(H, Kh, Sh, Ph), Wo = out_dim(W, Kw, Sw, Pw);
  const long long total = (long long)N * Co;
#pragma omp parallel for schedule(static)
  for (long long nc = 0; nc < total; ++nc) {
    const int n = (int)(nc / Co), co = (int)(nc % Co);
    for (int ho = 0; ho < Ho; ++ho)
      for (int wo = 0; wo < Wo; ++wo) {
        double acc = 0.0;
        for (int ci = 0; ci < C; ++ci)
          for (int kh = 0; kh < Kh; ++kh) {
            const int ih = ho * Sh - Ph + kh;
            if (ih < 0 || ih >= H) continue;
            for (int kw = 0; kw < Kw; ++kw) {
              const int iw = wo * Sw - Pw + kw;
              if (iw < 0 || iw >= W) continue;
              const double wv = w[(((size_t)co * C + ci) * Kh + kh) * Kw + kw];
              const double xv = x[(((size_t)n * C + ci) * H + ih) * W + iw];
              acc += mulp(wv, xv, absmode);
            }
          }
        if (b) acc += absmode ? fabs((double)b[co]) : (double)b[co];
        y[(((size_t)n * Co + co) * Ho + ho) * Wo + wo] = acc;
      }
  }
}

/* Alg. 2 (P101-121): GEMM W^T dy followed by col2im, written as a scatter-add over every
 * (co, ho, wo, ci, kh, kw).  One OpenMP task per sample n owns dx[n], so no races. */
void oracle_conv_bwd_data(int N, int C, int H, int W, int Co, int Kh, int Kw, int Sh, int Sw,
                          int Ph, int Pw, const float *dy, const float *w, double *dx,
                          int absmode) {
  const int Ho = out_dim(H, Kh, Sh, Ph), Wo = out_dim(W, Kw, Sw, Pw);
#pragma omp parallel for schedule(static)
  for (int n = 0; n < N; ++n) {
    double *dxn = dx + (size_t)n * C * H * W;
    for (size_t i = 0; i < (size_t)C * H * W; ++i) dxn[i] = 0.0;
    for (int co = 0; co < Co; ++co)
      for (int ho = 0; ho < Ho; ++ho)
        for (int wo = 0; wo < Wo; ++wo) {
          const double g = dy[(((size_t)n * Co + co) * Ho + ho) * Wo + wo];
          for (int ci = 0; ci < C; ++ci)
            for (int kh = 0; kh < Kh; ++kh) {
              const int ih = ho * Sh - Ph + kh;
              if (ih < 0 || ih >= H) continue;
              for (int kw = 0; kw < Kw; ++kw) {
                const int iw = wo * Sw - Pw + kw;
                if (iw < 0 || iw >= W) continue;
                const double wv = w[(((size_t)co * C + ci) * Kh + kh) * Kw + kw];
                dxn[((size_t)ci * H + ih) * W + iw] += mulp(wv, g, absmode);
              }
            }
        }
  }
}

/* Parameter gradients (P129; north_star "summed over the samples of a batch").
 * db may be NULL.  One OpenMP task per (co, ci) owns its dW entries. */
void oracle_conv_bwd_filter(int N, int C, int H, int W, int Co, int Kh, int Kw, int Sh, int Sw,
                            int Ph, int Pw, const float *x, const float *dy, double *dw,
                            double *db, int absmode) {
  const int Ho = out_dim(H, Kh, Sh, Ph), Wo = out_dim(W, Kw, Sw, Pw);
  const long long total = (long long)Co * C;
#pragma omp parallel for schedule(static)
  for (long long cc = 0; cc < total; ++cc) {
    const int co = (int)(cc / C), ci = (int)(cc % C);
    for (int kh = 0; kh < Kh; ++kh)
      for (int kw = 0; kw < Kw; ++kw) {
        double acc = 0.0;
        for (int n = 0; n < N; ++n)
          for (int ho = 0; ho < Ho; ++ho) {
            const int ih = ho * Sh - Ph + kh;
            if (ih < 0 || ih >= H) continue;
            for (int wo = 0; wo < Wo; ++wo) {
              const int iw = wo * Sw - Pw + kw;
              if (iw < 0 || iw >= W) continue;
              const double g = dy[(((size_t)n * Co + co) * Ho + ho) * Wo + wo];
              const double xv = x[(((size_t)n * C + ci) * H + ih) * W + iw];
              acc += mulp(g, xv, absmode);
            }
          }
        dw[(((size_t)co * C + ci) * Kh + kh) * Kw + kw] = acc;
      }
  }
  if (db) {
#pragma omp parallel for schedule(static)
    for (int co = 0; co < Co; ++co) {
      double acc = 0.0;
      for (int n = 0; n < N; ++n)
        for (int p = 0; p < Ho * Wo; ++p) {
          const double g = dy[((size_t)n * Co + co) * Ho * Wo + p];
          acc += absmode ? fabs(g) : g;
        }
      db[co] = acc;
    }
  }
}

/* Bias gradient alone (P129): db[co] = sum_{n,ho,wo} dy[n,co,ho,wo], the same loops as the db
 * part of oracle_conv_bwd_filter (for full-size checks where the whole dW would be too slow). */
void oracle_conv_db(int N, int Co, int Ho, int Wo, const float *dy, double *db) {
#pragma omp parallel for schedule(static)
  for (int co = 0; co < Co; ++co) {
    double acc = 0.0;
    for (int n = 0; n < N; ++n)
      for (int p = 0; p < Ho * Wo; ++p) acc += (double)dy[((size_t)n * Co + co) * Ho * Wo + p];
    db[co] = acc;
  }
}

/* Caffe im2col of ONE sample (P173 "im2col"): col[(ci*Kh+kh)*Kw+kw][ho*Wo+wo]. Pure data
 * movement, so the output keeps the input's fp32 values exactly. */
void oracle_im2col(int C, int H, int W, int Kh, int Kw, int Sh, int Sw, int Ph, int Pw,
                   const float *x_n, float *col) {
  const int Ho = out_dim(H, Kh, Sh, Ph), Wo = out_dim(W, Kw, Sw, Pw);
  for (int ci = 0; ci < C; ++ci)
    for (int kh = 0; kh < Kh; ++kh)
      for (int kw = 0; kw < Kw; ++kw) {
        const size_t row = ((size_t)ci * Kh + kh) * Kw + kw;
        for (int ho = 0; ho < Ho; ++ho)
          for (int wo = 0; wo < Wo; ++wo) {
            const int ih = ho * Sh - Ph + kh, iw = wo * Sw - Pw + kw;
            float v = 0.0f;
            if (ih >= 0 && ih < H && iw >= 0 && iw < W) v = x_n[((size_t)ci * H + ih) * W + iw];
            col[row * Ho * Wo + (size_t)ho * Wo + wo] = v;
          }
      }
}

/* One sampled element of the parameter gradient (same definition as oracle_conv_bwd_filter),
 * for parity at full benchmark sizes where the whole dW would take minutes. */
double oracle_conv_bwd_filter_at(int N, int C, int H, int W, int Co, int Kh, int Kw, int Sh,
                                 int Sw, int Ph, int Pw, const float *x, const float *dy, int co,
                                 int ci, int kh, int kw) {
  const int Ho = out_dim(H, Kh, Sh, Ph), Wo = out_dim(W, Kw, Sw, Pw);
  double acc = 0.0;
  for (int n = 0; n < N; ++n)
    for (int ho = 0; ho < Ho; ++ho) {
      const int ih = ho * Sh - Ph + kh;
      if (ih < 0 || ih >= H) continue;
      for (int wo = 0; wo < Wo; ++wo) {
        const int iw = wo * Sw - Pw + kw;
        if (iw < 0 || iw >= W) continue;
        acc += (double)dy[(((size_t)n * Co + co) * Ho + ho) * Wo + wo] *
               (double)x[(((size_t)n * C + ci) * H + ih) * W + iw];
      }
    }
  return acc;
}
