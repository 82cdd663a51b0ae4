// fp32 C++ CPU oracle of one decoder layer -- TEST / BASELINE INFRASTRUCTURE ONLY.
//
// The plain definition of the OPT-style pre-LN decoder layer (
// PAPER.md §4; reading R13), written out as loops in fp32 with
// OpenMP over independent outputs.  It exists for BASELINE.md's "CPU baseline plan"
// (C++17, -O3 -march=native -fopenmp, fp32 storage and accumulation, timed on the
// box's host cores) and is pinned against the fp64 numpy oracle (oracle/model.py,
// itself pinned to HF transformers) by tests/test_oracle_cpp.py.  It shares no code
// with the CUDA path; the product never loads it.
//
//   C2  LN(x) = (x - mean) / sqrt(var + eps) * g + b      (population variance)
//   C3  [q|k|v] = LN1(x) W_qkv + b_qkv ;  q *= d^-1/2      (after the bias)
//   C4  o_i = sum_j softmax_j(q_i . k_j, j <= pos(i)) v_j  (per head, max-subtracted)
//   C5  x1 = x + o W_o + b_o
//   C6  x2 = x1 + act(LN2(x1) W_1 + b_1) W_2 + b_2        act = ReLU | tanh-GELU
//
// Layout: every weight matrix is given as W^T, i.e. [N_out][K_in] row-major (row n holds
// the n-th column of the logical [K_in, N_out] matrix), so each output is one
// contiguous dot product; activations are [rows][features].  KV cache per sequence
// [heads][ctx][d].
//
// Two entry points:
//   ref_decoder_layer(...)  C ABI (ctypes) for the pin test;
//   main()                  the timing binary bench.py runs (weights from a hash).
#include <math.h>
#include <omp.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

#include <chrono>
#include <string>
#include <vector>

namespace {

// y[m][n] = sum_k x[m][k] * wt[n][k] + bias[n]     (C3/C5/C6 projections)
void linear(const float* x, int M, int K, const float* wt, const float* bias, int N, float* y) {
#pragma omp parallel for collapse(2) schedule(static)
  for (int n = 0; n < N; ++n)
    for (int m = 0; m < M; ++m) {
      const float* a = x + (size_t)m * K;
      const float* w = wt + (size_t)n * K;
      float acc = 0.f;
#pragma omp simd reduction(+ : acc)
      for (int k = 0; k < K; ++k) acc += a[k] * w[k];
      y[(size_t)m * N + n] = acc + (bias ? bias[n] : 0.f);
    }
}

// C2 LayerNorm of each row
void layer_norm(const float* x, int M, int H, const float* g, const float* b, float eps, float* y) {
#pragma omp parallel for schedule(static)
  for (int m = 0; m < M; ++m) {
    const float* r = x + (size_t)m * H;
    double s = 0;
    for (int i = 0; i < H; ++i) s += r[i];
    const float mean = (float)(s / H);
    double q = 0;
    for (int i = 0; i < H; ++i) q += (double)(r[i] - mean) * (r[i] - mean);
    const float rstd = 1.0f / sqrtf((float)(q / H) + eps);
    for (int i = 0; i < H; ++i) y[(size_t)m * H + i] = (r[i] - mean) * rstd * g[i] + b[i];
  }
}

float act_fn(float v, int act) {
  if (act == 1) return v > 0.f ? v : 0.f;                                                  // ReLU
  return 0.5f * v * (1.f + tanhf(0.7978845608028654f * (v + 0.044715f * v * v * v)));    // tanh-GELU
}

}  // namespace

extern "C" {

// One decoder layer over `s` new tokens per sequence at positions [start, start + s).
//   x [b*s][h] in, x2 [b*s][h] out; kcache / vcache [b][a][ctx_cap][d]: positions
//   [0, start) already hold the past, the new tokens' k, v are written at [start, start+s).
//   Weights transposed ([N_out][K_in]): wqkv_t [3h][h], wo_t [h][h], w1_t [f][h], w2_t [h][f].
int ref_decoder_layer(int b, int s, int start, int h, int a, int f, int act, float eps, const float* x,
                      const float* ln1_g, const float* ln1_b, const float* wqkv_t, const float* b_qkv,
                      const float* wo_t, const float* b_o, const float* ln2_g, const float* ln2_b,
                      const float* w1_t, const float* b_1, const float* w2_t, const float* b_2, float* kcache,
                      float* vcache, int ctx_cap, float* x2) {
  if (b <= 0 || s <= 0 || h % a || start + s > ctx_cap) return -22;
  const int M = b * s, d = h / a;
  std::vector<float> y((size_t)M * h), qkv((size_t)M * 3 * h), o((size_t)M * h), x1((size_t)M * h),
      z((size_t)M * f), p((size_t)M * h);
  layer_norm(x, M, h, ln1_g, ln1_b, eps, y.data());                       // C2
  linear(y.data(), M, h, wqkv_t, b_qkv, 3 * h, qkv.data());               // C3
  const float qs = 1.0f / sqrtf((float)d);
  for (int bi = 0; bi < b; ++bi)                                          // K/V of the new tokens
    for (int i = 0; i < s; ++i)
      for (int hd = 0; hd < a; ++hd)
        for (int e = 0; e < d; ++e) {
          const float* row = qkv.data() + (size_t)(bi * s + i) * 3 * h;
          const size_t c = (((size_t)bi * a + hd) * ctx_cap + start + i) * d + e;
          kcache[c] = row[h + hd * d + e];
          vcache[c] = row[2 * h + hd * d + e];
        }
#pragma omp parallel for collapse(3) schedule(static)
  for (int bi = 0; bi < b; ++bi)                                          // C4
    for (int hd = 0; hd < a; ++hd)
      for (int i = 0; i < s; ++i) {
        const float* q = qkv.data() + (size_t)(bi * s + i) * 3 * h + hd * d;
        const int n_keys = start + i + 1;                                 // causal: j <= pos(i)
        std::vector<float> sc(n_keys);
        float mx = -INFINITY;
        for (int j = 0; j < n_keys; ++j) {
          const float* k = kcache + (((size_t)bi * a + hd) * ctx_cap + j) * d;
          float acc = 0.f;
          for (int e = 0; e < d; ++e) acc += q[e] * qs * k[e];
          sc[j] = acc;
          mx = fmaxf(mx, acc);
        }
        float den = 0.f;
        for (int j = 0; j < n_keys; ++j) den += (sc[j] = expf(sc[j] - mx));
        float* out = o.data() + (size_t)(bi * s + i) * h + hd * d;
        for (int e = 0; e < d; ++e) out[e] = 0.f;
        for (int j = 0; j < n_keys; ++j) {
          const float* v = vcache + (((size_t)bi * a + hd) * ctx_cap + j) * d;
          const float pj = sc[j] / den;
          for (int e = 0; e < d; ++e) out[e] += pj * v[e];
        }
      }
  linear(o.data(), M, h, wo_t, b_o, h, p.data());                         // C5
  for (size_t i = 0; i < (size_t)M * h; ++i) x1[i] = x[i] + p[i];
  layer_norm(x1.data(), M, h, ln2_g, ln2_b, eps, y.data());               // C6
  linear(y.data(), M, h, w1_t, b_1, f, z.data());
  for (size_t i = 0; i < (size_t)M * f; ++i) z[i] = act_fn(z[i], act);
  linear(z.data(), M, f, w2_t, b_2, h, p.data());
  for (size_t i = 0; i < (size_t)M * h; ++i) x2[i] = x1[i] + p[i];
  return 0;
}

}  // extern "C"

#ifndef LAYER_REF_NO_MAIN
// Timing binary (BASELINE.md "CPU baseline plan"): one layer of the given shape with
// hashed weights (values do not change the work), a prefill over [batch, prompt] and
// decode steps at context `ctx`; prints one JSON line.
static void fill(std::vector<float>& v, uint64_t seed, float scale) {
#pragma omp parallel for schedule(static)
  for (size_t i = 0; i < v.size(); ++i) {
    uint64_t x = (i + 1) * 0x9E3779B97F4A7C15ull + seed;
    x ^= x >> 30; x *= 0xBF58476D1CE4E5B9ull; x ^= x >> 27; x *= 0x94D049BB133111EBull; x ^= x >> 31;
    v[i] = ((int64_t)(x >> 40) - (1 << 23)) * (scale / (1 << 23));
  }
}

int main(int argc, char** argv) {
  int h = 5120, a = 40, f = 20480, act = 1, b = 2, s = 128, steps = 4, ctx = 144;
  double budget = 12.0;
  for (int i = 1; i + 1 < argc; i += 2) {
    std::string k = argv[i];
    const char* v = argv[i + 1];
    if (k == "--hidden") h = atoi(v);
    else if (k == "--heads") a = atoi(v);
    else if (k == "--ffn") f = atoi(v);
    else if (k == "--act") act = std::string(v) == "relu" ? 1 : 2;
    else if (k == "--batch") b = atoi(v);
    else if (k == "--prompt") s = atoi(v);
    else if (k == "--decode-steps") steps = atoi(v);
    else if (k == "--ctx") ctx = atoi(v);
    else if (k == "--budget-s") budget = atof(v);
  }
  const int d = h / a, cap = (ctx > s ? ctx : s) + 1;
  std::vector<float> wqkv((size_t)3 * h * h), wo((size_t)h * h), w1((size_t)f * h), w2((size_t)h * f);
  std::vector<float> bq(3 * h), bo(h), b1(f), b2(h), g(h, 1.f), be(h, 0.f);
  fill(wqkv, 1, 0.02f); fill(wo, 2, 0.01f); fill(w1, 3, 0.02f); fill(w2, 4, 0.01f);
  fill(bq, 5, 0.01f); fill(bo, 6, 0.01f); fill(b1, 7, 0.01f); fill(b2, 8, 0.01f);
  std::vector<float> kc((size_t)b * a * cap * d), vc((size_t)b * a * cap * d);
  fill(kc, 9, 0.1f); fill(vc, 10, 0.1f);
  std::vector<float> x((size_t)b * s * h), out((size_t)b * s * h);
  fill(x, 11, 0.1f);
  using clk = std::chrono::steady_clock;
  // one untimed warm-up decode step, then the prefill, then the timed decode steps
  ref_decoder_layer(b, 1, ctx - 1, h, a, f, act, 1e-5f, x.data(), g.data(), be.data(), wqkv.data(), bq.data(),
                    wo.data(), bo.data(), g.data(), be.data(), w1.data(), b1.data(), w2.data(), b2.data(), kc.data(),
                    vc.data(), cap, out.data());
  auto t0 = clk::now();
  ref_decoder_layer(b, s, 0, h, a, f, act, 1e-5f, x.data(), g.data(), be.data(), wqkv.data(), bq.data(), wo.data(),
                    bo.data(), g.data(), be.data(), w1.data(), b1.data(), w2.data(), b2.data(), kc.data(), vc.data(),
                    cap, out.data());
  const double t_pf = std::chrono::duration<double>(clk::now() - t0).count();
  int n = 0;
  t0 = clk::now();
  while (n < steps) {
    ref_decoder_layer(b, 1, ctx - 1, h, a, f, act, 1e-5f, x.data(), g.data(), be.data(), wqkv.data(), bq.data(),
                      wo.data(), bo.data(), g.data(), be.data(), w1.data(), b1.data(), w2.data(), b2.data(),
                      kc.data(), vc.data(), cap, out.data());
    ++n;
    if (std::chrono::duration<double>(clk::now() - t0).count() > budget) break;
  }
  const double t_dc = std::chrono::duration<double>(clk::now() - t0).count() / n;
  printf("{\"threads\": %d, \"prefill_s\": %.6f, \"decode_step_s\": %.6f, \"decode_steps\": %d, \"hidden\": %d, "
         "\"batch\": %d, \"prompt\": %d, \"ctx\": %d}\n",
         omp_get_max_threads(), t_pf, t_dc, n, h, b, s, ctx);
  return 0;
}
#endif
