#include <initializer_list>
// banddiag.cpp — diagnostic (tooling): the loopback size-band parameters after
// mp_calibrate_bands next to the per-message time of back-to-back mp_xfer windows.
#include <cuda_runtime.h>

#include <chrono>
#include <cstdio>
#include <vector>

#include "mp.h"

int main() {
  mp_init_args a{};
  a.world = 1;
  a.n_loop_relays = 6;
  a.host_path = 1;
  a.heap_bytes = 16ull << 20;
  mp_ctx *ctx = nullptr;
  if (mp_init(&ctx, &a)) return 1;
  mp_model_opts o{};
  mp_get_options(ctx, &o);
  o.mode = MP_MODEL_B200;
  mp_set_options(ctx, &o);
  mp_calibrate_bands(ctx, nullptr, 0, 5);
  int nb = 0;
  mp_get_model_band(ctx, 0, 0, -1, nullptr, nullptr, nullptr, nullptr, &nb);
  for (int j = 0; j < nb; ++j) {
    uint64_t lo = 0;
    mp_path_params p[MP_MAX_PATHS];
    int np = 0;
    mp_port_params port;
    mp_get_model_band(ctx, 0, 0, j, &lo, p, &np, &port, nullptr);
    std::printf("{\"band\": %d, \"n_min\": %llu, \"direct_alpha_us\": %.3f, \"direct_beta_GBps\": %.1f}\n", j,
                static_cast<unsigned long long>(lo), p[0].alpha * 1e6, p[0].beta / 1e9);
  }
  const uint64_t maxn = 64ull << 20;
  void *s = nullptr, *d = nullptr;
  cudaMalloc(&s, maxn);
  cudaMalloc(&d, maxn);
  cudaStream_t st;
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  for (uint64_t n = 65536; n <= maxn; n <<= 4) {
    mp_config cfg;
    mp_select(ctx, 0, 0, n, 0, &cfg);
    for (int W : {1, 16, 64, 256}) {
      std::vector<float> v, hv;
      for (int r = 0; r < 8; ++r) {
        cudaEventRecord(e0, st);
        const auto h0 = std::chrono::steady_clock::now();
        for (int w = 0; w < W; ++w) mp_xfer(ctx, d, s, n, &cfg, st);
        const auto h1 = std::chrono::steady_clock::now();
        cudaEventRecord(e1, st);
        cudaEventSynchronize(e1);
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        v.push_back(ms * 1e3f / W);
        hv.push_back(static_cast<float>(std::chrono::duration<double>(h1 - h0).count() * 1e6 / W));
      }
      std::printf("{\"n\": %llu, \"W\": %d, \"us_per_msg\": [", static_cast<unsigned long long>(n), W);
      for (size_t i = 0; i < v.size(); ++i) std::printf("%s%.2f", i ? ", " : "", v[i]);
      std::printf("], \"host_us_per_launch\": [");
      for (size_t i = 0; i < hv.size(); ++i) std::printf("%s%.2f", i ? ", " : "", hv[i]);
      std::printf("], \"t_pred_us\": %.2f}\n", cfg.t_pred * 1e6);
    }
  }
  mp_finalize(ctx);
  return 0;
}
