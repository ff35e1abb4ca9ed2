// omb_window.cpp — NEXT f2 measurement (readings C24/C25): osu_bw's real loop on the
// loopback engine through the C ABI — per iteration a window of w back-to-back
// mp_xfer, then a 4-byte ack and a host wait (MPI_Waitall + the ack),
// timed with the host clock as OMB does — next to what the model predicts:
//   pred_msg_GBps   : the paper's per-message model (reading C15), n / T(mp_select config)
//   pred_win_GBps   : the window model, w·n / (T^w(mp_select_window config) + one ack)
// and the measured rate of both configs (mp_select vs mp_select_window).
//   g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include scripts/omb_window.cpp \
//       -L paper_conf_sc_sojoodiasfga25_b200/_lib -lmpx -L /usr/local/cuda/lib64 -lcudart \
//       -Wl,-rpath,'$ORIGIN/../paper_conf_sc_sojoodiasfga25_b200/_lib' -o scripts/omb_window
//   ./scripts/omb_window [bands]   → one JSON line of calibrated parameters, then one per (size, window)
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "mp.h"

#define CK(x)                                                                        \
  do {                                                                               \
    cudaError_t e = (x);                                                             \
    if (e != cudaSuccess) {                                                          \
      std::fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); \
      std::exit(1);                                                                  \
    }                                                                                \
  } while (0)
#define MK(x)                                                                                        \
  do {                                                                                               \
    int s = (x);                                                                                     \
    if (s) {                                                                                         \
      std::fprintf(stderr, "%s:%d %s %s\n", __FILE__, __LINE__, mp_strerror(s), mp_last_error(ctx)); \
      std::exit(1);                                                                                  \
    }                                                                                                \
  } while (0)

static void print_cfg(const char *key, const mp_config &c) {
  std::printf(", \"%s\": [", key);
  for (int i = 0; i < c.npaths; ++i)
    std::printf("%s[%llu, %u]", i ? ", " : "", static_cast<unsigned long long>(c.bytes[i]), c.chunks[i]);
  std::printf("]");
}

int main(int argc, char **argv) {
  const bool bands = argc > 1 && std::strcmp(argv[1], "bands") == 0;
  const uint64_t maxn = 1ull << 30;
  mp_init_args a{};
  a.world = 1;
  a.n_loop_relays = 6;
  a.host_path = 1;
  a.heap_bytes = 16ull << 20;
  mp_ctx *ctx = nullptr;
  if (int s = mp_init(&ctx, &a)) {
    std::fprintf(stderr, "mp_init: %s\n", mp_strerror(s));
    return 1;
  }
  mp_model_opts o{};
  MK(mp_get_options(ctx, &o));
  o.mode = MP_MODEL_B200;
  MK(mp_set_options(ctx, &o));
  if (bands) MK(mp_calibrate_bands(ctx, nullptr, 0, 5));
  MK(mp_calibrate_window(ctx, nullptr, 0, 16, 7));
  {
    double h[MP_MAX_PATHS], tau = 0, kappa = 0;
    int np = 0;
    MK(mp_get_window_model(ctx, 0, 0, h, &np, &tau));
    MK(mp_get_host_duplex(ctx, 0, &kappa));
    std::printf("{\"calibrated\": true, \"bands\": %s, \"tau_us\": %.3f, \"kappa\": %.4f, \"h_us\": [", bands ? "true" : "false",
                tau * 1e6, kappa);
    for (int i = 0; i < np; ++i) std::printf("%s%.3f", i ? ", " : "", h[i] * 1e6);
    std::printf("]}\n");
  }
  uint8_t *A = nullptr, *B = nullptr, *ack_s = nullptr, *ack_r = nullptr;
  CK(cudaMalloc(&A, maxn));
  CK(cudaMalloc(&B, maxn));
  CK(cudaMalloc(&ack_s, 256));
  CK(cudaMalloc(&ack_r, 256));
  CK(cudaMemset(A, 0x5a, maxn));
  CK(cudaMemset(ack_s, 1, 256));
  cudaStream_t s1;
  CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking));
  CK(cudaDeviceSynchronize());
  mp_config ack;
  MK(mp_select(ctx, 0, 0, 4, 1, &ack));
  double ack1 = 0, ack2 = 0;
  MK(mp_predict_window(ctx, 0, 0, 4, 1, &ack, &ack1));
  MK(mp_predict_window(ctx, 0, 0, 4, 2, &ack, &ack2));
  const double ack_inc = ack2 - ack1;  // one more (back-to-back) 4-byte message

  auto omb = [&](const mp_config &cfg, uint64_t n, int w, int it) {
    auto iter = [&] {
      for (int k = 0; k < w; ++k) MK(mp_xfer(ctx, B, A, n, &cfg, s1));
      MK(mp_xfer(ctx, ack_r, ack_s, 4, &ack, s1));
      CK(cudaStreamSynchronize(s1));
    };
    for (int i = 0; i < 2; ++i) iter();
    std::vector<double> ts;
    for (int r = 0; r < 3; ++r) {
      const auto t0 = std::chrono::steady_clock::now();
      for (int i = 0; i < it; ++i) iter();
      const auto t1 = std::chrono::steady_clock::now();
      ts.push_back(std::chrono::duration<double>(t1 - t0).count() / it);
    }
    std::sort(ts.begin(), ts.end());
    return static_cast<double>(n) * w / ts[1] / 1e9;  // GB/s of the median repeat
  };

  for (uint64_t n = 64 << 10; n <= maxn; n <<= 2) {
    mp_config c1;
    MK(mp_select(ctx, 0, 0, n, 0, &c1));
    for (int w : {1, 16, 64}) {
      mp_config cw;
      MK(mp_select_window(ctx, 0, 0, n, static_cast<uint32_t>(w), 0, &cw));
      const double per_iter_bytes = static_cast<double>(n) * w;
      const int it = std::max(3, static_cast<int>(std::min(400.0, 2e9 / per_iter_bytes)));
      const double bw_w = omb(cw, n, w, it);
      const bool same = std::memcmp(cw.bytes, c1.bytes, sizeof(c1.bytes)) == 0 &&
                        std::memcmp(cw.chunks, c1.chunks, sizeof(c1.chunks)) == 0;
      const double bw_1 = same ? bw_w : omb(c1, n, w, it);
      double tw = 0, tw1 = 0;
      MK(mp_predict_window(ctx, 0, 0, n, static_cast<uint32_t>(w), &cw, &tw));
      MK(mp_predict_window(ctx, 0, 0, n, static_cast<uint32_t>(w), &c1, &tw1));
      std::printf("{\"n\": %llu, \"w\": %d, \"bw_window_cfg_GBps\": %.4f, \"bw_msg_cfg_GBps\": %.4f, "
                  "\"pred_msg_GBps\": %.4f, \"pred_win_GBps\": %.4f, \"pred_win_msg_cfg_GBps\": %.4f, \"same_cfg\": %s",
                  static_cast<unsigned long long>(n), w, bw_w, bw_1, n / c1.t_pred / 1e9,
                  per_iter_bytes / (tw + ack_inc) / 1e9, per_iter_bytes / (tw1 + ack_inc) / 1e9,
                  same ? "true" : "false");
      print_cfg("cfg_window", cw);
      print_cfg("cfg_msg", c1);
      std::printf("}\n");
      std::fflush(stdout);
    }
  }
  MK(mp_sync(ctx));
  mp_finalize(ctx);
  return 0;
}
