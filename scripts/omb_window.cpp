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
//   ./scripts/omb_window [bands|asym] [max_bytes] [nobibw]
//       → one JSON line of calibrated parameters, then one per (size, window)
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
  const uint64_t maxn = argc > 2 ? std::strtoull(argv[2], nullptr, 10) : 1ull << 30;  // largest message
  const bool skip_bibw = argc > 3 && std::strcmp(argv[3], "nobibw") == 0;
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
    double h[MP_MAX_PATHS], tau = 0, kappa = 0, sub = 0;
    int np = 0;
    MK(mp_get_window_model(ctx, 0, 0, h, &np, &tau));
    MK(mp_get_host_duplex(ctx, 0, &kappa));
    MK(mp_get_submit_time(ctx, &sub));
    std::printf("{\"calibrated\": true, \"bands\": %s, \"tau_us\": %.3f, \"submit_us\": %.3f, \"kappa\": %.4f, \"h_us\": [",
                bands ? "true" : "false", tau * 1e6, sub * 1e6, kappa);
    for (int i = 0; i < np; ++i) std::printf("%s%.3f", i ? ", " : "", h[i] * 1e6);
    std::printf("]}\n");
  }
  {  // E5: the selector's own cost per call from C, cache miss / hit
    mp_config t;
    const int K = 20000;
    auto t0 = std::chrono::steady_clock::now();
    for (int i = 0; i < K; ++i) MK(mp_select(ctx, 0, 0, (1ull << 30) + 256ull * (i + 1), 0, &t));
    auto t1 = std::chrono::steady_clock::now();
    for (int i = 0; i < K; ++i) MK(mp_select(ctx, 0, 0, 1ull << 30, 0, &t));
    auto t2 = std::chrono::steady_clock::now();
    for (int i = 0; i < K; ++i) MK(mp_select_window(ctx, 0, 0, (1ull << 30) + 256ull * (i + 1), 16, 0, &t));
    auto t3 = std::chrono::steady_clock::now();
    std::printf("{\"select_miss_us\": %.3f, \"select_hit_us\": %.3f, \"select_window_us\": %.3f}\n",
                std::chrono::duration<double>(t1 - t0).count() / K * 1e6,
                std::chrono::duration<double>(t2 - t1).count() / K * 1e6,
                std::chrono::duration<double>(t3 - t2).count() / K * 1e6);
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

  {  // C27 cross-check: the marginal host cost of one more 64 KiB message, this process's loop
    mp_config c64;
    MK(mp_select(ctx, 0, 0, 65536, 1, &c64));
    auto burst = [&](int W) {  // mean of 100 consecutive windows (the loop osu_bw runs)
      for (int it = 0; it < 20; ++it) {
        for (int w = 0; w < W; ++w) MK(mp_xfer(ctx, B, A, 65536, &c64, s1));
        CK(cudaStreamSynchronize(s1));
      }
      const auto t0 = std::chrono::steady_clock::now();
      for (int it = 0; it < 100; ++it) {
        for (int w = 0; w < W; ++w) MK(mp_xfer(ctx, B, A, 65536, &c64, s1));
        CK(cudaStreamSynchronize(s1));
      }
      return std::chrono::duration<double>(std::chrono::steady_clock::now() - t0).count() / 100;
    };
    const double t16 = burst(16), t64 = burst(64);
    std::printf("{\"submit_check_us\": %.3f, \"t16_us\": %.3f, \"t64_us\": %.3f}\n", (t64 - t16) / 48 * 1e6,
                t16 * 1e6, t64 * 1e6);
  }

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

  // osu_bibw (Obs 1 and 5): both directions at once, four buffers, windows of
  // 16 per direction then a host wait.  Configs: the two flows selected jointly
  // (mp_select_flows, C19/C25) vs each selected alone (mp_select, the paper's
  // per-message model), with all paths and with {direct, host} only.
  uint8_t *Cb = nullptr, *D = nullptr;
  CK(cudaMalloc(&Cb, maxn));
  CK(cudaMalloc(&D, maxn));
  CK(cudaMemset(Cb, 0x3c, maxn));
  cudaStream_t s2;
  CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
  cudaEvent_t fork, join;
  CK(cudaEventCreateWithFlags(&fork, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&join, cudaEventDisableTiming));
  mp_path ps[MP_MAX_PATHS];
  int np = 0;
  MK(mp_paths(ctx, 0, 0, ps, &np));
  const uint32_t host_mask = 1u | (1u << (np - 1));
  auto bibw = [&](const mp_config &c1, const mp_config &c2, uint64_t n, int w, int it) {
    auto iter = [&] {
      CK(cudaEventRecord(fork, s1));
      CK(cudaStreamWaitEvent(s2, fork, 0));
      for (int k = 0; k < w; ++k) {
        MK(mp_xfer(ctx, B, A, n, &c1, s1));
        MK(mp_xfer(ctx, D, Cb, n, &c2, s2));
      }
      CK(cudaEventRecord(join, s2));
      CK(cudaStreamWaitEvent(s1, join, 0));
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
    return 2.0 * static_cast<double>(n) * w / ts[1] / 1e9;
  };
  for (uint64_t n = 16ull << 20; n <= maxn && !skip_bibw; n <<= 2)
    for (uint32_t mask : {0u, host_mask}) {
      const int w = 16;
      const int it = std::max(2, static_cast<int>(std::min(100.0, 4e9 / (2.0 * n * w))));
      mp_flow fl[2] = {{0, 0, mask, 0, n}, {0, 0, mask, 0, n}};
      mp_config fc[2], ind;
      MK(mp_select_flows(ctx, 2, fl, fc));
      MK(mp_select(ctx, 0, 0, n, mask, &ind));
      const double b_joint = bibw(fc[0], fc[1], n, w, it);
      const double b_ind = bibw(ind, ind, n, w, it);
      std::printf("{\"bibw\": true, \"n\": %llu, \"w\": %d, \"mask\": \"%s\", \"bibw_joint_GBps\": %.4f, "
                  "\"pred_joint_GBps\": %.4f, \"bibw_independent_GBps\": %.4f, \"pred_independent_GBps\": %.4f",
                  static_cast<unsigned long long>(n), w, mask ? "direct+host" : "all", b_joint,
                  2.0 * n / std::max(fc[0].t_pred, fc[1].t_pred) / 1e9, b_ind, 2.0 * n / ind.t_pred / 1e9);
      print_cfg("cfg_joint", fc[0]);
      print_cfg("cfg_independent", ind);
      std::printf("}\n");
      std::fflush(stdout);
    }
  MK(mp_sync(ctx));
  mp_finalize(ctx);
  return 0;
}
