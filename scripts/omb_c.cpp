// omb_c.cpp — the OMB-style loopback sweep (BASELINE.json config 4; osu_bw / osu_bibw /
// osu_latency methodology) driven from C through the public C ABI, as
// OSU's own harness is, so that small sizes measure the engine and not a Python loop.
//   g++ -O2 -std=c++17 -I include -I /usr/local/cuda/include scripts/omb_c.cpp \
//       -L paper_conf_sc_sojoodiasfga25_b200/_lib -lmpx -L /usr/local/cuda/lib64 -lcudart \
//       -Wl,-rpath,'$ORIGIN/../paper_conf_sc_sojoodiasfga25_b200/_lib' -o scripts/omb_c
//   ./scripts/omb_c [max_bytes]   → one JSON line per size
// Per size: bw (window 1, 16, 64 back-to-back model-selected mp_xfer) next to
// cudaMemcpyAsync D2D, bibw (two directions on two streams, four buffers as osu_bibw), one-way latency (median
// of single transfers), and the model's predicted bandwidth (size bands calibrated).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
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
#define MK(x)                                                                         \
  do {                                                                                \
    int s = (x);                                                                      \
    if (s) {                                                                          \
      std::fprintf(stderr, "%s:%d %s %s\n", __FILE__, __LINE__, mp_strerror(s), mp_last_error(ctx)); \
      std::exit(1);                                                                   \
    }                                                                                 \
  } while (0)

int main(int argc, char **argv) {
  const uint64_t maxn = argc > 1 ? std::strtoull(argv[1], nullptr, 10) : (2ull << 30);
  mp_init_args a{};
  a.rank = 0;
  a.world = 1;
  a.device = 0;
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
  MK(mp_calibrate_bands(ctx, nullptr, 0, 5));
  // osu_bibw: each side sends from its s_buf into the peer's r_buf — four buffers
  // (A→B one way, C→D the other)
  uint8_t *A = nullptr, *B = nullptr, *Cb = nullptr, *D = nullptr;
  CK(cudaMalloc(&A, maxn));
  CK(cudaMalloc(&B, maxn));
  CK(cudaMalloc(&Cb, maxn));
  CK(cudaMalloc(&D, maxn));
  CK(cudaMemset(A, 0x5a, maxn));
  CK(cudaMemset(B, 0xa5, maxn));
  CK(cudaMemset(Cb, 0x3c, maxn));
  CK(cudaMemset(D, 0xc3, maxn));
  cudaStream_t s1, s2;
  CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
  cudaEvent_t e0, e1, fork, join;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  CK(cudaEventCreateWithFlags(&fork, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&join, cudaEventDisableTiming));

  for (uint64_t n = 4096; n <= maxn; n <<= 1) {
    mp_config cfg;
    MK(mp_select(ctx, 0, 0, n, 0, &cfg));
    const int iters = n <= (1u << 20) ? 400 : (n <= (64u << 20) ? 60 : 8);
    auto timed = [&](auto &&fn, int w, int it) {
      for (int i = 0; i < 2; ++i) fn();
      CK(cudaEventRecord(e0, s1));
      for (int i = 0; i < it; ++i)
        for (int k = 0; k < w; ++k) fn();
      CK(cudaEventRecord(e1, s1));
      CK(cudaEventSynchronize(e1));
      float ms = 0;
      CK(cudaEventElapsedTime(&ms, e0, e1));
      return ms * 1e-3 / (static_cast<double>(it) * w);
    };
    auto mpx = [&] { MK(mp_xfer(ctx, B, A, n, nullptr, s1)); };
    auto ce = [&] { CK(cudaMemcpyAsync(B, A, n, cudaMemcpyDeviceToDevice, s1)); };
    std::printf("{\"n\": %llu, \"bytes\": [", static_cast<unsigned long long>(n));
    for (int i = 0; i < cfg.npaths; ++i)
      std::printf("%s%llu", i ? ", " : "", static_cast<unsigned long long>(cfg.bytes[i]));
    std::printf("], \"pred_GBps\": %.4f", n / cfg.t_pred / 1e9);
    {  // bibw as two concurrent flows of the same pair (NEXT f1/f2, reading C19)
      mp_flow fl[2] = {{0, 0, 0, 0, n}, {0, 0, 0, 0, n}};
      mp_config fc[2];
      MK(mp_select_flows(ctx, 2, fl, fc));
      std::printf(", \"pred_bibw_GBps\": %.4f", 2.0 * n / std::max(fc[0].t_pred, fc[1].t_pred) / 1e9);
    }
    for (int w : {1, 16, 64}) {
      const int it = std::max(2, iters / w);
      std::printf(", \"bw_w%d_GBps\": %.4f, \"ce_bw_w%d_GBps\": %.4f", w, n / timed(mpx, w, it) / 1e9, w,
                  n / timed(ce, w, it) / 1e9);
    }
    auto bibw = [&] {
      CK(cudaEventRecord(fork, s1));
      CK(cudaStreamWaitEvent(s2, fork, 0));
      MK(mp_xfer(ctx, B, A, n, nullptr, s1));
      MK(mp_xfer(ctx, D, Cb, n, nullptr, s2));
      CK(cudaEventRecord(join, s2));
      CK(cudaStreamWaitEvent(s1, join, 0));
    };
    auto cebibw = [&] {
      CK(cudaEventRecord(fork, s1));
      CK(cudaStreamWaitEvent(s2, fork, 0));
      CK(cudaMemcpyAsync(B, A, n, cudaMemcpyDeviceToDevice, s1));
      CK(cudaMemcpyAsync(D, Cb, n, cudaMemcpyDeviceToDevice, s2));
      CK(cudaEventRecord(join, s2));
      CK(cudaStreamWaitEvent(s1, join, 0));
    };
    const int itb = std::max(2, iters / 4);
    std::printf(", \"bibw_GBps\": %.4f, \"ce_bibw_GBps\": %.4f", 2.0 * n / timed(bibw, 1, itb) / 1e9,
                2.0 * n / timed(cebibw, 1, itb) / 1e9);
    if (n <= (4u << 20)) {
      auto lat = [&](auto &&fn) {
        std::vector<double> ts;
        for (int r = 0; r < 300; ++r) {
          CK(cudaEventRecord(e0, s1));
          fn();
          CK(cudaEventRecord(e1, s1));
          CK(cudaEventSynchronize(e1));
          float ms = 0;
          CK(cudaEventElapsedTime(&ms, e0, e1));
          ts.push_back(ms * 1e3);
        }
        std::sort(ts.begin(), ts.end());
        return ts[ts.size() / 2];
      };
      std::printf(", \"lat_us\": %.3f, \"ce_lat_us\": %.3f", lat(mpx), lat(ce));
    }
    std::printf("}\n");
    std::fflush(stdout);
  }
  MK(mp_sync(ctx));
  mp_finalize(ctx);
  return 0;
}
