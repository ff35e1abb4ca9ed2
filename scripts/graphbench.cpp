// graphbench.cpp — design experiment (tooling): a window of W direct-only mp_xfer
// messages enqueued from the host each time vs captured once in a CUDA graph and
// replayed (the engine's launches carry the PDL attribute, which a capture turns into
// programmatic graph edges).  µs per message, median of 7 timed windows.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <initializer_list>
#include <vector>

#include "mp.h"

int main() {
  mp_init_args a{};
  a.world = 1;
  a.n_loop_relays = 6;
  a.host_path = 1;
  a.heap_bytes = 16ull << 20;
  a.flags = MP_INIT_NO_CALIBRATE;
  mp_ctx *ctx = nullptr;
  if (mp_init(&ctx, &a)) return 1;
  const uint64_t maxn = 64ull << 20;
  void *s = nullptr, *d = nullptr;
  cudaMalloc(&s, maxn);
  cudaMalloc(&d, maxn);
  cudaStream_t st;
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const int W = 64;
  for (uint64_t n : {4096ull, 65536ull, 1ull << 20, 4ull << 20, 16ull << 20, 64ull << 20}) {
    mp_config cfg;
    mp_select(ctx, 0, 0, n, 1, &cfg);  // direct only
    auto time_it = [&](auto &&fn) {
      fn();
      cudaStreamSynchronize(st);
      std::vector<float> v;
      for (int r = 0; r < 7; ++r) {
        cudaEventRecord(e0, st);
        fn();
        cudaEventRecord(e1, st);
        cudaEventSynchronize(e1);
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        v.push_back(ms * 1e3f / W);
      }
      std::sort(v.begin(), v.end());
      return v[3];
    };
    const float host = time_it([&] {
      for (int w = 0; w < W; ++w) mp_xfer(ctx, d, s, n, &cfg, st);
    });
    cudaGraph_t g;
    cudaGraphExec_t ge;
    cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal);
    for (int w = 0; w < W; ++w) mp_xfer(ctx, d, s, n, &cfg, st);
    cudaStreamEndCapture(st, &g);
    cudaGraphInstantiate(&ge, g, 0);
    const float graph = time_it([&] { cudaGraphLaunch(ge, st); });
    cudaGraphExecDestroy(ge);
    cudaGraphDestroy(g);
    std::printf("{\"n\": %llu, \"W\": %d, \"host_enqueued_us\": %.3f, \"graph_us\": %.3f}\n",
                static_cast<unsigned long long>(n), W, host, graph);
    std::fflush(stdout);
  }
  if (int e = mp_sync(ctx)) std::printf("{\"error\": \"%s\"}\n", mp_strerror(e));
  mp_finalize(ctx);
  return 0;
}
