// bibwbench.cu — two concurrent large copies (osu_bibw on the loopback engine: A→B on
// one stream and B→A on another) for the engine's direct kernel at several grid
// sizes, the LDG/STG kernel, and the copy engine; swapped buffers (as the OMB bibw
// test) and four separate buffers.  Tooling, not the product.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o scripts/bibwbench scripts/bibwbench.cu
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <vector>

#include "../paper_conf_sc_sojoodiasfga25_b200/csrc/engine.cu"

#define CK(x)                                                                        \
  do {                                                                               \
    cudaError_t e = (x);                                                             \
    if (e != cudaSuccess) {                                                          \
      std::fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); \
      std::exit(1);                                                                  \
    }                                                                                \
  } while (0)

int main() {
  const uint64_t maxn = 1ull << 30;
  uint8_t *buf[4];
  for (auto &b : buf) {
    CK(cudaMalloc(&b, maxn));
    CK(cudaMemset(b, 1, maxn));
  }
  cudaStream_t s1, s2;
  CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
  cudaEvent_t e0, e1, fork, join;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  CK(cudaEventCreateWithFlags(&fork, cudaEventDisableTiming));
  CK(cudaEventCreateWithFlags(&join, cudaEventDisableTiming));
  CK(cudaFuncSetAttribute(mpx::direct_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, mpx::kBulkSmem));
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));

  auto run = [&](const char *name, uint64_t n, bool both, auto &&one) {
    auto step = [&] {
      CK(cudaEventRecord(fork, s1));
      CK(cudaStreamWaitEvent(s2, fork, 0));
      one(0, s1);
      if (both) one(1, s2);
      CK(cudaEventRecord(join, s2));
      CK(cudaStreamWaitEvent(s1, join, 0));
    };
    for (int i = 0; i < 3; ++i) step();
    const int it = n >= (512ull << 20) ? 6 : 20;
    CK(cudaEventRecord(e0, s1));
    for (int i = 0; i < it; ++i) step();
    CK(cudaEventRecord(e1, s1));
    CK(cudaEventSynchronize(e1));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    const double t = ms * 1e-3 / it;
    std::printf("{\"n\": %llu, \"variant\": \"%s\", \"GBps_total\": %.1f}\n", static_cast<unsigned long long>(n),
                name, (both ? 2.0 : 1.0) * n / t / 1e9);
    std::fflush(stdout);
  };

  for (uint64_t n : {64ull << 20, 256ull << 20, 1ull << 30}) {
    // pairs (dst, src) for direction 0 / 1: swapped = A→B, B→A; separate = A→B, C→D
    for (int sep = 0; sep < 2; ++sep) {
      uint8_t *d0 = buf[1], *s0 = buf[0], *d1 = sep ? buf[3] : buf[0], *s1p = sep ? buf[2] : buf[1];
      auto dst = [&](int k) { return k ? d1 : d0; };
      auto src = [&](int k) { return k ? s1p : s0; };
      char nm[96];
      std::snprintf(nm, sizeof nm, "ce_%s_one", sep ? "sep" : "swap");
      run(nm, n, false, [&](int k, cudaStream_t s) { CK(cudaMemcpyAsync(dst(k), src(k), n, cudaMemcpyDeviceToDevice, s)); });
      std::snprintf(nm, sizeof nm, "ce_%s", sep ? "sep" : "swap");
      run(nm, n, true, [&](int k, cudaStream_t s) { CK(cudaMemcpyAsync(dst(k), src(k), n, cudaMemcpyDeviceToDevice, s)); });
      for (int per : {2, 1}) {
        const uint32_t g = static_cast<uint32_t>(per * sms);
        std::snprintf(nm, sizeof nm, "tma_%s_g%u", sep ? "sep" : "swap", g);
        run(nm, n, true, [&](int k, cudaStream_t s) {
          const mpx::DirectArgs A{dst(k), src(k), n, 1, 4};
          mpx::direct_kernel<<<g, 256, mpx::kBulkSmem, s>>>(A);
        });
      }
      {
        const uint32_t g = static_cast<uint32_t>(4 * sms);
        std::snprintf(nm, sizeof nm, "reg_%s_g%u", sep ? "sep" : "swap", g);
        run(nm, n, true, [&](int k, cudaStream_t s) {
          const mpx::DirectArgs A{dst(k), src(k), n, 0, 4};
          mpx::direct_reg_kernel<<<g, 256, 0, s>>>(A);
        });
      }
      {  // one fused launch moving both directions (half the CTAs each)
        const uint32_t g = static_cast<uint32_t>(sms);
        std::snprintf(nm, sizeof nm, "tma_%s_serial_g%u", sep ? "sep" : "swap", 2 * g);
        run(nm, n, true, [&](int k, cudaStream_t s) {
          const mpx::DirectArgs A{dst(k), src(k), n, 1, 4};
          mpx::direct_kernel<<<2 * g, 256, mpx::kBulkSmem, s1>>>(A);  // both on s1: serialised
        });
      }
    }
  }
  return 0;
}
