// pdlbench.cu — programmatic dependent launch (PDL) design experiment (tooling, not
// the product).  Back-to-back copies of one buffer pair (a window, as osu_bw): the
// engine's one-shot small kernel and TMA direct kernel, launched plainly vs with
// cudaLaunchAttributeProgrammaticStreamSerialization, where each kernel first lets its
// successor launch (griddepcontrol.launch_dependents) and then waits for its
// predecessor to complete (griddepcontrol.wait) before touching memory.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o pdlbench scripts/pdlbench.cu
//   ./pdlbench  → one JSON line per size
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
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

using namespace mpx;

template <bool PDL>
__global__ void __launch_bounds__(256) small_k(uint8_t *dst, const uint8_t *src, uint64_t n) {
  if (PDL) {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    asm volatile("griddepcontrol.wait;" ::: "memory");
  }
  const uint64_t nvec = n >> 4;
  const uint64_t i = static_cast<uint64_t>(blockIdx.x) * 256 + threadIdx.x;
  if (i < nvec) reinterpret_cast<uint4 *>(dst)[i] = reinterpret_cast<const uint4 *>(src)[i];
}

template <bool PDL>
__global__ void __launch_bounds__(256, 4) tma_k(const __grid_constant__ DirectArgs A) {
  extern __shared__ __align__(128) uint8_t dyn_smem[];
  if (PDL) {
    asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
    asm volatile("griddepcontrol.wait;" ::: "memory");
  }
  bulk_copy<LD_SRC>(A.dst, A.src, A.bytes, blockIdx.x, gridDim.x, dyn_smem, A.stages, false);
}

template <typename K, typename... Args>
void launch(bool pdl, K kern, dim3 g, size_t smem, cudaStream_t s, Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = g;
  cfg.blockDim = dim3(256);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl ? 1 : 0;
  CK(cudaLaunchKernelEx(&cfg, kern, args...));
}

int main() {
  const uint64_t maxn = 256ull << 20;
  uint8_t *a, *b;
  CK(cudaMalloc(&a, maxn));
  CK(cudaMalloc(&b, maxn));
  CK(cudaMemset(a, 1, maxn));
  cudaStream_t s;
  CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  cudaEvent_t e0, e1, em;
  CK(cudaEventCreate(&em));
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  CK(cudaFuncSetAttribute(tma_k<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, kBulkSmem));
  CK(cudaFuncSetAttribute(tma_k<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, kBulkSmem));
  const int W = 64;
  auto timed = [&](auto &&fn) {
    for (int i = 0; i < 8; ++i) fn();
    std::vector<double> ts;
    for (int r = 0; r < 7; ++r) {
      CK(cudaEventRecord(e0, s));
      for (int i = 0; i < W; ++i) fn();
      CK(cudaEventRecord(e1, s));
      CK(cudaEventSynchronize(e1));
      float ms = 0;
      CK(cudaEventElapsedTime(&ms, e0, e1));
      ts.push_back(ms * 1e3 / W);
    }
    std::sort(ts.begin(), ts.end());
    return ts[ts.size() / 2];  // µs per message
  };
  std::vector<uint64_t> sizes = {4096, 65536, 1 << 20, 2 << 20, 4 << 20, 6 << 20, 8 << 20, 12 << 20, 16 << 20,
                                 32 << 20, 64 << 20, 256 << 20};
  for (uint64_t n : sizes) {
    const uint32_t gs = static_cast<uint32_t>(std::max<uint64_t>(1, (n / 16 + 255) / 256));
    const uint32_t gw = static_cast<uint32_t>(std::min<uint64_t>(2ull * sms, std::max<uint64_t>(1, n / 32768)));
    const DirectArgs A{b, a, n, 1, 4};
    std::printf("{\"n\": %llu, \"grid\": %u", static_cast<unsigned long long>(n), gw);
    if (n <= (8u << 20)) {
      std::printf(", \"small_us\": %.3f", timed([&] { launch(false, small_k<false>, dim3(gs), 0, s, b, (const uint8_t *)a, n); }));
      std::printf(", \"small_pdl_us\": %.3f", timed([&] { launch(true, small_k<true>, dim3(gs), 0, s, b, (const uint8_t *)a, n); }));
    }
    for (uint32_t gt : {gw, static_cast<uint32_t>(sms), static_cast<uint32_t>(2 * sms)}) {
      std::printf(", \"tma_g%u_us\": %.3f", gt, timed([&] { launch(false, tma_k<false>, dim3(gt), kBulkSmem, s, A); }));
      std::printf(", \"tma_pdl_g%u_us\": %.3f", gt, timed([&] { launch(true, tma_k<true>, dim3(gt), kBulkSmem, s, A); }));
    }
    std::printf(", \"tma_ev_us\": %.3f", timed([&] {  // an event record between launches
      launch(false, tma_k<false>, dim3(gw), kBulkSmem, s, A);
      CK(cudaEventRecord(em, s));
    }));
    std::printf(", \"tma_pdl_ev_us\": %.3f", timed([&] {
      launch(true, tma_k<true>, dim3(gw), kBulkSmem, s, A);
      CK(cudaEventRecord(em, s));
    }));
    std::printf(", \"ce_us\": %.3f", timed([&] { CK(cudaMemcpyAsync(b, a, n, cudaMemcpyDeviceToDevice, s)); }));
    std::printf("}\n");
    std::fflush(stdout);
  }
  return 0;
}
