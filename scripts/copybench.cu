// copybench.cu — design-space sweep for the direct-path copy on sm_100a (tooling,
// not the product): LDG/STG vector copies vs TMA bulk (cp.async.bulk) pipelines of
// different block sizes / depths / CTAs per SM / L2 hints, vs cudaMemcpyAsync.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o copybench scripts/copybench.cu
//   ./copybench [bytes]     → one line per variant: GB/s (payload) and % of memcpy
//   ./copybench [bytes] few → per-CTA rate of small grids (8/16/32 CTAs, as a staged
//                             stage group) vs issuing warps per CTA
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <string>
#include <vector>

#define CK(x)                                                                   \
  do {                                                                          \
    cudaError_t e = (x);                                                        \
    if (e != cudaSuccess) {                                                     \
      std::fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); \
      std::exit(1);                                                             \
    }                                                                           \
  } while (0)

template <int U>
__global__ void __launch_bounds__(256) reg_copy(uint4 *__restrict__ d, const uint4 *__restrict__ s, uint64_t n) {
  const uint64_t gt = blockIdx.x * 256ull + threadIdx.x, GT = gridDim.x * 256ull;
  uint64_t i = gt;
  for (; i + (U - 1) * GT < n; i += U * GT) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u)
      asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                   : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w)
                   : "l"(s + i + u * GT));
#pragma unroll
    for (int u = 0; u < U; ++u) d[i + u * GT] = v[u];
  }
  for (; i < n; i += GT) d[i] = s[i];
}

__device__ __forceinline__ uint32_t su32(const void *p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }

// TMA pipeline: each of `lanes` warps (lane 0) runs an independent D-stage pipeline of
// B-byte blocks; blocks are striped over (cta, warp) pairs.
__global__ void __launch_bounds__(256) tma_copy(uint8_t *d, const uint8_t *s, uint64_t n, uint32_t B, uint32_t D,
                                                uint32_t lanes, int hint) {
  extern __shared__ __align__(128) uint8_t sm[];
  const uint32_t w = threadIdx.x / 32;
  if (w >= lanes || (threadIdx.x & 31)) return;
  uint8_t *buf = sm + static_cast<uint64_t>(w) * B * D;
  uint64_t *bars = reinterpret_cast<uint64_t *>(sm + static_cast<uint64_t>(lanes) * B * D) + w * D;
  uint64_t pol = 0;
  if (hint) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  for (uint32_t i = 0; i < D; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(bars + i)));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  const uint64_t nblk = (n + B - 1) / B;
  const uint64_t me = static_cast<uint64_t>(blockIdx.x) * lanes + w, G = static_cast<uint64_t>(gridDim.x) * lanes;
  if (me >= nblk) return;
  const uint64_t mine = (nblk - me + G - 1) / G;
  auto load = [&](uint64_t it) {
    const uint64_t o = (me + it * G) * B;
    const uint32_t len = static_cast<uint32_t>(n - o < B ? n - o : B);
    const uint32_t st = it % D;
    const uint32_t bar = su32(bars + st);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(len) : "memory");
    if (hint)
      asm volatile(
          "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
              su32(buf + st * B)),
          "l"(s + o), "r"(len), "r"(bar), "l"(pol)
          : "memory");
    else
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                       su32(buf + st * B)),
                   "l"(s + o), "r"(len), "r"(bar)
                   : "memory");
  };
  const uint64_t pro = mine < D ? mine : D;
  for (uint64_t it = 0; it < pro; ++it) load(it);
  for (uint64_t it = 0; it < mine; ++it) {
    const uint32_t st = it % D;
    const uint32_t bar = su32(bars + st), par = (it / D) & 1;
    asm volatile(
        "{\n\t.reg .pred p;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n}" ::"r"(bar),
        "r"(par)
        : "memory");
    const uint64_t o = (me + it * G) * B;
    const uint32_t len = static_cast<uint32_t>(n - o < B ? n - o : B);
    if (hint)
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group.L2::cache_hint [%0], [%1], %2, %3;" ::"l"(d + o),
                   "r"(su32(buf + st * B)), "r"(len), "l"(pol)
                   : "memory");
    else
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(d + o), "r"(su32(buf + st * B)),
                   "r"(len)
                   : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    if (it >= 1 && it - 1 + D < mine) {
      asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      load(it - 1 + D);
    }
  }
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

// Same pipeline, one issuing thread per CTA, but the stage of block it-L is refilled
// after the store of block it (L stores may still be reading shared memory; loads run
// D-L blocks ahead).  L = 1 is tma_copy's schedule.
template <int L>
__global__ void __launch_bounds__(256) tma_lag(uint8_t *d, const uint8_t *s, uint64_t n, uint32_t B, uint32_t D) {
  extern __shared__ __align__(128) uint8_t sm[];
  if (threadIdx.x) return;
  uint64_t *bars = reinterpret_cast<uint64_t *>(sm + static_cast<uint64_t>(B) * D);
  for (uint32_t i = 0; i < D; ++i) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(bars + i)));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  const uint64_t nblk = (n + B - 1) / B, me = blockIdx.x, G = gridDim.x;
  if (me >= nblk) return;
  const uint64_t mine = (nblk - me + G - 1) / G;
  auto load = [&](uint64_t it) {
    const uint64_t o = (me + it * G) * B;
    const uint32_t len = static_cast<uint32_t>(n - o < B ? n - o : B);
    const uint32_t bar = su32(bars + it % D);
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(len) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     su32(sm + (it % D) * B)),
                 "l"(s + o), "r"(len), "r"(bar)
                 : "memory");
  };
  const uint64_t pro = mine < D ? mine : D;
  for (uint64_t it = 0; it < pro; ++it) load(it);
  for (uint64_t it = 0; it < mine; ++it) {
    const uint32_t st = it % D;
    asm volatile(
        "{\n\t.reg .pred p;\nW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t@!p bra W_%=;\n}" ::"r"(
            su32(bars + st)),
        "r"(static_cast<uint32_t>((it / D) & 1))
        : "memory");
    const uint64_t o = (me + it * G) * B;
    const uint32_t len = static_cast<uint32_t>(n - o < B ? n - o : B);
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(d + o), "r"(su32(sm + st * B)),
                 "r"(len)
                 : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    if (it >= L && it - L + D < mine) {
      asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(L) : "memory");
      load(it - L + D);
    }
  }
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

int main(int argc, char **argv) {
  const uint64_t n = argc > 1 ? std::strtoull(argv[1], nullptr, 0) : (1ull << 30);
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  uint8_t *s, *d;
  CK(cudaMalloc(&s, n));
  CK(cudaMalloc(&d, n));
  CK(cudaMemset(s, 0x3c, n));
  cudaStream_t st;
  CK(cudaStreamCreate(&st));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  auto timeit = [&](auto &&fn) {
    std::vector<float> t;
    for (int r = 0; r < 23; ++r) {
      CK(cudaEventRecord(e0, st));
      fn();
      CK(cudaEventRecord(e1, st));
      CK(cudaEventSynchronize(e1));
      float ms;
      CK(cudaEventElapsedTime(&ms, e0, e1));
      if (r >= 3) t.push_back(ms);
    }
    std::sort(t.begin(), t.end());
    return static_cast<double>(n) / (t[t.size() / 2] * 1e-3) / 1e9;
  };
  const double memcpy_gbs = timeit([&] { CK(cudaMemcpyAsync(d, s, n, cudaMemcpyDeviceToDevice, st)); });
  std::printf("{\"variant\": \"cudaMemcpyAsync\", \"GBps\": %.1f}\n", memcpy_gbs);
  for (int per_sm : {2, 4, 8}) {
    for (int U : {4, 8}) {
      const int grid = sms * per_sm;
      auto f = [&] {
        if (U == 4)
          reg_copy<4><<<grid, 256, 0, st>>>(reinterpret_cast<uint4 *>(d), reinterpret_cast<const uint4 *>(s), n / 16);
        else
          reg_copy<8><<<grid, 256, 0, st>>>(reinterpret_cast<uint4 *>(d), reinterpret_cast<const uint4 *>(s), n / 16);
      };
      const double g = timeit(f);
      std::printf("{\"variant\": \"reg U=%d ctas/sm=%d\", \"GBps\": %.1f, \"vs_memcpy\": %.3f}\n", U, per_sm, g,
                  g / memcpy_gbs);
    }
  }
  CK(cudaFuncSetAttribute(tma_copy, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024));
  if (argc > 2 && std::string(argv[2]) == "few") {
    for (uint32_t grid : {16u, 148u})
      for (uint32_t B : {8192u, 16384u})
        for (uint32_t D : {2u, 3u, 4u, 8u})
          for (uint32_t lanes : {1u, 2u, 4u}) {
            const uint64_t smem = static_cast<uint64_t>(B) * D * lanes + 8ull * D * lanes;
            if (smem > 220 * 1024) continue;
            const double g = timeit([&] { tma_copy<<<grid, 256, smem, st>>>(d, s, n, B, D, lanes, 0); });
            CK(cudaGetLastError());
            std::printf("{\"variant\": \"few grid=%u B=%u D=%u warps=%u\", \"GBps\": %.1f, \"GBps_per_cta\": %.2f}\n",
                        grid, B, D, lanes, g, g / grid);
          }
    CK(cudaFuncSetAttribute(tma_lag<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024));
    CK(cudaFuncSetAttribute(tma_lag<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024));
    CK(cudaFuncSetAttribute(tma_lag<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024));
    for (uint32_t grid : {16u, 148u, 296u})
      for (uint32_t B : {4096u, 8192u})
        for (uint32_t D : {4u, 8u})
          for (int L : {1, 2, 3}) {
            if (B * D > 32768u || L >= static_cast<int>(D)) continue;
            const uint64_t smem = static_cast<uint64_t>(B) * D + 8ull * D;
            const double g = timeit([&] {
              if (L == 1) tma_lag<1><<<grid, 256, smem, st>>>(d, s, n, B, D);
              if (L == 2) tma_lag<2><<<grid, 256, smem, st>>>(d, s, n, B, D);
              if (L == 3) tma_lag<3><<<grid, 256, smem, st>>>(d, s, n, B, D);
            });
            CK(cudaGetLastError());
            std::printf("{\"variant\": \"lag grid=%u B=%u D=%u L=%d\", \"GBps\": %.1f, \"GBps_per_cta\": %.2f}\n",
                        grid, B, D, L, g, g / grid);
          }
    return 0;
  }
  struct V {
    uint32_t B, D, lanes, per_sm;
    int hint;
  };
  std::vector<V> vs;
  for (uint32_t B : {8192u, 16384u, 32768u, 65536u})
    for (uint32_t D : {2u, 3u, 4u, 6u})
      for (uint32_t lanes : {1u, 2u, 4u})
        for (uint32_t per_sm : {1u, 2u, 4u})
          for (int hint : {0, 1}) {
            const uint64_t smem = static_cast<uint64_t>(B) * D * lanes + 8ull * D * lanes;
            if (smem * per_sm > 220 * 1024) continue;
            vs.push_back({B, D, lanes, per_sm, hint});
          }
  for (const V &v : vs) {
    const uint64_t smem = static_cast<uint64_t>(v.B) * v.D * v.lanes + 8ull * v.D * v.lanes;
    const int grid = sms * v.per_sm;
    const double g = timeit([&] { tma_copy<<<grid, 256, smem, st>>>(d, s, n, v.B, v.D, v.lanes, v.hint); });
    CK(cudaGetLastError());
    std::printf("{\"variant\": \"tma B=%u D=%u warps=%u ctas/sm=%u hint=%d\", \"GBps\": %.1f, \"vs_memcpy\": %.3f}\n",
                v.B, v.D, v.lanes, v.per_sm, v.hint, g, g / memcpy_gbs);
  }
  // correctness of the last variant
  std::vector<uint8_t> h(1 << 20);
  CK(cudaMemcpy(h.data(), d + n - h.size(), h.size(), cudaMemcpyDeviceToHost));
  for (uint8_t x : h)
    if (x != 0x3c) {
      std::printf("MISMATCH\n");
      return 1;
    }
  return 0;
}
