// smallbench.cu — small-message direct-copy design sweep (tooling, not the product).
// OMB-style per-message time of back-to-back launches (window 16 and 1) for the
// engine's direct kernel (TMA pipeline, one CTA per 32 KiB) against one-shot
// register-copy shapes (every CTA issues all its loads at once) and cudaMemcpyAsync.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o smallbench scripts/smallbench.cu
//   ./smallbench  → one JSON line per (size, variant)
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

// V vectors of 16 B per thread, all loads issued before any store.
template <int V>
__global__ void __launch_bounds__(256) oneshot(uint4 *__restrict__ d, const uint4 *__restrict__ s, uint64_t n) {
  const uint64_t base = static_cast<uint64_t>(blockIdx.x) * 256 * V + threadIdx.x;
  uint4 v[V];
#pragma unroll
  for (int u = 0; u < V; ++u)
    if (base + u * 256 < n)
      asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                   : "=r"(v[u].x), "=r"(v[u].y), "=r"(v[u].z), "=r"(v[u].w)
                   : "l"(s + base + u * 256));
#pragma unroll
  for (int u = 0; u < V; ++u)
    if (base + u * 256 < n) d[base + u * 256] = v[u];
}

__global__ void empty_kernel(int) {}

__global__ void __launch_bounds__(256) oneshot_gc(const __grid_constant__ mpx::DirectArgs A) {
  const uint64_t n = A.bytes / 16;
  const uint4 *s = reinterpret_cast<const uint4 *>(A.src);
  uint4 *d = reinterpret_cast<uint4 *>(A.dst);
  const uint64_t i = static_cast<uint64_t>(blockIdx.x) * 256 + threadIdx.x;
  if (i < n) d[i] = s[i];
}

__global__ void __launch_bounds__(256) oneshot_struct(mpx::DirectArgs A) {
  const uint64_t n = A.bytes / 16;
  const uint4 *s = reinterpret_cast<const uint4 *>(A.src);
  uint4 *d = reinterpret_cast<uint4 *>(A.dst);
  const uint64_t i = static_cast<uint64_t>(blockIdx.x) * 256 + threadIdx.x;
  if (i < n) d[i] = s[i];
}

__global__ void __launch_bounds__(256) reg_scalar(uint8_t *d, const uint8_t *s, uint64_t n) {
  mpx::group_copy<mpx::LD_SRC>(d, s, n, blockIdx.x, gridDim.x);
}

__global__ void __launch_bounds__(256) oneshot_asm(uint4 *d, const uint4 *s, uint64_t n) {
  const uint64_t i = static_cast<uint64_t>(blockIdx.x) * 256 + threadIdx.x;
  if (i < n) mpx::st16(d + i, mpx::ld16<mpx::LD_SRC>(s + i));
}

__global__ void __launch_bounds__(256) reg_nospill(const __grid_constant__ mpx::DirectArgs A) {
  mpx::group_copy<mpx::LD_SRC>(A.dst, A.src, A.bytes, blockIdx.x, gridDim.x);
}

// one TMA block (<= 8 KiB) per CTA, no pipeline: load, wait, store, wait
__global__ void __launch_bounds__(256) tma_one(uint8_t *d, const uint8_t *s, uint64_t n) {
  __shared__ __align__(128) uint8_t buf[8192];
  __shared__ __align__(8) uint64_t bar;
  if (threadIdx.x != 0) return;
  const uint64_t o = static_cast<uint64_t>(blockIdx.x) * 8192;
  if (o >= n) return;
  const uint32_t len = static_cast<uint32_t>(n - o < 8192 ? n - o : 8192);
  const uint32_t b = mpx::smem_u32(&bar), sb = mpx::smem_u32(buf);
  mpx::mbar_init(b);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  mpx::mbar_expect_tx(b, len);
  mpx::bulk_load(sb, s + o, len, b);
  mpx::mbar_wait(b, 0);
  mpx::bulk_store(d + o, sb, len);
  asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
}

int main() {
  const uint64_t maxn = 64ull << 20;
  uint8_t *src, *dst;
  CK(cudaMalloc(&src, maxn));
  CK(cudaMalloc(&dst, maxn));
  CK(cudaMemset(src, 1, maxn));
  cudaStream_t st;
  CK(cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking));
  cudaEvent_t e0, e1;
  CK(cudaEventCreate(&e0));
  CK(cudaEventCreate(&e1));
  CK(cudaFuncSetAttribute(mpx::direct_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, mpx::kBulkSmem));
  CK(cudaFuncSetAttribute(oneshot<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, mpx::kBulkSmem));
  int sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));

  auto run = [&](const char *name, uint64_t n, auto &&launch) {
    for (int i = 0; i < 20; ++i) launch();
    CK(cudaStreamSynchronize(st));
    // window 16 back to back, 50 windows
    const int W = 16, R = 50;
    CK(cudaEventRecord(e0, st));
    for (int r = 0; r < R; ++r)
      for (int w = 0; w < W; ++w) launch();
    CK(cudaEventRecord(e1, st));
    CK(cudaEventSynchronize(e1));
    float ms = 0;
    CK(cudaEventElapsedTime(&ms, e0, e1));
    const double t16 = ms * 1e-3 / (W * R);
    // single message latency (median of 200)
    std::vector<double> ts;
    for (int r = 0; r < 200; ++r) {
      CK(cudaEventRecord(e0, st));
      launch();
      CK(cudaEventRecord(e1, st));
      CK(cudaEventSynchronize(e1));
      CK(cudaEventElapsedTime(&ms, e0, e1));
      ts.push_back(ms * 1e-3);
    }
    std::sort(ts.begin(), ts.end());
    std::printf("{\"n\": %llu, \"variant\": \"%s\", \"us_w16\": %.3f, \"GBps_w16\": %.2f, \"lat_us\": %.3f}\n",
                static_cast<unsigned long long>(n), name, t16 * 1e6, n / t16 / 1e9, ts[ts.size() / 2] * 1e6);
    CK(cudaGetLastError());
  };

  for (uint64_t n = 4096; n <= maxn; n <<= 2) {
    run("memcpy", n, [&] { CK(cudaMemcpyAsync(dst, src, n, cudaMemcpyDeviceToDevice, st)); });
    {
      const uint32_t g = static_cast<uint32_t>(std::min<uint64_t>((n + 32767) / 32768, 2ull * sms));
      const mpx::DirectArgs A{dst, src, n, 1, 4};
      run("engine_tma_32k", n, [&] { mpx::direct_kernel<<<g, 256, mpx::kBulkSmem, st>>>(A); });
    }
    {
      const uint32_t g = static_cast<uint32_t>(std::min<uint64_t>((n + 16383) / 16384, 4ull * sms));
      const mpx::DirectArgs A{dst, src, n, 0, 4};
      run("engine_reg_16k", n, [&] { mpx::direct_reg_kernel<<<g, 256, 0, st>>>(A); });
    }
    if (n / 16 <= 256ull * 4 * 4 * sms) {
      const uint64_t nv = n / 16;
      run("oneshot_v4", n, [&] {
        oneshot<4><<<static_cast<uint32_t>((nv + 1023) / 1024), 256, 0, st>>>(
            reinterpret_cast<uint4 *>(dst), reinterpret_cast<const uint4 *>(src), nv);
      });
    }
    if (n / 16 <= 256ull * 8 * 4 * sms) {
      const uint64_t nv = n / 16;
      run("oneshot_v8", n, [&] {
        oneshot<8><<<static_cast<uint32_t>((nv + 2047) / 2048), 256, 0, st>>>(
            reinterpret_cast<uint4 *>(dst), reinterpret_cast<const uint4 *>(src), nv);
      });
    }
    if (n / 16 <= 256ull * 1 * 8 * sms) {
      const uint64_t nv = n / 16;
      run("oneshot_v1", n, [&] {
        oneshot<1><<<static_cast<uint32_t>((nv + 255) / 256), 256, 0, st>>>(
            reinterpret_cast<uint4 *>(dst), reinterpret_cast<const uint4 *>(src), nv);
      });
    }
    {  // the engine's own launcher (direct-only config): one-shot kernel up to kSmallMax
      mpx::XferParams P;
      std::memset(&P, 0, sizeof(P));
      P.copy_mode = 1;
      P.bulk_stages = 4;
      P.allow_small = 1;
      P.npaths = 1;
      P.p[0].kind = mpx::DK_DIRECT;
      P.p[0].bytes = n;
      P.p[0].src = src;
      P.p[0].dst = dst;
      P.p[0].align = 256;
      P.p[0].g_in = static_cast<uint32_t>(std::min<uint64_t>((n + 32767) / 32768, 2ull * sms));
      P.nblocks = P.p[0].g_in;
      run("engine_launch_xfer", n, [&] { CK(static_cast<cudaError_t>(mpx::launch_xfer(P, st))); });
    }
    run("empty", n, [&] { empty_kernel<<<1, 32, 0, st>>>(0); });
    if (n <= 4ull << 20) {
      const uint32_t g = static_cast<uint32_t>((n / 16 + 255) / 256);
      const mpx::DirectArgs A{dst, src, n, 0, 4};
      run("oneshot_gc", n, [&] { oneshot_gc<<<g, 256, 0, st>>>(A); });
      run("oneshot_struct", n, [&] { oneshot_struct<<<g, 256, 0, st>>>(A); });
      run("oneshot_asm", n, [&] { oneshot_asm<<<g, 256, 0, st>>>(reinterpret_cast<uint4 *>(dst), reinterpret_cast<const uint4 *>(src), n / 16); });
      run("reg_scalar_1shot", n, [&] { reg_scalar<<<g, 256, 0, st>>>(dst, src, n); });
    }
    {
      const uint32_t g = static_cast<uint32_t>(std::min<uint64_t>((n + 16383) / 16384, 4ull * sms));
      const mpx::DirectArgs A{dst, src, n, 0, 4};
      run("reg_nospill_16k", n, [&] { reg_nospill<<<g, 256, 0, st>>>(A); });
    }
    if (n <= 8192ull * 8 * sms)
      run("tma_one_8k", n, [&] { tma_one<<<static_cast<uint32_t>((n + 8191) / 8192), 256, 0, st>>>(dst, src, n); });
    if (n / 16 <= 256ull * 1 * 8 * sms) {
      const uint64_t nv = n / 16;
      run("oneshot_v1_smem32k", n, [&] {
        oneshot<1><<<static_cast<uint32_t>((nv + 255) / 256), 256, mpx::kBulkSmem, st>>>(
            reinterpret_cast<uint4 *>(dst), reinterpret_cast<const uint4 *>(src), nv);
      });
    }
    for (uint64_t per : {8192ull}) {
      const uint32_t g = static_cast<uint32_t>(std::min<uint64_t>((n + per - 1) / per, 2ull * sms));
      const mpx::DirectArgs A{dst, src, n, 1, 4};
      char nm[64];
      std::snprintf(nm, sizeof nm, "engine_tma_%lluk", static_cast<unsigned long long>(per / 1024));
      run(nm, n, [&] { mpx::direct_kernel<<<g, 256, mpx::kBulkSmem, st>>>(A); });
    }
  }
  return 0;
}
