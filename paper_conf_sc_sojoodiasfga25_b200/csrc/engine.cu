// engine.cu — sm_100a kernels of the multi-path transfer engine.
//
// The hot path of PAPER.md §3.4 on B200: every path of the chosen
// config is served by CTA groups of ONE fused launch (see engine.h):
//   * direct group   (A7): 128-bit vector copy source → destination;
//   * stage-in group (A8/A9 step 1): chunk → ring slot, then release per-CTA flags;
//   * forward group  (A8/A9 step 3): acquire the flags (step 2, the ε of Eq 2/12),
//                    slot → destination, release the slot.
// Memory ordering: the releasing CTA does bar.sync, then one thread issues
// fence.acq_rel.sys and a st.release.sys of its flag; the waiting CTA's warp 0
// polls with ld.acquire.sys, then bar.sync.  Ring data is read with L1-bypassing
// loads (.cg for device rings, .cv for host rings).  Every wait is bounded by
// %globaltimer and raises DERR_TIMEOUT instead of hanging.
#include <cuda_runtime.h>

#include "engine.h"

namespace mpx {

namespace {

// ------------------------------------------------------------------ PTX helpers

__device__ __forceinline__ uint64_t ld_acquire_sys(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void st_release_sys(uint64_t *p, uint64_t v) {
  asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void fence_acq_rel_sys() { asm volatile("fence.acq_rel.sys;" ::: "memory"); }

__device__ __forceinline__ uint64_t globaltimer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Load modes: user source (read-only for the kernel's lifetime), device ring
// (written by another CTA / GPU in this launch), host ring (PCIe, written by a GPU).
enum LoadMode { LD_SRC = 0, LD_RING = 1, LD_HOST = 2 };

template <int MODE>
__device__ __forceinline__ uint4 ld16(const uint4 *p) {
  uint4 r;
  if (MODE == LD_SRC)
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  else if (MODE == LD_RING)
    asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  else
    asm volatile("ld.global.cv.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

template <int MODE>
__device__ __forceinline__ uint8_t ld1(const uint8_t *p) {
  unsigned short v;
  if (MODE == LD_SRC)
    asm volatile("ld.global.nc.u8 %0, [%1];" : "=h"(v) : "l"(p));
  else if (MODE == LD_RING)
    asm volatile("ld.global.cg.u8 %0, [%1];" : "=h"(v) : "l"(p));
  else
    asm volatile("ld.global.cv.u8 %0, [%1];" : "=h"(v) : "l"(p));
  return static_cast<uint8_t>(v);
}

__device__ __forceinline__ void st16(uint4 *p, const uint4 &v) {
  asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}

// ------------------------------------------------------------------ group copy

// Copy len bytes src → dst cooperatively across a group of G CTAs (this CTA is
// number r of the group).  When src and dst are co-aligned mod 16 the body moves
// 16-byte vectors, 4 independent loads in flight per thread, each warp-coalesced;
// head/tail bytes go byte-wise.  Otherwise a byte-wise strided copy.
template <int MODE>
__device__ __forceinline__ void group_copy(uint8_t *dst, const uint8_t *src, uint64_t len, uint32_t r,
                                           uint32_t G) {
  const uint64_t gt = static_cast<uint64_t>(r) * blockDim.x + threadIdx.x;
  const uint64_t GT = static_cast<uint64_t>(G) * blockDim.x;
  if ((reinterpret_cast<uintptr_t>(dst) ^ reinterpret_cast<uintptr_t>(src)) & 15u) {
    for (uint64_t i = gt; i < len; i += GT) dst[i] = ld1<MODE>(src + i);
    return;
  }
  uint64_t head = (16u - (reinterpret_cast<uintptr_t>(src) & 15u)) & 15u;
  if (head > len) head = len;
  if (gt < head) dst[gt] = ld1<MODE>(src + gt);
  const uint64_t nvec = (len - head) >> 4;
  const uint4 *s4 = reinterpret_cast<const uint4 *>(src + head);
  uint4 *d4 = reinterpret_cast<uint4 *>(dst + head);
  constexpr int U = 4;
  uint64_t i = gt;
  for (; i + (U - 1) * GT < nvec; i += U * GT) {
    uint4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = ld16<MODE>(s4 + i + u * GT);
#pragma unroll
    for (int u = 0; u < U; ++u) st16(d4 + i + u * GT, v[u]);
  }
  for (; i < nvec; i += GT) st16(d4 + i, ld16<MODE>(s4 + i));
  const uint64_t t0 = head + (nvec << 4);
  if (gt < len - t0) dst[t0 + gt] = ld1<MODE>(src + t0 + gt);
}

// ------------------------------------------------------------------ flags

// Warp 0 polls `n` flag words until every one is >= target (ld.acquire.sys), then
// the CTA synchronises.  Returns false (and raises DERR_TIMEOUT) on timeout.
__device__ __forceinline__ bool wait_flags(const uint64_t *flags, uint32_t n, uint64_t target,
                                           const XferParams &P, int *s_abort) {
  if (threadIdx.x < 32) {
    const uint32_t lane = threadIdx.x;
    const uint64_t t_start = globaltimer();
    bool ok = true;
    for (;;) {
      const bool mine = lane >= n || ld_acquire_sys(flags + lane) >= target;
      if (__all_sync(0xffffffffu, mine)) break;
      if (globaltimer() - t_start > P.timeout_ns) {
        ok = false;
        break;
      }
      __nanosleep(64);
    }
    if (lane == 0) {
      if (!ok) {
        atomicExch(P.err, DERR_TIMEOUT);
        *s_abort = 1;
      }
      fence_acq_rel_sys();
    }
  }
  __syncthreads();
  return *s_abort == 0;
}

__device__ __forceinline__ void release_flag(uint64_t *flag, uint64_t value) {
  __syncthreads();
  if (threadIdx.x == 0) {
    fence_acq_rel_sys();
    st_release_sys(flag, value);
  }
}

// Reading C6: chunk j of a staged share [0, bytes) in units of A.
__device__ __forceinline__ void chunk_range(const DevPath &p, uint32_t j, uint64_t *off, uint64_t *len) {
  const uint64_t U = p.bytes / p.align, rem = p.bytes - U * p.align;
  const uint64_t s = p.align * ((j * U) / p.k);
  uint64_t e = p.align * (((j + 1) * U) / p.k);
  if (j + 1 == p.k) e += rem;
  *off = s;
  *len = e - s;
}

// ------------------------------------------------------------------ roles

__device__ void run_stage_in(const DevPath &p, uint32_t r, const XferParams &P, int *s_abort) {
  for (uint32_t j = 0; j < p.k; ++j) {
    uint64_t off, len;
    chunk_range(p, j, &off, &len);
    const uint64_t q = p.q0 + j, s = q % p.slots, u = q / p.slots;
    if (!wait_flags(p.freef + s * kFlagStride, p.g_out, u, P, s_abort)) return;
    const uint8_t *src = p.src + off;
    uint8_t *slot = p.ring + s * p.slot_stride + (reinterpret_cast<uintptr_t>(src) & 15u);
    // slice r of the chunk, split on 16-byte boundaries of the source
    const uint64_t a = ((len * r / p.g_in) + 15) & ~uint64_t(15);
    uint64_t b = ((len * (r + 1) / p.g_in) + 15) & ~uint64_t(15);
    if (r + 1 == p.g_in || b > len) b = len;
    if (a < b) group_copy<LD_SRC>(slot + a, src + a, b - a, 0, 1);
    release_flag(p.full + s * kFlagStride + r, u + 1);
  }
}

template <int MODE>
__device__ void run_forward(const DevPath &p, uint32_t r, const XferParams &P, int *s_abort) {
  for (uint32_t j = 0; j < p.k; ++j) {
    uint64_t off, len;
    chunk_range(p, j, &off, &len);
    const uint64_t q = p.q0 + j, s = q % p.slots, u = q / p.slots;
    if (!wait_flags(p.full + s * kFlagStride, p.g_in, u + 1, P, s_abort)) return;
    const uint8_t *slot =
        p.ring + s * p.slot_stride + (reinterpret_cast<uintptr_t>(p.src + off) & 15u);
    group_copy<MODE>(p.dst + off, slot, len, r, p.g_out);
    release_flag(p.freef + s * kFlagStride + r, u + 1);
  }
}

__global__ void __launch_bounds__(kThreads, 4) xfer_kernel(const __grid_constant__ XferParams P) {
  __shared__ int s_abort;
  if (threadIdx.x == 0) s_abort = 0;
  __syncthreads();
  const uint32_t b = blockIdx.x;
  for (uint32_t i = 0; i < P.npaths; ++i) {
    const DevPath &p = P.p[i];
    if (p.bytes == 0) continue;
    if (b >= p.cta0_in && b < p.cta0_in + p.g_in) {
      if (p.kind == DK_DIRECT)
        group_copy<LD_SRC>(p.dst, p.src, p.bytes, b - p.cta0_in, p.g_in);
      else
        run_stage_in(p, b - p.cta0_in, P, &s_abort);
      return;
    }
    if (p.kind == DK_STAGED && b >= p.cta0_out && b < p.cta0_out + p.g_out) {
      if (p.host_ring)
        run_forward<LD_HOST>(p, b - p.cta0_out, P, &s_abort);
      else
        run_forward<LD_RING>(p, b - p.cta0_out, P, &s_abort);
      return;
    }
  }
}

// Flag ping-pong between block 0 and block 1: ε probe (calibration, C12).
__global__ void pingpong_kernel(uint64_t *flags, int iters, uint64_t timeout_ns, int32_t *err) {
  if (threadIdx.x != 0) return;
  const uint64_t t0 = globaltimer();
  const int me = blockIdx.x;
  for (int i = 0; i < iters; ++i) {
    if (me == 0) {
      st_release_sys(flags + 0, 2 * i + 1);
      while (ld_acquire_sys(flags + 1) < static_cast<uint64_t>(2 * i + 1)) {
        if (globaltimer() - t0 > timeout_ns) {
          atomicExch(err, DERR_TIMEOUT);
          return;
        }
      }
    } else {
      while (ld_acquire_sys(flags + 0) < static_cast<uint64_t>(2 * i + 1)) {
        if (globaltimer() - t0 > timeout_ns) {
          atomicExch(err, DERR_TIMEOUT);
          return;
        }
      }
      st_release_sys(flags + 1, 2 * i + 1);
    }
  }
}

}  // namespace

int launch_xfer(const XferParams &P, void *stream) {
  if (P.nblocks == 0) return cudaSuccess;
  xfer_kernel<<<P.nblocks, kThreads, 0, static_cast<cudaStream_t>(stream)>>>(P);
  return static_cast<int>(cudaGetLastError());
}

int launch_pingpong(uint64_t *flags, int iters, uint64_t timeout_ns, int32_t *err, void *stream) {
  pingpong_kernel<<<2, 32, 0, static_cast<cudaStream_t>(stream)>>>(flags, iters, timeout_ns, err);
  return static_cast<int>(cudaGetLastError());
}

int xfer_capacity(int device, int *per_sm, int *sms) {
  int n = 0;
  cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, xfer_kernel, kThreads, 0);
  if (e != cudaSuccess) return static_cast<int>(e);
  int s = 0;
  e = cudaDeviceGetAttribute(&s, cudaDevAttrMultiProcessorCount, device);
  if (e != cudaSuccess) return static_cast<int>(e);
  *per_sm = n;
  *sms = s;
  return cudaSuccess;
}

}  // namespace mpx
