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
#include <cuda_bf16.h>
#include <cuda_runtime.h>

#include <utility>

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

// ------------------------------------------------------------------ TMA bulk copy

// Bulk-copy engine of one CTA: thread 0 streams BLK-byte blocks (8 KiB by default) global → shared →
// global with cp.async.bulk (TMA; SASS UBLKCP), kBulkStages blocks in flight, the
// load of each stage completing on an mbarrier (complete_tx) and each store tracked
// by a bulk group so a stage is only reloaded once its previous store has finished
// reading shared memory.  Blocks r, r+G, r+2G, … of the co-aligned 16-B body belong
// to CTA r; head/tail bytes go through group_copy.  Requires (dst ^ src) % 16 == 0.
// Sweep on B200 (scripts/copybench.cu, profiles/r01/copybench.jsonl): two pipelines
// per SM of 4 × 8 KiB beat both deeper/larger pipelines and cudaMemcpyAsync (+3.9 %).
constexpr uint32_t kBulkBlock = 8192;
constexpr uint32_t kBulkStages = 4;
constexpr uint32_t kBulkSmem = kBulkBlock * kBulkStages + 64;
// Staged legs of the loopback transfer kernel use 16 KiB blocks: one CTA's TMA rate is
// bound by the shared memory it keeps in flight (~32 KiB per ~1.5 µs round trip;
// few-CTA sweep, profiles/r01/copybench_few*.jsonl: 20 GB/s at 4 × 8 KiB, 40 GB/s at
// 4 × 16 KiB).  xfer_kernel launches with kXferSmem; residency drops from 4 to 3 CTAs
// per SM, and xfer_capacity() reports that, so the co-residency cap follows.
constexpr uint32_t kStagedBlock = 16384;
constexpr uint32_t kXferSmem = kStagedBlock * kBulkStages + 64;

__device__ __forceinline__ uint32_t smem_u32(const void *p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint32_t bar) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(bar) : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}

__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n}" ::"r"(bar),
      "r"(parity)
      : "memory");
}

__device__ __forceinline__ void bulk_load(uint32_t dst_smem, const void *src, uint32_t bytes, uint32_t bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst_smem),
      "l"(src), "r"(bytes), "r"(bar)
      : "memory");
}

__device__ __forceinline__ void bulk_store(void *dst, uint32_t src_smem, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst), "r"(src_smem), "r"(bytes)
               : "memory");
  asm volatile("cp.async.bulk.commit_group;" ::: "memory");
}

template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory");
}

__device__ __forceinline__ void bulk_wait_all() {
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
  asm volatile("fence.proxy.async.global;" ::: "memory");
}

template <int MODE, uint32_t BLK = kBulkBlock>
__device__ void bulk_copy(uint8_t *dst, const uint8_t *src, uint64_t len, uint32_t r, uint32_t G,
                          uint8_t *smem, uint32_t D, bool publish_after = true) {
  if ((reinterpret_cast<uintptr_t>(dst) ^ reinterpret_cast<uintptr_t>(src)) & 15u) {
    group_copy<MODE>(dst, src, len, r, G);
    return;
  }
  uint64_t head = (16u - (reinterpret_cast<uintptr_t>(src) & 15u)) & 15u;
  if (head > len) head = len;
  const uint64_t body = (len - head) & ~uint64_t(15);
  const uint64_t tail0 = head + body;
  // head and tail (< 16 B each) by CTA 0's threads
  if (r == 0) {
    if (threadIdx.x < head) dst[threadIdx.x] = ld1<MODE>(src + threadIdx.x);
    if (threadIdx.x < len - tail0) dst[tail0 + threadIdx.x] = ld1<MODE>(src + tail0 + threadIdx.x);
  }
  if (threadIdx.x != 0) return;
  // data published by another agent (acquired by this CTA before the barrier that
  // preceded this call) is about to be read through the async proxy
  if (MODE != LD_SRC) asm volatile("fence.proxy.async.global;" ::: "memory");
  const uint8_t *s = src + head;
  uint8_t *d = dst + head;
  const uint64_t nblk = (body + BLK - 1) / BLK;
  if (r >= nblk) return;
  const uint64_t mine = (nblk - r + G - 1) / G;  // blocks r, r+G, …
  if (D < 1 || D > kBulkStages) D = kBulkStages;
  uint64_t *bars = reinterpret_cast<uint64_t *>(smem + BLK * kBulkStages);
  for (uint32_t i = 0; i < D; ++i) mbar_init(smem_u32(bars + i));
  // make the initialised barriers visible to the async proxy (no cluster: CTA scope)
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  auto blk = [&](uint64_t it, uint64_t *off, uint32_t *bytes) {
    const uint64_t o = (r + it * G) * static_cast<uint64_t>(BLK);
    *off = o;
    *bytes = static_cast<uint32_t>(body - o < BLK ? body - o : BLK);
  };
  auto issue_load = [&](uint64_t it) {
    uint64_t o;
    uint32_t n;
    blk(it, &o, &n);
    const uint32_t st = static_cast<uint32_t>(it % D);
    const uint32_t bar = smem_u32(bars + st);
    mbar_expect_tx(bar, n);
    bulk_load(smem_u32(smem + st * BLK), s + o, n, bar);
  };
  const uint64_t pro = mine < D ? mine : D;
  for (uint64_t it = 0; it < pro; ++it) issue_load(it);
  for (uint64_t it = 0; it < mine; ++it) {
    const uint32_t st = static_cast<uint32_t>(it % D);
    mbar_wait(smem_u32(bars + st), static_cast<uint32_t>((it / D) & 1));
    uint64_t o;
    uint32_t n;
    blk(it, &o, &n);
    bulk_store(d + o, smem_u32(smem + st * BLK), n);
    // refill the stage used one iteration ago once its store has read shared memory
    if (it >= 1 && it - 1 + D < mine) {
      bulk_wait_read<1>();
      issue_load(it - 1 + D);
    }
  }
  if (publish_after) {
    bulk_wait_all();  // writes complete: a flag / byte count is released next
  } else {
    // nothing follows in this launch: only shared memory must outlive the reads
    // (kernel completion makes the global writes visible), as CUTLASS TMA epilogues do
    asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
  }
}

// ------------------------------------------------------------------ flags

// Warp 0 polls `n` flag words until every one is >= target (ld.acquire.sys), then
// the CTA synchronises.  Returns false (and raises DERR_TIMEOUT) on timeout, or when
// the optional host `stop` word becomes non-zero (persistent relay shutdown; then no
// error is raised and timeout_ns may be 0 = wait forever).
__device__ __forceinline__ bool wait_flags(const uint64_t *flags, uint32_t n, uint64_t target,
                                           uint64_t timeout_ns, int32_t *err, int *s_abort,
                                           const volatile int32_t *stop = nullptr) {
  if (threadIdx.x < 32) {
    const uint32_t lane = threadIdx.x;
    const uint64_t t_start = globaltimer();
    int why = 0;
    for (uint32_t it = 0;; ++it) {
      const bool mine = lane >= n || ld_acquire_sys(flags + lane) >= target;
      if (__all_sync(0xffffffffu, mine)) break;
      if (timeout_ns && globaltimer() - t_start > timeout_ns) {
        why = 1;
        break;
      }
      // fail fast: once any wait of this context has failed (sticky error word), the
      // flags this CTA waits for may never come — abort now instead of timing out in
      // turn behind it (the persistent relay, which passes `stop`, keeps serving)
      if (!stop && (it & 63u) == 63u &&
          __any_sync(0xffffffffu, lane == 0 && *reinterpret_cast<volatile int32_t *>(err) != 0)) {
        why = 3;
        break;
      }
      if (stop && (it & 255u) == 255u && *stop) {
        why = 2;
        break;
      }
      __nanosleep(stop ? 256 : 64);
    }
    if (lane == 0) {
      if (why == 1) atomicExch(err, DERR_TIMEOUT);
      if (why) *s_abort = 1;
    }
  }
  __syncthreads();
  return *s_abort == 0;
}

// Thread 0 polls one word until it equals / exceeds target, then the CTA syncs.
__device__ __forceinline__ bool wait_word(const uint64_t *w, uint64_t target, uint64_t timeout_ns,
                                          int32_t *err, int *s_abort) {
  if (threadIdx.x == 0) {
    const uint64_t t_start = globaltimer();
    for (uint32_t it = 0; ld_acquire_sys(w) < target; ++it) {
      if (globaltimer() - t_start > timeout_ns) {
        atomicExch(err, DERR_TIMEOUT);
        *s_abort = 1;
        break;
      }
      if ((it & 63u) == 63u && *reinterpret_cast<volatile int32_t *>(err) != 0) {  // fail fast
        *s_abort = 1;
        break;
      }
      __nanosleep(64);
    }
  }
  __syncthreads();
  return *s_abort == 0;
}

__device__ __forceinline__ void red_add_release_sys(uint64_t *p, uint64_t v) {
  asm volatile("red.release.sys.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ uint64_t ld_volatile(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.volatile.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

// One CTA copies its slice of a staged chunk: TMA pipeline (copy_mode 1) or LDG/STG.
template <int MODE, uint32_t BLK = kBulkBlock>
__device__ __forceinline__ void copy_slice(uint8_t *dst, const uint8_t *src, uint64_t len, uint8_t *smem,
                                           uint32_t copy_mode, uint32_t stages) {
  if (len == 0) return;
  if (copy_mode == 1)
    bulk_copy<MODE, BLK>(dst, src, len, 0, 1, smem, stages);
  else
    group_copy<MODE>(dst, src, len, 0, 1);
}

__device__ __forceinline__ void release_flag(uint64_t *flag, uint64_t value) {
  __syncthreads();
  if (threadIdx.x == 0) st_release_sys(flag, value);
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

// Slice r of G of [0, len), split on 16-byte boundaries.
__device__ __forceinline__ void slice_of(uint64_t len, uint32_t r, uint32_t G, uint64_t *a, uint64_t *b) {
  *a = ((len * r / G) + 15) & ~uint64_t(15);
  uint64_t e = ((len * (r + 1) / G) + 15) & ~uint64_t(15);
  if (r + 1 == G || e > len) e = len;
  if (*a > e) *a = e;
  *b = e;
}

// Programmatic dependent launch (PDL): let the stream's next kernel launch now (its
// CTAs become resident while this one runs), then wait until the stream's previous
// kernel has completed and its memory operations are visible.  Back-to-back messages
// (an OMB window, reading C24) then pay no launch gap.  Both instructions are no-ops
// for a kernel launched without the attribute.
__device__ __forceinline__ void pdl_enter() {
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  asm volatile("griddepcontrol.wait;" ::: "memory");
}

// ------------------------------------------------------------------ roles

__device__ void run_stage_in(const DevPath &p, uint32_t r, const XferParams &P, int *s_abort, uint8_t *smem) {
  for (uint32_t j = 0; j < p.k; ++j) {
    uint64_t off, len;
    chunk_range(p, j, &off, &len);
    const uint64_t q = p.q0 + j, s = q % p.slots, u = q / p.slots;
    if (!wait_flags(p.freef + s * kFlagStride, p.g_out, u, P.timeout_ns, P.err, s_abort)) return;
    const uint8_t *src = p.src + off;
    uint8_t *slot = p.ring + s * p.slot_stride + (reinterpret_cast<uintptr_t>(src) & 15u);
    uint64_t a, b;  // slice r of the chunk, split on 16-byte boundaries
    slice_of(len, r, p.g_in, &a, &b);
    copy_slice<LD_SRC, kStagedBlock>(slot + a, src + a, b - a, smem, P.copy_mode, P.bulk_stages);
    release_flag(p.full + s * kFlagStride + r, u + 1);
  }
}

template <int MODE>
__device__ void run_forward(const DevPath &p, uint32_t r, const XferParams &P, int *s_abort, uint8_t *smem) {
  for (uint32_t j = 0; j < p.k; ++j) {
    uint64_t off, len;
    chunk_range(p, j, &off, &len);
    const uint64_t q = p.q0 + j, s = q % p.slots, u = q / p.slots;
    if (!wait_flags(p.full + s * kFlagStride, p.g_in, u + 1, P.timeout_ns, P.err, s_abort)) return;
    const uint8_t *slot =
        p.ring + s * p.slot_stride + (reinterpret_cast<uintptr_t>(p.src + off) & 15u);
    uint64_t a, b;
    slice_of(len, r, p.g_out, &a, &b);
    copy_slice<MODE, kStagedBlock>(p.dst + off + a, slot + a, b - a, smem, P.copy_mode, P.bulk_stages);
    release_flag(p.freef + s * kFlagStride + r, u + 1);
  }
}

__global__ void __launch_bounds__(kThreads, 4) xfer_kernel(const __grid_constant__ XferParams P) {
  extern __shared__ __align__(128) uint8_t dyn_smem[];
  pdl_enter();
  __shared__ int s_abort;
  if (threadIdx.x == 0) s_abort = 0;
  __syncthreads();
  const uint32_t b = blockIdx.x;
  for (uint32_t i = 0; i < P.npaths; ++i) {
    const DevPath &p = P.p[i];
    if (p.bytes == 0) continue;
    if (b >= p.cta0_in && b < p.cta0_in + p.g_in) {
      if (p.kind == DK_DIRECT)
        if (P.copy_mode == 1)
          bulk_copy<LD_SRC>(p.dst, p.src, p.bytes, b - p.cta0_in, p.g_in, dyn_smem, P.bulk_stages, false);
        else
          group_copy<LD_SRC>(p.dst, p.src, p.bytes, b - p.cta0_in, p.g_in);
      else
        run_stage_in(p, b - p.cta0_in, P, &s_abort, dyn_smem);
      return;
    }
    if (p.kind == DK_STAGED && b >= p.cta0_out && b < p.cta0_out + p.g_out) {
      if (p.host_ring)
        run_forward<LD_HOST>(p, b - p.cta0_out, P, &s_abort, dyn_smem);
      else
        run_forward<LD_RING>(p, b - p.cta0_out, P, &s_abort, dyn_smem);
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


// ================================================================== multi-rank engine

__device__ __forceinline__ void chunk_of(uint64_t bytes, uint64_t align, uint32_t k, uint32_t j,
                                         uint64_t *off, uint64_t *len) {
  const uint64_t U = bytes / align, rem = bytes - U * align;
  const uint64_t s = align * ((j * U) / k);
  uint64_t e = align * (((j + 1) * U) / k);
  if (j + 1 == k) e += rem;
  *off = s;
  *len = e - s;
}

__device__ __forceinline__ MsgEntry *entry_at(uint8_t *ctrl, uint64_t base, uint32_t peer, uint64_t m) {
  return reinterpret_cast<MsgEntry *>(ctrl + base) + (static_cast<uint64_t>(peer) * kCtsRing + m % kCtsRing);
}

__device__ __forceinline__ uint64_t *done_at(uint8_t *ctrl, const CtrlLayout &L, uint32_t src) {
  return reinterpret_cast<uint64_t *>(ctrl + L.done + static_cast<uint64_t>(src) * 128);
}

// Base of rank `rank`'s receive region `region` in this process (see engine.h).
__device__ __forceinline__ uint8_t *region_base(const uint8_t *ctrl, const CtrlLayout &L, uint64_t region,
                                                uint32_t rank) {
  return reinterpret_cast<uint8_t *>(
      reinterpret_cast<const uint64_t *>(ctrl + L.regions)[region * L.world + rank]);
}

__device__ __forceinline__ uint64_t *flags_at(uint8_t *ctrl, uint64_t base, uint32_t who, uint32_t slots,
                                              uint64_t slot) {
  return reinterpret_cast<uint64_t *>(ctrl + base) + (static_cast<uint64_t>(who) * slots + slot) * kFlagStride;
}

// After a CTA's stores: make them visible system-wide, count `bytes` into a peer's
// done counter, optionally release a flag.
// The release operations carry the ordering themselves (bar.sync makes the CTA's
// prior writes precede thread 0's release, which is cumulative); no separate
// fence.acq_rel.sys — measured to cost ~18 µs per CTA per chunk on the multi-rank
// host path.  A byte counter on this same GPU only needs gpu scope.
__device__ __forceinline__ void red_add_release_gpu(uint64_t *p, uint64_t v) {
  asm volatile("red.release.gpu.global.add.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__device__ __forceinline__ void publish(uint64_t *done, uint64_t bytes, uint64_t *flag, uint64_t value,
                                        bool done_is_local = false) {
  __syncthreads();
  if (threadIdx.x == 0) {
    if (done && bytes) {
      if (done_is_local)
        red_add_release_gpu(done, bytes);
      else
        red_add_release_sys(done, bytes);
    }
    if (flag) st_release_sys(flag, value);
  }
}

// The rendezvous (P:62 analogue) runs in its own one-CTA launch ahead of the bulk
// send kernel on the same stream: the bulk kernel's hundreds of CTAs are only
// dispatched once the receiver's clear-to-send has arrived, so they never occupy SM
// slots spinning on it while a receive kernel on this GPU waits for room to run.
// PDL in the multi-rank engine: the gate waits for the stream's previous kernel, and
// lets the bulk send kernel launch only once the clear-to-send has arrived (no bulk
// CTA is ever resident during the rendezvous); send, receive and eager kernels let
// their successor launch at once and wait for their predecessor (pdl_enter).
__global__ void send_gate_kernel(const __grid_constant__ SendParams P) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  if (threadIdx.x != 0) return;
  MsgEntry *cts = entry_at(P.my_ctrl, P.L.cts, P.dst, P.seq);
  const uint64_t t_start = globaltimer();
  while (ld_acquire_sys(&cts->seq1) < P.seq + 1) {
    if (globaltimer() - t_start > P.timeout_ns) {
      atomicExch(P.err, DERR_TIMEOUT);
      return;
    }
    __nanosleep(64);
  }
  const uint64_t n = ld_volatile(&cts->b), tag = ld_volatile(&cts->c);
  const bool bad = (n != P.bytes) || (tag != P.tag);
  uint64_t host_k = 0, host_q0 = 0, host_off = 0, host_bytes = 0;
  for (uint32_t i = 0; i < P.npaths; ++i)
    if (P.sp[i].kind == 2) {
      host_k = P.sp[i].k;
      host_q0 = P.sp[i].q0;
      host_off = P.sp[i].off;
      host_bytes = P.sp[i].bytes;
    }
  // the receiver's host-ring consumers take the chunk layout from here (device
  // memory) — never from the slot headers in host memory, whose PCIe reads queue
  // behind the bulk traffic (measured ~18 µs per CTA per chunk)
  MsgEntry *h = entry_at(P.dst_ctrl, P.L.hdr, P.me, P.seq);
  h->a = bad ? 0 : host_k;
  h->b = host_q0;
  h->c = bad ? 2 : 0;
  h->d = host_off;
  h->e = host_bytes;
  h->f = reinterpret_cast<uintptr_t>(P.src + host_off) & 15u;
  st_release_sys(&h->seq1, P.seq + 1);
  if (bad) atomicExch(P.err, DERR_MISMATCH);
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

__global__ void __launch_bounds__(kThreads, 4) send_kernel(const __grid_constant__ SendParams P) {
  extern __shared__ __align__(128) uint8_t dyn_smem[];
  pdl_enter();
  __shared__ int s_abort;
  __shared__ uint64_t s_off, s_region;
  __shared__ uint8_t *s_dst;
  if (threadIdx.x == 0) s_abort = 0;
  __syncthreads();
  // the clear-to-send has arrived (send_gate_kernel ran first on this stream)
  MsgEntry *cts = entry_at(P.my_ctrl, P.L.cts, P.dst, P.seq);
  if (!wait_word(&cts->seq1, P.seq + 1, P.timeout_ns, P.err, &s_abort)) return;
  if (threadIdx.x == 0) {
    const uint64_t off = ld_volatile(&cts->a), n = ld_volatile(&cts->b), tag = ld_volatile(&cts->c);
    s_off = off;
    s_region = ld_volatile(&cts->d);
    if ((n != P.bytes) || (tag != P.tag) || s_region >= kMaxRegions) s_abort = 1;  // reported by the gate
    else s_dst = region_base(P.my_ctrl, P.L, s_region, P.dst) + off;
  }
  __syncthreads();
  if (s_abort) return;
  const uint64_t base = s_off;
  const uint32_t b = blockIdx.x;
  uint64_t *done = done_at(P.dst_ctrl, P.L, P.me);
  if (b < P.g_direct) {  // A7: direct NVLink stores into the receiver's heap
    if (P.copy_mode == 1)
      bulk_copy<LD_SRC>(s_dst, P.src, P.direct_bytes, b, P.g_direct, dyn_smem, P.bulk_stages);
    else
      group_copy<LD_SRC>(s_dst, P.src, P.direct_bytes, b, P.g_direct);
    const uint64_t share = P.direct_bytes * (b + 1) / P.g_direct - P.direct_bytes * b / P.g_direct;
    publish(done, share, nullptr, 0);
    return;
  }
  for (uint32_t i = 0; i < P.npaths; ++i) {
    const SendParams::StagedDesc &d = P.sp[i];
    if (b < d.cta0 || b >= d.cta0 + P.g_stage) continue;
    const uint32_t r = b - d.cta0;
    for (uint32_t j = 0; j < d.k; ++j) {  // A8/A9 step 1
      uint64_t off, len;
      chunk_of(d.bytes, 256, d.k, j, &off, &len);
      off += d.off;
      const uint64_t q = d.q0 + j;
      uint64_t *fr, *fl;
      uint8_t *slot;
      uint32_t nfree;
      if (d.kind == 1) {
        const uint64_t s = q % P.L.slots;
        fr = flags_at(P.my_ctrl, P.L.relay_free, d.relay, P.L.slots, s);
        fl = flags_at(d.ring_ctrl, P.L.ring_full, P.me, P.L.slots, s);
        slot = d.ring_ctrl + P.L.ring_data + (static_cast<uint64_t>(P.me) * P.L.slots + s) * P.L.stride;
        nfree = P.g_stage;
      } else {
        const uint64_t s = q % P.host_slots;
        fr = P.host.freef + s * kFlagStride;
        fl = P.host.full + s * kFlagStride;
        slot = P.host.data + s * P.host_stride;
        nfree = P.g_stage;
      }
      const uint64_t u = q / (d.kind == 1 ? P.L.slots : P.host_slots);
      if (!wait_flags(fr, nfree, u, P.timeout_ns, P.err, &s_abort)) return;
      const uint8_t *src = P.src + off;
      const uint64_t shift = reinterpret_cast<uintptr_t>(src) & 15u;
      uint8_t *data = slot + kSlotHdr + shift;
      uint64_t a, e;
      slice_of(len, r, P.g_stage, &a, &e);
      copy_slice<LD_SRC>(data + a, src + a, e - a, dyn_smem, P.copy_mode, P.bulk_stages);
      if (r == 0 && threadIdx.x == 0) {
        uint64_t *h = reinterpret_cast<uint64_t *>(slot);
        h[0] = P.dst;
        h[1] = base + off;
        h[2] = len;
        h[3] = shift;
        h[4] = s_region;
      }
      publish(nullptr, 0, fl + r, u + 1);
    }
    return;
  }
}

__global__ void __launch_bounds__(kThreads, 4) recv_kernel(const __grid_constant__ RecvParams P) {
  extern __shared__ __align__(128) uint8_t dyn_smem[];
  pdl_enter();
  __shared__ int s_abort;
  __shared__ uint64_t s_k, s_q0, s_hoff, s_hbytes, s_shift;
  if (threadIdx.x == 0) s_abort = 0;
  __syncthreads();
  MsgEntry *hdr = entry_at(P.my_ctrl, P.L.hdr, P.src, P.seq);
  if (blockIdx.x == 0) {
    if (threadIdx.x == 0) {  // post the clear-to-send into the sender's control block
      MsgEntry *cts = entry_at(P.src_ctrl, P.L.cts, P.me, P.seq);
      cts->a = P.region_off;
      cts->b = P.bytes;
      cts->c = P.tag;
      cts->d = P.region;
      fence_acq_rel_sys();
      st_release_sys(&cts->seq1, P.seq + 1);
      // A10: wait until every byte of the message has been counted in
      const uint64_t *done = done_at(P.my_ctrl, P.L, P.src);
      const uint64_t t_start = globaltimer();
      while (ld_acquire_sys(done) < P.done_target) {
        if (ld_acquire_sys(&hdr->seq1) == P.seq + 1 && ld_volatile(&hdr->c) == 2) {
          atomicExch(P.err, DERR_MISMATCH);
          break;
        }
        if (globaltimer() - t_start > P.timeout_ns) {
          atomicExch(P.err, DERR_TIMEOUT);
          break;
        }
        __nanosleep(128);
      }
      fence_acq_rel_sys();
    }
    return;
  }
  // A9 step 3: host-ring consumers
  const uint32_t r = blockIdx.x - 1;
  if (!wait_word(&hdr->seq1, P.seq + 1, P.timeout_ns, P.err, &s_abort)) return;
  if (threadIdx.x == 0) {
    s_k = ld_volatile(&hdr->c) ? 0 : ld_volatile(&hdr->a);
    s_q0 = ld_volatile(&hdr->b);
    s_hoff = ld_volatile(&hdr->d);
    s_hbytes = ld_volatile(&hdr->e);
    s_shift = ld_volatile(&hdr->f);
  }
  __syncthreads();
  uint64_t *done = done_at(P.my_ctrl, P.L, P.src);
  for (uint64_t j = 0; j < s_k; ++j) {
    const uint64_t q = s_q0 + j, s = q % P.host_slots, u = q / P.host_slots;
    if (!wait_flags(P.host.full + s * kFlagStride, P.g_host, u + 1, P.timeout_ns, P.err, &s_abort)) return;
    uint8_t *slot = P.host.data + s * P.host_stride;
    uint64_t off, len;
    chunk_of(s_hbytes, 256, static_cast<uint32_t>(s_k), static_cast<uint32_t>(j), &off, &len);
    uint64_t a, e;
    slice_of(len, r, P.g_host, &a, &e);
    copy_slice<LD_HOST>(P.buf + s_hoff + off + a, slot + kSlotHdr + s_shift + a, e - a, dyn_smem,
                        P.copy_mode, P.bulk_stages);
    publish(done, e - a, P.host.freef + s * kFlagStride + r, u + 1, /*done_is_local=*/true);
  }
}

// Persistent relay (A8 step 3): CTA group s (g CTAs) forwards sender s's ring.
__global__ void __launch_bounds__(kThreads, 4) relay_kernel(const __grid_constant__ RelayParams P) {
  extern __shared__ __align__(128) uint8_t dyn_smem[];
  __shared__ int s_abort;
  __shared__ uint64_t s_h[5];
  if (threadIdx.x == 0) s_abort = 0;
  __syncthreads();
  const uint32_t sender = blockIdx.x / P.g, r = blockIdx.x % P.g;
  if (sender == P.me || sender >= P.world) return;
  // ring position survives a stop/restart (mp_calibrate stops the relay)
  uint64_t *pos = reinterpret_cast<uint64_t *>(P.my_ctrl + P.L.relay_pos) + sender;
  for (uint64_t q = ld_volatile(pos);; ++q) {
    const uint64_t s = q % P.L.slots, u = q / P.L.slots;
    uint64_t *fl = flags_at(P.my_ctrl, P.L.ring_full, sender, P.L.slots, s);
    if (!wait_flags(fl, P.g, u + 1, 0, P.err, &s_abort, P.stop)) {
      if (r == 0 && threadIdx.x == 0) *pos = q;
      return;
    }
    uint8_t *slot = P.my_ctrl + P.L.ring_data + (static_cast<uint64_t>(sender) * P.L.slots + s) * P.L.stride;
    if (threadIdx.x < 5) s_h[threadIdx.x] = ld_volatile(reinterpret_cast<const uint64_t *>(slot) + threadIdx.x);
    __syncthreads();
    const uint32_t dst = static_cast<uint32_t>(s_h[0]);
    const uint64_t off = s_h[1], len = s_h[2], shift = s_h[3];
    uint64_t a, e;
    slice_of(len, r, P.g, &a, &e);
    copy_slice<LD_RING>(region_base(P.my_ctrl, P.L, s_h[4], dst) + off + a, slot + kSlotHdr + shift + a, e - a, dyn_smem, P.copy_mode,
                        P.bulk_stages);
    uint64_t *fr = flags_at(P.peer[sender].ctrl, P.L.relay_free, P.me, P.L.slots, s);
    publish(done_at(P.peer[dst].ctrl, P.L, sender), e - a, fr + r, u + 1);
  }
}


// Eager protocol (engine.h, reading C23).  Slot = [kEagerHdr header][shift][data]:
// header words 0/1 = bytes/tag (CTA 0), 16 + r = source shift of CTA r's slice, 8 + r =
// CTA r's sequence flag (seq + 1, released after its slice).
__global__ void __launch_bounds__(kThreads) eager_send_kernel(const __grid_constant__ EagerParams P) {
  pdl_enter();
  __shared__ int s_abort;
  if (threadIdx.x == 0) s_abort = 0;
  __syncthreads();
  const uint32_t r = blockIdx.x;
  // the slot is free once the receiver has returned message seq − kEagerSlots
  if (P.seq >= kEagerSlots && !wait_word(P.free_ctr, P.seq + 1 - kEagerSlots, P.timeout_ns, P.err, &s_abort))
    return;
  uint64_t *hdr = reinterpret_cast<uint64_t *>(P.slot);
  const uint64_t shift = reinterpret_cast<uintptr_t>(P.src) & 15u;
  uint8_t *data = P.slot + kEagerHdr + shift;
  const uint64_t a = static_cast<uint64_t>(r) * kEagerSlice;
  const uint64_t e = a + kEagerSlice < P.bytes ? a + kEagerSlice : P.bytes;
  if (a < e) group_copy<LD_SRC>(data + a, P.src + a, e - a, 0, 1);
  if (threadIdx.x == 0) {
    if (r == 0) {
      hdr[0] = P.bytes;
      hdr[1] = P.tag;
    }
    hdr[16 + r] = shift;
  }
  __syncthreads();  // the CTA's stores precede thread 0's release (cumulative)
  if (threadIdx.x == 0) st_release_sys(hdr + 8 + r, P.seq + 1);
}

__global__ void __launch_bounds__(kThreads) eager_recv_kernel(const __grid_constant__ EagerParams P) {
  pdl_enter();
  __shared__ int s_abort;
  if (threadIdx.x == 0) s_abort = 0;
  __syncthreads();
  const uint32_t r = blockIdx.x;
  const uint64_t *hdr = reinterpret_cast<const uint64_t *>(P.slot);
  if (!wait_word(hdr + 8 + r, P.seq + 1, P.timeout_ns, P.err, &s_abort)) return;
  if (r == 0 && threadIdx.x == 0 && (ld_volatile(hdr) != P.bytes || ld_volatile(hdr + 1) != P.tag))
    atomicExch(P.err, DERR_MISMATCH);
  const uint8_t *data = P.slot + kEagerHdr + ld_volatile(hdr + 16 + r);
  const uint64_t a = static_cast<uint64_t>(r) * kEagerSlice;
  const uint64_t e = a + kEagerSlice < P.bytes ? a + kEagerSlice : P.bytes;
  if (a < e) group_copy<LD_RING>(P.dst + a, data + a, e - a, 0, 1);
  __syncthreads();
  if (threadIdx.x == 0) {
    // the last CTA out returns the slot to the sender
    if (atomicAdd(P.cnt, 1u) == P.ctas - 1) {
      atomicExch(P.cnt, 0u);
      red_add_release_sys(P.free_ctr, 1);
    }
  }
}

// Direct-only messages (the B200-mode pick whenever the shared port is saturated by
// the direct path, and every calibration copy) get this small kernel instead of the
// fused one: ~30x less code, so a cold SM starts copying after far fewer instruction
// fetch misses (ncu on a 1 MiB fused launch: "no_instruction" was the top stall).
struct DirectArgs {
  uint8_t *dst;
  const uint8_t *src;
  uint64_t bytes;
  uint32_t copy_mode, stages;
};

__global__ void __launch_bounds__(kThreads, 4) direct_kernel(const __grid_constant__ DirectArgs A) {
  extern __shared__ __align__(128) uint8_t dyn_smem[];
  pdl_enter();
  bulk_copy<LD_SRC>(A.dst, A.src, A.bytes, blockIdx.x, gridDim.x, dyn_smem, A.stages, false);
}

// Step 1's timing copy of a loopback staged leg: the same striped TMA pipeline as
// direct_kernel, with the staged legs' block size (kStagedBlock), so the calibrated
// leg β is what a stage group of that many CTAs moves.
__global__ void __launch_bounds__(kThreads, 4) direct_leg_kernel(const __grid_constant__ DirectArgs A) {
  extern __shared__ __align__(128) uint8_t dyn_smem[];
  pdl_enter();
  bulk_copy<LD_SRC, kStagedBlock>(A.dst, A.src, A.bytes, blockIdx.x, gridDim.x, dyn_smem, A.stages, false);
}

// One-shot small copy (co-aligned src/dst): thread i of the grid moves vector i of the
// 16-B body; the last CTA also moves the < 16-byte head and tail.  Kept tiny and
// branch-light on purpose: at these sizes a launch on a cold SM is bound by its
// instruction fetches, not by the bytes.
__global__ void __launch_bounds__(kThreads) direct_small_kernel(uint8_t *dst, const uint8_t *src, uint64_t n) {
  pdl_enter();
  uint64_t head = (16u - (reinterpret_cast<uintptr_t>(src) & 15u)) & 15u;
  if (head > n) head = n;
  const uint64_t nvec = (n - head) >> 4;
  const uint64_t i = static_cast<uint64_t>(blockIdx.x) * kThreads + threadIdx.x;
  if (i < nvec)
    st16(reinterpret_cast<uint4 *>(dst + head) + i, ld16<LD_SRC>(reinterpret_cast<const uint4 *>(src + head) + i));
  if (blockIdx.x + 1 == gridDim.x) {
    const uint64_t t0 = head + (nvec << 4);
    if (threadIdx.x < head) dst[threadIdx.x] = ld1<LD_SRC>(src + threadIdx.x);
    if (threadIdx.x < n - t0) dst[t0 + threadIdx.x] = ld1<LD_SRC>(src + t0 + threadIdx.x);
  }
}

// LDG/STG direct copy (MPX_COPY=reg): no min-blocks bound, so the 4-deep unrolled
// vector loop gets the registers it needs (a 64-register cap made it spill).
__global__ void __launch_bounds__(kThreads) direct_reg_kernel(const __grid_constant__ DirectArgs A) {
  pdl_enter();
  group_copy<LD_SRC>(A.dst, A.src, A.bytes, blockIdx.x, gridDim.x);
}

// Elementwise dst += src (Allreduce, NEXT f3): grid-stride over 16-byte vectors when
// both pointers are 16-B aligned, element tail and unaligned inputs element-wise.
template <typename T>
__device__ __forceinline__ T add_elem(T a, T b) { return a + b; }
template <>
__device__ __forceinline__ __nv_bfloat16 add_elem(__nv_bfloat16 a, __nv_bfloat16 b) {
  return __float2bfloat16(__bfloat162float(a) + __bfloat162float(b));
}

template <typename T>
__global__ void __launch_bounds__(kThreads) reduce_add_kernel(T *dst, const T *src, uint64_t n) {
  constexpr int E = 16 / sizeof(T);
  const uint64_t gt = static_cast<uint64_t>(blockIdx.x) * kThreads + threadIdx.x;
  const uint64_t GT = static_cast<uint64_t>(gridDim.x) * kThreads;
  uint64_t done = 0;
  if (((reinterpret_cast<uintptr_t>(dst) | reinterpret_cast<uintptr_t>(src)) & 15u) == 0) {
    const uint64_t nv = n / E;
    for (uint64_t i = gt; i < nv; i += GT) {
      uint4 a = reinterpret_cast<const uint4 *>(dst)[i];
      const uint4 b = ld16<LD_RING>(reinterpret_cast<const uint4 *>(src) + i);
      T *pa = reinterpret_cast<T *>(&a);
      const T *pb = reinterpret_cast<const T *>(&b);
#pragma unroll
      for (int e = 0; e < E; ++e) pa[e] = add_elem(pa[e], pb[e]);
      reinterpret_cast<uint4 *>(dst)[i] = a;
    }
    done = nv * E;
  }
  for (uint64_t i = done + gt; i < n; i += GT) dst[i] = add_elem(dst[i], src[i]);
}

}  // namespace

int launch_reduce(int dtype, void *dst, const void *src, uint64_t bytes, void *stream) {
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  auto grid = [&](uint64_t vec) {
    const uint64_t g = (vec + kThreads - 1) / kThreads;
    return static_cast<uint32_t>(g < 1 ? 1 : (g > 1184 ? 1184 : g));
  };
  switch (dtype) {
    case 1:  // MP_DT_I32
      reduce_add_kernel<int32_t><<<grid(bytes / 16), kThreads, 0, s>>>(
          static_cast<int32_t *>(dst), static_cast<const int32_t *>(src), bytes / 4);
      break;
    case 2:  // MP_DT_I64
      reduce_add_kernel<long long><<<grid(bytes / 16), kThreads, 0, s>>>(
          static_cast<long long *>(dst), static_cast<const long long *>(src), bytes / 8);
      break;
    case 3:  // MP_DT_F32
      reduce_add_kernel<float><<<grid(bytes / 16), kThreads, 0, s>>>(static_cast<float *>(dst),
                                                                      static_cast<const float *>(src), bytes / 4);
      break;
    case 4:  // MP_DT_F64
      reduce_add_kernel<double><<<grid(bytes / 16), kThreads, 0, s>>>(static_cast<double *>(dst),
                                                                       static_cast<const double *>(src), bytes / 8);
      break;
    case 5:  // MP_DT_BF16
      reduce_add_kernel<__nv_bfloat16><<<grid(bytes / 16), kThreads, 0, s>>>(
          static_cast<__nv_bfloat16 *>(dst), static_cast<const __nv_bfloat16 *>(src), bytes / 2);
      break;
    default:
      return static_cast<int>(cudaErrorInvalidValue);
  }
  return static_cast<int>(cudaGetLastError());
}

namespace {
// <<<>>> with the PDL attribute when asked (cudaLaunchKernelEx).
template <typename... KArgs, typename... Args>
int launch_k(bool pdl, void (*kern)(KArgs...), uint32_t grid, uint32_t smem, void *stream, Args &&...args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = static_cast<cudaStream_t>(stream);
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl ? 1 : 0;
  return static_cast<int>(cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...));
}
}  // namespace

int launch_xfer(const XferParams &P, void *stream) {
  if (P.nblocks == 0) return cudaSuccess;
  const bool pdl = P.pdl != 0;
  bool direct_only = P.p[0].kind == DK_DIRECT && P.p[0].cta0_in == 0 && P.p[0].g_in == P.nblocks;
  for (uint32_t i = 1; i < P.npaths; ++i)
    if (P.p[i].bytes) direct_only = false;
  if (direct_only && P.allow_small && P.p[0].bytes <= kSmallMax &&
      ((reinterpret_cast<uintptr_t>(P.p[0].dst) ^ reinterpret_cast<uintptr_t>(P.p[0].src)) & 15u) == 0) {
    const uint64_t nvec = P.p[0].bytes >> 4;
    const uint32_t g = static_cast<uint32_t>(nvec ? (nvec + kThreads - 1) / kThreads : 1);
    return launch_k(pdl, direct_small_kernel, g, 0, stream, P.p[0].dst, static_cast<const uint8_t *>(P.p[0].src),
                    P.p[0].bytes);
  }
  if (direct_only) {
    const DirectArgs A{P.p[0].dst, P.p[0].src, P.p[0].bytes, P.copy_mode, P.bulk_stages};
    if (P.copy_mode == 1 && P.staged_blk) return launch_k(pdl, direct_leg_kernel, P.nblocks, kXferSmem, stream, A);
    if (P.copy_mode == 1) return launch_k(pdl, direct_kernel, P.nblocks, kBulkSmem, stream, A);
    return launch_k(pdl, direct_reg_kernel, P.nblocks, 0, stream, A);
  }
  return launch_k(pdl, xfer_kernel, P.nblocks, kXferSmem, stream, P);
}

int launch_send(const SendParams &P, void *stream) {
  const bool pdl = P.pdl != 0;
  cudaLaunchConfig_t cfg = {};  // the gate is one warp
  cfg.gridDim = dim3(1);
  cfg.blockDim = dim3(32);
  cfg.stream = static_cast<cudaStream_t>(stream);
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = pdl ? 1 : 0;
  if (int e = static_cast<int>(cudaLaunchKernelEx(&cfg, send_gate_kernel, P))) return e;
  return launch_k(pdl, send_kernel, P.nblocks, kBulkSmem, stream, P);
}

int launch_eager_send(const EagerParams &P, void *stream) {
  return launch_k(P.pdl != 0, eager_send_kernel, P.ctas, 0, stream, P);
}

int launch_eager_recv(const EagerParams &P, void *stream) {
  return launch_k(P.pdl != 0, eager_recv_kernel, P.ctas, 0, stream, P);
}

int launch_recv(const RecvParams &P, void *stream) {
  return launch_k(P.pdl != 0, recv_kernel, P.nblocks, kBulkSmem, stream, P);
}

int launch_relay(const RelayParams &P, void *stream) {
  relay_kernel<<<P.world * P.g, kThreads, kBulkSmem, static_cast<cudaStream_t>(stream)>>>(P);
  return static_cast<int>(cudaGetLastError());
}

int launch_pingpong(uint64_t *flags, int iters, uint64_t timeout_ns, int32_t *err, void *stream) {
  pingpong_kernel<<<2, 32, 0, static_cast<cudaStream_t>(stream)>>>(flags, iters, timeout_ns, err);
  return static_cast<int>(cudaGetLastError());
}

int preload_kernels() {
  // CUDA 12 loads kernels lazily, and loading may need a context synchronisation;
  // with the persistent relay kernel running that would deadlock the first launch of
  // any other engine kernel.  Force every kernel of this module to load up front.
  cudaFuncAttributes a;
  cudaError_t e = cudaFuncSetAttribute(xfer_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kXferSmem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(send_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kBulkSmem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(recv_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kBulkSmem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(relay_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kBulkSmem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(direct_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kBulkSmem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(direct_leg_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kXferSmem);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, direct_leg_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, xfer_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, direct_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, direct_reg_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, direct_small_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, eager_send_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, eager_recv_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, reduce_add_kernel<int32_t>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, reduce_add_kernel<long long>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, reduce_add_kernel<float>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, reduce_add_kernel<double>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, reduce_add_kernel<__nv_bfloat16>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, send_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, send_gate_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, recv_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, relay_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, pingpong_kernel);
  return static_cast<int>(e);
}

int xfer_capacity(int device, int *per_sm, int *sms) {
  int n = 0;
  cudaError_t e = cudaFuncSetAttribute(xfer_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kXferSmem);
  if (e != cudaSuccess) return static_cast<int>(e);
  e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, xfer_kernel, kThreads, kXferSmem);
  if (e != cudaSuccess) return static_cast<int>(e);
  int s = 0;
  e = cudaDeviceGetAttribute(&s, cudaDevAttrMultiProcessorCount, device);
  if (e != cudaSuccess) return static_cast<int>(e);
  *per_sm = n;
  *sms = s;
  return cudaSuccess;
}

}  // namespace mpx
