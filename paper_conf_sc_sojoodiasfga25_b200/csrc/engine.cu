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

// Polling and publishing under load: an acquire or release at system scope is a
// MEMBAR.SYS, which measured ~12 µs while the engine's streams are in flight
// (scripts/diag/lane_trace.py).  Polls are relaxed, with one acquire once the value has
// arrived; several flags published together share one fence, then relaxed stores
// (the PTX release pattern: a fence followed by a strong write).
__device__ __forceinline__ uint64_t ld_relaxed_sys(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

__device__ __forceinline__ void st_relaxed_sys(uint64_t *p, uint64_t v) {
  asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

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
// 4 × 16 KiB).  Kernels with staged CTAs launch with staged_smem<D>() (below); their
// residency (3 CTAs per SM at 4 stages, 2 at 6) comes from xfer_capacity().
constexpr uint32_t kStagedBlock = 16384;
// Stages of a staged lane's streamed pipeline (lane_stream) and of Step 1's staged-leg
// timing copy (direct_leg_kernel).  Deep (6 × 16 KiB = 96 KiB in flight per CTA) moves a
// lane ~19 % faster than 4 stages (relay ring alone, 16 lanes: 590-604 → 703-718 GB/s;
// profiles/r02/stages) but leaves 2 CTAs per SM instead of 3, so the host picks the
// depth per launch (deep when the staged CTAs leave every SM room for a direct CTA).
constexpr uint32_t kDeepStages = 6;
static_assert(kDeepStages >= kBulkStages, "staged CTAs also run the 4-stage per-chunk path");
// dynamic shared memory of a kernel with staged CTAs of depth D: the stages, then a
// full and an empty mbarrier per stage
template <uint32_t D>
constexpr uint32_t staged_smem() {
  return kStagedBlock * D + 16 * D + 64;
}

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

template <int MODE, uint32_t BLK = kBulkBlock, uint32_t MAXD = kBulkStages>
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
  if (D < 1 || D > MAXD) D = MAXD;
  uint64_t *bars = reinterpret_cast<uint64_t *>(smem + BLK * MAXD);
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
// the CTA synchronises.  Returns false (and raises DERR_TIMEOUT) on timeout, or once
// any other wait of the context has failed (the sticky error word is set).
__device__ __forceinline__ bool wait_flags(const uint64_t *flags, uint32_t n, uint64_t target,
                                           uint64_t timeout_ns, int32_t *err, int *s_abort) {
  if (threadIdx.x < 32) {
    const uint32_t lane = threadIdx.x;
    const uint64_t t_start = globaltimer();
    int why = 0;
    for (uint32_t it = 0;; ++it) {
      const bool mine = lane >= n || ld_relaxed_sys(flags + lane) >= target;
      if (__all_sync(0xffffffffu, mine)) {  // one acquire per flag once all have arrived
        if (lane < n) (void)ld_acquire_sys(flags + lane);
        break;
      }
      if (globaltimer() - t_start > timeout_ns) {
        why = 1;
        break;
      }
      // fail fast: once any wait of this context has failed (sticky error word), the
      // flags this CTA waits for may never come — abort now instead of timing out in
      // turn behind it
      if ((it & 63u) == 63u &&
          __any_sync(0xffffffffu, lane == 0 && *reinterpret_cast<volatile int32_t *>(err) != 0)) {
        why = 3;
        break;
      }
      __nanosleep(64);
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
    for (uint32_t it = 0; ld_relaxed_sys(w) < target || ld_acquire_sys(w) < target; ++it) {
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

// ------------------------------------------------------------------ streamed lanes
//
// One lane of a staged path (engine.h, lane_stride) moved through one TMA pipeline
// that runs across chunk boundaries: the loads of chunk j+1 are issued while the
// stores of chunk j are still in flight, and a chunk's flag is published once its
// stores have completed (a lag of kStreamLag store groups, or at once when the storer
// would otherwise block), so the pipeline never drains between chunks.  The handoff
// protocol is unchanged — chunk granularity: the full flag of a lane is released
// when its whole slice has landed and the free flag when it has been read (Eq 12-13's
// two-stage pipeline) — only the per-chunk restart and drain of the copy
// (profiles/r01 relay_sweep: ~5.6 µs per chunk per lane) are gone.
// Requires co-aligned source and destination slices (else the CTA-wide per-chunk
// path, copy_slice, is used).  A Role supplies, per chunk j:
//   int  wait(j)               watcher: block until chunk j may be read (consumer:
//                              full flag) / written (producer: free flag); 1 or -1
//   int  fetch(j, w)           watcher, after wait: up to 5 words for geom / stored
//                              (the relay's lane header); 1, or -1 when invalid
//   SliceGeo geom(j, w)        loader: source / destination / length of slice j
//   void before_store(j)       storer, producer: lane header (relay) — after wait
//   void loaded(j)             publisher: every load of slice j has landed
//                              (consumer: free flag)
//   void stored(j, w)          publisher: every store of slice j is complete and
//                              visible (producer: full flag; consumer: byte counters)
// Four threads, each one lane of its own warp: the loader (thread 0) enters chunks
// and issues the TMA loads, the storer (thread 96) issues the TMA stores and hands
// each stage back through an "empty" mbarrier once its store has read it out (the
// usual warp-specialised TMA pipeline: neither issue stream waits on the other's
// latencies), the watcher (thread 32) waits on the flags, the publisher (thread 64)
// issues the system-scope releases (each a MEMBAR.SYS of several µs).
constexpr uint32_t kStreamLag = 6;
constexpr uint32_t kStreamAhead = 8;  // chunks the watcher may run ahead of the publisher

struct SliceGeo {
  const uint8_t *src;
  uint8_t *dst;
  uint64_t len;
};

__device__ __forceinline__ void mbar_arrive(uint32_t bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(bar) : "memory");
}

__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }

// Non-blocking: has the phase with this parity completed?
__device__ __forceinline__ bool mbar_test(uint32_t bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2;\n\t"
      "selp.u32 %0, 1, 0, p;\n}"
      : "=r"(ok)
      : "r"(bar), "r"(parity)
      : "memory");
  return ok != 0;
}

// Wait for the phase, giving up (false) once *stop is set.
__device__ __forceinline__ bool mbar_wait_or_stop(uint32_t bar, uint32_t parity, const uint32_t *stop) {
  while (!mbar_test(bar, parity)) {
    if (*reinterpret_cast<const volatile uint32_t *>(stop)) return false;
    __nanosleep(20);
  }
  return true;
}


// Block one thread until *f >= target: 1, or -1 on timeout (DERR_TIMEOUT raised) or
// once the context's error word is set.  Polls relaxed (an acquire load invalidates
// the SM's L1 every time); one acquire on success.
__device__ __forceinline__ int poll_flag(const uint64_t *f, uint64_t target, uint64_t timeout_ns, int32_t *err) {
  const uint64_t t0 = globaltimer();
  for (uint32_t it = 0;; ++it) {
    if (ld_relaxed_sys(f) >= target && ld_acquire_sys(f) >= target) return 1;
    if (globaltimer() - t0 > timeout_ns) {
      atomicExch(err, DERR_TIMEOUT);
      return -1;
    }
    if ((it & 63u) == 63u && *reinterpret_cast<volatile int32_t *>(err) != 0) return -1;
    __nanosleep(128);
  }
}

// GPU scope: the loopback engine's device rings are written and read on one GPU, so
// their flags need only MEMBAR.GPU, not the MEMBAR.SYS that cross-GPU and host-memory
// handoffs need (µs under load).
__device__ __forceinline__ uint64_t ld_relaxed_gpu(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ uint64_t ld_acquire_gpu(const uint64_t *p) {
  uint64_t v;
  asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_gpu(uint64_t *p, uint64_t v) {
  asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
// poll_flag at GPU scope (gpu == true) or system scope
__device__ __forceinline__ int poll_flag_scoped(const uint64_t *f, uint64_t target, uint64_t timeout_ns, int32_t *err,
                                                bool gpu) {
  if (!gpu) return poll_flag(f, target, timeout_ns, err);
  const uint64_t t0 = globaltimer();
  for (uint32_t it = 0;; ++it) {
    if (ld_relaxed_gpu(f) >= target && ld_acquire_gpu(f) >= target) return 1;
    if (globaltimer() - t0 > timeout_ns) {
      atomicExch(err, DERR_TIMEOUT);
      return -1;
    }
    if ((it & 63u) == 63u && *reinterpret_cast<volatile int32_t *>(err) != 0) return -1;
    __nanosleep(128);
  }
}

__device__ __forceinline__ uint32_t ld_acquire_cta_shared(const uint32_t *p) {
  uint32_t v;
  asm volatile("ld.acquire.cta.shared::cta.u32 %0, [%1];" : "=r"(v) : "r"(smem_u32(p)) : "memory");
  return v;
}

__device__ __forceinline__ void st_release_cta_shared(uint32_t *p, uint32_t v) {
  asm volatile("st.release.cta.shared::cta.u32 [%0], %1;" ::"r"(smem_u32(p)), "r"(v) : "memory");
}

template <int MODE>
__device__ __forceinline__ void bytes_copy(uint8_t *d, const uint8_t *s, uint64_t n) {
  for (uint64_t i = 0; i < n; ++i) d[i] = ld1<MODE>(s + i);
}

#ifdef MPX_TRACE  // (design experiment: per-CTA, per-chunk timestamps of the streamed lanes)
__device__ uint64_t *g_mpx_trace;  // [CTA][128 chunks][4]: ready, loaded, stored, (unused)
__device__ __forceinline__ void trace(uint32_t j, uint32_t ev) {
  if (g_mpx_trace && j < 128) g_mpx_trace[(static_cast<uint64_t>(blockIdx.x) * 128 + j) * 4 + ev] = globaltimer();
}
#else
__device__ __forceinline__ void trace(uint32_t, uint32_t) {}
#endif

// The four roles; a thread returns from here when its role is done (threads other than
// 0, 32, 64 and 96 at once).
template <int MODE, uint32_t D, class Role>
__device__ void lane_stream_roles(Role &R, uint32_t nchunks, uint8_t *smem) {
  __shared__ uint32_t s_ready;    // chunks the watcher has found ready
  __shared__ uint32_t s_taken;    // chunks taken up (consumer: loader read the words; producer: storer)
  __shared__ uint32_t s_loaded;   // chunks whose loads have all landed (storer → publisher)
  __shared__ uint32_t s_stored;   // chunks whose stores are complete (storer → publisher)
  __shared__ uint32_t s_pub;      // chunks the publisher has finished (their words free)
  __shared__ uint32_t s_stop;     // 1: a wait failed
  __shared__ uint64_t s_words[kStreamAhead][5];
  constexpr uint32_t BLK = kStagedBlock;
  uint64_t *full = reinterpret_cast<uint64_t *>(smem + BLK * D);  // [D] loaded
  uint64_t *empty = full + D;                                      // [D] read out by its store
  const uint32_t full0 = smem_u32(full), empty0 = smem_u32(empty), smem0 = smem_u32(smem);
  if (threadIdx.x == 0) {
    s_ready = 0;
    s_taken = 0;
    s_loaded = 0;
    s_stored = 0;
    s_pub = 0;
    s_stop = 0;
    for (uint32_t i = 0; i < D; ++i) {
      mbar_init(full0 + 8 * i);
      mbar_init(empty0 + 8 * i);
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  __syncthreads();
  if (threadIdx.x == 32) {  // the watcher: flag waits (a global round trip per poll)
    for (uint32_t j = 0; j < nchunks; ++j) {
      while (ld_acquire_cta_shared(&s_pub) + kStreamAhead <= j) {
        if (*reinterpret_cast<volatile uint32_t *>(&s_stop)) return;
        __nanosleep(64);
      }
      if (R.wait(j) < 0 || R.fetch(j, s_words[j % kStreamAhead]) < 0) {
        st_release_cta_shared(&s_stop, 1);
        return;
      }
      trace(j, 0);
      st_release_cta_shared(&s_ready, j + 1);
    }
    return;
  }
  if (threadIdx.x == 64) {  // the publisher: system-scope releases (MEMBAR.SYS each) off the TMA issue
    uint32_t pl = 0, ps = 0;
    while (ps < nchunks || pl < nchunks) {
      const uint32_t a = ld_acquire_cta_shared(&s_loaded);
      const uint32_t b = ld_acquire_cta_shared(&s_stored);
      if (pl == a && ps == b) {
        if (*reinterpret_cast<volatile uint32_t *>(&s_stop)) return;
        __nanosleep(32);
        continue;
      }
      for (; pl < a; ++pl) {
        trace(pl, 1);
        R.loaded(pl);
      }
      for (; ps < b; ++ps) {
        trace(ps, 2);
        R.stored(ps, s_words[ps % kStreamAhead]);
      }
      st_release_cta_shared(&s_pub, ps);
    }
    return;
  }
  struct Geo {
    const uint8_t *s0;  // slice start (source), for the producer's head/tail
    const uint8_t *s;   // 16-B aligned body start (source)
    uint8_t *d;         // body start (destination)
    uint64_t len;       // slice bytes
    uint64_t body;      // body bytes (a multiple of 16)
    uint32_t steps;     // max(1, blocks of the body): a chunk without a body takes one empty step
  };
  // the geometry of the chunks between the store and the load cursor (<= D + 1),
  // written by the loader before it arms a chunk's first stage (mbarrier arrive =
  // release, the storer's wait = acquire)
  __shared__ Geo geo[kStreamAhead];
  if (threadIdx.x == 0) {
    // ---- the loader: chunk entry (consumer: readiness, geometry, head/tail), loads
    uint32_t gl = 0;
    for (uint32_t lc = 0; lc < nchunks; ++lc) {
      if (!R.producer) {
        // block: the storer publishes on its own (never waits on us with publications pending)
        int rdy = ld_acquire_cta_shared(&s_ready) > lc ? 1 : 0;
        while (!rdy) {
          if (*reinterpret_cast<volatile uint32_t *>(&s_stop)) rdy = -1;
          else if (ld_acquire_cta_shared(&s_ready) > lc) rdy = 1;
          else __nanosleep(32);
        }
        if (rdy < 0) return;
        asm volatile("fence.proxy.async.global;" ::: "memory");  // TMA reads what was acquired
      }
      const SliceGeo g = R.geom(lc, s_words[lc % kStreamAhead]);
      if (!R.producer) st_release_cta_shared(&s_taken, lc + 1);
      uint64_t h = (16u - (reinterpret_cast<uintptr_t>(g.src) & 15u)) & 15u;
      if (h > g.len) h = g.len;
      const uint64_t body = (g.len - h) & ~uint64_t(15);
      const uint32_t nblk = static_cast<uint32_t>((body + BLK - 1) / BLK);
      if (!R.producer) {  // consumer: head / tail bytes now (the lane is acquired)
        bytes_copy<MODE>(g.dst, g.src, h);
        bytes_copy<MODE>(g.dst + h + body, g.src + h + body, g.len - h - body);
      }
      // the stage of this chunk's first step is free (the store of step gl - D has read
      // it out); geo[lc % 8] was last read for chunk lc - 8, which the storer left
      // more than D steps ago
      if (gl >= D && !mbar_wait_or_stop(empty0 + 8 * (gl % D), ((gl / D) - 1) & 1u, &s_stop)) return;
      Geo &e = geo[lc % kStreamAhead];
      e.s0 = g.src;
      e.s = g.src + h;
      e.d = g.dst + h;
      e.len = g.len;
      e.body = body;
      e.steps = nblk ? nblk : 1;
      const uint8_t *src = g.src + h;
      uint64_t rem = body;
      for (uint32_t b = 0; b < e.steps; ++b, ++gl) {
        const uint32_t fb = full0 + 8 * (gl % D);
        if (b > 0 && gl >= D && !mbar_wait_or_stop(empty0 + 8 * (gl % D), ((gl / D) - 1) & 1u, &s_stop))
          return;
        if (rem) {
          const uint32_t n = rem < BLK ? static_cast<uint32_t>(rem) : BLK;
          mbar_expect_tx(fb, n);
          bulk_load(smem0 + (gl % D) * BLK, src, n, fb);
          src += n;
          rem -= n;
        } else {
          mbar_arrive(fb);
        }
      }
    }
    return;
  }
  if (threadIdx.x != 96) return;
  // ---- the storer: producer readiness + head/tail + lane header, stores, stage
  // release, publication of completed chunks
  // chunks [ph, pt) have their stores issued but are not yet published; the last
  // store step of chunk c is pend_last[c % 16] (at most kStreamLag + 1 are pending)
  __shared__ uint32_t pend_last[16];
  uint32_t ph = 0, pt = 0;
  uint32_t pub_at = 0xffffffffu;  // store step after which chunk ph is published
  auto flush = [&]() {            // every issued store complete; the publisher releases the chunks
    if (ph == pt) return;
    bulk_wait_all();
    ph = pt;
    st_release_cta_shared(&s_stored, pt);
    pub_at = 0xffffffffu;
  };
  uint32_t gs = 0;
  bool ok = true;
  for (uint32_t sc = 0; sc < nchunks && ok; ++sc) {
    if (R.producer) {
      if (ld_acquire_cta_shared(&s_ready) <= sc) {
        flush();  // never block with publications pending (the other side may wait on them)
        while (ld_acquire_cta_shared(&s_ready) <= sc) {
          if (*reinterpret_cast<volatile uint32_t *>(&s_stop)) {
            ok = false;
            break;
          }
          __nanosleep(32);
        }
        if (!ok) break;
      }
      st_release_cta_shared(&s_taken, sc + 1);
    }
    // the chunk's geometry: written by the loader before it armed this first step
    uint32_t fb = full0 + 8 * (gs % D);
    if (!mbar_test(fb, (gs / D) & 1u)) {
      flush();
      if (!mbar_wait_or_stop(fb, (gs / D) & 1u, &s_stop)) {
        ok = false;
        break;
      }
    }
    const Geo &e = geo[sc % kStreamAhead];
    if (R.producer) {
      const uint64_t h = static_cast<uint64_t>(e.s - e.s0);
      bytes_copy<MODE>(e.d - h, e.s0, h);
      bytes_copy<MODE>(e.d + e.body, e.s + e.body, e.len - h - e.body);
      R.before_store(sc);
    }
    uint8_t *dst = e.d;
    uint64_t rem = e.body;
    const uint32_t steps = e.steps;
    for (uint32_t b = 0; b < steps; ++b, ++gs) {
      fb = full0 + 8 * (gs % D);
      if (b > 0 && !mbar_test(fb, (gs / D) & 1u)) {
        flush();
        if (!mbar_wait_or_stop(fb, (gs / D) & 1u, &s_stop)) {
          ok = false;
          break;
        }
      }
      if (rem) {
        const uint32_t n = rem < BLK ? static_cast<uint32_t>(rem) : BLK;
        bulk_store(dst, smem0 + (gs % D) * BLK, n);
        dst += n;
        rem -= n;
      } else {
        bulk_commit();  // an empty group keeps group index == step index
      }
      // the previous step's store has read its stage: hand the stage back to the loader
      if (gs > 0) {
        bulk_wait_read<1>();
        mbar_arrive(empty0 + 8 * ((gs - 1) % D));
      }
      if (gs >= pub_at) {  // the oldest pending chunk's stores are kStreamLag groups back
        asm volatile("cp.async.bulk.wait_group %0;" ::"n"(kStreamLag) : "memory");
        asm volatile("fence.proxy.async.global;" ::: "memory");
        while (ph != pt && pend_last[ph % 16] + kStreamLag <= gs) ++ph;
        st_release_cta_shared(&s_stored, ph);
        pub_at = ph != pt ? pend_last[ph % 16] + kStreamLag : 0xffffffffu;
      }
    }
    if (!ok) break;
    // chunk sc fully loaded and its stores issued
    st_release_cta_shared(&s_loaded, sc + 1);
    pend_last[pt % 16] = gs - 1;  // pt == sc
    if (ph == pt) pub_at = gs - 1 + kStreamLag;
    ++pt;
  }
  if (ok) {
    flush();
    bulk_wait_read<0>();
  } else {
    st_release_cta_shared(&s_stop, 1);  // the watcher, loader and publisher stop too
    bulk_wait_all();
  }
}

// Called by every thread of the CTA: the roles, then every thread meets again and the
// stage barriers are invalidated, so the next call (a relay kernel streams one message
// after another) initialises fresh ones.
template <int MODE, uint32_t D, class Role>
__device__ void lane_stream(Role &R, uint32_t nchunks, uint8_t *smem) {
  lane_stream_roles<MODE, D>(R, nchunks, smem);
  __syncthreads();
  if (threadIdx.x == 0) {
    const uint32_t bars = smem_u32(smem + static_cast<uint64_t>(kStagedBlock) * D);
    for (uint32_t i = 0; i < 2 * D; ++i) asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(bars + 8 * i) : "memory");
  }
  __syncthreads();
}

// ------------------------------------------------------------------ roles

// Lane r of a staged path (stage-in CTA r and forward CTA r): slice r of every chunk
// goes through lane r of the chunk's slot, handed over by lane r's own full/free flag
// (engine.h, lane_stride) — an independent two-stage pipeline per lane.
__device__ __forceinline__ uint8_t *lane_at(const DevPath &p, uint64_t s, uint32_t r, const uint8_t *src) {
  return p.ring + s * p.slot_stride + r * p.lane + (reinterpret_cast<uintptr_t>(src) & 15u);
}

// Streamed roles of the loopback rings (lane_stream).
struct LoopProducer {
  static constexpr bool producer = true;
  const DevPath *p;
  uint32_t r;
  uint64_t timeout_ns;
  int32_t *err;
  __device__ SliceGeo geom(uint32_t j, const uint64_t *) const {
    uint64_t off, len, a, b;
    chunk_range(*p, j, &off, &len);
    slice_of(len, r, p->g_in, &a, &b);
    const uint8_t *src = p->src + off;
    return SliceGeo{src + a, lane_at(*p, (p->q0 + j) % p->slots, r, src), b - a};
  }
  __device__ int wait(uint32_t j) {
    const uint64_t q = p->q0 + j;
    return poll_flag_scoped(p->freef + (q % p->slots) * kFlagStride + r, q / p->slots, timeout_ns, err, !p->host_ring);
  }
  __device__ int fetch(uint32_t, uint64_t *) { return 1; }
  __device__ void before_store(uint32_t) {}
  __device__ void loaded(uint32_t) {}
  __device__ void stored(uint32_t j, const uint64_t *) {
    const uint64_t q = p->q0 + j;
    uint64_t *f = p->full + (q % p->slots) * kFlagStride + r;
    if (p->host_ring) st_release_sys(f, q / p->slots + 1);  // data in host memory
    else st_release_gpu(f, q / p->slots + 1);
  }
};

struct LoopConsumer {
  static constexpr bool producer = false;
  const DevPath *p;
  uint32_t r;
  uint64_t timeout_ns;
  int32_t *err;
  __device__ SliceGeo geom(uint32_t j, const uint64_t *) const {
    uint64_t off, len, a, b;
    chunk_range(*p, j, &off, &len);
    slice_of(len, r, p->g_out, &a, &b);
    return SliceGeo{lane_at(*p, (p->q0 + j) % p->slots, r, p->src + off), p->dst + off + a, b - a};
  }
  __device__ int wait(uint32_t j) {
    const uint64_t q = p->q0 + j;
    return poll_flag_scoped(p->full + (q % p->slots) * kFlagStride + r, q / p->slots + 1, timeout_ns, err, !p->host_ring);
  }
  __device__ int fetch(uint32_t, uint64_t *) { return 1; }
  __device__ void before_store(uint32_t) {}
  __device__ void loaded(uint32_t j) {
    const uint64_t q = p->q0 + j;
    uint64_t *f = p->freef + (q % p->slots) * kFlagStride + r;
    if (p->host_ring) st_release_sys(f, q / p->slots + 1);
    else st_release_gpu(f, q / p->slots + 1);
  }
  __device__ void stored(uint32_t, const uint64_t *) {}
};

template <uint32_t D>
__device__ void run_stage_in(const DevPath &p, uint32_t r, const XferParams &P, int *s_abort, uint8_t *smem) {
  if (P.copy_mode == 1) {  // streamed lane (the source slice and its lane are co-aligned)
    LoopProducer R{&p, r, P.timeout_ns, P.err};
    lane_stream<LD_SRC, D>(R, p.k, smem);
    return;
  }
  for (uint32_t j = 0; j < p.k; ++j) {
    uint64_t off, len;
    chunk_range(p, j, &off, &len);
    const uint64_t q = p.q0 + j, s = q % p.slots, u = q / p.slots;
    if (!wait_flags(p.freef + s * kFlagStride + r, 1, u, P.timeout_ns, P.err, s_abort)) return;
    const uint8_t *src = p.src + off;
    uint64_t a, b;  // slice r of the chunk, split on 16-byte boundaries
    slice_of(len, r, p.g_in, &a, &b);
    copy_slice<LD_SRC, kStagedBlock>(lane_at(p, s, r, src), src + a, b - a, smem, P.copy_mode, P.bulk_stages);
    release_flag(p.full + s * kFlagStride + r, u + 1);
  }
}

template <int MODE, uint32_t D>
__device__ void run_forward(const DevPath &p, uint32_t r, const XferParams &P, int *s_abort, uint8_t *smem) {
  if (P.copy_mode == 1 && ((reinterpret_cast<uintptr_t>(p.src) ^ reinterpret_cast<uintptr_t>(p.dst)) & 15u) == 0) {
    LoopConsumer R{&p, r, P.timeout_ns, P.err};
    lane_stream<MODE, D>(R, p.k, smem);
    return;
  }
  for (uint32_t j = 0; j < p.k; ++j) {
    uint64_t off, len;
    chunk_range(p, j, &off, &len);
    const uint64_t q = p.q0 + j, s = q % p.slots, u = q / p.slots;
    if (!wait_flags(p.full + s * kFlagStride + r, 1, u + 1, P.timeout_ns, P.err, s_abort)) return;
    uint64_t a, b;
    slice_of(len, r, p.g_out, &a, &b);
    copy_slice<MODE, kStagedBlock>(p.dst + off + a, lane_at(p, s, r, p.src + off), b - a, smem, P.copy_mode,
                                   P.bulk_stages);
    release_flag(p.freef + s * kFlagStride + r, u + 1);
  }
}

template <uint32_t D>
__global__ void __launch_bounds__(kThreads, D == kBulkStages ? 3 : 2) xfer_kernel(const __grid_constant__ XferParams P) {
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
        run_stage_in<D>(p, b - p.cta0_in, P, &s_abort, dyn_smem);
      return;
    }
    if (p.kind == DK_STAGED && b >= p.cta0_out && b < p.cta0_out + p.g_out) {
      if (p.host_ring)
        run_forward<LD_HOST, D>(p, b - p.cta0_out, P, &s_abort, dyn_smem);
      else
        run_forward<LD_RING, D>(p, b - p.cta0_out, P, &s_abort, dyn_smem);
      return;
    }
  }
}

// Holds a stream for `ns` nanoseconds (calibration of the host submission time, C27).
__global__ void spin_kernel(uint64_t ns) {
  const uint64_t t0 = globaltimer();
#ifdef MPX_SPIN_SLEEP  // (design experiment: the sleeping spin of round 2's first sessions)
  while (globaltimer() - t0 < ns) __nanosleep(1000);
#else
  // busy: a sleeping warp leaves the GPU idle for the spin's ~1 ms, and the launch-bound
  // small windows timed right after it then ran slower on some boxes (~1.5 µs per
  // 64 KiB message against ~1.1 µs behind a busy spin)
  while (globaltimer() - t0 < ns) {
  }
#endif
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

// Streamed roles of the multi-rank engine (lane_stream).
// Sender stage-in lane r of a relay or host path (A8/A9 step 1).
struct SendProducer {
  static constexpr bool producer = true;
  const SendParams *P;
  const SendParams::StagedDesc *d;
  uint32_t r;
  uint64_t lstride, base, region;
  __device__ void chunk(uint32_t j, uint64_t *off, uint64_t *a, uint64_t *e) const {
    uint64_t len;
    chunk_of(d->bytes, P->align, d->k, j, off, &len);
    *off += d->off;
    slice_of(len, r, d->g, a, e);
  }
  __device__ uint64_t slot(uint32_t j) const {
    const uint64_t q = d->q0 + j;
    return d->kind == 1 ? q % P->L.slots : q % P->host_slots;
  }
  __device__ uint64_t gen(uint32_t j) const {
    const uint64_t q = d->q0 + j;
    return d->kind == 1 ? q / P->L.slots : q / P->host_slots;
  }
  __device__ uint8_t *lane(uint32_t j) const {
    const uint64_t s = slot(j);
    return d->kind == 1 ? d->ring_ctrl + P->L.ring_data + (static_cast<uint64_t>(P->me) * P->L.slots + s) * P->L.stride +
                              r * lstride
                        : P->host.data + s * P->host_stride + r * lstride;
  }
  __device__ SliceGeo geom(uint32_t j, const uint64_t *) const {
    uint64_t off, a, e;
    chunk(j, &off, &a, &e);
    const uint8_t *src = P->src + off;
    return SliceGeo{src + a, lane(j) + kLaneHdr + (reinterpret_cast<uintptr_t>(src) & 15u), e - a};
  }
  __device__ int wait(uint32_t j) {
    const uint64_t *fr = d->kind == 1 ? flags_at(P->my_ctrl, P->L.relay_free, d->relay, P->L.slots, slot(j)) + r
                                      : P->host.freef + slot(j) * kFlagStride + r;
    return poll_flag(fr, gen(j), P->timeout_ns, P->err);
  }
  __device__ int fetch(uint32_t, uint64_t *) { return 1; }
  __device__ void before_store(uint32_t j) {
    if (d->kind != 1) return;
    uint64_t off, a, e;
    chunk(j, &off, &a, &e);
    uint64_t *h = reinterpret_cast<uint64_t *>(lane(j));  // the lane header the relay forwards by
    h[0] = P->dst;
    h[1] = base + off + a;
    h[2] = e - a;
    h[3] = reinterpret_cast<uintptr_t>(P->src + off) & 15u;
    h[4] = region;
  }
  __device__ void loaded(uint32_t) {}
  __device__ void stored(uint32_t j, const uint64_t *) {
    uint64_t *fl = d->kind == 1 ? flags_at(d->ring_ctrl, P->L.ring_full, P->me, P->L.slots, slot(j)) + r
                                : P->host.full + slot(j) * kFlagStride + r;
    st_release_sys(fl, gen(j) + 1);
  }
};

// Relay forward lane r (A8 step 3): the lane header names the destination.  The
// watcher copies it to shared memory (words: dst, region offset, len, shift, region).
struct RelayConsumer {
  static constexpr bool producer = false;
  const RelayParams *P;
  uint32_t r;
  uint64_t lstride;
  uint64_t q0;  // the message's first ring sequence
  uint64_t k;   // the message's chunks
  uint64_t acc; // bytes of this lane stored so far (counted once, after its last chunk)
  uint64_t m;   // the message's doorbell index on (sender, this relay)
  __device__ uint8_t *lane(uint32_t j) const {
    const uint64_t s = (q0 + j) % P->L.slots;
    return P->my_ctrl + P->L.ring_data + (static_cast<uint64_t>(P->sender) * P->L.slots + s) * P->L.stride +
           r * lstride;
  }
  __device__ int wait(uint32_t j) {
    const uint64_t q = q0 + j;
    return poll_flag(flags_at(P->my_ctrl, P->L.ring_full, P->sender, P->L.slots, q % P->L.slots) + r,
                     q / P->L.slots + 1, P->timeout_ns, P->err);
  }
  __device__ int fetch(uint32_t j, uint64_t *w) {
    const uint64_t *h = reinterpret_cast<const uint64_t *>(lane(j));
    for (int i = 0; i < 5; ++i) w[i] = ld_volatile(h + i);
    if (w[0] >= P->L.world || w[4] >= kMaxRegions || w[3] > 15) {  // never write through a torn lane
      atomicExch(P->err, DERR_MISMATCH);
      return -1;
    }
    return 1;
  }
  __device__ SliceGeo geom(uint32_t j, const uint64_t *w) const {
    return SliceGeo{lane(j) + kLaneHdr + w[3], region_base(P->my_ctrl, P->L, w[4], static_cast<uint32_t>(w[0])) + w[1],
                    w[2]};
  }
  __device__ void before_store(uint32_t) {}
  __device__ void loaded(uint32_t j) {
    const uint64_t q = q0 + j;
    st_release_sys(flags_at(P->sender_ctrl, P->L.relay_free, P->me, P->L.slots, q % P->L.slots) + r,
                   q / P->L.slots + 1);
  }
  // The receiver only waits for the message's whole byte count (A10).  After its last
  // chunk a lane adds (its bytes << 8 | 1) into the message's counter slot on this GPU
  // (GPU-scope acq_rel); the lane that completes the count releases the message's
  // relayed bytes into the destination's counter — one system-scope release per
  // relayed message, as the direct group's (§6).  Slot m % kBellRing is reused 64
  // messages later: a lane first waits until message m - 64 has been counted (rfree; a
  // relay's lanes drift at most a message or two apart, so this never waits in
  // practice: the sender's kernels on one relay ring run in order and wait for its
  // free flags).
  __device__ void stored(uint32_t j, const uint64_t *w) {
    acc += w[2];
    if (j + 1 != k) return;
    const uint64_t slot = static_cast<uint64_t>(P->sender) * kBellRing + m % kBellRing;
    uint64_t *cnt = reinterpret_cast<uint64_t *>(P->my_ctrl + P->L.rcnt) + slot;
    uint64_t *fr = reinterpret_cast<uint64_t *>(P->my_ctrl + P->L.rfree) + slot;
    if (m >= kBellRing && poll_flag_scoped(fr, m + 1 - kBellRing, P->timeout_ns, P->err, true) < 0) return;
    uint64_t old;
    asm volatile("atom.acq_rel.gpu.global.add.u64 %0, [%1], %2;"
                 : "=l"(old)
                 : "l"(cnt), "l"((acc << 8) | 1u)
                 : "memory");
    if ((old & 0xffu) + 1 == P->g) {
      *reinterpret_cast<volatile uint64_t *>(cnt) = 0;
      const uint64_t total = (old >> 8) + acc;
      if (total) red_add_release_sys(done_at(P->peer[w[0]].ctrl, P->L, P->sender), total);
      st_release_gpu(fr, m + 1);
    }
  }
};

// Receiver's host-ring consumer lane r (A9 step 3); the chunk layout comes from the
// message header in device memory.
struct HostConsumer {
  static constexpr bool producer = false;
  const RecvParams *P;
  uint32_t r;
  uint64_t lstride, k, q0, hoff, hbytes, shift, align;
  uint64_t *done;
  __device__ void chunk(uint32_t j, uint64_t *off, uint64_t *a, uint64_t *e) const {
    uint64_t len;
    chunk_of(hbytes, align, static_cast<uint32_t>(k), j, off, &len);
    slice_of(len, r, P->g_host, a, e);
  }
  __device__ SliceGeo geom(uint32_t j, const uint64_t *) const {
    uint64_t off, a, e;
    chunk(j, &off, &a, &e);
    const uint64_t s = (q0 + j) % P->host_slots;
    return SliceGeo{P->host.data + s * P->host_stride + r * lstride + kLaneHdr + ((shift + off) & 15u),
                    P->buf + hoff + off + a, e - a};
  }
  __device__ int wait(uint32_t j) {
    const uint64_t q = q0 + j;
    return poll_flag(P->host.full + (q % P->host_slots) * kFlagStride + r, q / P->host_slots + 1, P->timeout_ns,
                     P->err);
  }
  __device__ int fetch(uint32_t, uint64_t *) { return 1; }
  __device__ void before_store(uint32_t) {}
  __device__ void loaded(uint32_t j) {
    const uint64_t q = q0 + j;
    st_release_sys(P->host.freef + (q % P->host_slots) * kFlagStride + r, q / P->host_slots + 1);
  }
  __device__ void stored(uint32_t j, const uint64_t *) {
    uint64_t off, a, e;
    chunk(j, &off, &a, &e);
    red_add_release_gpu(done, e - a);
  }
};

// The rendezvous (P:62 analogue) runs in its own one-CTA launch ahead of the bulk
// send kernel on the same stream: the bulk kernel's hundreds of CTAs are only
// dispatched once the receiver's clear-to-send has arrived, so they never occupy SM
// slots spinning on it while a receive kernel on this GPU waits for room to run.
// The gate also rings the doorbell of every relay the message uses (engine.h): the
// relay rank's host thread then launches the relay kernel for the message's chunks,
// so a relay kernel only runs while the data it forwards is flowing.
// PDL in the multi-rank engine: the gate waits for the stream's previous kernel, and
// lets the bulk send kernel launch only once the clear-to-send has arrived (no bulk
// CTA is ever resident during the rendezvous); send, receive and eager kernels let
// their successor launch at once and wait for their predecessor (pdl_enter).
__device__ void send_gate_body(const SendParams &P) {
  if (threadIdx.x != 0) return;
  trace(126, 0);
  MsgEntry *cts = entry_at(P.my_ctrl, P.L.cts, P.dst, P.seq);
  const uint64_t t_start = globaltimer();
  uint64_t seen = 0;
  while (ld_relaxed_sys(&cts->seq1) < P.seq + 1 || (seen = ld_acquire_sys(&cts->seq1)) < P.seq + 1) {
    if (globaltimer() - t_start > P.timeout_ns) {
      atomicExch(P.err, DERR_TIMEOUT);
      return;
    }
    __nanosleep(64);
  }
  const uint64_t n = ld_volatile(&cts->b), tag = ld_volatile(&cts->c);
  // seen > seq + 1: the receiver posted a later receive into this CTS entry before
  // this send consumed it (more than kCtsRing outstanding receives from one peer) —
  // the entry no longer describes this message
  const bool bad = (n != P.bytes) || (tag != P.tag) || seen != P.seq + 1;
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
  h->g = P.align;
  if (bad) {
    st_release_sys(&h->seq1, P.seq + 1);
    atomicExch(P.err, DERR_MISMATCH);
    return;
  }
  // the direct group's completion counter slot: free once message seq - kCtsRing to the
  // same destination has been counted (only many streams of messages ever wait here)
  if (P.seq >= kCtsRing) {
    const uint64_t *fr = reinterpret_cast<const uint64_t *>(P.my_ctrl + P.L.dfree) +
                         static_cast<uint64_t>(P.dst) * kCtsRing + P.seq % kCtsRing;
    const uint64_t need = P.seq + 1 - kCtsRing, t0 = globaltimer();
    while (ld_relaxed_gpu(fr) < need || ld_acquire_gpu(fr) < need) {
      if (globaltimer() - t0 > P.timeout_ns) {
        atomicExch(P.err, DERR_TIMEOUT);
        break;
      }
      __nanosleep(256);
    }
  }
  // doorbells (relay rank's host thread): the fields of every one first, then ONE
  // system-scope fence for the message header and all of them, then their flags —
  // a release per flag cost a MEMBAR.SYS each (~12 µs under load), 7 for config 3
  for (uint32_t i = 0; i < P.npaths; ++i) {
    const SendParams::StagedDesc &d = P.sp[i];
    if (d.kind != 1) continue;
    BellEntry *e = d.bell + d.m % kBellRing;
    // flow control: the entry is reused only once the relay has taken the doorbell
    // kBellRing messages back (its kernels acknowledge into this rank's control
    // block); only more than kBellRing relayed messages in flight through one relay
    // (many streams) ever wait here
    if (d.m >= kBellRing) {
      const uint64_t *ack = reinterpret_cast<const uint64_t *>(P.my_ctrl + P.L.bell_ack) + d.relay * 16;
      const uint64_t need = d.m + 1 - kBellRing, t0 = globaltimer();
      while (ld_relaxed_sys(ack) < need || ld_acquire_sys(ack) < need) {
        if (globaltimer() - t0 > P.timeout_ns) {
          atomicExch(P.err, DERR_TIMEOUT);
          break;
        }
        __nanosleep(256);
      }
    }
    // co-alignment of source and target (mod 16 is the same in every process's
    // mapping: mapped bases are >= 256-B aligned) lets the relay stream its lanes
    const uint64_t region = ld_volatile(&cts->d);
    const bool aligned = region < kMaxRegions &&
                         ((reinterpret_cast<uintptr_t>(P.src) ^
                           (reinterpret_cast<uintptr_t>(region_base(P.my_ctrl, P.L, region, P.dst)) + ld_volatile(&cts->a))) &
                          15u) == 0;
    e->q0 = d.q0;
    e->k = d.k;
    e->g = d.g | (aligned ? (1ull << 32) : 0ull);
  }
  trace(126, 1);
  fence_acq_rel_sys();
  st_relaxed_sys(&h->seq1, P.seq + 1);
  for (uint32_t i = 0; i < P.npaths; ++i) {
    const SendParams::StagedDesc &d = P.sp[i];
    if (d.kind == 1) st_relaxed_sys(&(d.bell + d.m % kBellRing)->tag, d.m + 1);
  }
  trace(126, 2);
}

__global__ void send_gate_kernel(const __grid_constant__ SendParams P) {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  send_gate_body(P);
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

// CTA b of the send kernel's grid (the kernel below; one role of emu_kernel).
template <uint32_t D>
__device__ void send_body(const SendParams &P, const uint32_t b, uint8_t *dyn_smem) {
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
    if ((n != P.bytes) || (tag != P.tag) || s_region >= kMaxRegions || ld_volatile(&cts->seq1) != P.seq + 1)
      s_abort = 1;  // reported by the gate
    else
      s_dst = region_base(P.my_ctrl, P.L, s_region, P.dst) + off;
  }
  __syncthreads();
  if (s_abort) return;
  const uint64_t base = s_off;
  uint64_t *done = done_at(P.dst_ctrl, P.L, P.me);
  if (b < P.g_direct) {  // A7: direct NVLink stores into the receiver's heap
    if (threadIdx.x == 0) trace(120, 0);
    if (P.copy_mode == 1)
      bulk_copy<LD_SRC>(s_dst, P.src, P.direct_bytes, b, P.g_direct, dyn_smem, P.bulk_stages);
    else
      group_copy<LD_SRC>(s_dst, P.src, P.direct_bytes, b, P.g_direct);
    // Completion (A10): the group counts itself on this GPU (a GPU-scope acq_rel add per
    // CTA) and its last CTA adds the whole direct share into the receiver's counter —
    // one system-scope release per message instead of one per CTA (each a MEMBAR.SYS:
    // 16 MiB in the emulated world 28.2 -> 20.2 µs with the per-CTA releases dropped).
    // Cumulativity: every CTA's stores precede its release on the counter, which the
    // last CTA's RMW acquires before its system-scope release.  The counter slot is
    // reused kCtsRing messages later; the send gate waits for it (dfree).
    __syncthreads();
    if (threadIdx.x == 0) trace(120, 1);
    if (threadIdx.x == 0) {
      uint64_t *cnt = reinterpret_cast<uint64_t *>(P.my_ctrl + P.L.dcnt) +
                      static_cast<uint64_t>(P.dst) * kCtsRing + P.seq % kCtsRing;
      uint64_t old;
      asm volatile("atom.acq_rel.gpu.global.add.u64 %0, [%1], 1;" : "=l"(old) : "l"(cnt) : "memory");
      if (old + 1 == P.g_direct) {
        *reinterpret_cast<volatile uint64_t *>(cnt) = 0;
        trace(121, 0);
        if (P.direct_bytes) red_add_release_sys(done, P.direct_bytes);
        trace(121, 1);
        uint64_t *fr = reinterpret_cast<uint64_t *>(P.my_ctrl + P.L.dfree) +
                       static_cast<uint64_t>(P.dst) * kCtsRing + P.seq % kCtsRing;
        st_release_gpu(fr, P.seq + 1);
      }
    }
    return;
  }
  for (uint32_t i = 0; i < P.npaths; ++i) {
    const SendParams::StagedDesc &d = P.sp[i];
    if (b < d.cta0 || b >= d.cta0 + d.g) continue;
    const uint32_t r = b - d.cta0;  // lane r of every slot of this path
    const uint64_t lstride = lane_stride(P.L.slot_bytes, d.g);
    if (P.copy_mode == 1) {  // streamed lane (source slice and lane are co-aligned)
      SendProducer R{&P, &d, r, lstride, base, s_region};
      lane_stream<LD_SRC, D>(R, d.k, dyn_smem);
      return;
    }
    for (uint32_t j = 0; j < d.k; ++j) {  // A8/A9 step 1
      uint64_t off, len;
      chunk_of(d.bytes, P.align, d.k, j, &off, &len);
      off += d.off;
      const uint64_t q = d.q0 + j;
      uint64_t *fr, *fl;
      uint8_t *lane;
      uint64_t u;
      if (d.kind == 1) {
        const uint64_t s = q % P.L.slots;
        u = q / P.L.slots;
        fr = flags_at(P.my_ctrl, P.L.relay_free, d.relay, P.L.slots, s) + r;
        fl = flags_at(d.ring_ctrl, P.L.ring_full, P.me, P.L.slots, s) + r;
        lane = d.ring_ctrl + P.L.ring_data + (static_cast<uint64_t>(P.me) * P.L.slots + s) * P.L.stride + r * lstride;
      } else {
        const uint64_t s = q % P.host_slots;
        u = q / P.host_slots;
        fr = P.host.freef + s * kFlagStride + r;
        fl = P.host.full + s * kFlagStride + r;
        lane = P.host.data + s * P.host_stride + r * lstride;
      }
      if (!wait_flags(fr, 1, u, P.timeout_ns, P.err, &s_abort)) return;
      const uint8_t *src = P.src + off;
      const uint64_t shift = reinterpret_cast<uintptr_t>(src) & 15u;
      uint64_t a, e;
      slice_of(len, r, d.g, &a, &e);
      copy_slice<LD_SRC, kStagedBlock>(lane + kLaneHdr + shift, src + a, e - a, dyn_smem, P.copy_mode,
                                       P.bulk_stages);
      if (d.kind == 1 && threadIdx.x == 0) {  // the lane header the relay forwards by
        uint64_t *h = reinterpret_cast<uint64_t *>(lane);
        h[0] = P.dst;
        h[1] = base + off + a;
        h[2] = e - a;
        h[3] = shift;
        h[4] = s_region;
      }
      publish(nullptr, 0, fl, u + 1);
    }
    return;
  }
}

template <uint32_t D>
__global__ void __launch_bounds__(kThreads, D == kBulkStages ? 3 : 2) send_kernel(const __grid_constant__ SendParams P) {
  extern __shared__ __align__(128) uint8_t dyn_smem[];
  pdl_enter();
  send_body<D>(P, blockIdx.x, dyn_smem);
}

// CTA b of the receive kernel's grid (the kernel below; one role of emu_kernel).
template <uint32_t D>
__device__ void recv_body(const RecvParams &P, const uint32_t b, uint8_t *dyn_smem) {
  __shared__ int s_abort;
  __shared__ uint64_t s_k, s_q0, s_hoff, s_hbytes, s_shift, s_align;
  if (threadIdx.x == 0) s_abort = 0;
  __syncthreads();
  MsgEntry *hdr = entry_at(P.my_ctrl, P.L.hdr, P.src, P.seq);
  if (b == 0) {
    if (threadIdx.x == 0) {  // post the clear-to-send into the sender's control block
      MsgEntry *cts = entry_at(P.src_ctrl, P.L.cts, P.me, P.seq);
      cts->a = P.region_off;
      cts->b = P.bytes;
      cts->c = P.tag;
      cts->d = P.region;
      trace(125, 0);
      fence_acq_rel_sys();
      st_relaxed_sys(&cts->seq1, P.seq + 1);
      trace(125, 1);
      // A10: wait until every byte of the message has been counted in
      const uint64_t *done = done_at(P.my_ctrl, P.L, P.src);
      const uint64_t t_start = globaltimer();
      // polled relaxed, one acquire on success (an acquire load invalidates this SM's
      // L1 each time; poll_flag)
      while (ld_relaxed_sys(done) < P.done_target || ld_acquire_sys(done) < P.done_target) {
        if (ld_relaxed_sys(&hdr->seq1) == P.seq + 1 && ld_acquire_sys(&hdr->seq1) == P.seq + 1 &&
            ld_volatile(&hdr->c) == 2) {
          atomicExch(P.err, DERR_MISMATCH);
          break;
        }
        if (globaltimer() - t_start > P.timeout_ns) {
          atomicExch(P.err, DERR_TIMEOUT);
          break;
        }
        __nanosleep(128);
      }
      trace(123, 0);
      fence_acq_rel_sys();
      trace(123, 1);
    }
    return;
  }
  // A9 step 3: host-ring consumers, CTA r = lane r of every host slot
  const uint32_t r = b - 1;
  if (!wait_word(&hdr->seq1, P.seq + 1, P.timeout_ns, P.err, &s_abort)) return;
  if (threadIdx.x == 0) {
    s_k = ld_volatile(&hdr->c) ? 0 : ld_volatile(&hdr->a);
    s_q0 = ld_volatile(&hdr->b);
    s_hoff = ld_volatile(&hdr->d);
    s_hbytes = ld_volatile(&hdr->e);
    s_shift = ld_volatile(&hdr->f);
    s_align = ld_volatile(&hdr->g);
  }
  __syncthreads();
  uint64_t *done = done_at(P.my_ctrl, P.L, P.src);
  const uint64_t lstride = lane_stride(P.L.slot_bytes, P.g_host);
  if (P.copy_mode == 1 && ((reinterpret_cast<uintptr_t>(P.buf) + s_hoff) & 15u) == s_shift) {
    // streamed lane: the host slices and their destination are co-aligned
    HostConsumer R{&P, r, lstride, s_k, s_q0, s_hoff, s_hbytes, s_shift, s_align, done};
    lane_stream<LD_HOST, D>(R, static_cast<uint32_t>(s_k), dyn_smem);
    return;
  }
  for (uint64_t j = 0; j < s_k; ++j) {
    const uint64_t q = s_q0 + j, s = q % P.host_slots, u = q / P.host_slots;
    if (!wait_flags(P.host.full + s * kFlagStride + r, 1, u + 1, P.timeout_ns, P.err, &s_abort)) return;
    uint8_t *lane = P.host.data + s * P.host_stride + r * lstride;
    uint64_t off, len;
    chunk_of(s_hbytes, s_align, static_cast<uint32_t>(s_k), static_cast<uint32_t>(j), &off, &len);
    uint64_t a, e;
    slice_of(len, r, P.g_host, &a, &e);
    copy_slice<LD_HOST, kStagedBlock>(P.buf + s_hoff + off + a, lane + kLaneHdr + ((s_shift + off) & 15u), e - a,
                                      dyn_smem, P.copy_mode, P.bulk_stages);
    publish(done, e - a, P.host.freef + s * kFlagStride + r, u + 1, /*done_is_local=*/true);
  }
}

template <uint32_t D>
__global__ void __launch_bounds__(kThreads, D == kBulkStages ? 3 : 2) recv_kernel(const __grid_constant__ RecvParams P) {
  extern __shared__ __align__(128) uint8_t dyn_smem[];
  pdl_enter();
  recv_body<D>(P, blockIdx.x, dyn_smem);
}

// Relay (A8 step 3): CTA r forwards lane r of chunks [q0, q0 + k) of the sender's ring
// to the destination its lane header names, counts the bytes into the destination's
// `done` and returns the lane to the sender — for the launch's first message, then
// (lingering) for each next message of the sender whose doorbell CTA 0 sees within
// linger_ns, so back-to-back relayed messages pay no relaunch.  A relay kernel still
// ends once its sender goes quiet: nothing outlives the traffic by more than the linger.
template <uint32_t D>
__device__ bool relay_message(const RelayParams &P, const uint32_t r, uint64_t m, uint64_t q0, uint64_t k,
                              uint32_t aligned, int *s_abort, uint8_t *smem) {
  const uint64_t lstride = lane_stride(P.L.slot_bytes, P.g);
  if (P.copy_mode == 1 && aligned) {  // streamed lane (the sender found source and target co-aligned)
    RelayConsumer R{&P, r, lstride, q0, k, 0, m};
    lane_stream<LD_RING, D>(R, static_cast<uint32_t>(k), smem);
    return *reinterpret_cast<volatile int32_t *>(P.err) == 0;
  }
  __shared__ uint64_t s_h[5];
  for (uint64_t j = 0; j < k; ++j) {
    const uint64_t q = q0 + j, s = q % P.L.slots, u = q / P.L.slots;
    uint64_t *fl = flags_at(P.my_ctrl, P.L.ring_full, P.sender, P.L.slots, s) + r;
    if (!wait_flags(fl, 1, u + 1, P.timeout_ns, P.err, s_abort)) return false;
    uint8_t *lane =
        P.my_ctrl + P.L.ring_data + (static_cast<uint64_t>(P.sender) * P.L.slots + s) * P.L.stride + r * lstride;
    if (threadIdx.x < 5) s_h[threadIdx.x] = ld_volatile(reinterpret_cast<const uint64_t *>(lane) + threadIdx.x);
    __syncthreads();
    const uint32_t dst = static_cast<uint32_t>(s_h[0]);
    const uint64_t off = s_h[1], len = s_h[2], shift = s_h[3], region = s_h[4];
    if (dst >= P.L.world || region >= kMaxRegions) {  // a torn or foreign lane: never write through it
      if (threadIdx.x == 0) atomicExch(P.err, DERR_MISMATCH);
      return false;
    }
    copy_slice<LD_RING, kStagedBlock>(region_base(P.my_ctrl, P.L, region, dst) + off, lane + kLaneHdr + shift, len,
                                      smem, P.copy_mode, kBulkStages);
    uint64_t *fr = flags_at(P.sender_ctrl, P.L.relay_free, P.me, P.L.slots, s) + r;
    publish(done_at(P.peer[dst].ctrl, P.L, P.sender), len, fr, u + 1);
    __syncthreads();
  }
  // the per-chunk path counted its bytes chunk by chunk; the message still takes its
  // turn in the lanes' counter slot so that the streamed messages after it see it done
  if (threadIdx.x == 0) {
    const uint64_t slot = static_cast<uint64_t>(P.sender) * kBellRing + m % kBellRing;
    uint64_t *cnt = reinterpret_cast<uint64_t *>(P.my_ctrl + P.L.rcnt) + slot;
    uint64_t *rf = reinterpret_cast<uint64_t *>(P.my_ctrl + P.L.rfree) + slot;
    if (m >= kBellRing && poll_flag_scoped(rf, m + 1 - kBellRing, P.timeout_ns, P.err, true) < 0) return false;
    uint64_t old;
    asm volatile("atom.acq_rel.gpu.global.add.u64 %0, [%1], 1;" : "=l"(old) : "l"(cnt) : "memory");
    if ((old & 0xffu) + 1 == P.g) {
      *reinterpret_cast<volatile uint64_t *>(cnt) = 0;
      st_release_gpu(rf, m + 1);
    }
  }
  return true;
}

// CTA b of a relay launch; the launch's first message is chunks [q0, q0 + k) of
// doorbell P.m0 (the relay kernel below: read by the host thread; emu_kernel's relay
// role: read from the doorbell on the device).
template <uint32_t D>
__device__ void relay_body(const RelayParams &P, const uint32_t b, uint64_t q0, uint64_t k, uint32_t aligned,
                           uint8_t *dyn_smem) {
  __shared__ int s_abort;
  __shared__ uint64_t s_next[4];  // next message: tag, q0, k, flags (bit 0 aligned, bit 1 stop)
  if (threadIdx.x == 0) s_abort = 0;
  __syncthreads();
  uint64_t m = P.m0;
  // doorbell m is taken (the host thread read it for this launch): the sender may reuse
  // its ring entry kBellRing messages later (flow control in send_gate_kernel)
  uint64_t *ack = reinterpret_cast<uint64_t *>(P.sender_ctrl + P.L.bell_ack) + P.me * 16;
  if (b == 0 && threadIdx.x == 0) st_release_sys(ack, m + 1);
  for (;;) {
    if (!relay_message<D>(P, b, m, q0, k, aligned, &s_abort, dyn_smem)) break;
    // the sender's next message: CTA 0 looks for its doorbell for up to linger_ns and
    // publishes the decision; every CTA follows it
    uint64_t *dec = P.dec + ((m + 1) % kBellRing) * 4;
    if (b == 0 && threadIdx.x == 0) {
      const BellEntry *e = P.bells + (m + 1) % kBellRing;
      const uint64_t t0 = globaltimer();
      bool found = false;
      // max_msgs (emu_kernel): the launch serves exactly that many messages
      const bool more = P.max_msgs == 0 || m + 1 - P.m0 < P.max_msgs;
      while (more && P.linger_ns && globaltimer() - t0 < P.linger_ns) {
        if (ld_relaxed_sys(&e->tag) == m + 2) {
          found = ld_acquire_sys(&e->tag) == m + 2;
          break;
        }
        __nanosleep(256);
      }
      uint64_t nq = 0, nk = 0, flags = 2;  // stop
      if (found) {
        const uint64_t g = ld_volatile(&e->g);
        if (static_cast<uint32_t>(g & 0xffffffffu) == P.g) {  // same lanes: this launch serves it
          nq = ld_volatile(&e->q0);
          nk = ld_volatile(&e->k);
          flags = (g >> 32) & 1u;
          st_release_sys(ack, m + 2);  // doorbell m + 1 taken
        }
      }
      dec[1] = nq;
      dec[2] = nk;
      dec[3] = flags;
      st_release_sys(dec, m + 2);
    }
    if (threadIdx.x == 0) {
      const uint64_t t0 = globaltimer();
      while (ld_relaxed_sys(dec) != m + 2 || ld_acquire_sys(dec) != m + 2) {
        if (globaltimer() - t0 > P.linger_ns + P.timeout_ns) {
          atomicExch(P.err, DERR_TIMEOUT);
          s_abort = 1;
          break;
        }
        __nanosleep(128);
      }
      s_next[1] = ld_volatile(dec + 1);
      s_next[2] = ld_volatile(dec + 2);
      s_next[3] = ld_volatile(dec + 3);
    }
    __syncthreads();
    if (s_abort || (s_next[3] & 2u)) break;
    m += 1;
    q0 = s_next[1];
    k = s_next[2];
    aligned = static_cast<uint32_t>(s_next[3] & 1u);
    __syncthreads();
  }
  // the last CTA out hands the sender's doorbell position back to the host thread
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence_system();
    if (atomicAdd(P.exit_cnt, 1u) == P.g - 1) {
      atomicExch(P.exit_cnt, 0u);
      volatile uint64_t *st = P.state;
      st[0] = m + 1;                     // first message this launch did not serve
      st_release_sys(P.state + 1, 0);    // alive = 0
    }
  }
}

template <uint32_t D>
__global__ void __launch_bounds__(kThreads, D == kBulkStages ? 3 : 2) relay_kernel(const __grid_constant__ RelayParams P) {
  extern __shared__ __align__(128) uint8_t dyn_smem[];
  relay_body<D>(P, blockIdx.x, P.q0, P.k, P.aligned, dyn_smem);
}


// Eager protocol (engine.h, reading C23).  Slot = [kEagerHdr header][shift][data]:
// header words 0/1 = bytes/tag (CTA 0), kEagerShift0 + r = source shift of CTA r's
// slice, kEagerFlag0 + r = CTA r's sequence flag (seq + 1, released after its slice).
__device__ void eager_send_body(const EagerParams &P, const uint32_t r) {
  __shared__ int s_abort;
  if (threadIdx.x == 0) s_abort = 0;
  __syncthreads();
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
    hdr[kEagerShift0 + r] = shift;
  }
  __syncthreads();  // the CTA's stores precede thread 0's release (cumulative)
  if (threadIdx.x == 0) st_release_sys(hdr + kEagerFlag0 + r, P.seq + 1);
}

__global__ void __launch_bounds__(kThreads) eager_send_kernel(const __grid_constant__ EagerParams P) {
  pdl_enter();
  eager_send_body(P, blockIdx.x);
}

__device__ void eager_recv_body(const EagerParams &P, const uint32_t r) {
  __shared__ int s_abort;
  if (threadIdx.x == 0) s_abort = 0;
  __syncthreads();
  const uint64_t *hdr = reinterpret_cast<const uint64_t *>(P.slot);
  // every CTA first checks the sender's size and tag (CTA 0's flag): a receive posted
  // larger than the message would otherwise wait for slices that never come
  if (!wait_word(hdr + kEagerFlag0, P.seq + 1, P.timeout_ns, P.err, &s_abort)) return;
  if (ld_volatile(hdr) != P.bytes || ld_volatile(hdr + 1) != P.tag) {
    if (threadIdx.x == 0) atomicExch(P.err, DERR_MISMATCH);
    return;
  }
  if (r > 0 && !wait_word(hdr + kEagerFlag0 + r, P.seq + 1, P.timeout_ns, P.err, &s_abort)) return;
  const uint8_t *data = P.slot + kEagerHdr + ld_volatile(hdr + kEagerShift0 + r);
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

__global__ void __launch_bounds__(kThreads) eager_recv_kernel(const __grid_constant__ EagerParams P) {
  pdl_enter();
  eager_recv_body(P, blockIdx.x);
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
template <uint32_t D>
__global__ void __launch_bounds__(kThreads, D == kBulkStages ? 3 : 2) direct_leg_kernel(const __grid_constant__ DirectArgs A) {
  extern __shared__ __align__(128) uint8_t dyn_smem[];
  pdl_enter();
  bulk_copy<LD_SRC, kStagedBlock, D>(A.dst, A.src, A.bytes, blockIdx.x, gridDim.x, dyn_smem, D, false);
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

// ------------------------------------------------------------------ emulated world
//
// One cooperative grid plays every rank's kernels (engine.h: EmuTable).  The relay
// role stands in for the relay rank's service thread too: its CTAs read the sender's
// doorbell for the first message on the device, then run the relay kernel's body,
// which serves exactly max_msgs messages (the later doorbells through the same
// next-message decisions as a lingering relay kernel).
template <uint32_t D>
__device__ void relay_emu_body(const RelayParams &P, const uint32_t b, uint8_t *smem) {
  // CTA 0 alone polls the doorbell in pinned host memory (as the relay rank's one host
  // thread does) and hands {q0, k, g} to the role's other CTAs through device words:
  // sixteen CTAs polling host memory at system scope made every MEMBAR.SYS on the GPU
  // slower (a clear-to-send post 1.6 -> 9.7 µs; scripts/diag/bell_poll.sh)
  __shared__ uint64_t s_bell[3];
  __shared__ int s_ok;
  if (threadIdx.x == 0) trace(124, 0);
  if (threadIdx.x == 0) {
    const uint64_t t0 = globaltimer();
    int ok = 1;
    if (b == 0) {
      const BellEntry *e = P.bells + P.m0 % kBellRing;
      while (ld_relaxed_sys(&e->tag) != P.m0 + 1 || ld_acquire_sys(&e->tag) != P.m0 + 1) {
        if (*reinterpret_cast<volatile int32_t *>(P.err) != 0) {  // the relay rank already failed
          ok = 0;
          break;
        }
        if (globaltimer() - t0 > P.timeout_ns) {
          atomicExch(P.err, DERR_TIMEOUT);
          ok = 0;
          break;
        }
        __nanosleep(256);
      }
      P.first[1] = ok ? ld_volatile(&e->q0) : 0;
      P.first[2] = ok ? ld_volatile(&e->k) : 0;
      P.first[3] = ok ? ld_volatile(&e->g) : 0;
      asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(P.first), "l"(ok ? P.m0 + 1 : ~0ull) : "memory");
    }
    uint64_t tag;
    for (;;) {
      asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(tag) : "l"(P.first) : "memory");
      if (tag == P.m0 + 1) break;
      if (tag == ~0ull) {  // CTA 0 failed (already reported)
        ok = 0;
        break;
      }
      if (globaltimer() - t0 > P.timeout_ns) {
        atomicExch(P.err, DERR_TIMEOUT);
        ok = 0;
        break;
      }
      __nanosleep(128);
    }
    if (ok) {
      s_bell[0] = ld_volatile(P.first + 1);
      s_bell[1] = ld_volatile(P.first + 2);
      s_bell[2] = ld_volatile(P.first + 3);
      if (static_cast<uint32_t>(s_bell[2] & 0xffffffffu) != P.g) {  // the role's CTAs are the lanes
        atomicExch(P.err, DERR_MISMATCH);
        ok = 0;
      }
    }
    s_ok = ok;
  }
  __syncthreads();
  if (threadIdx.x == 0) trace(124, 1);
  if (!s_ok) return;
  relay_body<D>(P, b, s_bell[0], s_bell[1], static_cast<uint32_t>((s_bell[2] >> 32) & 1u), smem);
}

// A role's parameter block, copied from the table into shared memory before the body
// runs: the real kernels read theirs from the constant bank (__grid_constant__), and
// the bodies' acquires invalidate L1, so a block left in global memory would cost an
// L2 round trip per field access in the pipelines' geometry code.
constexpr size_t cmax(size_t a, size_t b) { return a > b ? a : b; }
constexpr size_t kEmuParamBytes =
    cmax(cmax(sizeof(SendParams), sizeof(RecvParams)), cmax(sizeof(RelayParams), sizeof(EagerParams)));

template <class T>
__device__ __forceinline__ const T &emu_stage_params(const T *g, uint64_t *sm) {
  static_assert(sizeof(T) % 8 == 0, "parameter blocks are 8-byte multiples");
  const uint64_t *src = reinterpret_cast<const uint64_t *>(g);
  for (uint32_t i = threadIdx.x; i < sizeof(T) / 8; i += blockDim.x) sm[i] = src[i];
  __syncthreads();
  return *reinterpret_cast<const T *>(sm);
}

template <uint32_t D>
__global__ void __launch_bounds__(kThreads, D == kBulkStages ? 3 : 2) emu_kernel(const __grid_constant__ EmuTable T) {
  extern __shared__ __align__(128) uint8_t dyn_smem[];
  __shared__ __align__(16) uint64_t s_par[kEmuParamBytes / 8 + 1];
  const uint32_t blk = blockIdx.x;
  for (uint32_t i = 0; i < T.nroles; ++i) {
    const EmuRole R = T.roles[i];
    if (blk < R.cta0 || blk >= R.cta0 + R.n) continue;
    const uint32_t b = blk - R.cta0;
    switch (R.kind) {
      case EMU_GATE: send_gate_body(emu_stage_params(T.send + R.idx, s_par)); break;
      case EMU_SEND: send_body<D>(emu_stage_params(T.send + R.idx, s_par), b, dyn_smem); break;
      case EMU_RECV: recv_body<D>(emu_stage_params(T.recv + R.idx, s_par), b, dyn_smem); break;
      case EMU_RELAY: relay_emu_body<D>(emu_stage_params(T.relay + R.idx, s_par), b, dyn_smem); break;
      case EMU_EAGER_SEND: eager_send_body(emu_stage_params(T.eager + R.idx, s_par), b); break;
      case EMU_EAGER_RECV: eager_recv_body(emu_stage_params(T.eager + R.idx, s_par), b); break;
      default: break;
    }
    return;
  }
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

// The kernels with staged CTAs come in two depths (kBulkStages = 4 / kDeepStages = 6):
// `stages` of the parameter block picks the instance and its shared memory.
int launch_xfer(const XferParams &P, void *stream) {
  if (P.nblocks == 0) return cudaSuccess;
  const bool pdl = P.pdl != 0;
  const bool deep = P.stages == kDeepStages;
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
    if (P.copy_mode == 1 && P.staged_blk)
      return deep ? launch_k(pdl, direct_leg_kernel<kDeepStages>, P.nblocks, staged_smem<kDeepStages>(), stream, A)
                  : launch_k(pdl, direct_leg_kernel<kBulkStages>, P.nblocks, staged_smem<kBulkStages>(), stream, A);
    if (P.copy_mode == 1) return launch_k(pdl, direct_kernel, P.nblocks, kBulkSmem, stream, A);
    return launch_k(pdl, direct_reg_kernel, P.nblocks, 0, stream, A);
  }
  return deep ? launch_k(pdl, xfer_kernel<kDeepStages>, P.nblocks, staged_smem<kDeepStages>(), stream, P)
              : launch_k(pdl, xfer_kernel<kBulkStages>, P.nblocks, staged_smem<kBulkStages>(), stream, P);
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
  return P.stages == kDeepStages
             ? launch_k(pdl, send_kernel<kDeepStages>, P.nblocks, staged_smem<kDeepStages>(), stream, P)
             : launch_k(pdl, send_kernel<kBulkStages>, P.nblocks, staged_smem<kBulkStages>(), stream, P);
}

int launch_eager_send(const EagerParams &P, void *stream) {
  return launch_k(P.pdl != 0, eager_send_kernel, P.ctas, 0, stream, P);
}

int launch_eager_recv(const EagerParams &P, void *stream) {
  return launch_k(P.pdl != 0, eager_recv_kernel, P.ctas, 0, stream, P);
}

int launch_recv(const RecvParams &P, void *stream) {
  return P.stages == kDeepStages
             ? launch_k(P.pdl != 0, recv_kernel<kDeepStages>, P.nblocks, staged_smem<kDeepStages>(), stream, P)
             : launch_k(P.pdl != 0, recv_kernel<kBulkStages>, P.nblocks, staged_smem<kBulkStages>(), stream, P);
}

int launch_relay(const RelayParams &P, void *stream) {
  if (P.stages == kDeepStages)
    relay_kernel<kDeepStages><<<P.g, kThreads, staged_smem<kDeepStages>(), static_cast<cudaStream_t>(stream)>>>(P);
  else
    relay_kernel<kBulkStages><<<P.g, kThreads, staged_smem<kBulkStages>(), static_cast<cudaStream_t>(stream)>>>(P);
  return static_cast<int>(cudaGetLastError());
}

namespace {
template <uint32_t D>
cudaError_t emu_occupancy(int *n) {
  const int smem = static_cast<int>(staged_smem<D>());
  cudaError_t e = cudaFuncSetAttribute(emu_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(n, emu_kernel<D>, kThreads, smem);
  return e;
}
}  // namespace

#ifdef MPX_TRACE
}  // namespace mpx
extern "C" int mpx_trace_set(void *p) {
  return static_cast<int>(cudaMemcpyToSymbol(mpx::g_mpx_trace, &p, sizeof(p)));
}
namespace mpx {
#endif

int emu_capacity(int *per_sm, int *per_sm_deep) {
  cudaError_t e = emu_occupancy<kBulkStages>(per_sm);
  if (e == cudaSuccess) e = emu_occupancy<kDeepStages>(per_sm_deep);
  return static_cast<int>(e);
}

int launch_emu(const EmuTable &T, uint32_t stages, void *stream) {
  const bool deep = stages == kDeepStages;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(T.nblocks);
  cfg.blockDim = dim3(kThreads);
  cfg.dynamicSmemBytes = deep ? staged_smem<kDeepStages>() : staged_smem<kBulkStages>();
  cfg.stream = static_cast<cudaStream_t>(stream);
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeCooperative;  // every CTA co-resident, or the launch fails
  at[0].val.cooperative = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return static_cast<int>(deep ? cudaLaunchKernelEx(&cfg, emu_kernel<kDeepStages>, T)
                               : cudaLaunchKernelEx(&cfg, emu_kernel<kBulkStages>, T));
}

int launch_spin(uint64_t ns, void *stream) {
  spin_kernel<<<1, 32, 0, static_cast<cudaStream_t>(stream)>>>(ns);
  return static_cast<int>(cudaGetLastError());
}

int launch_pingpong(uint64_t *flags, int iters, uint64_t timeout_ns, int32_t *err, void *stream) {
  pingpong_kernel<<<2, 32, 0, static_cast<cudaStream_t>(stream)>>>(flags, iters, timeout_ns, err);
  return static_cast<int>(cudaGetLastError());
}

namespace {
template <uint32_t D>
cudaError_t preload_staged() {
  cudaFuncAttributes a;
  const int smem = static_cast<int>(staged_smem<D>());
  cudaError_t e = cudaFuncSetAttribute(xfer_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(send_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(recv_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(relay_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(direct_leg_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, xfer_kernel<D>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, send_kernel<D>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, recv_kernel<D>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, relay_kernel<D>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, direct_leg_kernel<D>);
  return e;
}

template <uint32_t D>
cudaError_t occupancy(int *n) {
  const int smem = static_cast<int>(staged_smem<D>());
  cudaError_t e = cudaFuncSetAttribute(xfer_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(n, xfer_kernel<D>, kThreads, smem);
}
}  // namespace

int preload_kernels() {
  // CUDA 12 loads kernels lazily, and a first load may wait for the device to idle;
  // load every kernel of this module up front (the relay service thread launches
  // relay kernels while the user's streams are busy).
  cudaFuncAttributes a;
  cudaError_t e = preload_staged<kBulkStages>();
  if (e == cudaSuccess) e = preload_staged<kDeepStages>();
  if (e == cudaSuccess) e = cudaFuncSetAttribute(direct_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kBulkSmem);
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
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, send_gate_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, pingpong_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, spin_kernel);
  return static_cast<int>(e);
}

int xfer_capacity(int device, int *per_sm, int *per_sm_deep, int *sms) {
  int n = 0, nd = 0;
  cudaError_t e = occupancy<kBulkStages>(&n);
  if (e == cudaSuccess) e = occupancy<kDeepStages>(&nd);
  if (e != cudaSuccess) return static_cast<int>(e);
  int s = 0;
  e = cudaDeviceGetAttribute(&s, cudaDevAttrMultiProcessorCount, device);
  if (e != cudaSuccess) return static_cast<int>(e);
  *per_sm = n;
  *per_sm_deep = nd;
  *sms = s;
  return cudaSuccess;
}

uint32_t deep_stages() { return kDeepStages; }
uint32_t shallow_stages() { return kBulkStages; }

}  // namespace mpx
