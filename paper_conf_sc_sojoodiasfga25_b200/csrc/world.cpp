// world.cpp — multi-rank engine host side (one process per GPU).
//
// Bootstrap (§2.1: UCX cuda_ipc exchanges and caches IPC handles;
// here the exchange is one all-gather at mp_init): every rank exports its receive
// heap and control block with cudaIpcGetMemHandle and maps every peer's; every rank
// creates a POSIX shared-memory segment holding the pinned host rings of the
// messages it receives (A9), registered mapped+portable so both the sending and the
// receiving GPU address it, preceded by the rank's relay doorbells; with world >= 3
// every rank runs a relay service thread that launches bounded relay kernels (A8 step
// 3) when a sender's gate kernel rings one of its doorbells.
#include <fcntl.h>
#include <sys/mman.h>
#include <sys/prctl.h>
#include <time.h>
#include <unistd.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <condition_variable>
#include <functional>
#include <map>
#include <mutex>
#include <thread>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <random>
#include <string>
#include <vector>

#include "ctx.h"

namespace mpx {

namespace {

int wfail(mp_ctx *c, int code, const std::string &msg) {
  c->last_error = msg;
  return code;
}

#define CKW(call)                                                                                 \
  do {                                                                                            \
    cudaError_t e__ = (call);                                                                     \
    if (e__ != cudaSuccess) return wfail(c, MP_ERR_CUDA, std::string(#call) + ": " + cudaGetErrorString(e__)); \
  } while (0)

struct RankInfo {
  cudaIpcMemHandle_t heap;
  cudaIpcMemHandle_t ctrl;
  uint64_t jobid;
  uint64_t heap_addr;
  uint64_t ctrl_addr;  // emulated world: every rank's memory is this process's own
  uint64_t heap_bytes;
  int32_t device;
  int32_t relay_ctas;
  uint64_t slot_bytes;
  int32_t slots;
  int32_t host_path;
  uint64_t eager_max;
  mp_gpu_info gpu;   // topology (topo.cpp)
};

int allgather(mp_ctx *c, const void *in, void *out, uint64_t bytes) {
  if (!c->allgather) return wfail(c, MP_ERR_INVALID, "world > 1 needs an allgather callback");
  if (c->allgather(c->allgather_user, in, out, bytes) != 0)
    return wfail(c, MP_ERR_INVALID, "bootstrap all-gather failed");
  return MP_OK;
}

int barrier(mp_ctx *c) {
  std::vector<uint8_t> out(c->world);
  uint8_t one = 1;
  return allgather(c, &one, out.data(), 1);
}

CtrlLayout layout(uint32_t world, uint32_t slots, uint64_t slot_bytes) {
  CtrlLayout L;
  L.world = world;
  L.slots = slots;
  L.stride = slot_bytes + kSlotSlack;
  L.slot_bytes = slot_bytes;
  uint64_t off = 0;
  auto take = [&](uint64_t bytes) {
    const uint64_t o = off;
    off = (off + bytes + 255) & ~uint64_t(255);
    return o;
  };
  L.cts = take(static_cast<uint64_t>(world) * kCtsRing * sizeof(MsgEntry));
  L.hdr = take(static_cast<uint64_t>(world) * kCtsRing * sizeof(MsgEntry));
  L.done = take(static_cast<uint64_t>(world) * 128);
  L.relay_free = take(static_cast<uint64_t>(world) * slots * kFlagStride * 8);
  L.ring_full = take(static_cast<uint64_t>(world) * slots * kFlagStride * 8);
  L.host_full = take(static_cast<uint64_t>(world) * slots * kFlagStride * 8);
  L.host_free = take(static_cast<uint64_t>(world) * slots * kFlagStride * 8);
  L.probe = take(64);
  L.regions = take(static_cast<uint64_t>(kMaxRegions) * world * 8);
  L.eager = take(static_cast<uint64_t>(world) * kEagerSlots * kEagerStride);
  L.eager_free = take(static_cast<uint64_t>(world) * 128);
  L.eager_cnt = take(static_cast<uint64_t>(world) * kEagerSlots * 4);
  L.relay_dec = take(static_cast<uint64_t>(world) * kBellRing * 32);
  L.relay_exit = take(static_cast<uint64_t>(world) * 128);
  L.bell_ack = take(static_cast<uint64_t>(world) * 128);
  L.dcnt = take(static_cast<uint64_t>(world) * kCtsRing * 8);
  L.dfree = take(static_cast<uint64_t>(world) * kCtsRing * 8);
  L.rcnt = take(static_cast<uint64_t>(world) * kBellRing * 8);
  L.rfree = take(static_cast<uint64_t>(world) * kBellRing * 8);
  L.ring_data = take(world >= 3 ? static_cast<uint64_t>(world) * slots * L.stride : 0);
  L.total = off;
  return L;
}

std::string seg_name(uint64_t jobid, int rank) {
  char b[64];
  std::snprintf(b, sizeof(b), "/mpx_%016llx_%d", static_cast<unsigned long long>(jobid), rank);
  return b;
}

int map_segment(mp_ctx *c, int rank, bool create, uint8_t **out) {
  const std::string name = seg_name(c->jobid, rank);
  const int fd = shm_open(name.c_str(), create ? (O_CREAT | O_EXCL | O_RDWR) : O_RDWR, 0600);
  if (fd < 0) return wfail(c, MP_ERR_NOMEM, "shm_open " + name + " failed");
  if (create && ftruncate(fd, static_cast<off_t>(c->hseg_bytes)) != 0) {
    close(fd);
    return wfail(c, MP_ERR_NOMEM, "ftruncate " + name + " failed");
  }
  void *p = mmap(nullptr, c->hseg_bytes, PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
  close(fd);
  if (p == MAP_FAILED) return wfail(c, MP_ERR_NOMEM, "mmap " + name + " failed");
  if (create) {
    // the segment holds the host rings this rank's GPU reads (A9 step 3): first touch
    // on its NUMA node (NUMA effects on the host path)
    numa_prefer(p, c->hseg_bytes, c->topo.gpu[c->rank].numa_node);
    std::memset(p, 0, c->hseg_bytes);
  }
  cudaError_t e = cudaHostRegister(p, c->hseg_bytes, cudaHostRegisterMapped | cudaHostRegisterPortable);
  if (e != cudaSuccess) {
    munmap(p, c->hseg_bytes);
    return wfail(c, MP_ERR_CUDA, std::string("cudaHostRegister: ") + cudaGetErrorString(e));
  }
  void *d = nullptr;
  CKW(cudaHostGetDevicePointer(&d, p, 0));
  if (d != p) return wfail(c, MP_ERR_UNSUPPORTED, "mapped host pointer differs from its device pointer (no UVA)");
  *out = static_cast<uint8_t *>(p);
  return MP_OK;
}

// The host ring of pair (src, dst): data slots in the receiver's pinned segment; the
// flags live in device memory of the GPU that polls them — "full" in dst's control
// block (written by src over NVLink after its PCIe data writes, ordered by a sys-scope
// fence), "free" in src's (written by dst) — so no flag is ever polled over PCIe.
HostRingPtrs host_ring(const mp_ctx *c, int src, int dst) {
  HostRingPtrs h;
  h.data = c->hseg[dst] + bell_bytes(c->world) + static_cast<uint64_t>(src) * c->hseg_per_src;
  h.full = reinterpret_cast<uint64_t *>(c->peers[dst].ctrl + c->L.host_full) +
           static_cast<uint64_t>(src) * c->slots * kFlagStride;
  h.freef = reinterpret_cast<uint64_t *>(c->peers[src].ctrl + c->L.host_free) +
            static_cast<uint64_t>(dst) * c->slots * kFlagStride;
  return h;
}

}  // namespace

int world_barrier(mp_ctx *c) { return barrier(c); }
int world_allgather(mp_ctx *c, const void *in, void *out, uint64_t bytes) { return allgather(c, in, out, bytes); }

static bool debug_on() {
  const char *d = std::getenv("MPX_DEBUG");
  return d && d[0] == '1';
}

#define DBG(msg)                                                          \
  do {                                                                    \
    if (debug_on()) std::fprintf(stderr, "[mpx %d] %s\n", c->rank, msg); \
  } while (0)

int world_init(mp_ctx *c) {
  DBG("world_init begin");
  CKW(cudaSetDevice(c->device));
  const int W = c->world;
  c->L = layout(W, c->slots, c->slot_bytes);
  void *p = nullptr;
  CKW(cudaMalloc(&p, c->L.total));
  c->ctrl = static_cast<uint8_t *>(p);
  CKW(cudaMemset(c->ctrl, 0, c->L.total));

  RankInfo me;
  std::memset(&me, 0, sizeof(me));
  if (!c->emulated) {
    CKW(cudaIpcGetMemHandle(&me.heap, c->heap.base));
    CKW(cudaIpcGetMemHandle(&me.ctrl, c->ctrl));
  }
  me.ctrl_addr = reinterpret_cast<uintptr_t>(c->ctrl);
  me.jobid = std::random_device{}() ^ (static_cast<uint64_t>(std::random_device{}()) << 32) ^
             static_cast<uint64_t>(getpid());
  me.heap_addr = reinterpret_cast<uintptr_t>(c->heap.base);
  me.heap_bytes = c->heap.size;
  me.device = c->device;
  me.relay_ctas = c->relay_ctas;
  me.slot_bytes = c->slot_bytes;
  me.slots = c->slots;
  me.host_path = c->host_path ? 1 : 0;
  // MPX_EAGER: "0" = every message takes the rendezvous; a byte count = the eager limit
  // (<= kEagerMax); unset = kEagerMax
  const char *eg = std::getenv("MPX_EAGER");
  c->eager_max = kEagerMax;
  if (eg && eg[0]) c->eager_max = std::min<uint64_t>(kEagerMax, std::strtoull(eg, nullptr, 10));
  me.eager_max = c->eager_max;
  if (int s = topo_local(c, &me.gpu)) return s;
  std::vector<RankInfo> all(W);
  if (int s = allgather(c, &me, all.data(), sizeof(RankInfo))) return s;
  c->jobid = all[0].jobid;
  for (int r = 0; r < W; ++r)
    if (all[r].relay_ctas != c->relay_ctas || all[r].slot_bytes != c->slot_bytes ||
        all[r].slots != c->slots || all[r].host_path != me.host_path || all[r].eager_max != me.eager_max)
      return wfail(c, MP_ERR_INVALID, "ranks disagree on slots / slot_bytes / relay_ctas / host_path / MPX_EAGER");

  DBG("rank info exchanged");
  c->peers.assign(W, PeerPtrs{nullptr, nullptr});
  for (int r = 0; r < W; ++r) {
    if (r == c->rank) {
      c->peers[r] = PeerPtrs{c->heap.base, c->ctrl};
      continue;
    }
    if (c->emulated) {  // one process: a peer's memory is addressed as allocated
      c->peers[r] = PeerPtrs{reinterpret_cast<uint8_t *>(all[r].heap_addr), reinterpret_cast<uint8_t *>(all[r].ctrl_addr)};
      continue;
    }
    void *h = nullptr, *k = nullptr;
    cudaError_t e = cudaIpcOpenMemHandle(&h, all[r].heap, cudaIpcMemLazyEnablePeerAccess);
    if (e == cudaSuccess) e = cudaIpcOpenMemHandle(&k, all[r].ctrl, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess)
      return wfail(c, MP_ERR_TOPOLOGY, "cannot map rank " + std::to_string(r) + "'s memory: " + cudaGetErrorString(e));
    c->peers[r] = PeerPtrs{static_cast<uint8_t *>(h), static_cast<uint8_t *>(k)};
    c->ipc_maps[{r, all[r].heap_addr}] = mp_ctx::IpcMap{static_cast<uint8_t *>(h), 1};
  }
  // topology: GPUs, peer access (mapping every peer above succeeded, else
  // mp_init already failed with MP_ERR_TOPOLOGY), PCIe / NVLink / NUMA
  {
    std::vector<mp_gpu_info> gpus(W);
    for (int r = 0; r < W; ++r) gpus[r] = all[r].gpu;
    if (int s = topo_discover(c, gpus, std::vector<int>(W, 1))) return s;
  }
  // region 0 = the heaps
  c->regions.assign(kMaxRegions, mp_ctx::Region{});
  c->regions[0].used = true;
  c->regions[0].base = c->heap.base;
  c->regions[0].bytes = c->heap.size;
  c->regions[0].maps.assign(W, 0);
  {
    std::vector<uint64_t> row(W);
    for (int r = 0; r < W; ++r) row[r] = reinterpret_cast<uintptr_t>(c->peers[r].heap);
    CKW(cudaMemcpy(c->ctrl + c->L.regions, row.data(), W * 8, cudaMemcpyHostToDevice));
  }

  // One shared pinned segment per rank: its relay doorbells, then (host path) the host
  // rings of the messages it receives, one ring per sender.
  c->host_stride = c->slot_bytes + kSlotSlack;
  c->hseg_per_src = (static_cast<uint64_t>(c->slots) * c->host_stride + 4095) & ~uint64_t(4095);
  c->hseg_bytes = static_cast<size_t>(bell_bytes(W) + (c->host_path ? c->hseg_per_src * W : 0));
  c->hseg.assign(W, nullptr);
  if ((c->host_path || W >= 3) && c->emulated) {
    // one process: every rank registers its own segment once; the others use its address
    if (int s = map_segment(c, c->rank, true, &c->hseg[c->rank])) return s;
    shm_unlink(seg_name(c->jobid, c->rank).c_str());
    const uint64_t mine = reinterpret_cast<uintptr_t>(c->hseg[c->rank]);
    std::vector<uint64_t> segs(W);
    if (int s = allgather(c, &mine, segs.data(), sizeof(uint64_t))) return s;
    for (int r = 0; r < W; ++r) c->hseg[r] = reinterpret_cast<uint8_t *>(segs[r]);
  } else if (c->host_path || W >= 3) {
    if (int s = map_segment(c, c->rank, true, &c->hseg[c->rank])) return s;
    if (int s = barrier(c)) return s;
    for (int r = 0; r < W; ++r)
      if (r != c->rank)
        if (int s = map_segment(c, r, false, &c->hseg[r])) return s;
    if (int s = barrier(c)) return s;
    shm_unlink(seg_name(c->jobid, c->rank).c_str());
  }

  DBG("ipc + host segments mapped");
  c->send_seq.assign(W, 0);
  c->recv_seq.assign(W, 0);
  c->relay_q.assign(W, 0);
  c->relay_m.assign(W, 0);
  c->ring_order.assign(5 * static_cast<size_t>(W), mp_ctx::RingOrder{});
  c->host_q.assign(W, 0);
  c->done_target.assign(W, 0);
  c->eager_send_seq.assign(W, 0);
  c->eager_recv_seq.assign(W, 0);
  const int s = barrier(c);
  DBG("world_init done");
  return s;
}

// ---------------------------------------------------------------- relay service (A8 step 3)
//
// The relay rank's side of a GPU-staged path.  A sender's gate kernel rings a doorbell
// in this rank's shared pinned segment (BellEntry: ring sequence q0, chunk count k,
// lanes g) once the message's clear-to-send has arrived; this thread sees it and
// launches a relay kernel of g CTAs for those chunks on the sender's stream (stream
// order keeps a sender's ring positions in order).  The kernel also serves the
// sender's following messages whose doorbells arrive within the linger (200 µs;
// MPX_RELAY_LINGER_US), so back-to-back relayed messages pay no relaunch; its last
// CTA then records the first doorbell it left and clears `alive`, and this thread
// takes over from there.  Every relay kernel ends at most a linger after its sender's
// traffic, so nothing runs on this GPU without traffic to serve, and a device-wide
// synchronisation (torch.cuda.synchronize, cudaDeviceSynchronize, lazy module
// loading) completes on every rank.  The thread spins while traffic is recent and
// polls every ~20 µs after 50 ms of quiet.
struct RelayService {
  std::thread th;
  std::atomic<bool> stop{false};
  std::atomic<int> error{0};           // cudaError_t of a failed relay launch (sticky)
  std::atomic<uint64_t> launches{0};
  std::vector<cudaStream_t> streams;   // [world(sender)]
  BellEntry *bells = nullptr;          // this rank's doorbells [world(sender)][kBellRing]
  uint64_t *state = nullptr;           // mapped host [world(sender)][2]: first unserved
                                       // doorbell, a relay kernel alive (host sets, kernel clears)
  uint64_t linger_ns = 200000;         // a relay kernel waits this long for the next doorbell
};

namespace {
void relay_loop(mp_ctx *c, RelayService *S) {
  cudaSetDevice(c->device);
  prctl(PR_SET_TIMERSLACK, 1000UL);  // 1 µs: the idle poll's sleep stays short
  RelayParams base{};
  base.me = static_cast<uint32_t>(c->rank);
  base.copy_mode = c->copy_mode;
  base.timeout_ns = static_cast<uint64_t>(c->timeout_s * 1e9);
  base.stages = stages_for(c, static_cast<uint32_t>(c->relay_ctas));
  base.my_ctrl = c->ctrl;
  for (int r = 0; r < c->world; ++r) base.peer[r] = c->peers[r];
  base.L = c->L;
  base.err = c->d_err;
  base.linger_ns = S->linger_ns;
  auto last = std::chrono::steady_clock::now();
  while (!S->stop.load(std::memory_order_acquire)) {
    bool any = false;
    for (int s = 0; s < c->world; ++s) {
      if (s == c->rank) continue;
      uint64_t *st = S->state + 2 * static_cast<uint64_t>(s);
      if (__atomic_load_n(st + 1, __ATOMIC_ACQUIRE)) {  // a lingering relay kernel serves this sender
        any = true;
        continue;
      }
      const uint64_t n = __atomic_load_n(st, __ATOMIC_RELAXED);
      const BellEntry *e = S->bells + static_cast<uint64_t>(s) * kBellRing + n % kBellRing;
      if (__atomic_load_n(&e->tag, __ATOMIC_ACQUIRE) != n + 1) continue;
      RelayParams P = base;
      P.sender = static_cast<uint32_t>(s);
      P.sender_ctrl = c->peers[s].ctrl;
      P.m0 = n;
      P.q0 = __atomic_load_n(&e->q0, __ATOMIC_RELAXED);
      P.k = __atomic_load_n(&e->k, __ATOMIC_RELAXED);
      const uint64_t g = __atomic_load_n(&e->g, __ATOMIC_RELAXED);
      P.g = static_cast<uint32_t>(g & 0xffffffffu);
      P.aligned = static_cast<uint32_t>((g >> 32) & 1u);
      P.bells = S->bells + static_cast<uint64_t>(s) * kBellRing;
      P.dec = reinterpret_cast<uint64_t *>(c->ctrl + c->L.relay_dec) + static_cast<uint64_t>(s) * kBellRing * 4;
      P.exit_cnt = reinterpret_cast<uint32_t *>(c->ctrl + c->L.relay_exit + static_cast<uint64_t>(s) * 128);
      P.state = st;
      if (P.g < 1 || P.g > static_cast<uint32_t>(kFlagStride)) {
        S->error.store(static_cast<int>(cudaErrorInvalidValue));
        __atomic_store_n(st, n + 1, __ATOMIC_RELAXED);  // skip the malformed doorbell
        continue;
      }
      __atomic_store_n(st + 1, 1, __ATOMIC_RELEASE);
      if (int rc = launch_relay(P, S->streams[s])) {
        S->error.store(rc);
        __atomic_store_n(st + 1, 0, __ATOMIC_RELEASE);
      }
      S->launches.fetch_add(1, std::memory_order_relaxed);
      any = true;
    }
    const auto now = std::chrono::steady_clock::now();
    if (any) {
      last = now;
    } else if (now - last > std::chrono::milliseconds(50)) {
      timespec ts{0, 20000};
      nanosleep(&ts, nullptr);
    }
  }
}
}  // namespace

int world_start_relay(mp_ctx *c) {
  const char *no_relay = std::getenv("MPX_NO_RELAY");  // diagnostics: no relay service
  // an emulated world has no relay threads: mp_emu_run's relay roles read the doorbells
  if (c->world < 3 || c->relay_svc || c->emulated || (no_relay && no_relay[0] == '1')) return MP_OK;
  RelayService *S = new RelayService();
  S->streams.assign(c->world, nullptr);
  S->bells = reinterpret_cast<BellEntry *>(c->hseg[c->rank]);
  if (const char *l = std::getenv("MPX_RELAY_LINGER_US")) S->linger_ns = static_cast<uint64_t>(std::atof(l) * 1e3);
  {
    void *p = nullptr;
    cudaError_t e = cudaHostAlloc(&p, 16ull * c->world, cudaHostAllocMapped | cudaHostAllocPortable);
    if (e != cudaSuccess) {
      delete S;
      return wfail(c, MP_ERR_CUDA, std::string("relay state: ") + cudaGetErrorString(e));
    }
    std::memset(p, 0, 16ull * c->world);
    S->state = static_cast<uint64_t *>(p);
  }
  for (int r = 0; r < c->world; ++r) {
    if (r == c->rank) continue;
    cudaError_t e = cudaStreamCreateWithFlags(&S->streams[r], cudaStreamNonBlocking);
    if (e != cudaSuccess) {
      for (cudaStream_t st : S->streams)
        if (st) cudaStreamDestroy(st);
      delete S;
      return wfail(c, MP_ERR_CUDA, std::string("relay stream: ") + cudaGetErrorString(e));
    }
  }
  c->relay_svc = S;
  S->th = std::thread(relay_loop, c, S);
  DBG("relay service started");
  return MP_OK;
}

// Stop the service thread (finalize) and wait for every relay kernel it launched.
int world_stop_relay(mp_ctx *c) {
  RelayService *S = c->relay_svc;
  if (!S) return MP_OK;
  S->stop.store(true, std::memory_order_release);
  if (S->th.joinable()) S->th.join();
  for (cudaStream_t st : S->streams)
    if (st) {
      cudaStreamSynchronize(st);
      cudaStreamDestroy(st);
    }
  if (S->state) cudaFreeHost(S->state);
  c->relay_launches_done += S->launches.load();
  c->relay_svc = nullptr;
  delete S;
  DBG("relay service stopped");
  return MP_OK;
}

uint64_t world_relay_launches(const mp_ctx *c) {
  return c->relay_launches_done + (c->relay_svc ? c->relay_svc->launches.load() : 0);
}

int world_relay_error(const mp_ctx *c) { return c->relay_svc ? c->relay_svc->error.load() : 0; }

uint64_t world_relay_linger_ns(const mp_ctx *c) { return c->relay_svc ? c->relay_svc->linger_ns : 0; }

int world_finalize(mp_ctx *c) {
  int st = MP_OK;
  world_stop_relay(c);
  cudaDeviceSynchronize();  // every stream this process enqueued on (not a list of handles
                            // the caller may have destroyed since)
  for (mp_ctx::RingOrder &o : c->ring_order)
    if (o.done) cudaEventDestroy(o.done);
  c->ring_order.clear();
  if (c->allgather) st = barrier(c);
  for (int r = 0; r < static_cast<int>(c->peers.size()) && !c->emulated; ++r) {
    if (r == c->rank) continue;
    if (c->peers[r].ctrl) cudaIpcCloseMemHandle(c->peers[r].ctrl);
  }
  for (auto &m : c->ipc_maps) cudaIpcCloseMemHandle(m.second.mapped);  // heaps + registered regions
  c->ipc_maps.clear();
  c->regions.clear();
  c->peers.clear();
  for (size_t r = 0; r < c->hseg.size(); ++r)
    if (c->hseg[r] && (!c->emulated || static_cast<int>(r) == c->rank)) {  // emulated: own segment only
      cudaHostUnregister(c->hseg[r]);
      munmap(c->hseg[r], c->hseg_bytes);
    }
  c->hseg.clear();
  if (c->ctrl) cudaFree(c->ctrl);
  c->ctrl = nullptr;
  return st;
}


// Eager protocol (reading C23): 1..eager_max bytes, direct path, no rendezvous.
static EagerParams eager_params(mp_ctx *c, int sender, int receiver, uint64_t seq, uint64_t bytes, int tag) {
  EagerParams P{};
  P.seq = seq;
  P.bytes = bytes;
  P.tag = static_cast<uint64_t>(static_cast<int64_t>(tag));
  P.timeout_ns = static_cast<uint64_t>(c->timeout_s * 1e9);
  P.ctas = static_cast<uint32_t>((bytes + kEagerSlice - 1) / kEagerSlice);
  const uint64_t slot = seq % kEagerSlots;
  P.slot = c->peers[receiver].ctrl + c->L.eager + (static_cast<uint64_t>(sender) * kEagerSlots + slot) * kEagerStride;
  P.free_ctr = reinterpret_cast<uint64_t *>(c->peers[sender].ctrl + c->L.eager_free +
                                            static_cast<uint64_t>(receiver) * 128);
  P.cnt = reinterpret_cast<uint32_t *>(c->peers[receiver].ctrl + c->L.eager_cnt) +
          static_cast<uint64_t>(sender) * kEagerSlots + slot;
  P.err = c->d_err;
  P.pdl = c->pdl_world;
  return P;
}

// Ring order across streams (ctx.h: ring_order): wait for the ring's previous user when
// it ran on another stream; after the launch, record this one.
static int ring_wait(mp_ctx *c, size_t ring, cudaStream_t s) {
#ifdef MPX_NO_RING_ORDER  // (design experiment: the engine without it)
  return MP_OK;
#endif
  mp_ctx::RingOrder &o = c->ring_order[ring];
  if (o.done && o.stream != s) CKW(cudaStreamWaitEvent(s, o.done, 0));
  return MP_OK;
}
static int ring_mark(mp_ctx *c, size_t ring, cudaStream_t s) {
  mp_ctx::RingOrder &o = c->ring_order[ring];
  if (!o.done) CKW(cudaEventCreateWithFlags(&o.done, cudaEventDisableTiming));
  CKW(cudaEventRecord(o.done, s));
  o.stream = s;
  return MP_OK;
}

static int eager_send(mp_ctx *c, const void *buf, uint64_t bytes, int dst, int tag, void *stream) {
  EagerParams P = eager_params(c, c->rank, dst, c->eager_send_seq[dst], bytes, tag);
  P.peer = static_cast<uint32_t>(dst);
  P.src = static_cast<const uint8_t *>(buf);
  // the eager slots are a ring too (a send waits for its slot's previous message to be
  // copied out): same cross-stream order, per destination
  const size_t ring = 3 * static_cast<size_t>(c->world) + static_cast<size_t>(dst);
  if (int e = ring_wait(c, ring, static_cast<cudaStream_t>(stream))) return e;
  if (c->emulated) {
    c->emu_esend.push_back(P);
  } else if (int e = launch_eager_send(P, stream))
    return wfail(c, MP_ERR_CUDA, std::string("eager send launch: ") + cudaGetErrorString(static_cast<cudaError_t>(e)));
  if (int e = ring_mark(c, ring, static_cast<cudaStream_t>(stream))) return e;
  c->launches += 1;
  c->eager_send_seq[dst] += 1;
  return MP_OK;
}

static int eager_recv(mp_ctx *c, void *buf, uint64_t bytes, int src, int tag, void *stream) {
  EagerParams P = eager_params(c, src, c->rank, c->eager_recv_seq[src], bytes, tag);
  P.peer = static_cast<uint32_t>(src);
  P.dst = static_cast<uint8_t *>(buf);
  const size_t ring = 4 * static_cast<size_t>(c->world) + static_cast<size_t>(src);
  if (int e = ring_wait(c, ring, static_cast<cudaStream_t>(stream))) return e;
  if (c->emulated) {
    c->emu_erecv.push_back(P);
  } else if (int e = launch_eager_recv(P, stream))
    return wfail(c, MP_ERR_CUDA, std::string("eager recv launch: ") + cudaGetErrorString(static_cast<cudaError_t>(e)));
  if (int e = ring_mark(c, ring, static_cast<cudaStream_t>(stream))) return e;
  c->launches += 1;
  c->eager_recv_seq[src] += 1;
  return MP_OK;
}

int world_send(mp_ctx *c, const void *buf, uint64_t bytes, int dst, int tag, const mp_config &cfg,
               void *stream) {
  if (bytes > 0 && bytes <= c->eager_max) return eager_send(c, buf, bytes, dst, tag, stream);
  SendParams P{};
  P.me = static_cast<uint32_t>(c->rank);
  P.dst = static_cast<uint32_t>(dst);
  P.seq = c->send_seq[dst];
  P.bytes = bytes;
  P.tag = static_cast<uint64_t>(static_cast<int64_t>(tag));
  P.timeout_ns = static_cast<uint64_t>(c->timeout_s * 1e9);
  P.src = static_cast<const uint8_t *>(buf);
  P.my_ctrl = c->ctrl;
  P.dst_ctrl = c->peers[dst].ctrl;
  P.err = c->d_err;
  P.L = c->L;
  P.host_stride = c->host_stride;
  P.host_slots = static_cast<uint32_t>(c->slots);
  P.align = c->opts.align;
  P.copy_mode = c->copy_mode;
  P.pdl = c->pdl_world;
  P.bulk_stages = bulk_stages_for(cfg.bytes[0]);
  if (c->host_path) P.host = host_ring(c, c->rank, dst);
  P.direct_bytes = cfg.bytes[0];
  // Every staged path gets a stage group of relay_ctas CTAs (= lanes of its ring
  // slots; the receiver's host consumers and Step 1's leg timing use the same count).
  const uint32_t g_stage = static_cast<uint32_t>(c->relay_ctas);
  P.g_host = g_stage;
  uint32_t staged = 0;
  for (int i = 1; i < cfg.npaths; ++i)
    if (cfg.bytes[i]) staged += g_stage;
  P.stages = stages_for(c, staged);
  const int cap = std::max(1, per_sm_at(c, P.stages) * c->sms);
  P.g_direct = direct_ctas(c, cfg.bytes[0], cap - static_cast<int>(staged));
  if (staged && P.g_direct > static_cast<uint32_t>(c->sms))  // whole CTAs per SM beside staged groups
    P.g_direct = P.g_direct / static_cast<uint32_t>(c->sms) * static_cast<uint32_t>(c->sms);
  uint32_t next = P.g_direct;
  uint64_t off = cfg.bytes[0];
  uint32_t np = 0;
  std::vector<std::pair<int, uint32_t>> advance;
  for (int i = 1; i < cfg.npaths; ++i) {
    const uint64_t b = cfg.bytes[i];
    if (b) {
      SendParams::StagedDesc &d = P.sp[np++];
      d.kind = cfg.path[i].kind == MP_PATH_HOST ? 2 : 1;
      d.relay = d.kind == 1 ? static_cast<uint32_t>(cfg.path[i].via) : 0u;
      d.k = cfg.chunks[i];
      d.g = g_stage;
      d.cta0 = next;
      next += d.g;
      d.off = off;
      d.bytes = b;
      if (d.kind == 1) {
        if (!c->hseg[d.relay]) return wfail(c, MP_ERR_TOPOLOGY, "relay rank has no doorbell segment");
        d.q0 = c->relay_q[d.relay];
        d.ring_ctrl = c->peers[d.relay].ctrl;
        d.m = c->relay_m[d.relay];
        d.bell = reinterpret_cast<BellEntry *>(c->hseg[d.relay]) + static_cast<uint64_t>(c->rank) * kBellRing;
        advance.emplace_back(static_cast<int>(d.relay), d.k);
      } else {
        d.q0 = c->host_q[dst];
        advance.emplace_back(-1, d.k);
      }
    }
    off += b;
  }
  P.npaths = np;
  P.nblocks = next;
  const cudaStream_t cs = static_cast<cudaStream_t>(stream);
  const size_t W = static_cast<size_t>(c->world);
  for (auto &a : advance)
    if (int e = ring_wait(c, a.first < 0 ? W + static_cast<size_t>(dst) : static_cast<size_t>(a.first), cs)) return e;
  if (c->emulated) {
    c->emu_send.push_back(P);
  } else if (int e = launch_send(P, stream))
    return wfail(c, MP_ERR_CUDA, std::string("send launch: ") + cudaGetErrorString(static_cast<cudaError_t>(e)));
  for (auto &a : advance)
    if (int e = ring_mark(c, a.first < 0 ? W + static_cast<size_t>(dst) : static_cast<size_t>(a.first), cs)) return e;
  c->launches += 2;  // rendezvous gate + bulk send kernel
  c->send_seq[dst] += 1;
  for (auto &a : advance) {
    if (a.first < 0) {
      c->host_q[dst] += a.second;
    } else {
      c->relay_q[a.first] += a.second;
      c->relay_m[a.first] += 1;
    }
  }
  return MP_OK;
}

bool world_receivable(mp_ctx *c, const void *p, uint64_t n) {
  const uint8_t *b = static_cast<const uint8_t *>(p);
  for (const mp_ctx::Region &g : c->regions)
    if (g.used && g.base && b >= g.base && b + n <= g.base + g.bytes) return true;
  return false;
}

int world_recv(mp_ctx *c, void *buf, uint64_t bytes, int src, int tag, void *stream) {
  uint8_t *b = static_cast<uint8_t *>(buf);
  int region = -1;
  for (int i = 0; i < static_cast<int>(c->regions.size()) && bytes; ++i) {
    const mp_ctx::Region &g = c->regions[i];
    if (g.used && g.base && b >= g.base && b + bytes <= g.base + g.bytes) {
      region = i;
      break;
    }
  }
  if (!bytes) region = 0;
  if (region < 0)
    return wfail(c, MP_ERR_INVALID, "mp_recv buffer must come from mp_alloc or mp_register when world > 1");
  if (bytes > 0 && bytes <= c->eager_max) return eager_recv(c, buf, bytes, src, tag, stream);
  if (c->emulated) {  // every recorded receive posts its clear-to-send at once (mp_emu_run)
    uint32_t pending = 0;
    for (const RecvParams &R : c->emu_recv) pending += R.src == static_cast<uint32_t>(src) ? 1u : 0u;
    if (pending >= kCtsRing)
      return wfail(c, MP_ERR_INVALID, "mp_recv: at most " + std::to_string(kCtsRing) +
                                          " rendezvous messages of one pair per mp_emu_run");
  }
  RecvParams P{};
  P.me = static_cast<uint32_t>(c->rank);
  P.src = static_cast<uint32_t>(src);
  P.seq = c->recv_seq[src];
  P.bytes = bytes;
  P.tag = static_cast<uint64_t>(static_cast<int64_t>(tag));
  P.region = static_cast<uint64_t>(region);
  if (debug_on())
    std::fprintf(stderr, "[mpx %d] recv %llu B from %d into region %d + %llu\n", c->rank,
                 static_cast<unsigned long long>(bytes), src, region,
                 static_cast<unsigned long long>(bytes ? b - c->regions[region].base : 0));
  P.region_off = bytes ? static_cast<uint64_t>(b - c->regions[region].base) : 0;
  P.done_target = c->done_target[src] + bytes;
  P.timeout_ns = static_cast<uint64_t>(c->timeout_s * 1e9);
  P.my_ctrl = c->ctrl;
  P.buf = b;
  P.src_ctrl = c->peers[src].ctrl;
  P.err = c->d_err;
  P.L = c->L;
  P.host_stride = c->host_stride;
  P.host_slots = static_cast<uint32_t>(c->slots);
  P.g_host = c->host_path ? static_cast<uint32_t>(c->relay_ctas) : 0u;
  P.stages = stages_for(c, P.g_host);
  P.copy_mode = c->copy_mode;
  P.pdl = c->pdl_world;
  P.bulk_stages = bulk_stages_for(bytes);
  if (c->host_path) P.host = host_ring(c, src, c->rank);
  P.nblocks = 1 + P.g_host;
  const size_t ring = 2 * static_cast<size_t>(c->world) + static_cast<size_t>(src);
  const cudaStream_t cs = static_cast<cudaStream_t>(stream);
  if (c->host_path)
    if (int e = ring_wait(c, ring, cs)) return e;
  if (c->emulated) {
    c->emu_recv.push_back(P);
  } else if (int e = launch_recv(P, stream))
    return wfail(c, MP_ERR_CUDA, std::string("recv launch: ") + cudaGetErrorString(static_cast<cudaError_t>(e)));
  if (c->host_path)
    if (int e = ring_mark(c, ring, cs)) return e;
  c->launches += 1;
  c->recv_seq[src] += 1;
  c->done_target[src] += bytes;
  return MP_OK;
}

// ---------------------------------------------------------------- regions (mp_register)

namespace {
// cuMemGetAddressRange through the runtime's driver entry point (no -lcuda).
int alloc_range(mp_ctx *c, const void *p, uint64_t *base, uint64_t *size) {
  using Fn = int (*)(unsigned long long *, size_t *, unsigned long long);
  static Fn fn = nullptr;
  if (!fn) {
    void *f = nullptr;
    cudaDriverEntryPointQueryResult q{};
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &f, cudaEnableDefault, &q) != cudaSuccess || !f)
      return wfail(c, MP_ERR_CUDA, "cuMemGetAddressRange entry point not found");
    fn = reinterpret_cast<Fn>(f);
  }
  unsigned long long b = 0;
  size_t n = 0;
  if (fn(&b, &n, reinterpret_cast<uintptr_t>(p)) != 0)
    return wfail(c, MP_ERR_INVALID, "mp_register: not a device allocation");
  *base = b;
  *size = n;
  return MP_OK;
}

struct RegInfo {
  cudaIpcMemHandle_t h;
  uint64_t alloc_base, off;
  int32_t status;   // 0 nothing registered, 1 exported, < 0 MP_ERR_* of a local failure
  int32_t id;
};

int write_region_row(mp_ctx *c, int id, const std::vector<uint64_t> &row) {
  CKW(cudaMemcpy(c->ctrl + c->L.regions + static_cast<uint64_t>(id) * c->world * 8, row.data(),
                 c->world * 8, cudaMemcpyHostToDevice));
  // a pageable copy may return before its DMA lands (registration is collective and
  // no transfer is in flight, so no relay kernel runs: the device goes idle)
  CKW(cudaDeviceSynchronize());
  return MP_OK;
}

void unmap(mp_ctx *c, int r, uint64_t key) {
  auto it = c->ipc_maps.find({r, key});
  if (it == c->ipc_maps.end()) return;
  if (--it->second.refs == 0) {
    cudaIpcCloseMemHandle(it->second.mapped);
    c->ipc_maps.erase(it);
  }
}
}  // namespace

int world_register(mp_ctx *c, void *buf, uint64_t bytes, int *id) {
  if (c->emulated && !emu_rank_thread(c))
    return wfail(c, MP_ERR_UNSUPPORTED, "mp_register: in an emulated world, through mp_emu_register");
  const int W = c->world;
  int rid = -1;
  for (int i = 1; i < static_cast<int>(c->regions.size()); ++i)
    if (!c->regions[i].used) {
      rid = i;
      break;
    }
  RegInfo me;
  std::memset(&me, 0, sizeof(me));
  me.id = rid;
  std::string local_err;
  if (buf && bytes) {
    uint64_t base = 0, size = 0;
    if (int s = alloc_range(c, buf, &base, &size)) {
      me.status = s;
    } else if (reinterpret_cast<uintptr_t>(buf) + bytes > base + size) {
      me.status = MP_ERR_INVALID;
      c->last_error = "mp_register: buffer runs past its allocation";
    } else if (!c->emulated && cudaIpcGetMemHandle(&me.h, reinterpret_cast<void *>(base)) != cudaSuccess) {
      cudaGetLastError();
      me.status = MP_ERR_UNSUPPORTED;
      c->last_error = "mp_register: the allocation cannot be exported with cudaIpc (VMM / expandable segment?)";
    } else {
      me.status = 1;
      me.alloc_base = base;
      me.off = reinterpret_cast<uintptr_t>(buf) - base;
    }
  }
  std::vector<RegInfo> all(W);
  if (int s = allgather(c, &me, all.data(), sizeof(RegInfo))) return s;
  for (int r = 0; r < W; ++r) {
    if (all[r].id != rid) return wfail(c, MP_ERR_STATE, "mp_register / mp_deregister not called collectively");
    if (all[r].status < 0)
      return r == c->rank ? all[r].status
                          : wfail(c, all[r].status, "mp_register failed on rank " + std::to_string(r));
  }
  if (rid < 0) return wfail(c, MP_ERR_NOMEM, "mp_register: region table full");
  mp_ctx::Region g;
  g.used = true;
  g.base = static_cast<uint8_t *>(bytes ? buf : nullptr);
  g.bytes = bytes;
  g.maps.assign(W, 0);
  std::vector<uint64_t> row(W, 0);
  int st = MP_OK;
  for (int r = 0; r < W && st == MP_OK; ++r) {
    if (all[r].status != 1) continue;
    if (r == c->rank) {
      row[r] = reinterpret_cast<uintptr_t>(buf);
      continue;
    }
    if (c->emulated) {  // one process: the peer's buffer is addressed as allocated
      row[r] = all[r].alloc_base + all[r].off;
      continue;
    }
    auto it = c->ipc_maps.find({r, all[r].alloc_base});
    if (it == c->ipc_maps.end()) {
      void *h = nullptr;
      cudaError_t e = cudaIpcOpenMemHandle(&h, all[r].h, cudaIpcMemLazyEnablePeerAccess);
      if (e != cudaSuccess) {
        st = wfail(c, MP_ERR_CUDA, "mp_register: cannot map rank " + std::to_string(r) + ": " + cudaGetErrorString(e));
        break;
      }
      it = c->ipc_maps.emplace(std::make_pair(r, all[r].alloc_base), mp_ctx::IpcMap{static_cast<uint8_t *>(h), 0}).first;
    }
    it->second.refs += 1;
    g.maps[r] = all[r].alloc_base;
    row[r] = reinterpret_cast<uintptr_t>(it->second.mapped) + all[r].off;
  }
  if (st == MP_OK) st = write_region_row(c, rid, row);
  if (debug_on())
    for (int r = 0; r < W; ++r)
      std::fprintf(stderr, "[mpx %d] region %d rank %d -> %p (status %d, alloc %llx + %llu)\n", c->rank, rid, r,
                   reinterpret_cast<void *>(row[r]), all[r].status,
                   static_cast<unsigned long long>(all[r].alloc_base), static_cast<unsigned long long>(all[r].off));
  if (st == MP_OK) {
    c->regions[rid] = g;
    *id = rid;
  } else {
    for (int r = 0; r < W; ++r)
      if (g.maps[r]) unmap(c, r, g.maps[r]);
  }
  // every rank's table holds the row before anyone sends into the region
  if (int s = barrier(c)) return s;
  return st;
}

int world_deregister(mp_ctx *c, int id) {
  if (c->emulated && !emu_rank_thread(c))
    return wfail(c, MP_ERR_UNSUPPORTED, "mp_deregister: in an emulated world, through mp_emu_deregister");
  const int W = c->world;
  if (id <= 0 || id >= static_cast<int>(c->regions.size()) || !c->regions[id].used)
    return wfail(c, MP_ERR_INVALID, "mp_deregister: unknown region id");
  RegInfo me;
  std::memset(&me, 0, sizeof(me));
  me.id = id;
  CKW(cudaDeviceSynchronize());  // our receives into it are done
  std::vector<RegInfo> all(W);
  if (int s = allgather(c, &me, all.data(), sizeof(RegInfo))) return s;
  for (int r = 0; r < W; ++r)
    if (all[r].id != id) return wfail(c, MP_ERR_STATE, "mp_register / mp_deregister not called collectively");
  int st = write_region_row(c, id, std::vector<uint64_t>(W, 0));
  for (int r = 0; r < W; ++r)
    if (c->regions[id].maps[r]) unmap(c, r, c->regions[id].maps[r]);
  c->regions[id] = mp_ctx::Region{};
  if (int s = barrier(c)) return s;
  return st;
}

// A device-wide wait: every stream this process used (relay kernels are bounded
// launches, §7, so nothing outlives the traffic by more than the linger).  The engine
// keeps no list of the caller's streams: a handle destroyed after mp_send would make
// such a list unusable.
int world_sync(mp_ctx *c) {
  CKW(cudaDeviceSynchronize());
  if (int e = world_relay_error(c))
    return wfail(c, MP_ERR_CUDA, std::string("relay launch: ") + cudaGetErrorString(static_cast<cudaError_t>(e)));
  int32_t e = 0;
  CKW(cudaMemcpy(&e, c->d_err, sizeof(e), cudaMemcpyDeviceToHost));
  if (e == DERR_TIMEOUT) return wfail(c, MP_ERR_TIMEOUT, "a device-side wait timed out");
  if (e == DERR_MISMATCH) return wfail(c, MP_ERR_MISMATCH, "send/recv size or tag mismatch");
  return MP_OK;
}


// ---------------------------------------------------------------- emulated world
//
// MP_INIT_EMULATED (include/mp.h): the ranks of a world are contexts of ONE process on
// ONE GPU.  mp_init_emulated bootstraps them on one thread each through an in-process
// all-gather (the same world_init as a real job, with the IPC exchange replaced by
// the allocations' own addresses); mp_send / mp_recv record their parameter blocks;
// mp_emu_run launches everything recorded as one cooperative grid (engine.h EmuTable)
// — the B200 guide's rule for ranks whose kernels wait on one another when there are
// fewer GPUs than ranks.

struct EmuWorld {
  int world = 0;
  std::mutex mu;
  std::condition_variable cv;
  uint64_t gen = 0;
  int arrived = 0;
  bool aborted = false;
  std::vector<uint8_t> buf, out;
  std::vector<mp_ctx *> ctxs;
};

namespace {
thread_local int t_emu_rank = -1;

// The in-process all-gather: rank t_emu_rank's bytes into slot t_emu_rank; the last
// arrival publishes the gathered block; a rank whose mp_init failed aborts every
// pending and later all-gather (no rank waits forever for it).
int emu_allgather(void *user, const void *in, void *out, uint64_t bytes) {
  EmuWorld *w = static_cast<EmuWorld *>(user);
  const int r = t_emu_rank;
  if (r < 0 || r >= w->world) return -1;
  std::unique_lock<std::mutex> lk(w->mu);
  if (w->aborted) return -1;
  const uint64_t g = w->gen;
  if (w->arrived == 0) w->buf.assign(bytes * w->world, 0);
  if (w->buf.size() != bytes * w->world) return -1;
  std::memcpy(w->buf.data() + bytes * r, in, bytes);
  if (++w->arrived == w->world) {
    w->out = w->buf;
    w->arrived = 0;
    w->gen += 1;
    w->cv.notify_all();
  } else {
    w->cv.wait(lk, [&] { return w->gen != g || w->aborted; });
    if (w->gen == g) return -1;  // aborted
  }
  std::memcpy(out, w->out.data(), bytes * w->world);
  return 0;
}

void emu_abort(EmuWorld *w) {
  std::lock_guard<std::mutex> lk(w->mu);
  w->aborted = true;
  w->cv.notify_all();
}
}  // namespace

int emu_init_world(mp_ctx **ctxs, const mp_init_args *a) {
  const int W = a->world;
  EmuWorld *w = new EmuWorld();
  w->world = W;
  w->ctxs.assign(W, nullptr);
  std::vector<int> st(W, MP_OK);
  std::vector<std::thread> th;
  for (int r = 0; r < W; ++r)
    th.emplace_back([&, r] {
      t_emu_rank = r;
      mp_init_args ar = *a;
      ar.rank = r;
      ar.flags = (a->flags | MP_INIT_EMULATED | MP_INIT_NO_CALIBRATE) & ~MP_INIT_MODEL_ONLY;
      ar.allgather = emu_allgather;
      ar.allgather_user = w;
      st[r] = mp_init(&w->ctxs[r], &ar);
      if (st[r] != MP_OK) emu_abort(w);
    });
  for (std::thread &t : th) t.join();
  int bad = MP_OK;
  for (int r = 0; r < W; ++r)
    if (st[r] != MP_OK && bad == MP_OK) bad = st[r];
  if (bad != MP_OK) {  // ranks that did come up: finalize them without the collective part
    for (int r = 0; r < W; ++r)
      if (w->ctxs[r]) {
        w->ctxs[r]->emu_world = nullptr;
        w->ctxs[r]->allgather = nullptr;
        mp_finalize(w->ctxs[r]);
      }
    delete w;
    return bad;
  }
  for (int r = 0; r < W; ++r) {
    w->ctxs[r]->emu_world = w;
    ctxs[r] = w->ctxs[r];
  }
  return MP_OK;
}

int emu_finalize_world(mp_ctx **ctxs, int n) {
  EmuWorld *w = ctxs[0]->emu_world;
  if (!w || n != w->world) return MP_ERR_INVALID;
  for (int r = 0; r < n; ++r)
    if (!ctxs[r] || ctxs[r]->emu_world != w || ctxs[r]->rank != r) return MP_ERR_INVALID;
  std::vector<std::thread> th;
  for (int r = 0; r < n; ++r)
    th.emplace_back([=] {
      t_emu_rank = r;
      ctxs[r]->emu_world = nullptr;  // mp_finalize's collective part runs on this thread
      mp_finalize(ctxs[r]);
    });
  for (std::thread &t : th) t.join();
  delete w;
  return MP_OK;
}

bool emu_thread() { return t_emu_rank >= 0; }
bool emu_rank_thread(const mp_ctx *c) { return t_emu_rank == c->rank; }

// A collective call of every rank of an emulated world, each on its own thread (the
// in-process all-gather needs all of them at once); the first failure is returned.
int emu_each_rank(mp_ctx **ctxs, int n, const std::function<int(int)> &fn) {
  EmuWorld *w = ctxs[0]->emu_world;
  if (!w || n != w->world) return MP_ERR_INVALID;
  for (int r = 0; r < n; ++r)
    if (!ctxs[r] || ctxs[r]->emu_world != w || ctxs[r]->rank != r) return MP_ERR_INVALID;
  std::vector<int> st(n, MP_OK);
  std::vector<std::thread> th;
  for (int r = 0; r < n; ++r)
    th.emplace_back([&, r] {
      t_emu_rank = r;
      cudaSetDevice(ctxs[r]->device);
      st[r] = fn(r);
      if (st[r] != MP_OK) emu_abort(w);
    });
  for (std::thread &t : th) t.join();
  {
    std::lock_guard<std::mutex> lk(w->mu);  // a failed call aborted the all-gathers: reset for later calls
    w->aborted = false;
    w->arrived = 0;
  }
  for (int r = 0; r < n; ++r)
    if (st[r] != MP_OK) return st[r];
  return MP_OK;
}

int emu_run(mp_ctx **ctxs, int n, void *stream, double *kernel_s) {
  mp_ctx *c = ctxs[0];
  EmuWorld *w = c->emu_world;
  if (!w || n != w->world) return wfail(c, MP_ERR_INVALID, "mp_emu_run: pass every context of one emulated world");
  for (int r = 0; r < n; ++r)
    if (!ctxs[r] || ctxs[r]->emu_world != w || ctxs[r]->rank != r)
      return wfail(c, MP_ERR_INVALID, "mp_emu_run: contexts must be the world's, in rank order");
  c = w->ctxs[0];
  CKW(cudaSetDevice(c->device));
  // whatever happens below, the recorded work is consumed by this call
  auto clear = [&] {
    for (int r = 0; r < n; ++r) {
      ctxs[r]->emu_send.clear();
      ctxs[r]->emu_recv.clear();
      ctxs[r]->emu_esend.clear();
      ctxs[r]->emu_erecv.clear();
    }
  };
  std::vector<SendParams> send;
  std::vector<RecvParams> recv;
  std::vector<EagerParams> eager;
  std::vector<RelayParams> relay;
  std::vector<EmuRole> roles;
  for (int r = 0; r < n; ++r) {
    mp_ctx *cr = ctxs[r];
    send.insert(send.end(), cr->emu_send.begin(), cr->emu_send.end());
    recv.insert(recv.end(), cr->emu_recv.begin(), cr->emu_recv.end());
  }
  // every recorded receive posts its clear-to-send at once: at most kCtsRing messages
  // of one ordered pair per run (a real receiver's stream posts them one at a time)
  {
    std::map<std::pair<uint32_t, uint32_t>, uint32_t> per_pair;
    for (const RecvParams &P : recv)
      if (++per_pair[{P.src, P.me}] > kCtsRing) {
        clear();
        return wfail(c, MP_ERR_INVALID, "mp_emu_run: more than " + std::to_string(kCtsRing) +
                                            " rendezvous messages of one pair in one run");
      }
  }
  // relay roles: one per (relay rank, sender), serving that sender's recorded doorbells
  // m0 .. m0 + count - 1 (what the relay's service thread and its lingering kernels do)
  std::map<std::pair<uint32_t, uint32_t>, std::vector<std::pair<uint64_t, uint32_t>>> bells;  // -> (m, g)
  for (const SendParams &P : send)
    for (uint32_t i = 0; i < P.npaths; ++i)
      if (P.sp[i].kind == 1) bells[{P.sp[i].relay, P.me}].emplace_back(P.sp[i].m, P.sp[i].g);
  for (auto &kv : bells) {
    std::vector<std::pair<uint64_t, uint32_t>> &v = kv.second;
    std::sort(v.begin(), v.end());
    for (size_t j = 1; j < v.size(); ++j)
      if (v[j].first != v[j - 1].first + 1 || v[j].second != v[0].second) {
        clear();
        return wfail(c, MP_ERR_INVALID, "mp_emu_run: a relay's doorbells must be consecutive with equal lanes");
      }
    mp_ctx *rc = w->ctxs[kv.first.first];
    const uint32_t snd = kv.first.second;
    RelayParams P{};
    P.me = static_cast<uint32_t>(rc->rank);
    P.sender = snd;
    P.g = v[0].second;
    P.copy_mode = rc->copy_mode;
    P.timeout_ns = static_cast<uint64_t>(rc->timeout_s * 1e9);
    P.m0 = v[0].first;
    P.max_msgs = v.size();
    P.linger_ns = P.timeout_ns;  // the next doorbell of a recorded message does come
    P.bells = reinterpret_cast<const BellEntry *>(rc->hseg[rc->rank]) + static_cast<uint64_t>(snd) * kBellRing;
    P.dec = reinterpret_cast<uint64_t *>(rc->ctrl + rc->L.relay_dec) + static_cast<uint64_t>(snd) * kBellRing * 4;
    P.exit_cnt = reinterpret_cast<uint32_t *>(rc->ctrl + rc->L.relay_exit + static_cast<uint64_t>(snd) * 128);
    P.my_ctrl = rc->ctrl;
    P.sender_ctrl = rc->peers[snd].ctrl;
    for (int r = 0; r < rc->world; ++r) P.peer[r] = rc->peers[r];
    P.L = rc->L;
    P.err = rc->d_err;
    relay.push_back(P);
  }
  for (int r = 0; r < n; ++r) {
    mp_ctx *cr = ctxs[r];
    eager.insert(eager.end(), cr->emu_esend.begin(), cr->emu_esend.end());
  }
  const size_t n_esend = eager.size();
  for (int r = 0; r < n; ++r) {
    mp_ctx *cr = ctxs[r];
    eager.insert(eager.end(), cr->emu_erecv.begin(), cr->emu_erecv.end());
  }
  // Grid: every role co-resident.  Only the direct groups are elastic (any CTA count
  // moves the same bytes): they share what the fixed roles leave, in proportion to
  // the CTA counts the real launches would have used.  Staged pipelines run at the
  // deep depth when the whole grid fits its occupancy (as the real launches choose per
  // launch, stages_for), else at 4 stages; MPX_STAGES forces one.
  int per_sm = 0, per_sm_deep = 0;
  if (int e = emu_capacity(&per_sm, &per_sm_deep)) {
    clear();
    return wfail(c, MP_ERR_CUDA, std::string("emu_capacity: ") + cudaGetErrorString(static_cast<cudaError_t>(e)));
  }
  uint64_t fixed = 0, want = 0;
  for (const SendParams &P : send) {
    fixed += 1 + (P.nblocks - P.g_direct);
    want += P.g_direct;
  }
  for (const RecvParams &P : recv) fixed += P.nblocks;
  for (const RelayParams &P : relay) fixed += P.g;
  for (const EagerParams &P : eager) fixed += P.ctas;
  const uint64_t sms = static_cast<uint64_t>(c->sms);
  uint32_t stages = fixed + want <= static_cast<uint64_t>(per_sm_deep) * sms ? deep_stages() : shallow_stages();
  if (c->force_stages) stages = c->force_stages;
  const uint64_t cap = static_cast<uint64_t>(stages == deep_stages() ? per_sm_deep : per_sm) * sms;
  if (fixed + send.size() > cap) {
    clear();
    return wfail(c, MP_ERR_INVALID, "mp_emu_run: the recorded kernels do not fit one co-resident grid (" +
                                         std::to_string(fixed + send.size()) + " > " + std::to_string(cap) + " CTAs)");
  }
  if (fixed + want > cap)
    for (SendParams &P : send) {
      const uint32_t gd = std::max<uint32_t>(1, static_cast<uint32_t>(P.g_direct * (cap - fixed) / want));
      uint32_t next = gd;
      for (uint32_t i = 0; i < P.npaths; ++i) {
        P.sp[i].cta0 = next;
        next += P.sp[i].g;
      }
      P.g_direct = gd;
      P.nblocks = next;
    }
  uint32_t cta = 0;
  auto add = [&](uint32_t kind, uint32_t cnt, uint32_t idx) {
    roles.push_back(EmuRole{kind, cta, cnt, idx});
    cta += cnt;
  };
  for (uint32_t i = 0; i < recv.size(); ++i) add(EMU_RECV, recv[i].nblocks, i);
  for (uint32_t i = 0; i < relay.size(); ++i) add(EMU_RELAY, relay[i].g, i);
  for (uint32_t i = 0; i < send.size(); ++i) {
    add(EMU_GATE, 1, i);
    add(EMU_SEND, send[i].nblocks, i);
  }
  for (uint32_t i = 0; i < eager.size(); ++i) add(i < n_esend ? EMU_EAGER_SEND : EMU_EAGER_RECV, eager[i].ctas, i);
  clear();
  if (kernel_s) *kernel_s = 0;
  if (roles.empty()) return MP_OK;
  // one device block: roles, then the parameter arrays (16-B aligned)
  auto al = [](size_t x) { return (x + 255) & ~size_t(255); };
  const size_t o_roles = 0, o_send = al(o_roles + roles.size() * sizeof(EmuRole)),
               o_recv = al(o_send + send.size() * sizeof(SendParams)),
               o_relay = al(o_recv + recv.size() * sizeof(RecvParams)),
               o_eager = al(o_relay + relay.size() * sizeof(RelayParams)),
               o_state = al(o_eager + eager.size() * sizeof(EagerParams)),
               o_first = al(o_state + std::max<size_t>(1, relay.size()) * 2 * sizeof(uint64_t)),
               total = al(o_first + std::max<size_t>(1, relay.size()) * 4 * sizeof(uint64_t));
  std::vector<uint8_t> h(total, 0);
  void *d = nullptr;
  CKW(cudaMalloc(&d, total));
  uint8_t *db = static_cast<uint8_t *>(d);
  for (size_t i = 0; i < relay.size(); ++i) {
    relay[i].state = reinterpret_cast<uint64_t *>(db + o_state) + 2 * i;  // the relay's exit record (unread)
    relay[i].first = reinterpret_cast<uint64_t *>(db + o_first) + 4 * i;  // zeroed by the upload below
  }
  std::memcpy(h.data() + o_roles, roles.data(), roles.size() * sizeof(EmuRole));
  if (!send.empty()) std::memcpy(h.data() + o_send, send.data(), send.size() * sizeof(SendParams));
  if (!recv.empty()) std::memcpy(h.data() + o_recv, recv.data(), recv.size() * sizeof(RecvParams));
  if (!relay.empty()) std::memcpy(h.data() + o_relay, relay.data(), relay.size() * sizeof(RelayParams));
  if (!eager.empty()) std::memcpy(h.data() + o_eager, eager.data(), eager.size() * sizeof(EagerParams));
  EmuTable T{};
  T.roles = reinterpret_cast<const EmuRole *>(db + o_roles);
  T.send = reinterpret_cast<const SendParams *>(db + o_send);
  T.recv = reinterpret_cast<const RecvParams *>(db + o_recv);
  T.relay = reinterpret_cast<const RelayParams *>(db + o_relay);
  T.eager = reinterpret_cast<const EagerParams *>(db + o_eager);
  T.nroles = static_cast<uint32_t>(roles.size());
  T.nblocks = cta;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  cudaEvent_t ev[2] = {nullptr, nullptr};
  cudaError_t e = cudaMemcpyAsync(d, h.data(), total, cudaMemcpyHostToDevice, st);
  if (e == cudaSuccess && kernel_s) e = cudaEventCreate(&ev[0]);
  if (e == cudaSuccess && kernel_s) e = cudaEventCreate(&ev[1]);
  if (e == cudaSuccess && kernel_s) e = cudaEventRecord(ev[0], st);
  if (e == cudaSuccess) e = static_cast<cudaError_t>(launch_emu(T, stages, stream));
  if (e == cudaSuccess && kernel_s) e = cudaEventRecord(ev[1], st);
  if (e == cudaSuccess) e = cudaStreamSynchronize(st);
  if (e == cudaSuccess && kernel_s) {
    float ms = 0;
    e = cudaEventElapsedTime(&ms, ev[0], ev[1]);
    *kernel_s = ms * 1e-3;
  }
  for (cudaEvent_t x : ev)
    if (x) cudaEventDestroy(x);
  cudaFree(d);
  if (e != cudaSuccess) return wfail(c, MP_ERR_CUDA, std::string("mp_emu_run: ") + cudaGetErrorString(e));
  for (int r = 0; r < n; ++r) {
    int32_t de = 0;
    CKW(cudaMemcpy(&de, ctxs[r]->d_err, sizeof(de), cudaMemcpyDeviceToHost));
    if (de == DERR_TIMEOUT) return wfail(c, MP_ERR_TIMEOUT, "rank " + std::to_string(r) + ": a device-side wait timed out");
    if (de == DERR_MISMATCH)
      return wfail(c, MP_ERR_MISMATCH, "rank " + std::to_string(r) + ": send/recv size or tag mismatch");
  }
  return MP_OK;
}

}  // namespace mpx
