// ctx.h — the library context behind the opaque mp_ctx (internal).
#pragma once
#include <cuda_runtime.h>

#include <algorithm>

#include <cstdint>
#include <deque>
#include <functional>
#include <map>
#include <string>
#include <unordered_map>
#include <vector>

#include "../../include/mp.h"
#include "engine.h"
#include "model.h"

namespace mpx {

struct CollState;     // collectives (coll.cpp): internal streams, events, heap scratch
struct RelayService;  // world.cpp: the relay rank's doorbell thread and streams

// A staging ring (D8): S slots of slot_stride bytes + per-CTA flag words.
struct Ring {
  uint8_t *data = nullptr;     // device memory (relay) or mapped pinned host memory (host)
  uint64_t *full = nullptr;    // [slots][kFlagStride]
  uint64_t *freef = nullptr;   // [slots][kFlagStride]
  bool host = false;
  bool registered = false;     // host data from mmap + cudaHostRegister (diagnostics)
  uint64_t data_bytes = 0;
  uint64_t q = 0;              // next ring sequence number (chunks issued so far)
};

// First-fit allocator over one device region (the registered heap).
struct Heap {
  uint8_t *base = nullptr;
  uint64_t size = 0;
  std::map<uint64_t, uint64_t> free_;  // offset -> length
  std::map<uint64_t, uint64_t> used_;  // offset -> length
  void reset(uint8_t *b, uint64_t n);
  void *alloc(uint64_t n);
  bool release(void *p);
};

struct PendingSend {           // loopback mp_send waiting for its mp_recv
  const void *buf;
  uint64_t bytes;
  int tag;
  bool has_cfg;
  mp_config cfg;
  cudaEvent_t ready;
};

struct CacheKey {
  int src, dst;
  uint32_t mask;
  uint64_t n;
  bool operator==(const CacheKey &o) const {
    return src == o.src && dst == o.dst && mask == o.mask && n == o.n;
  }
};
struct CacheKeyHash {
  size_t operator()(const CacheKey &k) const {
    uint64_t h = k.n * 0x9E3779B97F4A7C15ull;
    h ^= (static_cast<uint64_t>(k.src) << 40) ^ (static_cast<uint64_t>(k.dst) << 20) ^ k.mask;
    return static_cast<size_t>(h ^ (h >> 29));
  }
};

}  // namespace mpx

namespace mpx {
struct EmuWorld;  // world.cpp
}

struct mp_ctx {
  int rank = 0, world = 1, device = 0, flags = 0;
  bool model_only = true;
  std::string last_error;
  mpx::ModelOpts opts;
  std::map<std::pair<int, int>, mpx::PairModel> models;
  // NEXT f4 size bands (reading C20): per pair, (n_min, model) ascending, n_min > 0;
  // the base model (models) is band 0 with n_min = 0.
  std::map<std::pair<int, int>, std::vector<std::pair<uint64_t, mpx::PairModel>>> bands;
  // NEXT f2 (readings C24, C25): per-pair window parameters and per-GPU host duplex
  // factors (absent = h 0, τ 0; κ 1).
  std::map<std::pair<int, int>, mpx::WindowModel> windows;
  std::vector<double> kappa;
  double submit = 0.0;             // reading C27: host submission time per message [s]
  std::unordered_map<mpx::CacheKey, mpx::Selection, mpx::CacheKeyHash> cache;
  mp_topology topo{};              // topo.cpp: found by mp_init or injected (model-only)
  bool have_topo = false;
  uint32_t env_kinds = 0x7u;       // path kinds allowed by MPX_PATHS (bit = MP_PATH_*)

  // engine
  int n_loop_relays = 6;
  bool host_path = true;
  int slots = 4;
  int relay_ctas = 16;
  uint64_t slot_bytes = 32ull << 20;
  double timeout_s = 20.0;
  int per_sm = 0, per_sm_deep = 0, sms = 0;  // co-resident staged-kernel CTAs per SM (4 / 6 stages)
  uint32_t force_stages = 0;       // env MPX_STAGES=4|6: every staged launch at that depth
  uint32_t pdl = 1;                // loopback launches use PDL (env MPX_PDL=0: off)
  uint32_t pdl_world = 0;          // multi-rank launches use PDL (env MPX_PDL_WORLD=1: on)
  uint32_t copy_mode = 1;          // direct-path copy: 1 = TMA bulk, 0 = LDG/STG (env MPX_COPY=reg)
  int32_t *d_err = nullptr;
  std::vector<mpx::Ring> rings;   // loopback: [0..V) relays, [V] host (if enabled)
  mpx::Heap heap;
  std::deque<mpx::PendingSend> pending;
  uint64_t launches = 0;
  // the last large loopback transfer (concurrency-aware direct grid)
  cudaEvent_t big_ev = nullptr;
  cudaStream_t big_stream = nullptr;
  bool big_valid = false;
  // the last loopback launch that used the staging rings: ring slots are handed out in
  // launch order, so a staged launch on another stream runs after it (no two kernels
  // ever wait on each other's ring slots)
  cudaEvent_t ring_ev = nullptr;
  cudaStream_t ring_stream = nullptr;
  bool ring_valid = false;
  uint64_t *d_probe = nullptr;    // calibration flag words (device)
  uint64_t *h_probe = nullptr;    // calibration flag words (mapped host)

  // multi-rank engine (world > 1), see engine.h / world.cpp
  mp_allgather_fn allgather = nullptr;
  void *allgather_user = nullptr;
  uint64_t jobid = 0;
  mpx::CtrlLayout L;
  uint8_t *ctrl = nullptr;                  // this rank's control block (device)
  std::vector<mpx::PeerPtrs> peers;         // [world]: heap/ctrl of every rank (self = local)
  uint64_t host_stride = 0;
  uint64_t hseg_per_src = 0;                // bytes of one pair's host ring in a segment
  size_t hseg_bytes = 0;
  std::vector<uint8_t *> hseg;              // [world]: mapped host segment of each receiver
  std::vector<uint64_t> send_seq, recv_seq, relay_q, host_q, done_target;
  std::vector<uint64_t> relay_m;            // [world(relay)]: relayed messages sent via each relay
  // Ring order across streams: ring positions are assigned in call order, so a staged
  // send (recv with host consumers) on another stream than the previous user of the
  // same ring waits for it — a later message's CTAs spinning on slots could otherwise
  // hold the SMs its predecessor needs.  [5·world]: relay ring r (sender side), host
  // ring to d (sender side, world + d), host ring from s (receiver side, 2·world + s),
  // eager slots to d (3·world + d) and from s (4·world + s).
  struct RingOrder {
    cudaStream_t stream = nullptr;
    cudaEvent_t done = nullptr;
  };
  std::vector<RingOrder> ring_order;
  mpx::CollState *coll = nullptr;           // created by the first collective
  std::vector<uint64_t> eager_send_seq, eager_recv_seq;  // eager protocol (reading C23)
  uint64_t eager_max = 0;                   // messages of 1..eager_max bytes go eager
  mpx::RelayService *relay_svc = nullptr;   // world >= 3: launches relay kernels on doorbells
  uint64_t relay_launches_done = 0;         // relay launches of stopped services
  // receive regions (mp_register): [kMaxRegions], region 0 = the heap
  struct Region {
    bool used = false;
    uint8_t *base = nullptr;                // this rank's buffer (nullptr: none registered)
    uint64_t bytes = 0;
    std::vector<uint64_t> maps;             // [world]: key into ipc_maps (0 = none)
  };
  std::vector<Region> regions;
  // IPC mapping cache: (rank, remote allocation base) -> {mapped base, refs}
  struct IpcMap {
    uint8_t *mapped = nullptr;
    int refs = 0;
  };
  std::map<std::pair<int, uint64_t>, IpcMap> ipc_maps;
  // emulated world (MP_INIT_EMULATED; engine.h EmuTable): the kernels mp_send / mp_recv
  // would launch, recorded for the next mp_emu_run
  bool emulated = false;
  mpx::EmuWorld *emu_world = nullptr;       // shared by the world's contexts (world.cpp)
  std::vector<mpx::SendParams> emu_send;
  std::vector<mpx::RecvParams> emu_recv;
  std::vector<mpx::EagerParams> emu_esend, emu_erecv;
};

namespace mpx {
// TMA pipeline shape of a direct group: 2 CTAs per SM × 4 stages of 8 KiB at every
// size.  (scripts/copybench.cu favoured 4 CTAs/SM × 3 stages for L2-resident sizes in
// single-launch timings, but inside the engine that shape measured slower at every
// size in the OMB sweep — profiles/r01/omb_*.jsonl — so it is not used.)
inline uint32_t bulk_stages_for(uint64_t /*bytes*/) { return 4u; }

// CTAs of a direct group: one per 32 KiB, at most 2 per SM (TMA) or 4 per SM
// (LDG/STG), and at most `room` (what is left of the co-resident capacity).  With PDL
// (full_grid: loopback launches) a TMA group always takes the full 2 per SM: a grid that is not a multiple of the SM
// count lands unevenly on the SMs its predecessor still occupies (8 MiB, 256 CTAs:
// 5.2 µs per back-to-back message vs 3.1 µs with 296; scripts/pdlbench.cu).
inline uint32_t direct_ctas(const mp_ctx *c, uint64_t bytes, int room, bool full_grid = false) {
  uint64_t want = bytes ? (bytes + (32u << 10) - 1) / (32u << 10) : 1;
  const int per_sm = c->copy_mode == 1 ? 2 : 4;
  const int lim = std::max(1, std::min(room, per_sm * c->sms));
  if (full_grid && c->copy_mode == 1) want = static_cast<uint64_t>(lim);
  return static_cast<uint32_t>(std::min<uint64_t>(want, static_cast<uint64_t>(lim)));
}

// Staged pipeline depth of a launch with `staged` staged CTAs (engine.cu): the deep
// pipeline (6 × 16 KiB, 2 CTAs per SM) when those CTAs leave every SM room for at least
// one more CTA (the direct group), else 4 stages (3 CTAs per SM).
inline uint32_t stages_for(const mp_ctx *c, uint32_t staged) {
  if (c->force_stages) return c->force_stages;
  return staged + static_cast<uint32_t>(c->sms) <= static_cast<uint32_t>(c->per_sm_deep * c->sms) ? deep_stages()
                                                                                                    : shallow_stages();
}
inline int per_sm_at(const mp_ctx *c, uint32_t stages) { return stages == deep_stages() ? c->per_sm_deep : c->per_sm; }

// One direct-path fused launch dst ← src (any world; dst may be peer or mapped host).
// ctas > 0 fixes the CTA count (calibration of a staged leg uses the staged group's).
int launch_direct_copy(mp_ctx *c, void *dst, const void *src, uint64_t n, void *stream, int ctas = 0);
int world_barrier(mp_ctx *c);
int world_allgather(mp_ctx *c, const void *in, void *out, uint64_t bytes);
int world_init(mp_ctx *c);
int world_start_relay(mp_ctx *c);
int world_stop_relay(mp_ctx *c);
uint64_t world_relay_launches(const mp_ctx *c);  // relay kernels this rank launched
int world_relay_error(const mp_ctx *c);          // cudaError_t of a failed relay launch, 0 if none
uint64_t world_relay_linger_ns(const mp_ctx *c);  // the relay kernels' linger, 0 without a service
int world_finalize(mp_ctx *c);
int world_send(mp_ctx *c, const void *buf, uint64_t bytes, int dst, int tag, const mp_config &cfg,
               void *stream);
int world_recv(mp_ctx *c, void *buf, uint64_t bytes, int src, int tag, void *stream);
int world_sync(mp_ctx *c);
// emulated world (world.cpp): bootstrap / teardown of all ranks on one thread each,
// the one cooperative launch of what they recorded, and whether this thread is one of
// the bootstrap's rank threads
int emu_init_world(mp_ctx **ctxs, const mp_init_args *a);
int emu_finalize_world(mp_ctx **ctxs, int n);
int emu_run(mp_ctx **ctxs, int n, void *stream, double *kernel_s);
bool emu_thread();
bool emu_rank_thread(const mp_ctx *c);  // this thread runs c's rank inside emu_each_rank
int emu_each_rank(mp_ctx **ctxs, int n, const std::function<int(int)> &fn);
int world_register(mp_ctx *c, void *buf, uint64_t bytes, int *id);
// true when [p, p + n) lies in a receive region (heap or mp_register) of this rank
bool world_receivable(mp_ctx *c, const void *p, uint64_t n);
// collectives (coll.cpp): release the per-context streams, events and heap scratch
void coll_release(mp_ctx *c);
int world_deregister(mp_ctx *c, int id);
// topology (topo.cpp)
int topo_local(mp_ctx *c, mp_gpu_info *g);
int topo_discover(mp_ctx *c, const std::vector<mp_gpu_info> &gpus, const std::vector<int> &mapped);
uint64_t topo_fingerprint(const mp_topology &t);
void numa_prefer(void *p, size_t n, int node);
}  // namespace mpx
