// engine.h — device-side transfer engine: parameter blocks shared by the host
// launcher (capi.cpp) and the kernels (engine.cu).  Internal; not part of the ABI.
//
// One message is cut into per-path byte ranges (reading C6).  Every path is served
// by CTA *groups* of one fused kernel launch:
//   direct path : one group copies its range straight to the destination (A7).
//   staged path : a stage-in group copies chunk j into ring slot (q0+j) % S and
//                 releases per-CTA "full" flags; a forward group acquires them,
//                 copies the slot to the destination and releases per-CTA "free"
//                 flags (A8 relays, A9 host).  This is the three-step pipeline of
//                 P:224-228 with the flag handoff standing for the synchronisation ε.
// Flags are 64-bit generation words, one per CTA (no atomics, so they also work in
// pinned host memory where PCIe gives no atomics): chunk q uses slot s = q % S for
// the u = q / S-th time; producers wait free[s][*] >= u, consumers full[s][*] >= u+1.
#pragma once
#include <cstdint>

#ifdef __CUDACC__
#define MPX_HD __host__ __device__
#else
#define MPX_HD
#endif

namespace mpx {

constexpr int kMaxPaths = 16;
constexpr int kFlagStride = 32;    // flag words per slot (max CTAs per staged group)
constexpr int kThreads = 256;      // threads per CTA of every engine kernel
// A staging slot is cut into per-lane regions, one per CTA of the stage group (see
// lane_stride): lane r of a slot only ever holds slice r of a chunk, written by
// stage-in CTA r and read by forward CTA r, so each lane is an independent two-stage
// pipeline with its own full/free flag (no CTA waits for another CTA's slice).
// Slack per slot: lanes round up (<= 144 B each for <= kFlagStride lanes).
constexpr uint32_t kSlotSlack = 8192;
constexpr uint32_t kLaneHdr = 64;     // per-lane header (multi-rank relay rings)

// Bytes between lanes of a slot of slot_bytes payload cut into g lanes: a slice of a
// chunk <= slot_bytes is at most ceil(slot_bytes/g) + 16 bytes (slice_of rounds its
// ends up to 16 B), plus the <= 15-byte co-alignment shift and the lane header.
MPX_HD inline uint64_t lane_stride(uint64_t slot_bytes, uint32_t g) {
  return (((slot_bytes + g - 1) / g + 15) / 16) * 16 + 128;
}

enum : int32_t { DK_DIRECT = 0, DK_STAGED = 1 };

// Error codes raised by kernels into the context's device error word.
enum : int32_t { DERR_NONE = 0, DERR_TIMEOUT = 1, DERR_MISMATCH = 2 };

struct DevPath {
  int32_t kind;          // DK_DIRECT / DK_STAGED
  uint32_t g_in;         // direct: CTAs; staged: stage-in CTAs = lanes (<= kFlagStride)
  uint32_t g_out;        // staged: forward CTAs (== g_in: lane r is served by CTA r of each)
  uint32_t cta0_in;      // first blockIdx.x of the direct / stage-in group
  uint32_t cta0_out;     // first blockIdx.x of the forward group
  uint32_t k;            // chunks
  uint32_t slots;        // ring slots S
  uint32_t host_ring;    // 1 when ring + flags live in pinned host memory
  uint64_t q0;           // ring sequence number of chunk 0
  uint64_t bytes;        // bytes on this path
  uint64_t align;        // chunk unit A (reading C6)
  uint64_t slot_stride;  // bytes between slots (slot_bytes + kSlotSlack)
  uint64_t lane;         // bytes between the lanes of a slot (lane_stride(slot_bytes, g))
  const uint8_t *src;    // source + path offset
  uint8_t *dst;          // destination + path offset (local, peer or mapped)
  uint8_t *ring;         // slot 0
  uint64_t *full;        // [slots][kFlagStride], written by the stage-in group
  uint64_t *freef;       // [slots][kFlagStride], written by the forward group
};

struct XferParams {
  uint32_t npaths;
  uint32_t nblocks;
  uint32_t copy_mode;    // direct group: 0 = LDG/STG vectors, 1 = TMA bulk (cp.async.bulk)
  uint32_t bulk_stages;  // TMA pipeline depth per CTA (1..4)
  uint32_t allow_small;  // 1: a small direct-only message may use the one-shot kernel
  uint32_t pdl;          // 1: launched with programmatic stream serialization (PDL)
  uint32_t staged_blk;   // 1: a direct-only copy timing a loopback staged leg (Step 1):
                         //    moved with the staged legs' TMA block size
  uint32_t stages;       // staged pipeline depth: shallow_stages() or deep_stages()
  uint64_t timeout_ns;
  int32_t *err;          // device (or mapped host) error word
  DevPath p[kMaxPaths];
};

// Direct-only messages up to this size (co-aligned mod 16) go to the one-shot kernel:
// one 16-B vector per thread, every load in flight at once, ~20 instructions of
// straight-line code (profiles/r01/smallbench*.jsonl: 2.1-3.1 µs per back-to-back
// message vs 4.1 µs for the TMA pipeline kernel, whose cold instruction fetches
// dominate at these sizes).
constexpr uint64_t kSmallMax = 4ull << 20;

// Launch the fused transfer kernel (engine.cu).  Returns a cudaError_t value.
int launch_xfer(const XferParams &P, void *stream);

// ---------------------------------------------------------------- multi-rank engine
//
// One process per GPU.  Every rank exports (cudaIpc) its receive heap and its
// control block; every rank maps every peer's.  A message src → dst:
//   receiver (mp_recv):  recv kernel CTA 0 posts a CTS entry {seq+1, region offset,
//                        bytes, tag, region id} into the sender's control block, then waits for
//                        its per-src byte counter `done` to reach the target; CTAs
//                        1.. consume the message's host-ring chunks (A9 step 3).
//   sender   (mp_send):  a one-CTA gate kernel waits for the CTS, writes the message
//                        header {seq+1, host_k, host_q0, status, ...} into the
//                        receiver's control block and rings the doorbell of every
//                        relay the message uses; then the bulk send kernel's direct
//                        group stores into the target region (A7), its stage-in
//                        groups fill relay rings (A8 step 1) and the host ring (A9
//                        step 1); every byte delivered is counted into the
//                        receiver's `done` with red.release.sys.
//   relay    (on demand): a host thread of the relay rank watches its doorbells (in
//                        its shared pinned segment, written by the senders' gate
//                        kernels over PCIe) and launches one bounded relay kernel per
//                        relayed message range, on a per-sender stream; CTA r forwards
//                        lane r of every chunk of the range to the destination named
//                        in the lane header (A8 step 3), then the kernel ends.  No
//                        kernel outlives the traffic it serves, so a device-wide
//                        synchronisation on any rank completes.
// Relay slot = kFlagStride-many lanes (lane_stride); lane header = {dst rank, region
// offset of the slice, slice length, shift, region}.
// A receive target is (region id, offset): every rank's control block holds the table
// regions[id][rank] = base of rank's region `id` as mapped in THIS process (region 0
// = the heaps, 1.. = mp_register), so a sender or relay resolves it locally.

constexpr uint32_t kCtsRing = 64;     // outstanding messages per ordered pair
constexpr uint32_t kBellRing = 64;    // outstanding relayed messages per (sender, relay)

// Eager protocol (NEXT f4's low-latency protocol, reading C23): a message of
// 1..kEagerMax bytes skips the rendezvous — the sender writes it, with per-CTA
// sequence flags, into one of kEagerSlots slots the receiver owns per sender, the
// receiver copies it out and returns the slot with a counter.  One kernel per side,
// no clear-to-send round trip.
// Round 2 raised kEagerMax from 64 KiB to 1 MiB: a rendezvous costs a clear-to-send
// round trip per message (the receive holds its stream until the message lands), far
// more than the eager copy-out of ≤ 1 MiB.
constexpr uint32_t kEagerSlots = 8;
constexpr uint64_t kEagerMax = 1ull << 20;
constexpr uint32_t kEagerSlice = 16384;           // bytes per CTA (≤ 64 CTAs)
constexpr uint32_t kEagerCtas = kEagerMax / kEagerSlice;
constexpr uint32_t kEagerFlag0 = 64;              // header word of CTA r's sequence flag: 64 + r
constexpr uint32_t kEagerShift0 = 128;            // header word of CTA r's source shift: 128 + r
constexpr uint32_t kEagerHdr = 2048;              // {bytes, tag, …, flags[64], shifts[64]} before the data
constexpr uint64_t kEagerStride = kEagerHdr + kEagerMax + 256;  // + co-alignment shift
static_assert(kEagerCtas <= 64, "eager header holds 64 flags and 64 shifts");
constexpr uint32_t kMaxRegions = 64;  // receive regions: 0 = heap, 1.. = mp_register

struct MsgEntry {                      // CTS and message-header entries (64 B)
  uint64_t seq1;                       // sequence + 1 (written last, with release)
  uint64_t a, b, c;                    // CTS: region offset, bytes, tag; HDR: host_k, host_q0, status
  uint64_t d, e, f, g;                 // CTS: region id; HDR: host range message offset, host bytes,
                                       //      src shift (mod 16), chunk unit A
};

// Doorbell of one relayed message (sender → relay rank's host thread), in the relay's
// shared pinned segment.  Written by the sender's gate kernel; tag last (release).
struct BellEntry {
  uint64_t tag;                        // message index on (sender, relay) + 1
  uint64_t q0;                         // ring sequence of the message's first chunk
  uint64_t k;                          // chunks
  uint64_t g;                          // lanes (stage-group CTAs); bit 32: source and
                                       // target co-aligned mod 16
};
inline uint64_t bell_bytes(uint32_t world) {
  return (static_cast<uint64_t>(world) * kBellRing * sizeof(BellEntry) + 4095) & ~uint64_t(4095);
}

struct PeerPtrs {
  uint8_t *heap;                       // peer's receive heap (mapped)
  uint8_t *ctrl;                       // peer's control block (mapped)
};

// Byte offsets inside every rank's control block (identical on all ranks).
struct CtrlLayout {
  uint32_t world = 0, slots = 0;
  uint64_t stride = 0;                 // relay slot stride (slot_bytes + kSlotSlack)
  uint64_t slot_bytes = 0;             // payload bytes per relay slot (lane_stride input)
  uint64_t cts = 0;                    // [world(src=receiver)][kCtsRing] MsgEntry — on the sender
  uint64_t hdr = 0;                    // [world(src=sender)][kCtsRing] MsgEntry   — on the receiver
  uint64_t done = 0;                   // [world(src)] u64, 128-B padded         — on the receiver
  uint64_t relay_free = 0;             // [world(relay)][slots][kFlagStride]      — on the sender
  uint64_t ring_full = 0;              // [world(sender)][slots][kFlagStride]     — on the relay
  uint64_t ring_data = 0;              // [world(sender)][slots][stride]          — on the relay
  uint64_t host_full = 0;              // [world(sender)][slots][kFlagStride]     — on the receiver
  uint64_t host_free = 0;              // [world(receiver)][slots][kFlagStride]   — on the sender
  uint64_t probe = 0;                  // 64 B of flag words for the ε ping-pong of the predecessor
  uint64_t regions = 0;                // [kMaxRegions][world] u64: mapped region bases (local)
  uint64_t eager = 0;                  // [world(sender)][kEagerSlots][kEagerStride]   — on the receiver
  uint64_t eager_free = 0;             // [world(receiver)] u64, 128-B padded: slots returned — on the sender
  uint64_t eager_cnt = 0;              // [world(sender)][kEagerSlots] u32: CTAs done copying out — on the receiver
  uint64_t relay_dec = 0;              // [world(sender)][kBellRing][4] u64: a relay kernel's next-message decisions
  uint64_t relay_exit = 0;             // [world(sender)] u32, 128-B padded: relay CTAs that have left
  uint64_t bell_ack = 0;               // [world(relay)] u64, 128-B padded: doorbells the relay has taken — on the sender
  uint64_t dcnt = 0;                   // [world(dst)][kCtsRing] u64: direct CTAs of message m done — on the sender
  uint64_t dfree = 0;                  // [world(dst)][kCtsRing] u64: last message whose direct CTAs were counted + 1
  uint64_t rcnt = 0;                   // [world(sender)][kBellRing] u64: relay lanes of message m done
                                       //   (bytes << 8 | lanes) — on the relay
  uint64_t rfree = 0;                  // [world(sender)][kBellRing] u64: last relayed message counted + 1
  uint64_t total = 0;
};

// Host ring of one ordered pair (lives in the receiver's shared pinned segment).
struct HostRingPtrs {
  uint8_t *data;                       // [slots][host_stride]
  uint64_t *full;                      // [slots][kFlagStride]
  uint64_t *freef;                     // [slots][kFlagStride]
};

struct SendParams {
  uint32_t me, dst, nblocks, g_direct, npaths, copy_mode, bulk_stages, g_host;
  uint32_t stages, pad_;     // staged pipeline depth (shallow_stages() / deep_stages())
  uint64_t seq, bytes, tag, timeout_ns, align;
  const uint8_t *src;
  uint8_t *my_ctrl;
  uint8_t *dst_ctrl;
  int32_t *err;
  CtrlLayout L;
  uint64_t host_stride;
  uint32_t host_slots;
  uint32_t pdl;          // 1: launched with programmatic stream serialization (PDL)
  struct StagedDesc {
    int32_t kind;            // 1 relay, 2 host
    uint32_t relay;          // relay rank
    uint32_t k;              // chunks
    uint32_t cta0;           // first block of the stage-in group
    uint32_t g;              // CTAs of the stage-in group = lanes of the ring slots
    uint32_t pad_;
    uint64_t off, bytes;     // message byte range of this path
    uint64_t q0;             // ring sequence of chunk 0
    uint64_t m;              // relay: message index on (me, relay) (doorbell entry)
    uint8_t *ring_ctrl;      // relay's control block (relay) — full flags + ring data
    BellEntry *bell;         // relay: the doorbell ring for (me) in the relay's segment (mapped)
  } sp[kMaxPaths];
  uint64_t direct_bytes;
  HostRingPtrs host;         // this pair's host ring (mapped)
};

struct RecvParams {
  uint32_t me, src, nblocks, g_host, copy_mode, bulk_stages;
  uint32_t stages, pad_;     // staged pipeline depth
  uint64_t seq, bytes, tag, region, region_off, done_target, timeout_ns;
  uint8_t *my_ctrl;
  uint8_t *buf;              // the receive buffer (host-ring consumers write here)
  uint8_t *src_ctrl;
  int32_t *err;
  CtrlLayout L;
  uint64_t host_stride;
  uint32_t host_slots;
  uint32_t pdl;          // 1: launched with programmatic stream serialization (PDL)
  HostRingPtrs host;
};

// One relay launch: forward chunks [q0, q0 + k) of `sender`'s ring (its doorbell
// message m0), g lanes (grid = g CTAs, CTA r = lane r); then, while the sender's next
// doorbell arrives within linger_ns with the same g, its message too, and so on; the
// last CTA out records the first message it did not serve and clears `alive`.
struct RelayParams {
  uint32_t me, sender, g, copy_mode;
  uint32_t aligned;            // 1: source and target co-aligned (streamed lanes)
  uint32_t stages;             // staged pipeline depth
  uint64_t q0, k, timeout_ns;
  uint64_t m0;                 // doorbell index of the first message
  uint64_t linger_ns;          // how long CTA 0 waits for the next doorbell (0: one message)
  uint64_t max_msgs;           // > 0 (emu_kernel): serve exactly this many messages; 0: linger rule
  uint64_t *first;             // emu_kernel: device words {tag, q0, k, g} of the first doorbell,
                               // read from host memory by CTA 0 alone and handed to the others
  const BellEntry *bells;      // the sender's doorbell row in this rank's segment (mapped host)
  uint64_t *dec;               // [kBellRing][4] device words: CTA 0's next-message decisions
  uint32_t *exit_cnt;          // device word: CTAs that have left
  uint64_t *state;             // mapped host [2]: first unserved message, alive (host sets 1)
  uint8_t *my_ctrl;
  uint8_t *sender_ctrl;        // the sender's control block (mapped): relay_free flags
  PeerPtrs peer[kMaxPaths];    // ctrl of every rank (self: local): destinations' done counters
  CtrlLayout L;
  int32_t *err;
};

struct EagerParams {
  uint32_t peer;             // receiver (send) / sender (recv)
  uint32_t ctas;             // ⌈bytes / kEagerSlice⌉ (>= 1)
  uint64_t seq;              // eager sequence number of this message on the pair
  uint64_t bytes, tag, timeout_ns;
  const uint8_t *src;        // send: the user buffer
  uint8_t *dst;              // recv: the user buffer
  uint8_t *slot;             // the slot (receiver's control block; mapped on the sender)
  uint64_t *free_ctr;        // eager_free word of the pair (sender's control block)
  uint32_t *cnt;             // recv: eager_cnt word of the slot (receiver-local)
  int32_t *err;
  uint32_t pdl;              // 1: launched with programmatic stream serialization (PDL)
};

// Emulated world (MP_INIT_EMULATED, include/mp.h): every rank is a context of one
// process on one GPU, and mp_send / mp_recv record their kernels' parameter blocks
// instead of launching them.  mp_emu_run then launches ONE cooperative grid whose CTA
// ranges (roles) run those kernels' bodies — the send gate, the send kernel, the
// receive kernel, the eager kernels and, for every (relay rank, sender) pair, the relay
// kernel that rank's service thread would have launched (it reads its doorbells on
// the device instead).  Kernels of different ranks that wait on one another are then
// co-resident by construction (a cooperative launch), never separate launches sharing
// a GPU.
enum EmuKind : uint32_t { EMU_GATE = 0, EMU_SEND, EMU_RECV, EMU_RELAY, EMU_EAGER_SEND, EMU_EAGER_RECV };
struct EmuRole {
  uint32_t kind;             // EmuKind
  uint32_t cta0, n;          // CTA range [cta0, cta0 + n) of the grid
  uint32_t idx;              // index into the parameter array of its kind
};
struct EmuTable {
  const EmuRole *roles;      // device arrays
  const SendParams *send;
  const RecvParams *recv;
  const RelayParams *relay;
  const EagerParams *eager;
  uint32_t nroles, nblocks;
};
// Co-resident CTAs per SM of emu_kernel at 4 and at 6 staged-pipeline stages (its grid
// must not exceed that x SMs).
int emu_capacity(int *per_sm, int *per_sm_deep);
// Cooperative launch of emu_kernel over T.nblocks CTAs (T's arrays in device memory);
// `stages` = shallow_stages() or deep_stages(): the depth of every role's staged pipeline.
int launch_emu(const EmuTable &T, uint32_t stages, void *stream);

int launch_send(const SendParams &P, void *stream);
int launch_eager_send(const EagerParams &P, void *stream);
int launch_eager_recv(const EagerParams &P, void *stream);
int launch_recv(const RecvParams &P, void *stream);
int launch_relay(const RelayParams &P, void *stream);

// Collectives (coll.cpp): dst[i] += src[i] over `bytes` bytes of `dtype` elements
// (MP_DT_* of include/mp.h; bf16 added in fp32 and rounded).  Returns a cudaError_t.
int launch_reduce(int dtype, void *dst, const void *src, uint64_t bytes, void *stream);

// Calibration probes (engine.cu).
// Flag ping-pong between two CTAs through `flags` (2 words, device or mapped host):
// `iters` round trips; the measured time is read with events by the caller.
int launch_pingpong(uint64_t *flags, int iters, uint64_t timeout_ns, int32_t *err, void *stream);
// A one-warp kernel that holds `stream` for `ns` nanoseconds (Step 1 of C27).
int launch_spin(uint64_t ns, void *stream);

// Co-resident CTAs per SM of the kernels with staged CTAs at 4 stages (per_sm) and at
// the deep 6 (per_sm_deep), and the SM count.
int xfer_capacity(int device, int *per_sm, int *per_sm_deep, int *sms);
// The two staged-pipeline depths (engine.cu): `stages` of XferParams / SendParams /
// RecvParams / RelayParams must be one of them.
uint32_t deep_stages();
uint32_t shallow_stages();

// Load every engine kernel now (no lazy loading once persistent kernels run).
int preload_kernels();

}  // namespace mpx
