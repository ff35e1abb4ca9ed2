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

namespace mpx {

constexpr int kMaxPaths = 16;
constexpr int kFlagStride = 32;    // flag words per slot (max CTAs per staged group)
constexpr int kThreads = 256;      // threads per CTA of every engine kernel
constexpr uint32_t kSlotSlack = 256;  // bytes of slack per slot (co-alignment shift)

enum : int32_t { DK_DIRECT = 0, DK_STAGED = 1 };

// Error codes raised by kernels into the context's device error word.
enum : int32_t { DERR_NONE = 0, DERR_TIMEOUT = 1, DERR_MISMATCH = 2 };

struct DevPath {
  int32_t kind;          // DK_DIRECT / DK_STAGED
  uint32_t g_in;         // direct: CTAs; staged: stage-in CTAs (<= kFlagStride)
  uint32_t g_out;        // staged: forward CTAs (<= kFlagStride)
  uint32_t cta0_in;      // first blockIdx.x of the direct / stage-in group
  uint32_t cta0_out;     // first blockIdx.x of the forward group
  uint32_t k;            // chunks
  uint32_t slots;        // ring slots S
  uint32_t host_ring;    // 1 when ring + flags live in pinned host memory
  uint64_t q0;           // ring sequence number of chunk 0
  uint64_t bytes;        // bytes on this path
  uint64_t align;        // chunk unit A (reading C6)
  uint64_t slot_stride;  // bytes between slots (slot_bytes + kSlotSlack)
  const uint8_t *src;    // source + path offset
  uint8_t *dst;          // destination + path offset (local, peer or mapped)
  uint8_t *ring;         // slot 0
  uint64_t *full;        // [slots][kFlagStride], written by the stage-in group
  uint64_t *freef;       // [slots][kFlagStride], written by the forward group
};

struct XferParams {
  uint32_t npaths;
  uint32_t nblocks;
  uint64_t timeout_ns;
  int32_t *err;          // device (or mapped host) error word
  DevPath p[kMaxPaths];
};

// Launch the fused transfer kernel (engine.cu).  Returns a cudaError_t value.
int launch_xfer(const XferParams &P, void *stream);

// Calibration probes (engine.cu).
// Flag ping-pong between two CTAs through `flags` (2 words, device or mapped host):
// `iters` round trips; the measured time is read with events by the caller.
int launch_pingpong(uint64_t *flags, int iters, uint64_t timeout_ns, int32_t *err, void *stream);

// Max co-resident CTAs of the transfer kernel on this device (occupancy × SMs).
int xfer_capacity(int device, int *per_sm, int *sms);

}  // namespace mpx
