// ctx.h — the library context behind the opaque mp_ctx (internal).
#pragma once
#include <cuda_runtime.h>

#include <cstdint>
#include <deque>
#include <map>
#include <string>
#include <unordered_map>
#include <vector>

#include "../../include/mp.h"
#include "engine.h"
#include "model.h"

namespace mpx {

// A staging ring (D8): S slots of slot_stride bytes + per-CTA flag words.
struct Ring {
  uint8_t *data = nullptr;     // device memory (relay) or mapped pinned host memory (host)
  uint64_t *full = nullptr;    // [slots][kFlagStride]
  uint64_t *freef = nullptr;   // [slots][kFlagStride]
  bool host = false;
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

struct mp_ctx {
  int rank = 0, world = 1, device = 0, flags = 0;
  bool model_only = true;
  std::string last_error;
  mpx::ModelOpts opts;
  std::map<std::pair<int, int>, mpx::PairModel> models;
  std::unordered_map<mpx::CacheKey, mpx::Selection, mpx::CacheKeyHash> cache;

  // engine
  int n_loop_relays = 6;
  bool host_path = true;
  int slots = 4;
  int relay_ctas = 16;
  uint64_t slot_bytes = 32ull << 20;
  double timeout_s = 20.0;
  int per_sm = 0, sms = 0;
  int32_t *d_err = nullptr;
  std::vector<mpx::Ring> rings;   // loopback: [0..V) relays, [V] host (if enabled)
  mpx::Heap heap;
  std::deque<mpx::PendingSend> pending;
  uint64_t launches = 0;
  uint64_t *d_probe = nullptr;    // calibration flag words (device)
  uint64_t *h_probe = nullptr;    // calibration flag words (mapped host)
};
