// capi.cpp — the C ABI of include/mp.h: context lifetime, model calls, heap,
// loopback transfer launcher.  PAPER.md §4 (Steps 1-5; Alg 1).
#include <sys/mman.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <limits>
#include <new>
#include <string>

#include "ctx.h"

using namespace mpx;

namespace {

int fail(mp_ctx *c, int code, const std::string &msg) {
  if (c) c->last_error = msg;
  return code;
}

int cuda_fail(mp_ctx *c, cudaError_t e, const char *what) {
  return fail(c, MP_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

#define CK(call)                                        \
  do {                                                  \
    cudaError_t e__ = (call);                           \
    if (e__ != cudaSuccess) return cuda_fail(c, e__, #call); \
  } while (0)

// Default model parameters before calibration (B200-like guesses, not from the
// paper; replaced by mp_calibrate / mp_load_params / mp_set_model).
PathModel default_path(int kind, int via, bool loopback) {
  PathModel p;
  p.kind = kind;
  p.via = via;
  p.c = 1.0;
  if (kind == K_DIRECT) {
    p.alpha = 4e-6;
    p.beta = loopback ? 3.0e12 : 7.5e11;
    p.w = loopback ? 2.0 : 1.0;
  } else if (kind == K_GPU) {
    p.alpha = 4e-6;
    p.beta = loopback ? 3.0e12 : 7.5e11;
    p.alpha2 = 1e-6;
    p.beta2 = loopback ? 3.0e12 : 7.5e11;
    p.eps = 2e-6;
    p.w = loopback ? 4.0 : 1.0;
  } else {
    p.alpha = 5e-6;
    p.beta = 5.0e10;
    p.alpha2 = 2e-6;
    p.beta2 = 5.0e10;
    p.eps = 3e-6;
    p.w = loopback ? 2.0 : 0.0;
  }
  return p;
}

// Reading A1: direct, GPU relays by ascending rank (loopback: ring index), host.
PairModel default_pair(const mp_ctx *c, int src, int dst) {
  PairModel m;
  const bool loop = (src == dst);
  m.paths.push_back(default_path(K_DIRECT, -1, loop));
  if (loop) {
    for (int r = 0; r < c->n_loop_relays; ++r) m.paths.push_back(default_path(K_GPU, r, true));
  } else {
    // a relay r needs peer access src -> r and r -> dst (topology, mp_init)
    for (int r = 0; r < c->world; ++r)
      if (r != src && r != dst &&
          (!c->have_topo || (c->topo.peer_access[src][r] && c->topo.peer_access[r][dst])))
        m.paths.push_back(default_path(K_GPU, r, false));
  }
  if (c->host_path) m.paths.push_back(default_path(K_HOST, -1, loop));
  m.port_alpha = 4e-6;
  m.port_beta = loop ? 6.5e12 : 9.0e11;
  return m;
}

bool pair_ok(const mp_ctx *c, int src, int dst) {
  if (src < 0 || dst < 0 || src >= c->world || dst >= c->world) return false;
  if (src != dst && c->have_topo && !c->topo.peer_access[src][dst]) return false;  // no direct path
  return true;
}

PairModel *pair_model(mp_ctx *c, int src, int dst) {
  auto key = std::make_pair(src, dst);
  auto it = c->models.find(key);
  if (it == c->models.end()) it = c->models.emplace(key, default_pair(c, src, dst)).first;
  return &it->second;
}

// The model of the band holding a message of n bytes (reading C20): the last band
// with n_min <= n, else the base model.
const PairModel *model_for(mp_ctx *c, int src, int dst, uint64_t n) {
  const PairModel *m = pair_model(c, src, dst);
  auto it = c->bands.find(std::make_pair(src, dst));
  if (it == c->bands.end()) return m;
  for (const auto &b : it->second)
    if (b.first <= n) m = &b.second;
  return m;
}

void fill_config(const PairModel &m, const Selection &s, mp_config *out) {
  std::memset(out, 0, sizeof(*out));
  out->npaths = static_cast<int32_t>(m.paths.size());
  for (size_t i = 0; i < m.paths.size(); ++i) {
    out->path[i].kind = m.paths[i].kind;
    out->path[i].via = m.paths[i].via;
    out->theta[i] = s.theta[i];
    out->bytes[i] = s.bytes[i];
    out->chunks[i] = s.chunks[i];
  }
  out->t_pred = s.t_pred;
  out->t_level = s.t_level;
}

// Engine-side validation of a config against the pair's paths (mp_send/mp_xfer).
int check_config(mp_ctx *c, const PairModel &m, uint64_t n, const mp_config *cfg) {
  if (cfg->npaths != static_cast<int32_t>(m.paths.size()))
    return fail(c, MP_ERR_INVALID, "config npaths does not match the pair's paths");
  uint64_t sum = 0;
  for (int i = 0; i < cfg->npaths; ++i) {
    if (cfg->path[i].kind != m.paths[i].kind || cfg->path[i].via != m.paths[i].via)
      return fail(c, MP_ERR_TOPOLOGY, "config path " + std::to_string(i) + " is not available");
    const uint64_t b = cfg->bytes[i];
    sum += b;
    if (i == 0 || b == 0) continue;
    const uint64_t A = c->opts.align, U = b / A, rem = b - U * A;
    const uint64_t k = cfg->chunks[i];
    if (k < 1 || k > std::max<uint64_t>(1, U))
      return fail(c, MP_ERR_INVALID, "chunk count out of range on path " + std::to_string(i));
    const uint64_t max_chunk = A * ((U + k - 1) / k) + rem;
    if (max_chunk > c->slot_bytes)
      return fail(c, MP_ERR_INVALID, "chunk larger than a staging slot on path " + std::to_string(i));
  }
  if (sum != n) return fail(c, MP_ERR_INVALID, "config bytes do not sum to the message size");
  return MP_OK;
}

int check_err(mp_ctx *c) {
  if (!c->d_err) return MP_OK;
  int32_t e = 0;
  CK(cudaMemcpy(&e, c->d_err, sizeof(e), cudaMemcpyDeviceToHost));
  if (e == DERR_TIMEOUT) return fail(c, MP_ERR_TIMEOUT, "a device-side wait timed out");
  if (e == DERR_MISMATCH) return fail(c, MP_ERR_MISMATCH, "send/recv mismatch detected on the device");
  return MP_OK;
}

void free_engine(mp_ctx *c) {
  for (auto &r : c->rings) {
    if (r.host) {
      if (r.data && r.registered) {
        cudaHostUnregister(r.data);
        munmap(r.data, r.data_bytes);
      } else if (r.data) {
        cudaFreeHost(r.data);
      }
      if (r.full) cudaFree(r.full);
    } else {
      if (r.data) cudaFree(r.data);
      if (r.full) cudaFree(r.full);
    }
  }
  c->rings.clear();
  if (c->heap.base) cudaFree(c->heap.base);
  c->heap = Heap();
  if (c->d_err) cudaFree(c->d_err);
  c->d_err = nullptr;
  if (c->d_probe) cudaFree(c->d_probe);
  c->d_probe = nullptr;
  if (c->h_probe) cudaFreeHost(c->h_probe);
  c->h_probe = nullptr;
  for (auto &p : c->pending) cudaEventDestroy(p.ready);
  c->pending.clear();
  if (c->big_ev) cudaEventDestroy(c->big_ev);
  c->big_ev = nullptr;
  c->big_valid = false;
  if (c->ring_ev) cudaEventDestroy(c->ring_ev);
  c->ring_ev = nullptr;
  c->ring_valid = false;
}

int alloc_ring(mp_ctx *c, bool host, Ring *r) {
  const uint64_t stride = c->slot_bytes + kSlotSlack;
  const uint64_t data_bytes = stride * static_cast<uint64_t>(c->slots);
  const uint64_t flag_bytes = 2ull * c->slots * kFlagStride * sizeof(uint64_t);
  r->host = host;
  if (host) {
    // data in pinned host memory (the PCIe leg); the flags in device memory, so that
    // polling never crosses PCIe (measured: host-resident flags polled by 16-32 CTAs
    // cut the host path to 9-22 GB/s, profiles/r01/diag_host.jsonl)
    void *d = nullptr, *f = nullptr;
    const char *reg = std::getenv("MPX_HOSTRING_REGISTER");  // diagnostics: shm-like pages
    if (reg && reg[0] == '1') {
      d = mmap(nullptr, data_bytes, PROT_READ | PROT_WRITE, MAP_SHARED | MAP_ANONYMOUS, -1, 0);
      if (d == MAP_FAILED) return fail(c, MP_ERR_NOMEM, "mmap host ring");
      CK(cudaHostRegister(d, data_bytes, cudaHostRegisterMapped | cudaHostRegisterPortable));
      r->registered = true;
    } else {
      CK(cudaHostAlloc(&d, data_bytes, cudaHostAllocMapped | cudaHostAllocPortable));
    }
    r->data_bytes = data_bytes;
    r->data = static_cast<uint8_t *>(d);
    CK(cudaMalloc(&f, flag_bytes));
    CK(cudaMemset(f, 0, flag_bytes));
    r->full = static_cast<uint64_t *>(f);
  } else {
    void *d = nullptr, *f = nullptr;
    CK(cudaMalloc(&d, data_bytes));
    r->data = static_cast<uint8_t *>(d);
    CK(cudaMalloc(&f, flag_bytes));
    CK(cudaMemset(f, 0, flag_bytes));
    r->full = static_cast<uint64_t *>(f);
  }
  r->freef = r->full + static_cast<uint64_t>(c->slots) * kFlagStride;
  r->q = 0;
  return MP_OK;
}

int init_engine(mp_ctx *c) {
  CK(cudaSetDevice(c->device));
  if (int e = xfer_capacity(c->device, &c->per_sm, &c->per_sm_deep, &c->sms))
    return cuda_fail(c, static_cast<cudaError_t>(e), "occupancy query");
  if (const char *m = std::getenv("MPX_STAGES"))  // design experiments: one staged depth for every launch
    c->force_stages = std::strcmp(m, "4") == 0 ? shallow_stages() : (std::strcmp(m, "6") == 0 ? deep_stages() : 0u);
  if (int e = preload_kernels()) return cuda_fail(c, static_cast<cudaError_t>(e), "kernel preload");
  if (const char *m = std::getenv("MPX_COPY")) c->copy_mode = std::strcmp(m, "reg") == 0 ? 0u : 1u;
  if (const char *m = std::getenv("MPX_PDL")) c->pdl = std::strcmp(m, "0") == 0 ? 0u : 1u;
  // multi-rank PDL is opt-in: with both ranks on one GPU under MPS it cost 10-18 % on
  // direct messages of 1-16 MiB (profiles/r01/world_pdl); unmeasured across GPUs
  if (const char *m = std::getenv("MPX_PDL_WORLD")) c->pdl_world = std::strcmp(m, "1") == 0 ? 1u : 0u;
  void *p = nullptr;
  CK(cudaMalloc(&p, sizeof(int32_t)));
  c->d_err = static_cast<int32_t *>(p);
  CK(cudaMemset(c->d_err, 0, sizeof(int32_t)));
  CK(cudaMalloc(&p, 64));
  c->d_probe = static_cast<uint64_t *>(p);
  CK(cudaHostAlloc(&p, 64, cudaHostAllocMapped | cudaHostAllocPortable));
  c->h_probe = static_cast<uint64_t *>(p);
  if (c->heap.size) {
    void *h = nullptr;
    cudaError_t e = cudaMalloc(&h, c->heap.size);
    if (e != cudaSuccess) return fail(c, MP_ERR_NOMEM, "heap allocation failed");
    c->heap.reset(static_cast<uint8_t *>(h), c->heap.size);
  }
  if (c->world == 1) {  // topology of the loopback job: this GPU alone
    std::vector<mp_gpu_info> g(1);
    if (int s = topo_local(c, &g[0])) return s;
    if (int s = topo_discover(c, g, std::vector<int>(1, 1))) return s;
    c->rings.resize(c->n_loop_relays + (c->host_path ? 1 : 0));
    for (int r = 0; r < c->n_loop_relays; ++r)
      if (int s = alloc_ring(c, false, &c->rings[r])) return s;
    if (c->host_path)
      if (int s = alloc_ring(c, true, &c->rings[c->n_loop_relays])) return s;
  }
  return MP_OK;
}

// Builds the fused launch of one loopback message (A7-A9) and enqueues it.
int launch_loopback(mp_ctx *c, void *dst, const void *src, uint64_t n, const mp_config &cfg,
                    void *stream) {
  XferParams P;
  std::memset(&P, 0, sizeof(P));
  P.timeout_ns = static_cast<uint64_t>(c->timeout_s * 1e9);
  P.err = c->d_err;
  P.copy_mode = c->copy_mode;
  P.pdl = c->pdl;
  P.bulk_stages = bulk_stages_for(cfg.bytes[0]);
  P.allow_small = 1;
  uint32_t staged_ctas = 0;
  for (int i = 1; i < cfg.npaths; ++i)
    if (cfg.bytes[i]) staged_ctas += 2u * static_cast<uint32_t>(c->relay_ctas);
  P.stages = stages_for(c, staged_ctas);
  const int cap = std::max(1, per_sm_at(c, P.stages) * c->sms);
  // direct group sized by direct_ctas(), leaving room for every staged group to be
  // co-resident.
  uint32_t g_direct = direct_ctas(c, cfg.bytes[0], cap - static_cast<int>(staged_ctas), c->pdl != 0);
  // beside staged groups, a whole number of CTAs per SM (an uneven grid lands unevenly
  // on the SMs a PDL predecessor still holds)
  if (staged_ctas && g_direct > static_cast<uint32_t>(c->sms))
    g_direct = g_direct / static_cast<uint32_t>(c->sms) * static_cast<uint32_t>(c->sms);
  // Two large copies running at once (osu_bibw's two directions on two streams) do
  // best with one TMA pipeline per SM each — 64 KiB in flight per SM in total, as one
  // copy with two (profiles/r01/bibw.jsonl).  A large direct-only launch that finds
  // the previous one, from another stream, still running takes one CTA per SM.
  cudaStreamCaptureStatus capst = cudaStreamCaptureStatusNone;
  const bool big = staged_ctas == 0 && cfg.bytes[0] >= (16ull << 20) &&
                   cudaStreamIsCapturing(static_cast<cudaStream_t>(stream), &capst) == cudaSuccess &&
                   capst == cudaStreamCaptureStatusNone;  // (not inside a CUDA-graph capture)
  if (big && c->big_valid && c->big_stream != static_cast<cudaStream_t>(stream) &&
      cudaEventQuery(c->big_ev) == cudaErrorNotReady)
    g_direct = std::min<uint32_t>(g_direct, static_cast<uint32_t>(c->sms));
  uint32_t next = 0;
  uint64_t off = 0;
  P.npaths = static_cast<uint32_t>(cfg.npaths);
  for (int i = 0; i < cfg.npaths; ++i) {
    DevPath &d = P.p[i];
    const uint64_t b = cfg.bytes[i];
    d.bytes = b;
    d.src = static_cast<const uint8_t *>(src) + off;
    d.dst = static_cast<uint8_t *>(dst) + off;
    d.align = c->opts.align;
    off += b;
    if (b == 0) continue;
    if (i == 0) {
      d.kind = DK_DIRECT;
      d.g_in = g_direct;
      d.cta0_in = next;
      next += g_direct;
      continue;
    }
    const int ring_idx = cfg.path[i].kind == MP_PATH_HOST ? c->n_loop_relays : cfg.path[i].via;
    Ring &r = c->rings[ring_idx];
    d.kind = DK_STAGED;
    d.k = cfg.chunks[i];
    d.slots = static_cast<uint32_t>(c->slots);
    d.host_ring = r.host ? 1u : 0u;
    d.q0 = r.q;
    d.slot_stride = c->slot_bytes + kSlotSlack;
    d.lane = lane_stride(c->slot_bytes, static_cast<uint32_t>(c->relay_ctas));
    d.ring = r.data;
    d.full = r.full;
    d.freef = r.freef;
    d.g_out = static_cast<uint32_t>(c->relay_ctas);
    d.g_in = static_cast<uint32_t>(c->relay_ctas);
    d.cta0_out = next;  // consumers before producers (deadlock-free dispatch order)
    next += d.g_out;
    d.cta0_in = next;
    next += d.g_in;
    r.q += d.k;
  }
  P.nblocks = next;
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  if (staged_ctas && c->ring_valid && c->ring_stream != st) CK(cudaStreamWaitEvent(st, c->ring_ev, 0));
  const int e = launch_xfer(P, stream);
  if (e != cudaSuccess) return cuda_fail(c, static_cast<cudaError_t>(e), "xfer launch");
  c->launches += 1;
  if (staged_ctas) {
    if (!c->ring_ev) CK(cudaEventCreateWithFlags(&c->ring_ev, cudaEventDisableTiming));
    CK(cudaEventRecord(c->ring_ev, st));
    c->ring_stream = st;
    c->ring_valid = true;
  }
  if (big) {
    if (!c->big_ev) CK(cudaEventCreateWithFlags(&c->big_ev, cudaEventDisableTiming));
    CK(cudaEventRecord(c->big_ev, static_cast<cudaStream_t>(stream)));
    c->big_stream = static_cast<cudaStream_t>(stream);
    c->big_valid = true;
  }
  return MP_OK;
}

}  // namespace

int mpx::launch_direct_copy(mp_ctx *c, void *dst, const void *src, uint64_t n, void *stream, int ctas) {
  XferParams P;
  std::memset(&P, 0, sizeof(P));
  P.timeout_ns = static_cast<uint64_t>(c->timeout_s * 1e9);
  P.err = c->d_err;
  P.copy_mode = c->copy_mode;
  P.pdl = c->pdl;
  P.bulk_stages = bulk_stages_for(n);
  P.allow_small = ctas > 0 ? 0u : 1u;  // a staged leg's calibration times its group's CTAs
  P.staged_blk = ctas > 0 ? 1u : 0u;  // staged lanes move 16 KiB TMA blocks in every engine
  // a staged leg is timed at the depth a staged path alone runs at (one group of CTAs)
  P.stages = ctas > 0 ? stages_for(c, 2u * static_cast<uint32_t>(ctas)) : shallow_stages();
  P.npaths = 1;
  DevPath &d = P.p[0];
  d.kind = DK_DIRECT;
  d.bytes = n;
  d.src = static_cast<const uint8_t *>(src);
  d.dst = static_cast<uint8_t *>(dst);
  d.align = c->opts.align;
  d.g_in = ctas > 0 ? static_cast<uint32_t>(ctas) : direct_ctas(c, n, c->per_sm * c->sms, c->pdl != 0);
  P.nblocks = d.g_in;
  const int e = launch_xfer(P, stream);
  if (e != cudaSuccess) return cuda_fail(c, static_cast<cudaError_t>(e), "copy launch");
  c->launches += 1;
  return MP_OK;
}

// ------------------------------------------------------------------ Heap

void mpx::Heap::reset(uint8_t *b, uint64_t n) {
  base = b;
  size = n;
  free_.clear();
  used_.clear();
  if (n) free_[0] = n;
}

void *mpx::Heap::alloc(uint64_t n) {
  n = (std::max<uint64_t>(n, 1) + 255) & ~uint64_t(255);
  for (auto it = free_.begin(); it != free_.end(); ++it) {
    if (it->second < n) continue;
    const uint64_t off = it->first, len = it->second;
    free_.erase(it);
    if (len > n) free_[off + n] = len - n;
    used_[off] = n;
    return base + off;
  }
  return nullptr;
}

bool mpx::Heap::release(void *p) {
  if (!base) return false;
  const uint64_t off = static_cast<uint64_t>(static_cast<uint8_t *>(p) - base);
  auto it = used_.find(off);
  if (it == used_.end()) return false;
  uint64_t o = off, len = it->second;
  used_.erase(it);
  auto nx = free_.lower_bound(o);
  if (nx != free_.end() && nx->first == o + len) {
    len += nx->second;
    free_.erase(nx);
  }
  auto pv = free_.lower_bound(o);
  if (pv != free_.begin()) {
    --pv;
    if (pv->first + pv->second == o) {
      o = pv->first;
      len += pv->second;
      free_.erase(pv);
    }
  }
  free_[o] = len;
  return true;
}

// ------------------------------------------------------------------ ABI

extern "C" {

int mp_abi_version(void) { return MP_ABI_VERSION; }

const char *mp_strerror(int s) {
  switch (s) {
    case MP_OK: return "MP_OK";
    case MP_ERR_INVALID: return "MP_ERR_INVALID";
    case MP_ERR_CUDA: return "MP_ERR_CUDA";
    case MP_ERR_TOPOLOGY: return "MP_ERR_TOPOLOGY";
    case MP_ERR_NOMEM: return "MP_ERR_NOMEM";
    case MP_ERR_STATE: return "MP_ERR_STATE";
    case MP_ERR_UNSUPPORTED: return "MP_ERR_UNSUPPORTED";
    case MP_ERR_TIMEOUT: return "MP_ERR_TIMEOUT";
    case MP_ERR_MISMATCH: return "MP_ERR_MISMATCH";
    default: return "MP_ERR_UNKNOWN";
  }
}

const char *mp_last_error(mp_ctx *c) { return c ? c->last_error.c_str() : "null context"; }

int mp_init(mp_ctx **out, const mp_init_args *a) {
  if (!out || !a) return MP_ERR_INVALID;
  *out = nullptr;
  if (a->world < 1 || a->rank < 0 || a->rank >= a->world) return MP_ERR_INVALID;
  mp_ctx *c = new (std::nothrow) mp_ctx();
  if (!c) return MP_ERR_NOMEM;
  c->rank = a->rank;
  c->world = a->world;
  c->device = a->device;
  c->flags = a->flags;
  c->model_only = (a->flags & MP_INIT_MODEL_ONLY) != 0;
  c->emulated = (a->flags & MP_INIT_EMULATED) != 0;
  if (c->emulated && (!mpx::emu_thread() || a->world < 2 || c->model_only)) {  // only through mp_init_emulated
    delete c;
    return MP_ERR_INVALID;
  }
  c->n_loop_relays = a->n_loop_relays < 0 ? 6 : std::min(a->n_loop_relays, MP_MAX_PATHS - 2);
  c->host_path = a->host_path < 0 ? true : a->host_path != 0;
  c->slots = a->slots > 0 ? a->slots : 4;
  c->relay_ctas = a->relay_ctas > 0 ? std::min(a->relay_ctas, kFlagStride) : 16;
  c->slot_bytes = a->slot_bytes ? ((a->slot_bytes + 255) & ~uint64_t(255)) : (32ull << 20);
  c->timeout_s = a->timeout_s > 0 ? a->timeout_s : 20.0;
  c->heap.size = a->heap_bytes ? a->heap_bytes : (2304ull << 20);
  c->opts.slot_bytes = c->slot_bytes > 2 * c->opts.align ? c->slot_bytes - 2 * c->opts.align : 0;
  if (c->world > MP_MAX_PATHS) {
    delete c;
    return MP_ERR_INVALID;
  }
  if (const char *ps = std::getenv("MPX_PATHS")) {  // e.g. "direct,host"
    const std::string s(ps);
    c->env_kinds = 1u << MP_PATH_DIRECT;
    if (s.find("gpu") != std::string::npos || s.find("relay") != std::string::npos) c->env_kinds |= 1u << MP_PATH_GPU;
    if (s.find("host") != std::string::npos) c->env_kinds |= 1u << MP_PATH_HOST;
    if (s.empty() || s == "all") c->env_kinds = 0x7u;
  }
  c->allgather = a->allgather;
  c->allgather_user = a->allgather_user;
  if (!c->model_only) {
    int s = init_engine(c);
    if (!s && c->world > 1) s = world_init(c);
    if (s) {
      std::string msg = c->last_error;
      if (c->world > 1) world_finalize(c);
      free_engine(c);
      delete c;
      std::fprintf(stderr, "mp_init: %s\n", msg.c_str());
      return s;
    }
  }
  if (a->param_file && a->param_file[0]) {
    FILE *f = std::fopen(a->param_file, "r");
    if (f) {
      std::fclose(f);
      if (int s = mp_load_params(c, a->param_file)) {
        mp_finalize(c);
        return s;
      }
    }
  }
  if (!c->model_only && !(a->flags & MP_INIT_NO_CALIBRATE)) {
    if (int s = mp_calibrate(c, nullptr, 0, 0)) {
      std::fprintf(stderr, "mp_init: calibration failed: %s\n", c->last_error.c_str());
      mp_finalize(c);
      return s;
    }
  }
  if (!c->model_only && c->world > 1) {
    if (int s = world_start_relay(c)) {
      std::fprintf(stderr, "mp_init: %s\n", c->last_error.c_str());
      mp_finalize(c);
      return s;
    }
    // reading C28: the relays' start time, once their service runs
    if (c->world >= 3 && !(a->flags & MP_INIT_NO_CALIBRATE) && c->relay_svc) {
      if (int s = mp_calibrate_wake(c, 0, 0)) {
        std::fprintf(stderr, "mp_init: wake calibration failed: %s\n", c->last_error.c_str());
        mp_finalize(c);
        return s;
      }
    }
  }
  *out = c;
  return MP_OK;
}

int mp_finalize(mp_ctx *c) {
  if (!c) return MP_OK;
  if (c->emulated && c->emu_world) return MP_ERR_STATE;  // mp_finalize_emulated tears the world down
  if (!c->model_only) {
    cudaSetDevice(c->device);
    coll_release(c);
    if (c->world > 1) world_finalize(c);  // stops the persistent relay kernel first
    cudaDeviceSynchronize();
    free_engine(c);
  }
  delete c;
  return MP_OK;
}

int mp_init_emulated(mp_ctx **ctxs, const mp_init_args *args) {
  if (!ctxs || !args || args->world < 2 || args->world > MP_MAX_PATHS) return MP_ERR_INVALID;
  if (args->flags & MP_INIT_MODEL_ONLY) return MP_ERR_INVALID;
  for (int r = 0; r < args->world; ++r) ctxs[r] = nullptr;
  return mpx::emu_init_world(ctxs, args);
}

int mp_finalize_emulated(mp_ctx **ctxs, int n) {
  if (!ctxs || n < 2 || !ctxs[0] || !ctxs[0]->emulated) return MP_ERR_INVALID;
  return mpx::emu_finalize_world(ctxs, n);
}

int mp_emu_register(mp_ctx **ctxs, int n, void *const *bufs, const uint64_t *bytes, int *ids) {
  if (!ctxs || n < 2 || !ctxs[0] || !bufs || !bytes || !ids || !ctxs[0]->emulated) return MP_ERR_INVALID;
  return mpx::emu_each_rank(ctxs, n, [&](int r) { return mp_register(ctxs[r], bufs[r], bytes[r], &ids[r]); });
}

int mp_emu_deregister(mp_ctx **ctxs, int n, const int *ids) {
  if (!ctxs || n < 2 || !ctxs[0] || !ids || !ctxs[0]->emulated) return MP_ERR_INVALID;
  return mpx::emu_each_rank(ctxs, n, [&](int r) { return mp_deregister(ctxs[r], ids[r]); });
}

int mp_emu_run(mp_ctx **ctxs, int n, void *stream, double *kernel_s) {
  if (!ctxs || n < 2 || !ctxs[0]) return MP_ERR_INVALID;
  if (!ctxs[0]->emulated) return fail(ctxs[0], MP_ERR_STATE, "mp_emu_run: not an emulated world");
  return mpx::emu_run(ctxs, n, stream, kernel_s);
}

int mp_paths(mp_ctx *c, int src, int dst, mp_path *out, int *npaths) {
  if (!c || !out || !npaths) return fail(c, MP_ERR_INVALID, "null argument");
  if (!pair_ok(c, src, dst)) return fail(c, MP_ERR_TOPOLOGY, "no such pair");
  const PairModel *m = pair_model(c, src, dst);
  for (size_t i = 0; i < m->paths.size(); ++i) {
    out[i].kind = m->paths[i].kind;
    out[i].via = m->paths[i].via;
  }
  *npaths = static_cast<int>(m->paths.size());
  return MP_OK;
}

int mp_set_model(mp_ctx *c, int src, int dst, const mp_path *paths, const mp_path_params *prm,
                 int npaths, const mp_port_params *port) {
  if (!c || !paths || !prm) return fail(c, MP_ERR_INVALID, "null argument");
  if (!pair_ok(c, src, dst)) return fail(c, MP_ERR_TOPOLOGY, "no such pair");
  if (npaths < 1 || npaths > MP_MAX_PATHS) return fail(c, MP_ERR_INVALID, "npaths out of range");
  PairModel m;
  for (int i = 0; i < npaths; ++i) {
    PathModel p;
    p.kind = paths[i].kind;
    p.via = paths[i].via;
    p.alpha = prm[i].alpha;
    p.beta = prm[i].beta;
    p.alpha2 = prm[i].alpha2;
    p.beta2 = prm[i].beta2;
    p.eps = prm[i].eps;
    p.c = prm[i].c;
    p.sigma = prm[i].sigma;
    p.w = prm[i].w;
    p.wake = prm[i].wake;
    m.paths.push_back(p);
  }
  if (port) {
    m.port_alpha = port->alpha;
    m.port_beta = port->beta;
  }
  const std::string why = validate_model(m);
  if (!why.empty()) return fail(c, MP_ERR_INVALID, why);
  if (!c->model_only && src == dst) {  // loopback paths must map onto existing rings
    for (const PathModel &p : m.paths) {
      if (p.kind == K_GPU && (p.via < 0 || p.via >= c->n_loop_relays))
        return fail(c, MP_ERR_TOPOLOGY, "loopback relay ring does not exist");
      if (p.kind == K_HOST && !c->host_path) return fail(c, MP_ERR_TOPOLOGY, "host path disabled");
    }
  }
  c->models[std::make_pair(src, dst)] = m;
  c->bands.erase(std::make_pair(src, dst));  // a new base model drops the pair's bands
  auto wt = c->windows.find(std::make_pair(src, dst));  // … and window params of another path list
  if (wt != c->windows.end() && wt->second.h.size() != m.paths.size()) c->windows.erase(wt);
  c->cache.clear();
  return MP_OK;
}

int mp_set_model_band(mp_ctx *c, int src, int dst, uint64_t n_min, const mp_path_params *prm, int npaths,
                      const mp_port_params *port) {
  if (!c || !prm) return fail(c, MP_ERR_INVALID, "null argument");
  if (!pair_ok(c, src, dst)) return fail(c, MP_ERR_TOPOLOGY, "no such pair");
  if (n_min == 0) return fail(c, MP_ERR_INVALID, "band n_min must be > 0 (band 0 is mp_set_model)");
  const PairModel *base = pair_model(c, src, dst);
  if (npaths != static_cast<int>(base->paths.size()))
    return fail(c, MP_ERR_INVALID, "band path count must equal the pair's");
  PairModel m = *base;
  for (int i = 0; i < npaths; ++i) {
    PathModel &p = m.paths[i];
    p.alpha = prm[i].alpha;
    p.beta = prm[i].beta;
    p.alpha2 = prm[i].alpha2;
    p.beta2 = prm[i].beta2;
    p.eps = prm[i].eps;
    p.c = prm[i].c;
    p.sigma = prm[i].sigma;
    p.w = prm[i].w;
    p.wake = prm[i].wake;
  }
  m.port_alpha = port ? port->alpha : 0.0;
  m.port_beta = port ? port->beta : 0.0;
  const std::string why = validate_model(m);
  if (!why.empty()) return fail(c, MP_ERR_INVALID, why);
  auto &v = c->bands[std::make_pair(src, dst)];
  auto it = std::find_if(v.begin(), v.end(),
                         [&](const std::pair<uint64_t, PairModel> &b) { return b.first >= n_min; });
  if (it != v.end() && it->first == n_min)
    it->second = m;
  else
    v.insert(it, std::make_pair(n_min, m));
  c->cache.clear();
  return MP_OK;
}

int mp_get_model_band(mp_ctx *c, int src, int dst, int band, uint64_t *n_min, mp_path_params *prm,
                      int *npaths, mp_port_params *port, int *nbands) {
  if (!c) return MP_ERR_INVALID;
  if (!pair_ok(c, src, dst)) return fail(c, MP_ERR_TOPOLOGY, "no such pair");
  const PairModel *m = pair_model(c, src, dst);
  auto it = c->bands.find(std::make_pair(src, dst));
  const int nb = 1 + (it == c->bands.end() ? 0 : static_cast<int>(it->second.size()));
  if (nbands) *nbands = nb;
  if (band < 0) return MP_OK;  // count only
  if (band >= nb) return fail(c, MP_ERR_INVALID, "no such band");
  uint64_t lo = 0;
  if (band > 0) {
    lo = it->second[band - 1].first;
    m = &it->second[band - 1].second;
  }
  if (n_min) *n_min = lo;
  if (npaths) *npaths = static_cast<int>(m->paths.size());
  if (prm)
    for (size_t i = 0; i < m->paths.size(); ++i) {
      const PathModel &p = m->paths[i];
      prm[i] = mp_path_params{p.alpha, p.beta, p.alpha2, p.beta2, p.eps, p.c, p.sigma, p.w, p.wake};
    }
  if (port) {
    port->alpha = m->port_alpha;
    port->beta = m->port_beta;
  }
  return MP_OK;
}

int mp_get_model(mp_ctx *c, int src, int dst, mp_path *paths, mp_path_params *prm, int *npaths,
                 mp_port_params *port) {
  if (!c || !npaths) return fail(c, MP_ERR_INVALID, "null argument");
  if (!pair_ok(c, src, dst)) return fail(c, MP_ERR_TOPOLOGY, "no such pair");
  const PairModel *m = pair_model(c, src, dst);
  *npaths = static_cast<int>(m->paths.size());
  for (size_t i = 0; i < m->paths.size(); ++i) {
    const PathModel &p = m->paths[i];
    if (paths) {
      paths[i].kind = p.kind;
      paths[i].via = p.via;
    }
    if (prm) prm[i] = mp_path_params{p.alpha, p.beta, p.alpha2, p.beta2, p.eps, p.c, p.sigma, p.w, p.wake};
  }
  if (port) {
    port->alpha = m->port_alpha;
    port->beta = m->port_beta;
  }
  return MP_OK;
}

int mp_set_options(mp_ctx *c, const mp_model_opts *o) {
  if (!c || !o) return fail(c, MP_ERR_INVALID, "null argument");
  if (o->mode != MP_MODEL_PAPER && o->mode != MP_MODEL_B200) return fail(c, MP_ERR_INVALID, "bad mode");
  if (o->align < 1 || o->k_max < 1) return fail(c, MP_ERR_INVALID, "align and k_max must be >= 1");
  ModelOpts m;
  m.mode = o->mode;
  m.stagger = o->stagger ? 1 : 0;
  m.refine = o->refine < 0 ? -1 : (o->refine ? 1 : 0);
  m.align = o->align;
  m.c_min = o->c_min;
  m.k_max = o->k_max;
  m.slot_bytes = o->slot_bytes;
  if (o->window < 0) return fail(c, MP_ERR_INVALID, "window must be >= 0");
  m.window = o->window > 1 ? static_cast<uint32_t>(o->window) : 1u;
  if (!c->model_only) {  // chunks must fit the engine's staging slots
    const uint64_t lim = c->slot_bytes > 2 * m.align ? c->slot_bytes - 2 * m.align : 1;
    if (m.slot_bytes == 0 || m.slot_bytes > lim) m.slot_bytes = lim;
  }
  c->opts = m;
  c->cache.clear();
  return MP_OK;
}

int mp_get_options(mp_ctx *c, mp_model_opts *o) {
  if (!c || !o) return fail(c, MP_ERR_INVALID, "null argument");
  std::memset(o, 0, sizeof(*o));
  o->mode = c->opts.mode;
  o->stagger = c->opts.stagger;
  o->refine = c->opts.refine;
  o->align = c->opts.align;
  o->c_min = c->opts.c_min;
  o->k_max = c->opts.k_max;
  o->slot_bytes = c->opts.slot_bytes;
  o->window = static_cast<int32_t>(c->opts.window);
  return MP_OK;
}

int mp_predict(mp_ctx *c, int src, int dst, uint64_t bytes, const mp_config *cfg, double *seconds) {
  if (!c || !cfg || !seconds) return fail(c, MP_ERR_INVALID, "null argument");
  if (!pair_ok(c, src, dst)) return fail(c, MP_ERR_TOPOLOGY, "no such pair");
  const PairModel *m = model_for(c, src, dst, bytes);
  if (cfg->npaths != static_cast<int32_t>(m->paths.size()))
    return fail(c, MP_ERR_INVALID, "config npaths does not match the pair's paths");
  uint64_t sum = 0;
  for (int i = 0; i < cfg->npaths; ++i) {
    sum += cfg->bytes[i];
    if (i > 0 && cfg->bytes[i] && cfg->chunks[i] < 1)
      return fail(c, MP_ERR_INVALID, "staged path with bytes needs chunks >= 1");
  }
  if (sum != bytes) return fail(c, MP_ERR_INVALID, "config bytes do not sum to the message size");
  *seconds = predict(*m, bytes, cfg->bytes, cfg->chunks, c->opts);
  return MP_OK;
}

// The pair's window model with the context's host submission time (reading C27).
static WindowModel window_of_pair(mp_ctx *c, int src, int dst) {
  auto it = c->windows.find(std::make_pair(src, dst));
  WindowModel w = it == c->windows.end() ? WindowModel() : it->second;
  w.submit = c->submit;
  return w;
}

int mp_select(mp_ctx *c, int src, int dst, uint64_t bytes, uint32_t mask, mp_config *out) {
  if (!c || !out) return fail(c, MP_ERR_INVALID, "null argument");
  if (!pair_ok(c, src, dst)) return fail(c, MP_ERR_TOPOLOGY, "no such pair");
  const PairModel *m = model_for(c, src, dst, bytes);
  // environment variables include/exclude path kinds (MPX_PATHS).
  if (c->env_kinds != 0x7u) {
    uint32_t eff = 0;
    for (size_t i = 0; i < m->paths.size(); ++i) {
      const bool asked = mask == 0 || ((mask >> i) & 1u);
      if (i == 0 || (asked && ((c->env_kinds >> m->paths[i].kind) & 1u))) eff |= 1u << i;
    }
    mask = eff;
  }
  const CacheKey key{src, dst, mask, bytes};
  auto it = c->cache.find(key);  // Alg 1 lines 4-6 (C10)
  if (it == c->cache.end()) {
    Selection s;
    if (c->opts.window > 1)  // NEXT f2: window-aware auto-selection (C24)
      select_window(*m, window_of_pair(c, src, dst), bytes, c->opts.window, mask, c->opts, &s);
    else
      select(*m, bytes, mask, c->opts, &s);
    it = c->cache.emplace(key, std::move(s)).first;  // Alg 1 line 29
  }
  fill_config(*m, it->second, out);
  return MP_OK;
}

int mp_select_flows(mp_ctx *c, int nflows, const mp_flow *flows, mp_config *out) {
  if (!c || (nflows > 0 && (!flows || !out)) || nflows < 0) return fail(c, MP_ERR_INVALID, "bad arguments");
  std::vector<const PairModel *> models;
  std::vector<FlowSpec> specs;
  for (int f = 0; f < nflows; ++f) {
    if (!pair_ok(c, flows[f].src, flows[f].dst)) return fail(c, MP_ERR_TOPOLOGY, "no such pair");
    models.push_back(model_for(c, flows[f].src, flows[f].dst, flows[f].bytes));
    FlowSpec s;
    s.src = flows[f].src;
    s.dst = flows[f].dst;
    s.bytes = flows[f].bytes;
    s.mask = flows[f].path_mask;
    specs.push_back(s);
  }
  std::vector<WindowModel> wcopy;
  for (int f = 0; f < nflows; ++f) wcopy.push_back(window_of_pair(c, flows[f].src, flows[f].dst));
  std::vector<const WindowModel *> wms;
  for (int f = 0; f < nflows; ++f) wms.push_back(&wcopy[f]);
  std::vector<Selection> sel;
  select_flows(models, specs, c->opts, &sel, &c->kappa, &wms);
  for (int f = 0; f < nflows; ++f) fill_config(*models[f], sel[f], &out[f]);
  return MP_OK;
}

// ------------------------------------------------------------------ NEXT f2 (C24, C25)

int mp_set_window_model(mp_ctx *c, int src, int dst, const double *h, int npaths, double tau) {
  if (!c || (npaths > 0 && !h)) return fail(c, MP_ERR_INVALID, "null argument");
  if (!pair_ok(c, src, dst)) return fail(c, MP_ERR_TOPOLOGY, "no such pair");
  const PairModel *m = pair_model(c, src, dst);
  if (npaths != static_cast<int>(m->paths.size()))
    return fail(c, MP_ERR_INVALID, "window npaths must equal the pair's path count");
  if (!(tau >= 0.0) || !std::isfinite(tau)) return fail(c, MP_ERR_INVALID, "tau must be finite and >= 0");
  WindowModel w;
  for (int i = 0; i < npaths; ++i) {
    if (!(h[i] >= 0.0) || !std::isfinite(h[i])) return fail(c, MP_ERR_INVALID, "h must be finite and >= 0");
    w.h.push_back(h[i]);
  }
  w.tau = tau;
  c->windows[std::make_pair(src, dst)] = w;
  c->cache.clear();  // mp_select depends on it when opts.window > 1
  return MP_OK;
}

int mp_get_window_model(mp_ctx *c, int src, int dst, double *h, int *npaths, double *tau) {
  if (!c) return MP_ERR_INVALID;
  if (!pair_ok(c, src, dst)) return fail(c, MP_ERR_TOPOLOGY, "no such pair");
  const PairModel *m = pair_model(c, src, dst);
  auto it = c->windows.find(std::make_pair(src, dst));
  if (npaths) *npaths = static_cast<int>(m->paths.size());
  if (h)
    for (size_t i = 0; i < m->paths.size(); ++i)
      h[i] = (it != c->windows.end() && i < it->second.h.size()) ? it->second.h[i] : 0.0;
  if (tau) *tau = it != c->windows.end() ? it->second.tau : 0.0;
  return MP_OK;
}

int mp_predict_window(mp_ctx *c, int src, int dst, uint64_t bytes, uint32_t window, const mp_config *cfg,
                      double *seconds) {
  if (!c || !cfg || !seconds) return fail(c, MP_ERR_INVALID, "null argument");
  if (window < 1) return fail(c, MP_ERR_INVALID, "window must be >= 1");
  double t1 = 0.0;
  if (int s = mp_predict(c, src, dst, bytes, cfg, &t1)) return s;  // validates the config
  *seconds = predict_window(*model_for(c, src, dst, bytes), window_of_pair(c, src, dst), bytes, window,
                            cfg->bytes, cfg->chunks, c->opts);
  return MP_OK;
}

int mp_select_window(mp_ctx *c, int src, int dst, uint64_t bytes, uint32_t window, uint32_t mask,
                     mp_config *out) {
  if (!c || !out) return fail(c, MP_ERR_INVALID, "null argument");
  if (window < 1) return fail(c, MP_ERR_INVALID, "window must be >= 1");
  if (!pair_ok(c, src, dst)) return fail(c, MP_ERR_TOPOLOGY, "no such pair");
  const PairModel *m = model_for(c, src, dst, bytes);
  if (c->env_kinds != 0x7u) {  // MPX_PATHS, as in mp_select
    uint32_t eff = 0;
    for (size_t i = 0; i < m->paths.size(); ++i) {
      const bool asked = mask == 0 || ((mask >> i) & 1u);
      if (i == 0 || (asked && ((c->env_kinds >> m->paths[i].kind) & 1u))) eff |= 1u << i;
    }
    mask = eff;
  }
  Selection s;
  select_window(*m, window_of_pair(c, src, dst), bytes, window, mask, c->opts, &s);
  fill_config(*m, s, out);
  return MP_OK;
}

int mp_set_submit_time(mp_ctx *c, double seconds) {
  if (!c) return MP_ERR_INVALID;
  if (!(seconds >= 0.0) || !std::isfinite(seconds)) return fail(c, MP_ERR_INVALID, "submit time must be finite and >= 0");
  c->submit = seconds;
  c->cache.clear();  // mp_select depends on it when opts.window > 1
  return MP_OK;
}

int mp_get_submit_time(mp_ctx *c, double *seconds) {
  if (!c || !seconds) return MP_ERR_INVALID;
  *seconds = c->submit;
  return MP_OK;
}

int mp_set_host_duplex(mp_ctx *c, int gpu, double kappa) {
  if (!c) return MP_ERR_INVALID;
  if (gpu < 0 || gpu >= MP_MAX_PATHS) return fail(c, MP_ERR_TOPOLOGY, "gpu out of range");
  if (!(kappa > 0.0) || !(kappa <= 1.0)) return fail(c, MP_ERR_INVALID, "kappa must be in (0, 1]");
  if (static_cast<int>(c->kappa.size()) <= gpu) c->kappa.resize(gpu + 1, 1.0);
  c->kappa[gpu] = kappa;
  c->cache.clear();
  return MP_OK;
}

int mp_get_host_duplex(mp_ctx *c, int gpu, double *kappa) {
  if (!c || !kappa) return MP_ERR_INVALID;
  if (gpu < 0 || gpu >= MP_MAX_PATHS) return fail(c, MP_ERR_TOPOLOGY, "gpu out of range");
  *kappa = gpu < static_cast<int>(c->kappa.size()) ? c->kappa[gpu] : 1.0;
  return MP_OK;
}

int mp_alloc(mp_ctx *c, uint64_t bytes, void **dptr) {
  if (!c || !dptr) return fail(c, MP_ERR_INVALID, "null argument");
  if (c->model_only) return fail(c, MP_ERR_STATE, "model-only context");
  void *p = c->heap.alloc(bytes);
  if (!p) return fail(c, MP_ERR_NOMEM, "heap exhausted");
  *dptr = p;
  return MP_OK;
}

int mp_free(mp_ctx *c, void *dptr) {
  if (!c) return MP_ERR_INVALID;
  if (!dptr) return MP_OK;
  if (!c->heap.release(dptr)) return fail(c, MP_ERR_INVALID, "pointer not from mp_alloc");
  return MP_OK;
}

int mp_peer_base(mp_ctx *c, int rank, void **base) {
  if (!c || !base) return fail(c, MP_ERR_INVALID, "null argument");
  if (c->model_only) return fail(c, MP_ERR_STATE, "model-only context");
  if (rank < 0 || rank >= c->world) return fail(c, MP_ERR_TOPOLOGY, "no such rank");
  if (rank == c->rank || c->peers.empty()) {
    if (rank != c->rank) return fail(c, MP_ERR_TOPOLOGY, "no such rank");
    *base = c->heap.base;
  } else {
    *base = c->peers[rank].heap;
  }
  return MP_OK;
}

int mp_register(mp_ctx *c, void *buf, uint64_t bytes, int *id) {
  if (!c || !id) return fail(c, MP_ERR_INVALID, "null argument");
  if (c->model_only) return fail(c, MP_ERR_STATE, "model-only context");
  if ((bytes == 0) != (buf == nullptr)) return fail(c, MP_ERR_INVALID, "buf and bytes must both be set or both 0");
  if (c->world == 1) {  // loopback receives into any device buffer: nothing to map
    if (c->regions.empty()) c->regions.assign(mpx::kMaxRegions, mp_ctx::Region{});
    for (int i = 1; i < static_cast<int>(c->regions.size()); ++i)
      if (!c->regions[i].used) {
        c->regions[i].used = true;
        c->regions[i].base = static_cast<uint8_t *>(buf);
        c->regions[i].bytes = bytes;
        *id = i;
        return MP_OK;
      }
    return fail(c, MP_ERR_NOMEM, "mp_register: region table full");
  }
  return mpx::world_register(c, buf, bytes, id);
}

int mp_deregister(mp_ctx *c, int id) {
  if (!c) return MP_ERR_INVALID;
  if (c->model_only) return fail(c, MP_ERR_STATE, "model-only context");
  if (c->world == 1) {
    if (id <= 0 || id >= static_cast<int>(c->regions.size()) || !c->regions[id].used)
      return fail(c, MP_ERR_INVALID, "mp_deregister: unknown region id");
    c->regions[id] = mp_ctx::Region{};
    return MP_OK;
  }
  return mpx::world_deregister(c, id);
}

int mp_xfer(mp_ctx *c, void *dst, const void *src, uint64_t bytes, const mp_config *cfg,
            void *stream) {
  if (!c) return MP_ERR_INVALID;
  if (c->model_only) return fail(c, MP_ERR_STATE, "model-only context");
  if (c->world != 1) return fail(c, MP_ERR_STATE, "mp_xfer is the single-GPU engine");
  if (bytes == 0) return MP_OK;
  if (!dst || !src) return fail(c, MP_ERR_INVALID, "null buffer");
  const PairModel *m = pair_model(c, 0, 0);
  mp_config sel;
  if (!cfg) {
    if (int s = mp_select(c, 0, 0, bytes, 0, &sel)) return s;
    cfg = &sel;
  }
  if (int s = check_config(c, *m, bytes, cfg)) return s;
  // CUDA-graph capture: a direct-only transfer is a pure kernel and replays
  // correctly; a staged one advances the rings' sequence numbers on the host at
  // launch, which a replay would not repeat, so it is refused while capturing.
  // (only staged configs need the query: it costs host time on every small message)
  bool staged = false;
  for (int i = 1; i < cfg->npaths; ++i) staged = staged || cfg->bytes[i] != 0;
  cudaStreamCaptureStatus cap = cudaStreamCaptureStatusNone;
  if (staged && cudaStreamIsCapturing(static_cast<cudaStream_t>(stream), &cap) == cudaSuccess &&
      cap != cudaStreamCaptureStatusNone)
    return fail(c, MP_ERR_UNSUPPORTED, "staged paths cannot be captured in a CUDA graph (direct-only can)");
  return launch_loopback(c, dst, src, bytes, *cfg, stream);
}

int mp_send(mp_ctx *c, const void *buf, uint64_t bytes, int dst, int tag, const mp_config *cfg,
            void *stream) {
  if (!c) return MP_ERR_INVALID;
  if (c->model_only) return fail(c, MP_ERR_STATE, "model-only context");
  if (dst < 0 || dst >= c->world) return fail(c, MP_ERR_TOPOLOGY, "no such rank");
  if (bytes && !buf) return fail(c, MP_ERR_INVALID, "null buffer");
  if (c->world != 1) {
    if (dst == c->rank) return fail(c, MP_ERR_TOPOLOGY, "send to self needs world == 1 (loopback)");
    const PairModel *m = pair_model(c, c->rank, dst);
    mp_config sel;
    if (!cfg) {
      if (int s = mp_select(c, c->rank, dst, bytes, 0, &sel)) return s;
      cfg = &sel;
    }
    if (int s = check_config(c, *m, bytes, cfg)) return s;
    return world_send(c, buf, bytes, dst, tag, *cfg, stream);
  }
  PendingSend ps;
  ps.buf = buf;
  ps.bytes = bytes;
  ps.tag = tag;
  ps.has_cfg = cfg != nullptr;
  if (cfg) {
    ps.cfg = *cfg;
    if (int s = check_config(c, *pair_model(c, 0, 0), bytes, cfg)) return s;
  }
  CK(cudaEventCreateWithFlags(&ps.ready, cudaEventDisableTiming));
  CK(cudaEventRecord(ps.ready, static_cast<cudaStream_t>(stream)));
  c->pending.push_back(ps);
  return MP_OK;
}

int mp_recv(mp_ctx *c, void *buf, uint64_t bytes, int src, int tag, void *stream) {
  if (!c) return MP_ERR_INVALID;
  if (c->model_only) return fail(c, MP_ERR_STATE, "model-only context");
  if (src < 0 || src >= c->world) return fail(c, MP_ERR_TOPOLOGY, "no such rank");
  if (c->world != 1) {
    if (src == c->rank) return fail(c, MP_ERR_TOPOLOGY, "recv from self needs world == 1 (loopback)");
    if (bytes && !buf) return fail(c, MP_ERR_INVALID, "null buffer");
    return world_recv(c, buf, bytes, src, tag, stream);
  }
  if (c->pending.empty()) return fail(c, MP_ERR_STATE, "loopback recv without a posted send");
  PendingSend ps = c->pending.front();
  if (ps.bytes != bytes || ps.tag != tag) {
    return fail(c, MP_ERR_MISMATCH, "loopback send/recv size or tag mismatch");
  }
  c->pending.pop_front();
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  cudaError_t e = cudaStreamWaitEvent(st, ps.ready, 0);
  cudaEventDestroy(ps.ready);
  if (e != cudaSuccess) return cuda_fail(c, e, "cudaStreamWaitEvent");
  return mp_xfer(c, buf, ps.buf, bytes, ps.has_cfg ? &ps.cfg : nullptr, stream);
}

int mp_sync(mp_ctx *c) {
  if (!c) return MP_ERR_INVALID;
  if (c->model_only) return MP_OK;
  CK(cudaSetDevice(c->device));
  if (c->world > 1) return world_sync(c);
  CK(cudaDeviceSynchronize());
  return check_err(c);
}

int mp_stats(mp_ctx *c, uint64_t *launches) {
  if (!c || !launches) return MP_ERR_INVALID;
  *launches = c->launches + (c->world > 1 && !c->model_only ? world_relay_launches(c) : 0);
  return MP_OK;
}

int mp_save_params(mp_ctx *c, const char *path) {
  if (!c || !path) return MP_ERR_INVALID;
  FILE *f = std::fopen(path, "w");
  if (!f) return fail(c, MP_ERR_INVALID, std::string("cannot write ") + path);
  std::fprintf(f, "mpx-params 1\n");
  if (c->have_topo) {  // Step 1's parameters belong to this topology
    const mp_topology &T = c->topo;
    std::fprintf(f, "topology %016llx %d\n", static_cast<unsigned long long>(T.fingerprint), T.world);
    for (int r = 0; r < T.world; ++r) {
      const mp_gpu_info &g = T.gpu[r];
      std::fprintf(f, "gpu %d ", r);
      for (int i = 0; i < 16; ++i) std::fprintf(f, "%02x", static_cast<unsigned char>(g.uuid[i]));
      std::fprintf(f, " %d %d %d %d %d\n", g.sms, g.nvlinks, g.pcie_gen, g.pcie_width, g.numa_node);
    }
  }
  for (const auto &kv : c->models) {
    const PairModel &m = kv.second;
    std::fprintf(f, "pair %d %d %zu %.17g %.17g\n", kv.first.first, kv.first.second, m.paths.size(),
                 m.port_alpha, m.port_beta);
    for (const PathModel &p : m.paths)
      std::fprintf(f, "path %d %d %.17g %.17g %.17g %.17g %.17g %.17g %.17g %.17g %.17g\n", p.kind, p.via,
                   p.alpha, p.beta, p.alpha2, p.beta2, p.eps, p.c, p.sigma, p.w, p.wake);
    auto wt = c->windows.find(kv.first);
    if (wt != c->windows.end()) {
      std::fprintf(f, "window %d %d %zu %.17g", kv.first.first, kv.first.second, wt->second.h.size(), wt->second.tau);
      for (double h : wt->second.h) std::fprintf(f, " %.17g", h);
      std::fprintf(f, "\n");
    }
    auto bt = c->bands.find(kv.first);
    if (bt == c->bands.end()) continue;
    for (const auto &b : bt->second) {
      std::fprintf(f, "band %d %d %zu %llu %.17g %.17g\n", kv.first.first, kv.first.second, b.second.paths.size(),
                   static_cast<unsigned long long>(b.first), b.second.port_alpha, b.second.port_beta);
      for (const PathModel &p : b.second.paths)
        std::fprintf(f, "path %d %d %.17g %.17g %.17g %.17g %.17g %.17g %.17g %.17g %.17g\n", p.kind, p.via,
                     p.alpha, p.beta, p.alpha2, p.beta2, p.eps, p.c, p.sigma, p.w, p.wake);
    }
  }
  for (size_t g = 0; g < c->kappa.size(); ++g)
    if (c->kappa[g] != 1.0) std::fprintf(f, "duplex %zu 0 1 %.17g\n", g, c->kappa[g]);
  if (c->submit > 0.0) std::fprintf(f, "submit %.17g\n", c->submit);
  std::fclose(f);
  return MP_OK;
}

int mp_load_params(mp_ctx *c, const char *path) {
  if (!c || !path) return MP_ERR_INVALID;
  FILE *f = std::fopen(path, "r");
  if (!f) return fail(c, MP_ERR_INVALID, std::string("cannot read ") + path);
  std::vector<std::string> lines;
  char buf[4096];
  while (std::fgets(buf, sizeof(buf), f)) lines.push_back(buf);
  std::fclose(f);
  char tag[32];
  int ver = 0;
  if (lines.empty() || std::sscanf(lines[0].c_str(), "%31s %d", tag, &ver) != 2 || std::strcmp(tag, "mpx-params") != 0 ||
      ver != 1)
    return fail(c, MP_ERR_INVALID, "not an mpx parameter file");
  // Step 2 loads only what Step 1 measured on this topology
  for (const std::string &ln : lines) {
    unsigned long long fp = 0;
    int w = 0;
    if (std::sscanf(ln.c_str(), "topology %llx %d", &fp, &w) == 2 && c->have_topo &&
        (fp != c->topo.fingerprint || w != c->topo.world)) {
      char msg[160];
      std::snprintf(msg, sizeof(msg), "parameter file topology %016llx (world %d) is not this job's %016llx (world %d)",
                    fp, w, static_cast<unsigned long long>(c->topo.fingerprint), c->topo.world);
      return fail(c, MP_ERR_TOPOLOGY, msg);
    }
  }
  auto truncated = [&]() { return fail(c, MP_ERR_INVALID, "truncated parameter file"); };
  size_t i = 1;
  while (i < lines.size()) {
    const char *ln = lines[i].c_str();
    int src = 0, dst = 0;
    size_t np = 0;
    if (std::sscanf(ln, "%31s", tag) != 1) {
      ++i;
      continue;
    }
    if (!std::strcmp(tag, "topology") || !std::strcmp(tag, "gpu")) {
      ++i;
      continue;
    }
    if (!std::strcmp(tag, "submit")) {  // reading C27
      double v = 0.0;
      if (std::sscanf(ln, "%31s %lf", tag, &v) != 2) return truncated();
      if (int s = mp_set_submit_time(c, v)) return s;
      ++i;
      continue;
    }
    if (!std::strcmp(tag, "window") || !std::strcmp(tag, "duplex")) {  // NEXT f2
      const bool win = tag[0] == 'w';
      double tau = 0.0, h[MP_MAX_PATHS];
      int used = 0;
      if (std::sscanf(ln, "%31s %d %d %zu %lf%n", tag, &src, &dst, &np, &tau, &used) != 5 || np < 1 ||
          np > MP_MAX_PATHS)
        return truncated();
      if (win) {
        const char *q = ln + used;
        for (size_t k = 0; k < np; ++k) {
          int u = 0;
          if (std::sscanf(q, "%lf%n", &h[k], &u) != 1) return truncated();
          q += u;
        }
      }
      int s = MP_OK;
      if (win && pair_ok(c, src, dst)) s = mp_set_window_model(c, src, dst, h, static_cast<int>(np), tau);
      if (!win) s = mp_set_host_duplex(c, src, tau);
      if (s) return s;
      ++i;
      continue;
    }
    const bool band = !std::strcmp(tag, "band");
    if (!band && std::strcmp(tag, "pair")) return fail(c, MP_ERR_INVALID, std::string("unknown line: ") + tag);
    unsigned long long n_min = 0;
    double pa = 0.0, pb = 0.0;
    const int got = band ? std::sscanf(ln, "%31s %d %d %zu %llu %lf %lf", tag, &src, &dst, &np, &n_min, &pa, &pb)
                         : std::sscanf(ln, "%31s %d %d %zu %lf %lf", tag, &src, &dst, &np, &pa, &pb);
    if (got != (band ? 7 : 6) || np < 1 || np > MP_MAX_PATHS || i + np >= lines.size()) return truncated();
    mp_path paths[MP_MAX_PATHS];
    mp_path_params prm[MP_MAX_PATHS];
    for (size_t k = 0; k < np; ++k) {
      mp_path_params &q = prm[k];
      q.wake = 0.0;  // a round-2 file has no 12th field (C28)
      const int got_p = std::sscanf(lines[i + 1 + k].c_str(), "%31s %d %d %lf %lf %lf %lf %lf %lf %lf %lf %lf", tag,
                                    &paths[k].kind, &paths[k].via, &q.alpha, &q.beta, &q.alpha2, &q.beta2, &q.eps,
                                    &q.c, &q.sigma, &q.w, &q.wake);
      if (got_p != 11 && got_p != 12) return truncated();
    }
    mp_port_params port{pa, pb};
    if (pair_ok(c, src, dst)) {
      const int s = band ? mp_set_model_band(c, src, dst, n_min, prm, static_cast<int>(np), &port)
                         : mp_set_model(c, src, dst, paths, prm, static_cast<int>(np), &port);
      if (s) return s;
    }
    i += 1 + np;
  }
  return MP_OK;
}

}  // extern "C"
