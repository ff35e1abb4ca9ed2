// coll.cpp — collectives over multi-path P2P (§5.3,
// P:389-393): MPI_Alltoall (Bruck / pairwise) and MPI_Allreduce (radix-2 K-nomial =
// recursive halving + doubling / ring), each P2P step one model-selected multi-path
// mp_send/mp_recv pair (mp_select_flows over the step's pattern, host path excluded
// per P:393).  A schedule is data (mp_coll_plan, see include/mp.h); the executor below
// runs any plan on two internal streams.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <map>
#include <new>
#include <string>
#include <tuple>
#include <vector>

#include "ctx.h"

using namespace mpx;

namespace {

int cfail(mp_ctx *c, int code, const std::string &msg) {
  if (c) c->last_error = msg;
  return code;
}

bool pow2(int w) { return w > 0 && (w & (w - 1)) == 0; }

int elem_bytes(int dtype) {
  switch (dtype) {
    case MP_DT_U8: return 1;
    case MP_DT_I32: return 4;
    case MP_DT_I64: return 8;
    case MP_DT_F32: return 4;
    case MP_DT_F64: return 8;
    case MP_DT_BF16: return 2;
    default: return 0;
  }
}

// Plan under construction (bounds checked at the end).
struct Builder {
  mp_coll_plan *p;
  bool overflow = false;
  void pre(int sb, uint64_t so, int db, uint64_t dof, uint64_t len) { copy(p->pre, &p->npre, sb, so, db, dof, len); }
  void post(int sb, uint64_t so, int db, uint64_t dof, uint64_t len) { copy(p->post, &p->npost, sb, so, db, dof, len); }
  void copy(mp_coll_copy *arr, int32_t *n, int sb, uint64_t so, int db, uint64_t dof, uint64_t len) {
    if (len == 0) return;
    if (*n >= MP_COLL_MAX_COPIES) {
      overflow = true;
      return;
    }
    arr[(*n)++] = mp_coll_copy{sb, db, so, dof, len};
  }
  mp_coll_step *step(int to, int from, int reduce) {
    if (p->nsteps >= MP_COLL_MAX_STEPS) {
      overflow = true;
      return nullptr;
    }
    mp_coll_step *s = &p->step[p->nsteps++];
    *s = mp_coll_step{to, from, reduce, 0, static_cast<uint32_t>(p->nsegs), 0, 0, 0, 0};
    return s;
  }
  void send_seg(mp_coll_step *s, int buf, uint64_t off, uint64_t len) {
    if (!s || !seg(buf, off, len)) return;
    s->send_nseg += 1;
    s->bytes += len;
  }
  void begin_recv(mp_coll_step *s) {
    if (s) s->recv_seg0 = static_cast<uint32_t>(p->nsegs);
  }
  void recv_seg(mp_coll_step *s, int buf, uint64_t off, uint64_t len) {
    if (!s || !seg(buf, off, len)) return;
    s->recv_nseg += 1;
  }
  bool seg(int buf, uint64_t off, uint64_t len) {
    if (p->nsegs >= MP_COLL_MAX_SEGS) {
      overflow = true;
      return false;
    }
    p->seg[p->nsegs++] = mp_coll_seg{buf, 0, off, len};
    return true;
  }
};

// Bruck (UCC's Alltoall).  TMP holds W blocks: (1) TMP[i] = SEND[(r+i) mod W];
// (2) for d = 1, 2, 4, … < W: send the blocks i with (i & d) != 0 to r+d, receive the
// same block positions from r−d; (3) RECV[(r−i) mod W] = TMP[i].
void plan_bruck(Builder &b, int W, int r, uint64_t B) {
  b.p->tmp_bytes = B * static_cast<uint64_t>(W);
  for (int i = 0; i < W; ++i) b.pre(MP_BUF_SEND, B * ((r + i) % W), MP_BUF_TMP, B * i, B);
  for (int d = 1; d < W; d <<= 1) {
    mp_coll_step *s = b.step((r + d) % W, (r - d + W) % W, 0);
    for (int i = 1; i < W; ++i)
      if (i & d) b.send_seg(s, MP_BUF_TMP, B * i, B);
    b.begin_recv(s);
    for (int i = 1; i < W; ++i)
      if (i & d) b.recv_seg(s, MP_BUF_TMP, B * i, B);
  }
  for (int i = 0; i < W; ++i) b.post(MP_BUF_TMP, B * i, MP_BUF_RECV, B * ((r - i + W) % W), B);
}

// Pairwise exchange: step i sends block r+i to rank r+i, receives block r−i from r−i.
void plan_pairwise(Builder &b, int W, int r, uint64_t B) {
  b.pre(MP_BUF_SEND, B * r, MP_BUF_RECV, B * r, B);
  for (int i = 1; i < W; ++i) {
    const int to = (r + i) % W, from = (r - i + W) % W;
    mp_coll_step *s = b.step(to, from, 0);
    b.send_seg(s, MP_BUF_SEND, B * to, B);
    b.begin_recv(s);
    b.recv_seg(s, MP_BUF_RECV, B * from, B);
  }
}

// Block k of an Allreduce vector of n elements (elem bytes each): elements
// [k·n/W, (k+1)·n/W) — byte range [lo, hi).
void block_range(uint64_t n, uint32_t elem, int W, int k0, int k1, uint64_t *lo, uint64_t *hi) {
  *lo = elem * (static_cast<uint64_t>(k0) * n / W);
  *hi = elem * (static_cast<uint64_t>(k1) * n / W);
}

// Radix-2 K-nomial: recursive halving reduce-scatter — the block range
// [lo, hi) halves every step, rank r keeps the half holding block r and exchanges
// the other with r ^ d — then recursive doubling allgather in reverse.  W = 2^m.
void plan_knomial(Builder &b, int W, int r, uint64_t n, uint32_t elem) {
  const uint64_t bytes = n * elem;
  b.pre(MP_BUF_SEND, 0, MP_BUF_RECV, 0, bytes);
  int lo = 0, hi = W;
  for (int d = W / 2; d >= 1; d /= 2) {
    const int mid = lo + (hi - lo) / 2;
    const bool low = r < mid;
    const int klo = low ? lo : mid, khi = low ? mid : hi;  // keep
    const int glo = low ? mid : lo, ghi = low ? hi : mid;  // give
    uint64_t a, e;
    mp_coll_step *s = b.step(r ^ d, r ^ d, 1);
    block_range(n, elem, W, glo, ghi, &a, &e);
    b.send_seg(s, MP_BUF_RECV, a, e - a);
    b.begin_recv(s);
    block_range(n, elem, W, klo, khi, &a, &e);
    b.recv_seg(s, MP_BUF_RECV, a, e - a);
    lo = klo;
    hi = khi;
  }
  for (int d = 1; d < W; d *= 2) {
    const int size = hi - lo, sib = lo ^ size;
    uint64_t a, e;
    mp_coll_step *s = b.step(r ^ d, r ^ d, 0);
    block_range(n, elem, W, lo, hi, &a, &e);
    b.send_seg(s, MP_BUF_RECV, a, e - a);
    b.begin_recv(s);
    block_range(n, elem, W, sib, sib + size, &a, &e);
    b.recv_seg(s, MP_BUF_RECV, a, e - a);
    lo = std::min(lo, sib);
    hi = lo + 2 * size;
  }
}

// Ring: W−1 reduce-scatter steps (send block r−s, receive and add block r−s−1), then
// W−1 allgather steps (send block r+1−s, receive block r−s).
void plan_ring(Builder &b, int W, int r, uint64_t n, uint32_t elem) {
  b.pre(MP_BUF_SEND, 0, MP_BUF_RECV, 0, n * elem);
  const int to = (r + 1) % W, from = (r - 1 + W) % W;
  auto blk = [&](int k, uint64_t *a, uint64_t *e) {
    k = ((k % W) + W) % W;
    block_range(n, elem, W, k, k + 1, a, e);
  };
  for (int s = 0; s < W - 1; ++s) {
    uint64_t a, e;
    mp_coll_step *st = b.step(to, from, 1);
    blk(r - s, &a, &e);
    b.send_seg(st, MP_BUF_RECV, a, e - a);
    b.begin_recv(st);
    blk(r - s - 1, &a, &e);
    b.recv_seg(st, MP_BUF_RECV, a, e - a);
  }
  for (int s = 0; s < W - 1; ++s) {
    uint64_t a, e;
    mp_coll_step *st = b.step(to, from, 0);
    blk(r + 1 - s, &a, &e);
    b.send_seg(st, MP_BUF_RECV, a, e - a);
    b.begin_recv(st);
    blk(r - s, &a, &e);
    b.recv_seg(st, MP_BUF_RECV, a, e - a);
  }
}

int resolve_algo(int coll, int algo, int W, uint64_t bytes) {
  if (algo != MP_ALGO_AUTO) return algo;
  if (coll == MP_COLL_ALLTOALL) return bytes < (256u << 10) ? MP_ALGO_BRUCK : MP_ALGO_PAIRWISE;
  return pow2(W) ? MP_ALGO_KNOMIAL : MP_ALGO_RING;
}

}  // namespace

extern "C" int mp_coll_plan_build(int coll, int algo, int world, int rank, uint64_t bytes, uint32_t elem_size,
                                  mp_coll_plan *out) {
  if (!out || world < 1 || world > MP_MAX_PATHS || rank < 0 || rank >= world || elem_size < 1)
    return MP_ERR_INVALID;
  if (bytes % elem_size) return MP_ERR_INVALID;
  algo = resolve_algo(coll, algo, world, bytes);
  std::memset(out, 0, sizeof(*out));
  out->coll = coll;
  out->algo = algo;
  out->world = world;
  out->rank = rank;
  Builder b{out};
  if (coll == MP_COLL_ALLTOALL) {
    if (world == 1 || bytes == 0) {
      b.pre(MP_BUF_SEND, 0, MP_BUF_RECV, 0, bytes);
    } else if (algo == MP_ALGO_BRUCK) {
      plan_bruck(b, world, rank, bytes);
    } else if (algo == MP_ALGO_PAIRWISE) {
      plan_pairwise(b, world, rank, bytes);
    } else {
      return MP_ERR_INVALID;
    }
  } else if (coll == MP_COLL_ALLREDUCE) {
    const uint64_t n = bytes / elem_size;
    if (world == 1 || bytes == 0) {
      b.pre(MP_BUF_SEND, 0, MP_BUF_RECV, 0, bytes);
    } else if (algo == MP_ALGO_KNOMIAL) {
      if (!pow2(world)) return MP_ERR_INVALID;
      plan_knomial(b, world, rank, n, elem_size);
    } else if (algo == MP_ALGO_RING) {
      plan_ring(b, world, rank, n, elem_size);
    } else {
      return MP_ERR_INVALID;
    }
  } else {
    return MP_ERR_INVALID;
  }
  return b.overflow ? MP_ERR_INVALID : MP_OK;
}

// ------------------------------------------------------------------ executor

namespace mpx {
struct CollState {
  cudaStream_t s = nullptr, r = nullptr;   // internal send / receive streams
  std::vector<cudaEvent_t> ev;             // event pool
  void *scratch = nullptr;                 // heap scratch: [tmp | send staging | recv staging]
  uint64_t scratch_bytes = 0;
  uint64_t seq = 0;
  std::map<std::tuple<int, int, uint64_t, uint32_t>, std::vector<mp_config>> cfgs;  // per-step configs
};
}  // namespace mpx

namespace {

int ensure(mp_ctx *c, CollState &st, uint64_t need, int nev) {
  if (!st.s) {
    if (cudaStreamCreateWithFlags(&st.s, cudaStreamNonBlocking) != cudaSuccess ||
        cudaStreamCreateWithFlags(&st.r, cudaStreamNonBlocking) != cudaSuccess)
      return cfail(c, MP_ERR_CUDA, "collective streams");
  }
  while (static_cast<int>(st.ev.size()) < nev) {
    cudaEvent_t e;
    if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess)
      return cfail(c, MP_ERR_CUDA, "collective events");
    st.ev.push_back(e);
  }
  if (need > st.scratch_bytes) {
    // the old scratch may still be read by an earlier collective on these streams
    cudaStreamSynchronize(st.s);
    cudaStreamSynchronize(st.r);
    if (st.scratch) mp_free(c, st.scratch);
    st.scratch = nullptr;
    st.scratch_bytes = 0;
    if (int e = mp_alloc(c, need, &st.scratch)) return e;
    st.scratch_bytes = need;
  }
  return MP_OK;
}

// Per-step multi-path configs: mp_select_flows over every rank's message of the step
// (the pattern is known ahead of time; reading C19), host path excluded.
int step_configs(mp_ctx *c, CollState &st, const mp_coll_plan &me, uint64_t bytes, uint32_t elem,
                 const std::vector<mp_config> **out) {
  const auto key = std::make_tuple(me.coll, me.algo, bytes, elem);
  auto it = st.cfgs.find(key);
  if (it != st.cfgs.end()) {
    *out = &it->second;
    return MP_OK;
  }
  const int W = c->world;
  std::vector<mp_coll_plan> plans(W);
  for (int r = 0; r < W; ++r)
    if (int e = mp_coll_plan_build(me.coll, me.algo, W, r, bytes, elem, &plans[r])) return cfail(c, e, "plan");
  std::vector<mp_config> mine(me.nsteps);
  for (int j = 0; j < me.nsteps; ++j) {
    std::vector<mp_flow> flows;
    int my = -1;
    for (int r = 0; r < W; ++r) {
      const mp_coll_step &s = plans[r].step[j];
      mp_path ps[MP_MAX_PATHS];
      int np = 0;
      if (int e = mp_paths(c, r, s.send_to, ps, &np)) return e;
      uint32_t mask = 0;
      for (int i = 0; i < np; ++i)
        if (ps[i].kind != MP_PATH_HOST) mask |= 1u << i;
      if (r == c->rank) my = static_cast<int>(flows.size());
      flows.push_back(mp_flow{r, s.send_to, mask, 0, s.bytes});
    }
    std::vector<mp_config> cf(flows.size());
    // one message per pair and step: never the window-aware selection (C24)
    const uint32_t w = c->opts.window;
    c->opts.window = 1;
    const int e = mp_select_flows(c, static_cast<int>(flows.size()), flows.data(), cf.data());
    c->opts.window = w;
    if (e) return e;
    mine[j] = cf[my];
  }
  *out = &st.cfgs.emplace(key, std::move(mine)).first->second;
  return MP_OK;
}

int launch_reduce_sum(mp_ctx *c, int dtype, void *dst, const void *src, uint64_t bytes, cudaStream_t s) {
  const int e = launch_reduce(dtype, dst, src, bytes, s);
  if (e) return cfail(c, MP_ERR_CUDA, std::string("reduce launch: ") + cudaGetErrorString(static_cast<cudaError_t>(e)));
  c->launches += 1;
  return MP_OK;
}

int local_copy(mp_ctx *c, void *dst, const void *src, uint64_t n, cudaStream_t s) {
  if (n == 0 || dst == src) return MP_OK;
  return launch_direct_copy(c, dst, src, n, s);
}

// One rank's execution of a plan, in pieces.  The real executor (run_plan) chains
// them on two internal streams with events; the emulated world's executor
// (emu_collective) runs every rank's pieces step by step around one cooperative grid
// per step.
struct PlanExec {
  mp_ctx *c = nullptr;
  const mp_coll_plan *P = nullptr;
  const void *sendbuf = nullptr;
  void *recvbuf = nullptr;
  int dtype = 0;
  uint8_t *tmpb = nullptr, *stg_s = nullptr, *stg_r = nullptr;
  const std::vector<mp_config> *cfgs = nullptr;
  uint64_t seq = 0;

  uint8_t *buf(int id) const {
    return id == MP_BUF_SEND ? const_cast<uint8_t *>(static_cast<const uint8_t *>(sendbuf))
                             : (id == MP_BUF_RECV ? static_cast<uint8_t *>(recvbuf) : tmpb);
  }
  int tag(int j) const { return 0x3C000000 | static_cast<int>((seq & 0xFFFF) << 8) | (j & 0xFF); }

  // scratch [tmp | send staging | recv staging] in the heap, events, per-step configs
  int setup(uint64_t bytes, uint32_t elem) {
    if (!c->coll) c->coll = new (std::nothrow) CollState();
    if (!c->coll) return MP_ERR_NOMEM;
    CollState &st = *c->coll;
    uint64_t maxmsg = 0;
    for (int j = 0; j < P->nsteps; ++j) maxmsg = std::max(maxmsg, P->step[j].bytes);
    const uint64_t align = 256;
    const uint64_t tmp = (P->tmp_bytes + align - 1) / align * align, stg = (maxmsg + align - 1) / align * align;
    if (int e = ensure(c, st, std::max<uint64_t>(tmp + 2 * stg, 256), 2 + 2 * P->nsteps)) return e;
    uint8_t *base = static_cast<uint8_t *>(st.scratch);
    tmpb = base;
    stg_s = base + tmp;
    stg_r = base + tmp + stg;
    if (c->world > 1 && P->nsteps)
      if (int e = step_configs(c, st, *P, bytes, elem, &cfgs)) return e;
    seq = st.seq++;
    return MP_OK;
  }
  int copies(const mp_coll_copy *k, int n, cudaStream_t s) {
    for (int i = 0; i < n; ++i)
      if (int e = local_copy(c, buf(k[i].dst_buf) + k[i].dst_off, buf(k[i].src_buf) + k[i].src_off, k[i].len, s))
        return e;
    return MP_OK;
  }
  int pre(cudaStream_t s) { return copies(P->pre, P->npre, s); }
  int post(cudaStream_t s) { return copies(P->post, P->npost, s); }
  // send side of step j: pack its segments (one segment is sent in place), mp_send
  int send(int j, cudaStream_t s) {
    const mp_coll_step &t = P->step[j];
    const uint8_t *msg = nullptr;
    if (t.send_nseg == 1) {
      const mp_coll_seg &g = P->seg[t.send_seg0];
      msg = buf(g.buf) + g.off;
    } else {
      uint64_t o = 0;
      for (uint32_t k = 0; k < t.send_nseg; ++k) {
        const mp_coll_seg &g = P->seg[t.send_seg0 + k];
        if (int e = local_copy(c, stg_s + o, buf(g.buf) + g.off, g.len, s)) return e;
        o += g.len;
      }
      msg = stg_s;
    }
    return mp_send(c, msg, t.bytes, t.send_to, tag(j), &(*cfgs)[j], s);
  }
  uint64_t recv_bytes(int j) const {
    const mp_coll_step &t = P->step[j];
    uint64_t n = 0;
    for (uint32_t k = 0; k < t.recv_nseg; ++k) n += P->seg[t.recv_seg0 + k].len;
    return n;
  }
  // step j's message lands straight in its target: one receivable segment, no
  // reduction, and not overlapping what the step still sends (Bruck sends and receives
  // the same TMP block positions)
  bool direct_recv(int j) const {
    const mp_coll_step &t = P->step[j];
    const mp_coll_seg *g0 = t.recv_nseg ? &P->seg[t.recv_seg0] : nullptr;
    bool overlap = false;
    for (uint32_t k = 0; k < t.send_nseg && g0; ++k) {
      const mp_coll_seg &g = P->seg[t.send_seg0 + k];
      const uint8_t *a0 = buf(g.buf) + g.off, *b0 = buf(g0->buf) + g0->off;
      if (a0 < b0 + g0->len && b0 < a0 + g.len) overlap = true;
    }
    return t.recv_nseg == 1 && !t.reduce && !overlap &&
           (g0->buf == MP_BUF_TMP || world_receivable(c, buf(g0->buf) + g0->off, g0->len));
  }
  int recv(int j, cudaStream_t s) {
    const mp_coll_step &t = P->step[j];
    uint8_t *dst = stg_r;
    if (direct_recv(j)) {
      const mp_coll_seg &g0 = P->seg[t.recv_seg0];
      dst = buf(g0.buf) + g0.off;
    }
    return mp_recv(c, dst, recv_bytes(j), t.recv_from, tag(j), s);
  }
  // a staged receive of step j: its segments copied (or reduced) out of the staging
  int unpack(int j, cudaStream_t s) {
    const mp_coll_step &t = P->step[j];
    uint64_t o = 0;
    for (uint32_t k = 0; k < t.recv_nseg; ++k) {
      const mp_coll_seg &g = P->seg[t.recv_seg0 + k];
      const int e = t.reduce ? launch_reduce_sum(c, dtype, buf(g.buf) + g.off, stg_r + o, g.len, s)
                             : local_copy(c, buf(g.buf) + g.off, stg_r + o, g.len, s);
      if (e) return e;
      o += g.len;
    }
    return MP_OK;
  }
};

int run_plan(mp_ctx *c, const mp_coll_plan &P, const void *sendbuf, void *recvbuf, uint64_t bytes, uint32_t elem,
             int dtype, void *ustream) {
  PlanExec X;
  X.c = c;
  X.P = &P;
  X.sendbuf = sendbuf;
  X.recvbuf = recvbuf;
  X.dtype = dtype;
  if (int e = X.setup(bytes, elem)) return e;
  CollState &st = *c->coll;
  cudaStream_t us = static_cast<cudaStream_t>(ustream);
  cudaEvent_t *ev = st.ev.data();
  // fork
  if (cudaEventRecord(ev[0], us) != cudaSuccess || cudaStreamWaitEvent(st.s, ev[0], 0) != cudaSuccess ||
      cudaStreamWaitEvent(st.r, ev[0], 0) != cudaSuccess)
    return cfail(c, MP_ERR_CUDA, "collective fork");
  if (int e = X.pre(st.s)) return e;
  cudaEvent_t prev_r = nullptr;
  for (int j = 0; j < P.nsteps; ++j) {
    cudaEvent_t sent = ev[2 + 2 * j], done_r = ev[3 + 2 * j];
    // send side: after the previous step's receive (its data may be sent now)
    if (prev_r) cudaStreamWaitEvent(st.s, prev_r, 0);
    if (int e = X.send(j, st.s)) return e;
    cudaEventRecord(sent, st.s);  // the send kernel has consumed its source
    if (prev_r) cudaStreamWaitEvent(st.r, prev_r, 0);
    if (int e = X.recv(j, st.r)) return e;
    if (!X.direct_recv(j)) {
      cudaStreamWaitEvent(st.r, sent, 0);  // this step's send has read what the unpack overwrites
      if (int e = X.unpack(j, st.r)) return e;
    }
    cudaEventRecord(done_r, st.r);
    prev_r = done_r;
  }
  if (prev_r) cudaStreamWaitEvent(st.s, prev_r, 0);
  if (int e = X.post(st.s)) return e;
  // join: the receive stream's work is already ordered before the send stream's tail
  cudaEventRecord(ev[1], st.s);
  if (cudaStreamWaitEvent(us, ev[1], 0) != cudaSuccess) return cfail(c, MP_ERR_CUDA, "collective join");
  return MP_OK;
}

// The emulated world's executor: every rank's plan in lock step on `stream` — every
// rank's pre copies; per step, every rank's packing and recorded send / receive, ONE
// cooperative grid for all of them (mp_emu_run), every rank's unpacking; every rank's
// post copies.
int emu_collective(mp_ctx **ctxs, int n, int coll, int algo, const void *const *sendbufs, void *const *recvbufs,
                   uint64_t bytes, uint32_t elem, int dtype, void *stream) {
  mp_ctx *c0 = ctxs[0];
  if (!c0->emu_world) return cfail(c0, MP_ERR_STATE, "not an emulated world");
  for (int r = 0; r < n; ++r)
    if (!ctxs[r] || ctxs[r]->rank != r || ctxs[r]->world != n || !sendbufs[r] || !recvbufs[r])
      return cfail(c0, MP_ERR_INVALID, "emulated collective: every rank's context and buffers, in rank order");
  if (bytes == 0) return MP_OK;
  std::vector<mp_coll_plan> plans(static_cast<size_t>(n));
  std::vector<PlanExec> X(static_cast<size_t>(n));
  cudaStream_t s = static_cast<cudaStream_t>(stream);
  auto discard = [&](int e) {  // nothing recorded may outlive a failed collective
    cudaStreamSynchronize(s);
    for (int r = 0; r < n; ++r) {
      ctxs[r]->emu_send.clear();
      ctxs[r]->emu_recv.clear();
      ctxs[r]->emu_esend.clear();
      ctxs[r]->emu_erecv.clear();
    }
    return e;
  };
  for (int r = 0; r < n; ++r) {
    if (int e = mp_coll_plan_build(coll, algo, n, r, bytes, elem, &plans[r]))
      return cfail(c0, e, "collective plan: invalid algorithm / size for this world");
    X[r].c = ctxs[r];
    X[r].P = &plans[r];
    X[r].sendbuf = sendbufs[r];
    X[r].recvbuf = recvbufs[r];
    X[r].dtype = dtype;
    if (int e = X[r].setup(bytes, elem)) return discard(e);
    if (plans[r].nsteps != plans[0].nsteps) return discard(cfail(c0, MP_ERR_INVALID, "ranks' plans differ in steps"));
  }
  for (int r = 0; r < n; ++r)
    if (int e = X[r].pre(s)) return discard(e);
  for (int j = 0; j < plans[0].nsteps; ++j) {
    for (int r = 0; r < n; ++r) {
      if (int e = X[r].send(j, s)) return discard(e);
      if (int e = X[r].recv(j, s)) return discard(e);
    }
    if (int e = mp_emu_run(ctxs, n, stream, nullptr)) return discard(e);
    for (int r = 0; r < n; ++r)
      if (!X[r].direct_recv(j))
        if (int e = X[r].unpack(j, s)) return discard(e);
  }
  for (int r = 0; r < n; ++r)
    if (int e = X[r].post(s)) return discard(e);
  if (cudaStreamSynchronize(s) != cudaSuccess) return cfail(c0, MP_ERR_CUDA, "emulated collective");
  return MP_OK;
}

int collective(mp_ctx *c, int coll, int algo, const void *sendbuf, void *recvbuf, uint64_t bytes, uint32_t elem,
               int dtype, void *stream) {
  if (!c) return MP_ERR_INVALID;
  if (c->model_only) return cfail(c, MP_ERR_STATE, "model-only context");
  // an emulated world runs everything recorded as one grid: a plan's later steps
  // depend on its earlier ones (and on local kernels in between)
  if (c->emulated) return cfail(c, MP_ERR_UNSUPPORTED, "collectives: not in an emulated world");
  if (bytes == 0) return MP_OK;
  if (!sendbuf || !recvbuf) return cfail(c, MP_ERR_INVALID, "null buffer");
  mp_coll_plan *P = new (std::nothrow) mp_coll_plan;
  if (!P) return MP_ERR_NOMEM;
  int e = mp_coll_plan_build(coll, algo, c->world, c->rank, bytes, elem, P);
  if (e) {
    delete P;
    return cfail(c, e, "collective plan: invalid algorithm / size for this world");
  }
  e = run_plan(c, *P, sendbuf, recvbuf, bytes, elem, dtype, stream);
  delete P;
  return e;
}

}  // namespace

void mpx::coll_release(mp_ctx *c) {
  if (!c->coll) return;
  CollState &st = *c->coll;
  if (st.s) cudaStreamSynchronize(st.s);
  if (st.r) cudaStreamSynchronize(st.r);
  for (cudaEvent_t e : st.ev) cudaEventDestroy(e);
  if (st.s) cudaStreamDestroy(st.s);
  if (st.r) cudaStreamDestroy(st.r);
  if (st.scratch) mp_free(c, st.scratch);
  delete c->coll;
  c->coll = nullptr;
}

extern "C" int mp_alltoall(mp_ctx *c, const void *sendbuf, void *recvbuf, uint64_t bytes_per_rank, int algo,
                           void *stream) {
  return collective(c, MP_COLL_ALLTOALL, algo, sendbuf, recvbuf, bytes_per_rank, 1, MP_DT_U8, stream);
}

extern "C" int mp_allreduce(mp_ctx *c, const void *sendbuf, void *recvbuf, uint64_t count, int dtype, int op,
                            int algo, void *stream) {
  if (!c) return MP_ERR_INVALID;
  const int eb = elem_bytes(dtype);
  if (eb == 0 || dtype == MP_DT_U8) return cfail(c, MP_ERR_INVALID, "allreduce: unsupported dtype");
  if (op != MP_OP_SUM) return cfail(c, MP_ERR_INVALID, "allreduce: unsupported op");
  return collective(c, MP_COLL_ALLREDUCE, algo, sendbuf, recvbuf, count * eb, static_cast<uint32_t>(eb), dtype,
                    stream);
}

extern "C" int mp_emu_alltoall(mp_ctx **ctxs, int n, const void *const *sendbufs, void *const *recvbufs,
                               uint64_t bytes_per_rank, int algo, void *stream) {
  if (!ctxs || n < 2 || !ctxs[0] || !sendbufs || !recvbufs) return MP_ERR_INVALID;
  return emu_collective(ctxs, n, MP_COLL_ALLTOALL, algo, sendbufs, recvbufs, bytes_per_rank, 1, MP_DT_U8, stream);
}

extern "C" int mp_emu_allreduce(mp_ctx **ctxs, int n, const void *const *sendbufs, void *const *recvbufs,
                                uint64_t count, int dtype, int op, int algo, void *stream) {
  if (!ctxs || n < 2 || !ctxs[0] || !sendbufs || !recvbufs) return MP_ERR_INVALID;
  const int eb = elem_bytes(dtype);
  if (eb == 0 || dtype == MP_DT_U8) return cfail(ctxs[0], MP_ERR_INVALID, "allreduce: unsupported dtype");
  if (op != MP_OP_SUM) return cfail(ctxs[0], MP_ERR_INVALID, "allreduce: unsupported op");
  return emu_collective(ctxs, n, MP_COLL_ALLREDUCE, algo, sendbufs, recvbufs, count * eb, static_cast<uint32_t>(eb),
                        dtype, stream);
}
