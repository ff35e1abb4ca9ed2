// calib.cpp — Step 1 of PAPER.md §4: extract the model parameters of every
// path once per topology, with the engine's own kernels (reading C12).
//
// Single-GPU loopback: the "links" are
//   direct        src HBM  → dst HBM
//   relay leg 1   src      → relay ring      leg 2  relay ring → dst
//   host leg 1    src      → pinned host ring (PCIe writes)   leg 2  host ring → dst (PCIe reads)
// Each link is timed with a direct-only fused launch between the two buffers
// (median of `reps` CUDA-event timings per size, L2 flushed before each), and
// T(n) = α + n/β is fitted by least squares weighted by 1/T² over the sizes.
// ε of a staging device is half the round trip of a flag ping-pong between two CTAs
// through that device's flag memory (the same release/acquire the pipeline uses).
#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstring>
#include <string>
#include <thread>
#include <vector>

#include "ctx.h"

using namespace mpx;

namespace {

int cfail(mp_ctx *c, int code, const std::string &msg) {
  c->last_error = msg;
  return code;
}

#define CKC(call)                                                                          \
  do {                                                                                     \
    cudaError_t e__ = (call);                                                              \
    if (e__ != cudaSuccess) return cfail(c, MP_ERR_CUDA, std::string(#call) + ": " + cudaGetErrorString(e__)); \
  } while (0)

struct Fit {
  double alpha, beta;
};

// Weighted least squares of T = α + n·g (g = 1/β), weights 1/T² (relative error).
Fit fit_hockney(const std::vector<double> &n, const std::vector<double> &t) {
  double s00 = 0, s01 = 0, s11 = 0, r0 = 0, r1 = 0;
  for (size_t i = 0; i < n.size(); ++i) {
    const double w = 1.0 / (t[i] * t[i]);
    s00 += w;
    s01 += w * n[i];
    s11 += w * n[i] * n[i];
    r0 += w * t[i];
    r1 += w * n[i] * t[i];
  }
  const double det = s00 * s11 - s01 * s01;
  double a = (r0 * s11 - r1 * s01) / det;
  double g = (s00 * r1 - s01 * r0) / det;
  if (!(a > 1e-7)) {
    // constraint α >= 1e-7 (Eq 14 needs α > 0): the convex objective's constrained
    // optimum is on the bound — refit the slope with α fixed there
    a = 1e-7;
    g = (r1 - a * s01) / s11;
  }
  if (!(g > 0)) g = t.back() / n.back();
  return Fit{a, 1.0 / g};
}

double median(std::vector<double> v) {
  std::sort(v.begin(), v.end());
  return v[v.size() / 2];
}

struct Bench {
  mp_ctx *c;
  cudaStream_t s = nullptr;
  cudaEvent_t e0 = nullptr, e1 = nullptr;
  void *flush = nullptr;
  uint64_t flush_bytes = 256ull << 20;
};

// One direct-only fused launch dst ← src of n bytes; returns seconds.
int time_copy(Bench &b, void *dst, const void *src, uint64_t n, int reps, double *out, int ctas = 0) {
  mp_ctx *c = b.c;
  std::vector<double> ts;
  for (int r = 0; r < reps + 1; ++r) {
    CKC(cudaMemsetAsync(b.flush, r & 0xff, b.flush_bytes, b.s));
    CKC(cudaEventRecord(b.e0, b.s));
    if (int st = launch_direct_copy(c, dst, src, n, b.s, ctas)) return st;
    CKC(cudaEventRecord(b.e1, b.s));
    CKC(cudaEventSynchronize(b.e1));
    float ms = 0;
    CKC(cudaEventElapsedTime(&ms, b.e0, b.e1));
    if (r > 0) ts.push_back(ms * 1e-3);  // first launch is a warm-up
  }
  *out = median(ts);
  return MP_OK;
}

// OMB-style timing (reading C21): `W` back-to-back copies of n bytes between the
// same buffers (no flush — a window of repeated sends), median over
// `reps` windows; returns seconds per message.  Each window is enqueued behind a spin
// kernel that outlasts the host's enqueue (~3 µs per launch), so its copies run back
// to back at GPU speed — launched from a stream, as a caller's messages are.  (Round 2
// first replayed the window from a CUDA graph: also GPU-speed, but a graph launches
// each kernel ~0.8 µs sooner than a stream does, and the bands then over-predicted
// stream-launched windows by 16-33 % at 4-16 MiB.)  Enqueued without the spin, a small
// message would be timed at the host's 2-3 µs per call instead (C27 models
// that part separately).
int time_window(Bench &b, void *dst, const void *src, uint64_t n, int reps, int W, double *out, int ctas = 0) {
  mp_ctx *c = b.c;
  std::vector<double> ts;
#ifdef MPX_GRAPH_WINDOWS  // (design experiment: the window replayed from a CUDA graph)
  {
    cudaGraph_t g = nullptr;
    cudaGraphExec_t ge = nullptr;
    CKC(cudaStreamBeginCapture(b.s, cudaStreamCaptureModeThreadLocal));
    int st = MP_OK;
    for (int w = 0; w < W && st == MP_OK; ++w) st = launch_direct_copy(c, dst, src, n, b.s, ctas);
    const cudaError_t ce = cudaStreamEndCapture(b.s, &g);
    if (st) {
      if (g) cudaGraphDestroy(g);
      return st;
    }
    CKC(ce);
    const cudaError_t ie = cudaGraphInstantiate(&ge, g, 0);
    cudaGraphDestroy(g);
    CKC(ie);
    for (int r = 0; r < reps + 1; ++r) {
      CKC(cudaEventRecord(b.e0, b.s));
      CKC(cudaGraphLaunch(ge, b.s));
      CKC(cudaEventRecord(b.e1, b.s));
      CKC(cudaEventSynchronize(b.e1));
      float ms = 0;
      CKC(cudaEventElapsedTime(&ms, b.e0, b.e1));
      if (r > 0) ts.push_back(ms * 1e-3 / W);
    }
    cudaGraphExecDestroy(ge);
    *out = median(ts);
    return MP_OK;
  }
#endif
  uint64_t spin_ns = 100000ull + 10000ull * static_cast<uint64_t>(W);
  for (int r = 0, redo = 0; r < reps + 1; ++r) {
    if (launch_spin(spin_ns, b.s) != 0) return cfail(c, MP_ERR_CUDA, "window spin launch");
    CKC(cudaEventRecord(b.e0, b.s));
    for (int w = 0; w < W; ++w)
      if (int st = launch_direct_copy(c, dst, src, n, b.s, ctas)) return st;
    CKC(cudaEventRecord(b.e1, b.s));
    // the spin must still be running once the whole window is enqueued (else the GPU
    // waited for the host inside the window): if not, redo with a longer spin
    const bool covered = cudaEventQuery(b.e0) == cudaErrorNotReady;
    CKC(cudaEventSynchronize(b.e1));
    if (!covered && redo < 4) {
      spin_ns *= 2;
      ++redo;
      --r;
      continue;
    }
    float ms = 0;
    CKC(cudaEventElapsedTime(&ms, b.e0, b.e1));
    if (r > 0) ts.push_back(ms * 1e-3 / W);  // first window is a warm-up
  }
  *out = median(ts);
  return MP_OK;
}

// Samples (n, t) of one link over `sizes` (<= cap): window-timed when `window`,
// else single copies with the L2 flushed before each.
int sample_link(Bench &b, void *dst, const void *src, const std::vector<uint64_t> &sizes, uint64_t cap, int reps,
                int ctas, bool window, std::vector<double> *n, std::vector<double> *t) {
  // long windows at small sizes: the events around a window cost a few µs of stream
  // time, which must not land in the per-message time (PDL makes a back-to-back small
  // message ~2 µs)
  auto win = [](uint64_t s) { return s <= (4ull << 20) ? 64 : (s <= (64ull << 20) ? 16 : 4); };
  const size_t first = n->size();
  for (uint64_t s : sizes) {
    if (s > cap) continue;
    double sec = 0;
    if (window) {
      if (int st = time_window(b, dst, src, s, reps, win(s), &sec, ctas)) return st;
    } else {
      if (int st = time_copy(b, dst, src, s, reps, &sec, ctas)) return st;
    }
    n->push_back(static_cast<double>(s));
    t->push_back(sec);
  }
  // A larger copy is never faster than a smaller one on the same link, so a window
  // that took more than 5 % longer than the next size's was disturbed (measured on
  // B200: a 64 KiB window at 1.45 µs beside 1.2 µs at 128 KiB, once in several fresh
  // boxes, which tilted its size band's fit by 25 %).  Such samples are re-timed (at
  // most twice each, keeping the faster), smallest size first.
  if (window)
    for (int pass = 0; pass < 2; ++pass) {
      bool again = false;
      for (size_t i = first; i + 1 < n->size(); ++i) {
        if ((*t)[i] <= 1.05 * (*t)[i + 1]) continue;
        double sec = 0;
        const uint64_t s = static_cast<uint64_t>((*n)[i]);
        if (int st = time_window(b, dst, src, s, reps, win(s), &sec, ctas)) return st;
        (*t)[i] = std::min((*t)[i], sec);
        again = true;
      }
      if (!again) break;
    }
  return MP_OK;
}

// Reading C20: band j is fitted on the samples with e_j <= n <= e_{j+1} (both
// inclusive; the last band unbounded); a band without two samples takes the fit of
// the nearest band above it that has two, else of the nearest below.  Returns false
// when no band has two samples.
bool fit_bands_impl(const std::vector<double> &n, const std::vector<double> &t, const std::vector<double> &edges,
                    std::vector<Fit> *out) {
  const int B = static_cast<int>(edges.size());
  std::vector<int> own(B, 0);
  std::vector<Fit> fits(B, Fit{0, 0});
  for (int j = 0; j < B; ++j) {
    const double lo = edges[j], hi = j + 1 < B ? edges[j + 1] : HUGE_VAL;
    std::vector<double> bn, bt;
    for (size_t i = 0; i < n.size(); ++i)
      if (n[i] >= lo && n[i] <= hi) {
        bn.push_back(n[i]);
        bt.push_back(t[i]);
      }
    if (bn.size() >= 2) {
      fits[j] = fit_hockney(bn, bt);
      own[j] = 1;
    }
  }
  for (int j = 0; j < B; ++j) {
    if (own[j]) continue;
    int from = -1;
    for (int i = j + 1; i < B && from < 0; ++i)
      if (own[i]) from = i;
    for (int i = j - 1; i >= 0 && from < 0; --i)
      if (own[i]) from = i;
    if (from < 0) return false;
    fits[j] = fits[from];
  }
  *out = fits;
  return true;
}

int fit_samples(mp_ctx *c, const std::vector<double> &n, const std::vector<double> &t,
                const std::vector<double> &edges, std::vector<Fit> *out) {
  if (!fit_bands_impl(n, t, edges, out))
    return cfail(c, MP_ERR_INVALID, "calibration needs at least two sizes in some band");
  return MP_OK;
}

// Fit one link.  ctas > 0 times the copy with that many CTAs: a staged leg is moved
// by a stage group of relay_ctas CTAs, so its β is what that group achieves.
int fit_link(Bench &b, void *dst, const void *src, const std::vector<uint64_t> &sizes, uint64_t cap,
             int reps, Fit *f, int ctas = 0) {
  std::vector<double> n, t;
  for (uint64_t s : sizes) {
    if (s > cap) continue;
    double sec = 0;
    if (int st = time_copy(b, dst, src, s, reps, &sec, ctas)) return st;
    n.push_back(static_cast<double>(s));
    t.push_back(sec);
  }
  if (n.size() < 2) return cfail(b.c, MP_ERR_INVALID, "calibration needs at least two sizes");
  *f = fit_hockney(n, t);
  return MP_OK;
}

// Two links timed concurrently (dst1 ← src1 on one stream, dst2 ← src2 on another,
// launched together), each fitted on its own times.
int sample_links_duplex(Bench &b, void *dst1, const void *src1, void *dst2, const void *src2,
                        const std::vector<uint64_t> &sizes, int reps, int ctas, bool flush, std::vector<double> *pn,
                        std::vector<double> *pt1, std::vector<double> *pt2) {
  mp_ctx *c = b.c;
  cudaStream_t s2 = nullptr;
  cudaEvent_t fork = nullptr, e2a = nullptr, e2b = nullptr;
  CKC(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
  CKC(cudaEventCreateWithFlags(&fork, cudaEventDisableTiming));
  CKC(cudaEventCreate(&e2a));
  CKC(cudaEventCreate(&e2b));
  std::vector<double> n, t1, t2;
  int st = MP_OK;
  for (uint64_t s : sizes) {
    std::vector<double> a, bb;
    for (int r = 0; r < reps + 1 && st == MP_OK; ++r) {
      if (flush) cudaMemsetAsync(b.flush, r & 0xff, b.flush_bytes, b.s);
      cudaEventRecord(fork, b.s);
      cudaStreamWaitEvent(s2, fork, 0);
      cudaEventRecord(b.e0, b.s);
      cudaEventRecord(e2a, s2);
      st = launch_direct_copy(c, dst1, src1, s, b.s, ctas);
      if (!st) st = launch_direct_copy(c, dst2, src2, s, s2, ctas);
      cudaEventRecord(b.e1, b.s);
      cudaEventRecord(e2b, s2);
      cudaEventSynchronize(b.e1);
      cudaEventSynchronize(e2b);
      float ms1 = 0, ms2 = 0;
      cudaEventElapsedTime(&ms1, b.e0, b.e1);
      cudaEventElapsedTime(&ms2, e2a, e2b);
      if (r > 0) {
        a.push_back(ms1 * 1e-3);
        bb.push_back(ms2 * 1e-3);
      }
    }
    if (st) break;
    n.push_back(static_cast<double>(s));
    t1.push_back(median(a));
    t2.push_back(median(bb));
  }
  cudaStreamSynchronize(s2);
  cudaStreamDestroy(s2);
  cudaEventDestroy(fork);
  cudaEventDestroy(e2a);
  cudaEventDestroy(e2b);
  if (st) return st;
  *pn = n;
  *pt1 = t1;
  *pt2 = t2;
  return MP_OK;
}

int fit_links_duplex(Bench &b, void *dst1, const void *src1, void *dst2, const void *src2,
                     const std::vector<uint64_t> &sizes, int reps, Fit *f1, Fit *f2, int ctas) {
  std::vector<double> n, t1, t2;
  if (int st = sample_links_duplex(b, dst1, src1, dst2, src2, sizes, reps, ctas, true, &n, &t1, &t2)) return st;
  if (n.size() < 2) return cfail(b.c, MP_ERR_INVALID, "calibration needs at least two sizes");
  *f1 = fit_hockney(n, t1);
  *f2 = fit_hockney(n, t2);
  return MP_OK;
}

int time_pingpong(Bench &b, uint64_t *flags, bool host, int iters, double *eps) {
  mp_ctx *c = b.c;
  if (host)
    std::memset(flags, 0, 16);
  else
    CKC(cudaMemsetAsync(flags, 0, 16, b.s));
  CKC(cudaEventRecord(b.e0, b.s));
  int e = launch_pingpong(flags, iters, static_cast<uint64_t>(c->timeout_s * 1e9), c->d_err, b.s);
  if (e) return cfail(c, MP_ERR_CUDA, "pingpong launch");
  c->launches += 1;
  CKC(cudaEventRecord(b.e1, b.s));
  CKC(cudaEventSynchronize(b.e1));
  float ms = 0;
  CKC(cudaEventElapsedTime(&ms, b.e0, b.e1));
  *eps = ms * 1e-3 / (2.0 * iters);
  return MP_OK;
}

// Time the staged path `idx` of the loopback pair alone carrying n bytes in k chunks
// for every k of a grid; return c = k_best / k* (clamped to [0.1, 10]).
int fit_phi(mp_ctx *c, int idx, uint64_t n, int reps, double *c_out) {
  mp_path paths[MP_MAX_PATHS];
  mp_path_params prm[MP_MAX_PATHS];
  int np = 0;
  mp_port_params port;
  if (int s = mp_get_model(c, 0, 0, paths, prm, &np, &port)) return s;
  PathModel pm;
  pm.kind = paths[idx].kind;
  pm.alpha = prm[idx].alpha;
  pm.beta = prm[idx].beta;
  pm.alpha2 = prm[idx].alpha2;
  pm.beta2 = prm[idx].beta2;
  pm.eps = prm[idx].eps;
  const double ks = k_star(pm, static_cast<double>(n), M_B200);
  Bench b;
  b.c = c;
  void *src = nullptr, *dst = nullptr;
  CKC(cudaStreamCreateWithFlags(&b.s, cudaStreamNonBlocking));
  CKC(cudaEventCreate(&b.e0));
  CKC(cudaEventCreate(&b.e1));
  CKC(cudaMalloc(&b.flush, b.flush_bytes));
  CKC(cudaMalloc(&src, n));
  CKC(cudaMalloc(&dst, n));
  mp_config cfg;
  std::memset(&cfg, 0, sizeof(cfg));
  cfg.npaths = np;
  for (int i = 0; i < np; ++i) cfg.path[i] = paths[i];
  cfg.bytes[idx] = n;
  double best_t = 1e30;
  uint32_t best_k = 1;
  int st = MP_OK;
  for (uint32_t k : {1u, 2u, 3u, 4u, 6u, 8u, 12u, 16u, 24u, 32u, 48u, 64u}) {
    const uint64_t A = c->opts.align, U = n / A;
    if (k > U || A * ((U + k - 1) / k) + (n - U * A) > c->slot_bytes) continue;
    cfg.chunks[idx] = k;
    std::vector<double> ts;
    for (int r = 0; r < reps + 1 && st == MP_OK; ++r) {
      cudaMemsetAsync(b.flush, r & 0xff, b.flush_bytes, b.s);
      cudaEventRecord(b.e0, b.s);
      st = mp_xfer(c, dst, src, n, &cfg, b.s);
      cudaEventRecord(b.e1, b.s);
      cudaEventSynchronize(b.e1);
      float ms = 0;
      cudaEventElapsedTime(&ms, b.e0, b.e1);
      if (r > 0) ts.push_back(ms * 1e-3);
    }
    if (st) break;
    const double t = median(ts);
    if (t < best_t) {
      best_t = t;
      best_k = k;
    }
  }
  cudaStreamSynchronize(b.s);
  cudaFree(src);
  cudaFree(dst);
  cudaFree(b.flush);
  cudaEventDestroy(b.e0);
  cudaEventDestroy(b.e1);
  cudaStreamDestroy(b.s);
  if (st) return st;
  const double cc = ks > 0 ? static_cast<double>(best_k) / ks : 1.0;
  *c_out = std::min(10.0, std::max(0.1, cc));
  return MP_OK;
}

// Multi-rank Step 1 (collective): every rank measures its own links — the NVLink
// put into its successor's heap (direct link and both relay legs, which are the same
// kind of link through NVSwitch), the host legs into/out of its own pinned segment,
// ε of a GPU stage by a flag ping-pong through the successor's memory, ε of the host
// stage through pinned memory — then all ranks exchange their measurements and
// install a model for every ordered pair (s, d): direct and leg 1 from s, relay leg 2
// and ε from the relay r, host leg 2 and ε from d; the shared port is s's egress.
struct LinkMeas {
  double da, db;          // NVLink put α, β (direct group)
  double ra, rb;          // NVLink put α, β with a stage group's CTAs (relay legs)
  double h1a, h1b;        // GPU → host α, β
  double h2a, h2b;        // host → GPU α, β
  double eps_dev, eps_host;
  double kappa;           // host duplex factor of this GPU (reading C25)
  double egress_b;        // C14 shared port: this GPU writing to every peer at once [B/s]
  double ingress_b;       // every peer writing into this GPU at once [B/s]
};

// Reading C14's shared port across GPUs: on NVSwitch every NVLink path of a pair leaves
// through the source's egress and enters through the destination's ingress, so the
// port of (s, d) is min(egress(s), ingress(d)) — measured here as aggregates, not as
// the one-destination direct copy (which would leave no room for a relay even where
// one peer stream cannot fill the links).  Egress of rank s: s copies n bytes into
// every peer's heap at once (one stream per peer), rounds serialised over s.  Ingress
// of rank d: every other rank copies n bytes into d's heap at once after a barrier;
// the aggregate is (W − 1)·n over the slowest copy.  Medians of `reps` rounds.
int aggregate_ports(mp_ctx *c, uint64_t n, int reps, double *egress, double *ingress) {
  const int W = c->world, me = c->rank;
  *egress = *ingress = 0.0;
  if (W < 2 || n == 0) return MP_OK;
  std::vector<cudaStream_t> st(W, nullptr);
  std::vector<cudaEvent_t> e0(W, nullptr), e1(W, nullptr);
  void *src = nullptr;
  int rc = MP_OK;
  auto ck = [&](cudaError_t e, const char *what) {
    if (e != cudaSuccess && rc == MP_OK) rc = cfail(c, MP_ERR_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
    return e == cudaSuccess;
  };
  ck(cudaMalloc(&src, n), "cudaMalloc");
  for (int r = 0; r < W && rc == MP_OK; ++r) {
    ck(cudaStreamCreateWithFlags(&st[r], cudaStreamNonBlocking), "stream");
    ck(cudaEventCreate(&e0[r]), "event");
    ck(cudaEventCreate(&e1[r]), "event");
  }
  if (rc == MP_OK) ck(cudaMemset(src, 0x6b, n), "memset");
  if (rc == MP_OK) ck(cudaDeviceSynchronize(), "sync");
  // every rank takes part in every barrier, even after a local failure (no hang)
  std::vector<double> eg, in;
  for (int rep = 0; rep < reps; ++rep) {
    for (int s = 0; s < W; ++s) {  // egress rounds
      if (int b = world_barrier(c)) return b;
      double t = 0.0;
      if (me == s && rc == MP_OK) {
        for (int r = 0; r < W; ++r)
          if (r != me) {
            ck(cudaEventRecord(e0[r], st[r]), "record");
            if (rc == MP_OK) rc = launch_direct_copy(c, c->peers[r].heap, src, n, st[r]);
            ck(cudaEventRecord(e1[r], st[r]), "record");
          }
        for (int r = 0; r < W; ++r)
          if (r != me && rc == MP_OK) ck(cudaEventSynchronize(e1[r]), "sync");
        // first start to last end across the streams
        float lo = 0, hi = 0;
        int first = -1;
        for (int r = 0; r < W && rc == MP_OK; ++r) {
          if (r == me) continue;
          if (first < 0) first = r;
          float a = 0, b = 0;
          ck(cudaEventElapsedTime(&a, e0[first], e0[r]), "elapsed");
          ck(cudaEventElapsedTime(&b, e0[first], e1[r]), "elapsed");
          lo = std::min(lo, a);
          hi = std::max(hi, b);
        }
        t = (hi - lo) * 1e-3;
        if (t > 0) eg.push_back(static_cast<double>(W - 1) * n / t);
      }
    }
    for (int d = 0; d < W; ++d) {  // ingress rounds
      if (int b = world_barrier(c)) return b;
      double t = 0.0;
      if (me != d && rc == MP_OK) {
        ck(cudaEventRecord(e0[d], st[d]), "record");
        if (rc == MP_OK) rc = launch_direct_copy(c, c->peers[d].heap, src, n, st[d]);
        ck(cudaEventRecord(e1[d], st[d]), "record");
        ck(cudaEventSynchronize(e1[d]), "sync");
        float ms = 0;
        ck(cudaEventElapsedTime(&ms, e0[d], e1[d]), "elapsed");
        t = ms * 1e-3;
      }
      std::vector<double> all(W);
      if (int b = world_allgather(c, &t, all.data(), sizeof(double))) return b;
      const double tmax = *std::max_element(all.begin(), all.end());
      if (me == d && tmax > 0) in.push_back(static_cast<double>(W - 1) * n / tmax);
    }
  }
  if (src) cudaFree(src);
  for (int r = 0; r < W; ++r) {
    if (st[r]) cudaStreamDestroy(st[r]);
    if (e0[r]) cudaEventDestroy(e0[r]);
    if (e1[r]) cudaEventDestroy(e1[r]);
  }
  if (rc) return rc;
  *egress = eg.empty() ? 0.0 : median(eg);
  *ingress = in.empty() ? 0.0 : median(in);
  return MP_OK;
}

// Sizes the band fits sample (C20/C21): powers of two from 4 KiB to 1 GiB, plus 1.5×
// powers of two from 6 to 96 MiB, where the loopback working set crosses the 126 MB L2
// and the per-message rate is furthest from a line.
std::vector<uint64_t> band_sizes() {
  std::vector<uint64_t> sizes;
  for (uint64_t s = 4096; s <= (1024ull << 20); s <<= 1) {
    sizes.push_back(s);
    if (s >= (4ull << 20) && s <= (64ull << 20)) sizes.push_back(s + s / 2);
  }
  return sizes;
}

// edges = {0}: the plain Step-1 fit (flushed single copies); more edges: one
// parameter set per size band (reading C20), window-timed (reading C21).
int calibrate_world(mp_ctx *c, std::vector<uint64_t> sizes, int reps, const std::vector<double> &edges,
                    bool window) {
  const int W = c->world, me = c->rank, succ = (c->rank + 1) % c->world;
  const int B = static_cast<int>(edges.size());
  // the successor's heap is used as the put target: nobody may have live buffers yet
  int32_t busy = c->heap.used_.empty() ? 0 : 1;
  std::vector<int32_t> all_busy(W);
  if (int s = world_allgather(c, &busy, all_busy.data(), sizeof(busy))) return s;
  for (int32_t v : all_busy)
    if (v) return cfail(c, MP_ERR_STATE, "multi-rank calibration needs empty receive heaps (call it before mp_alloc)");
  const uint64_t cap = std::min<uint64_t>(c->heap.size, 1024ull << 20);
  std::vector<uint64_t> sz;
  for (uint64_t s : sizes)
    if (s <= cap) sz.push_back(s);
  if (sz.size() < 2) sz = {cap / 4, cap / 2, cap};
  const uint64_t big = *std::max_element(sz.begin(), sz.end());

  Bench b;
  b.c = c;
  CKC(cudaSetDevice(c->device));
  CKC(cudaStreamCreateWithFlags(&b.s, cudaStreamNonBlocking));
  CKC(cudaEventCreate(&b.e0));
  CKC(cudaEventCreate(&b.e1));
  void *src = nullptr;
  CKC(cudaMalloc(&b.flush, b.flush_bytes));
  CKC(cudaMalloc(&src, big));
  CKC(cudaMemset(src, 0x5a, big));
  std::vector<LinkMeas> m(B, LinkMeas{});
  // Ranks sharing one GPU (several processes per device, e.g. under MPS) measure in
  // turn: measured at once they would share its HBM and every link would be fitted
  // at a fraction of its rate.  Ranks on distinct GPUs measure concurrently (each
  // link is used once: rank r puts into r + 1).
  bool shared_gpu = false;
  if (c->have_topo)
    for (int r = 0; r < W; ++r)
      for (int q = r + 1; q < W; ++q)
        shared_gpu = shared_gpu || std::memcmp(c->topo.gpu[r].uuid, c->topo.gpu[q].uuid, 16) == 0;
  auto measure = [&]() -> int {
    int st = MP_OK;
    std::vector<double> n, t;
    std::vector<Fit> fd, fr, fh1, fh2;
    if ((st = sample_link(b, c->peers[succ].heap, src, sz, big, reps, 0, window, &n, &t))) return st;
    if ((st = fit_samples(c, n, t, edges, &fd))) return st;
    n.clear();
    t.clear();
    if ((st = sample_link(b, c->peers[succ].heap, src, sz, big, reps, c->relay_ctas, window, &n, &t))) return st;
    if ((st = fit_samples(c, n, t, edges, &fr))) return st;
    double eps_host = 0, eps_dev = 0, kappa = 1.0;
    if (c->host_path) {
      // the own segment's ring of sender == me is never used for traffic
      uint8_t *hr = c->hseg[me] + bell_bytes(static_cast<uint32_t>(W)) + static_cast<uint64_t>(me) * c->hseg_per_src;
      const uint64_t hcap = static_cast<uint64_t>(c->slots) * c->host_stride;
      std::vector<uint64_t> hs;
      for (uint64_t s : sz)
        if (s <= std::min<uint64_t>(hcap, 64ull << 20)) hs.push_back(s);
      if (hs.size() < 2) hs = {hcap / 4, hcap / 2};
      const int hr_reps = std::max(3, reps / 2);
      n.clear();
      t.clear();
      if ((st = sample_link(b, hr, src, hs, hcap, hr_reps, c->relay_ctas, window, &n, &t))) return st;
      if ((st = fit_samples(c, n, t, edges, &fh1))) return st;
      n.clear();
      t.clear();
      if ((st = sample_link(b, src, hr, hs, hcap, hr_reps, c->relay_ctas, window, &n, &t))) return st;
      if ((st = fit_samples(c, n, t, edges, &fh2))) return st;
      if ((st = time_pingpong(b, c->h_probe, true, 500, &eps_host))) return st;
      // κ (reading C25, NEXT f2): both host legs of this GPU alone, then at once
      const uint64_t hk = std::min<uint64_t>(hcap / 2, 32ull << 20);
      if (big >= 2 * hk && hk >= (1u << 20)) {
        double up = 0, down = 0;
        std::vector<double> kn, k1, k2;
        uint8_t *sb = static_cast<uint8_t *>(src);
        if ((st = time_copy(b, hr, sb, hk, hr_reps, &up, c->relay_ctas))) return st;
        if ((st = time_copy(b, sb + big - hk, hr + hcap / 2, hk, hr_reps, &down, c->relay_ctas))) return st;
        if ((st = sample_links_duplex(b, hr, sb, sb + big - hk, hr + hcap / 2, {hk}, hr_reps, c->relay_ctas, true,
                                      &kn, &k1, &k2)))
          return st;
        kappa = std::min(1.0, 0.5 * (up / k1[0] + down / k2[0]));
      }
    }
    uint64_t *pf = reinterpret_cast<uint64_t *>(c->peers[succ].ctrl + c->L.probe);
    if ((st = time_pingpong(b, pf, false, 1000, &eps_dev))) return st;
    for (int j = 0; j < B; ++j) {
      m[j].da = fd[j].alpha;
      m[j].db = fd[j].beta;
      m[j].ra = fr[j].alpha;
      m[j].rb = fr[j].beta;
      if (c->host_path) {
        m[j].h1a = fh1[j].alpha;
        m[j].h1b = fh1[j].beta;
        m[j].h2a = fh2[j].alpha;
        m[j].h2b = fh2[j].beta;
      }
      m[j].eps_dev = eps_dev;
      m[j].eps_host = eps_host;
      m[j].kappa = std::max(kappa, 1e-3);
    }
    return st;
  };
  int st = MP_OK;
  if (shared_gpu) {
    for (int t = 0; t < W; ++t) {
      if (int e = world_barrier(c)) return e;
      if (t == me) st = measure();
    }
    if (int e = world_barrier(c)) return e;
  } else {
    st = measure();
  }
  cudaStreamSynchronize(b.s);
  cudaFree(src);
  cudaFree(b.flush);
  cudaEventDestroy(b.e0);
  cudaEventDestroy(b.e1);
  cudaStreamDestroy(b.s);
  int32_t ok = st == MP_OK ? 0 : 1;
  std::vector<int32_t> all_ok(W);
  if (int s = world_allgather(c, &ok, all_ok.data(), sizeof(ok))) return s;
  if (st) return st;
  for (int32_t v : all_ok)
    if (v) return cfail(c, MP_ERR_STATE, "calibration failed on another rank");
  {  // C14's shared port as aggregates (egress, ingress); heaps are still empty
    double eg = 0.0, in = 0.0;
    const uint64_t n_each = std::min<uint64_t>(cap, 256ull << 20);
    const int ae = aggregate_ports(c, n_each, std::max(3, reps / 2), &eg, &in);
    int32_t aok = ae ? 1 : 0;  // agree before the next collective: a local failure must not strand the peers
    std::vector<int32_t> all_aok(W);
    if (int s = world_allgather(c, &aok, all_aok.data(), sizeof(aok))) return s;
    if (ae) return ae;
    for (int32_t v : all_aok)
      if (v) return cfail(c, MP_ERR_STATE, "port calibration failed on another rank");
    for (int j = 0; j < B; ++j) {
      m[j].egress_b = eg;
      m[j].ingress_b = in;
    }
  }
  std::vector<LinkMeas> lm(static_cast<size_t>(W) * B);  // [rank][band]
  if (int s = world_allgather(c, m.data(), lm.data(), sizeof(LinkMeas) * B)) return s;

  for (int g = 0; g < W; ++g)  // reading C25: every GPU's duplex factor
    if (int e = mp_set_host_duplex(c, g, lm[static_cast<size_t>(g) * B].kappa)) return e;
  for (int s = 0; s < W; ++s)
    for (int d = 0; d < W; ++d) {
      if (s == d) continue;
      // φ multipliers of an existing model are kept (Step-1 band fits replace α, β only)
      mp_path_params old[MP_MAX_PATHS];
      int nold = 0;
      const bool keep_c = B > 1 && mp_get_model(c, s, d, nullptr, old, &nold, nullptr) == MP_OK;
      for (int j = 0; j < B; ++j) {
        const LinkMeas &S = lm[static_cast<size_t>(s) * B + j], &D = lm[static_cast<size_t>(d) * B + j];
        mp_path paths[MP_MAX_PATHS];
        mp_path_params prm[MP_MAX_PATHS];
        int np = 0;
        paths[np] = mp_path{MP_PATH_DIRECT, -1};
        prm[np++] = mp_path_params{S.da, S.db, 0, 0, 0, 1, 0, 1, 0};
        for (int r = 0; r < W; ++r) {
          if (r == s || r == d) continue;
          const LinkMeas &R = lm[static_cast<size_t>(r) * B + j];
          paths[np] = mp_path{MP_PATH_GPU, r};
          prm[np++] = mp_path_params{S.ra, S.rb, R.ra, R.rb, std::max(R.eps_dev, 1e-8), 1, 0, 1, 0};
        }
        if (c->host_path) {
          paths[np] = mp_path{MP_PATH_HOST, -1};
          prm[np++] = mp_path_params{S.h1a, S.h1b, D.h2a, D.h2b, std::max(D.eps_host, 1e-8), 1, 0, 0, 0};
        }
        if (keep_c && nold == np)
          for (int i = 0; i < np; ++i) prm[i].c = old[i].c;
        // the port of (s, d): min(egress(s), ingress(d)) (C14); the direct copy's β when
        // an aggregate is missing or lower (the port is never below one stream)
        double pb = S.db;
        if (S.egress_b > 0 && D.ingress_b > 0) pb = std::max(S.db, std::min(S.egress_b, D.ingress_b));
        mp_port_params port{S.da, pb};
        const int e = j == 0 ? mp_set_model(c, s, d, paths, prm, np, &port)
                             : mp_set_model_band(c, s, d, static_cast<uint64_t>(edges[j]), prm, np, &port);
        if (e) return e;
      }
    }
  if (c->relay_svc && W >= 3) return mp_calibrate_wake(c, 0, 0);  // C28 (mp_init: after the service starts)
  return world_barrier(c);
}

// Loopback size bands (reading C20/C21): every link of the pair (0, 0) is sampled
// window-timed over 4 KiB .. 1 GiB and fitted per band; ε, φ multipliers c, σ and w
// are kept from the installed model (mp_calibrate / mp_load_params).
int calibrate_loop_bands(mp_ctx *c, const std::vector<double> &edges, int reps) {
  const int B = static_cast<int>(edges.size());
  mp_path paths[MP_MAX_PATHS];
  mp_path_params base[MP_MAX_PATHS];
  int np = 0;
  if (int s = mp_get_model(c, 0, 0, paths, base, &np, nullptr)) return s;
  const std::vector<uint64_t> sizes = band_sizes();
  const uint64_t big = sizes.back();
  const uint64_t ring_cap = static_cast<uint64_t>(c->slots) * c->slot_bytes;
  Bench b;
  b.c = c;
  CKC(cudaSetDevice(c->device));
  CKC(cudaStreamCreateWithFlags(&b.s, cudaStreamNonBlocking));
  CKC(cudaEventCreate(&b.e0));
  CKC(cudaEventCreate(&b.e1));
  void *src = nullptr, *dst = nullptr;
  CKC(cudaMalloc(&b.flush, b.flush_bytes));
  CKC(cudaMalloc(&src, big));
  CKC(cudaMalloc(&dst, big));
  CKC(cudaMemset(src, 0x5a, big));
  int st = MP_OK;
  std::vector<Fit> fd, f1, f2, fh1, fh2;
  do {
    std::vector<double> n, t, t2;
    if ((st = sample_link(b, dst, src, sizes, big, reps, 0, true, &n, &t))) break;
    if ((st = fit_samples(c, n, t, edges, &fd))) break;
    if (c->n_loop_relays > 0) {
      uint8_t *ring = c->rings[0].data;
      n.clear();
      t.clear();
      if ((st = sample_link(b, ring, src, sizes, ring_cap, reps, c->relay_ctas, true, &n, &t))) break;
      if ((st = fit_samples(c, n, t, edges, &f1))) break;
      n.clear();
      t.clear();
      if ((st = sample_link(b, dst, ring, sizes, ring_cap, reps, c->relay_ctas, true, &n, &t))) break;
      if ((st = fit_samples(c, n, t, edges, &f2))) break;
    }
    if (c->host_path) {
      uint8_t *hr = c->rings[c->n_loop_relays].data;
      std::vector<uint64_t> hs;
      for (uint64_t s : sizes)
        if (s <= std::min<uint64_t>(ring_cap / 2, 64ull << 20)) hs.push_back(s);
      n.clear();
      t.clear();
      if ((st = sample_links_duplex(b, hr, src, dst, hr + ring_cap / 2, hs, std::max(3, reps / 2), c->relay_ctas,
                                    false, &n, &t, &t2)))
        break;
      if ((st = fit_samples(c, n, t, edges, &fh1))) break;
      if ((st = fit_samples(c, n, t2, edges, &fh2))) break;
    }
  } while (false);
  cudaStreamSynchronize(b.s);
  cudaFree(src);
  cudaFree(dst);
  cudaFree(b.flush);
  cudaEventDestroy(b.e0);
  cudaEventDestroy(b.e1);
  cudaStreamDestroy(b.s);
  if (st) return st;
  int32_t derr = 0;
  CKC(cudaMemcpy(&derr, c->d_err, sizeof(derr), cudaMemcpyDeviceToHost));
  if (derr) return cfail(c, MP_ERR_TIMEOUT, "calibration copy timed out");
  for (int j = 0; j < B; ++j) {
    mp_path_params prm[MP_MAX_PATHS];
    for (int i = 0; i < np; ++i) {
      prm[i] = base[i];
      if (paths[i].kind == MP_PATH_DIRECT) {
        prm[i].alpha = fd[j].alpha;
        prm[i].beta = fd[j].beta;
      } else if (paths[i].kind == MP_PATH_GPU) {
        prm[i].alpha = f1[j].alpha;
        prm[i].beta = f1[j].beta;
        prm[i].alpha2 = f2[j].alpha;
        prm[i].beta2 = f2[j].beta;
      } else {
        prm[i].alpha = fh1[j].alpha;
        prm[i].beta = fh1[j].beta;
        prm[i].alpha2 = fh2[j].alpha;
        prm[i].beta2 = fh2[j].beta;
      }
    }
    mp_port_params port{fd[j].alpha, 2.0 * fd[j].beta};  // HBM: read + write per direct byte
    const int e = j == 0 ? mp_set_model(c, 0, 0, paths, prm, np, &port)
                         : mp_set_model_band(c, 0, 0, static_cast<uint64_t>(edges[j]), prm, np, &port);
    if (e) return e;
  }
  return MP_OK;
}

}  // namespace

extern "C" int mp_calibrate_bands(mp_ctx *c, const uint64_t *edges_in, int nedges, int reps) {
  if (!c) return MP_ERR_INVALID;
  if (c->model_only) return cfail(c, MP_ERR_STATE, "model-only context");
  if (c->emulated) return cfail(c, MP_ERR_UNSUPPORTED, "calibration: not in an emulated world (no links to time)");
  if (reps <= 0) reps = 5;
  std::vector<double> edges;
  if (edges_in && nedges > 0) {
    if (edges_in[0] != 0) return cfail(c, MP_ERR_INVALID, "band edges must start at 0");
    for (int j = 0; j < nedges; ++j) {
      if (j > 0 && edges_in[j] <= edges_in[j - 1]) return cfail(c, MP_ERR_INVALID, "band edges must increase");
      edges.push_back(static_cast<double>(edges_in[j]));
    }
  } else {
    for (uint64_t e : {0ull, 64ull << 10, 256ull << 10, 4ull << 20, 8ull << 20, 16ull << 20, 32ull << 20, 48ull << 20,
                       64ull << 20, 128ull << 20})
      edges.push_back(static_cast<double>(e));
  }
  if (c->world != 1) {
    if (int s = calibrate_world(c, band_sizes(), reps, edges, true)) return s;
    int32_t derr = 0;
    CKC(cudaMemcpy(&derr, c->d_err, sizeof(derr), cudaMemcpyDeviceToHost));
    if (derr) return cfail(c, MP_ERR_TIMEOUT, "calibration probe timed out");
    return MP_OK;
  }
  return calibrate_loop_bands(c, edges, reps);
}

// NEXT f2 window / duplex calibration (readings C24, C25, C27), loopback pair (0, 0).
//   h_sub (C27) = the host's time per mp_xfer call: the marginal host-clock cost of
//                 one more 64 KiB direct-only message in an OMB-style window (enqueue,
//                 wait): (t(64 calls) − t(16 calls)) / 48, medians of 2·reps;
//   per path alone and per size: T1 = one message on an idle stream, TW = W messages
//   back to back (CUDA events around the enqueue, a stream sync before each window);
//   (h_i, τ) = mp_fit_window(h_sub): τ = median(T1 − mp_predict) over the direct
//   path's sizes, clamped >= 0; the steady per-message time s = (TW − T1)/(W − 1) =
//   max(a, T1 − τ − a, h_sub), read in the serve-bound branch (s > h_sub):
//   a = T1 − τ − s; h_i = median over those sizes of max(0, a);
//   then τ += the host's completion overhead of a window, as osu_bw sees it (its
//   wait-all): the median over the direct path's sizes of the host-clock time
//   of one message (enqueue + stream synchronisation) minus its device time.
// κ of this GPU = the host legs' duplex / simplex rate (D2H and H2D alone, then both at
// once, 64 MiB).
extern "C" int mp_calibrate_window(mp_ctx *c, const uint64_t *sizes_in, int nsizes, int window, int reps) {
  if (!c) return MP_ERR_INVALID;
  if (c->model_only) return cfail(c, MP_ERR_STATE, "model-only context");
  if (c->emulated) return cfail(c, MP_ERR_UNSUPPORTED, "calibration: not in an emulated world (no links to time)");
  if (c->world != 1) return cfail(c, MP_ERR_UNSUPPORTED, "mp_calibrate_window: loopback contexts only");
  if (window <= 0) window = 16;
  if (window < 2) return cfail(c, MP_ERR_INVALID, "window must be >= 2");
  if (reps <= 0) reps = 7;
  std::vector<uint64_t> sizes;
  if (sizes_in && nsizes > 0)
    sizes.assign(sizes_in, sizes_in + nsizes);
  else
    sizes = {64ull << 10, 1ull << 20, 4ull << 20, 16ull << 20, 64ull << 20};
  uint64_t big = 0;
  for (uint64_t s : sizes) big = std::max(big, s);
  if (big == 0) return cfail(c, MP_ERR_INVALID, "sizes must be > 0");
  const uint64_t ring_cap = static_cast<uint64_t>(c->slots) * c->slot_bytes;
  const uint64_t hn = std::min<uint64_t>(64ull << 20, ring_cap / 2);  // κ probe size
  if (c->host_path) big = std::max(big, hn);
  mp_path paths[MP_MAX_PATHS];
  int np = 0;
  if (int s = mp_paths(c, 0, 0, paths, &np)) return s;
  Bench b;
  b.c = c;
  CKC(cudaSetDevice(c->device));
  CKC(cudaStreamCreateWithFlags(&b.s, cudaStreamNonBlocking));
  CKC(cudaEventCreate(&b.e0));
  CKC(cudaEventCreate(&b.e1));
  void *src = nullptr, *dst = nullptr;
  CKC(cudaMalloc(&b.flush, b.flush_bytes));
  CKC(cudaMalloc(&src, big));
  CKC(cudaMalloc(&dst, big));
  CKC(cudaMemset(src, 0x3c, big));
  CKC(cudaDeviceSynchronize());
  int st = MP_OK;
  using clk = std::chrono::steady_clock;
  auto timed = [&](const mp_config &cfg, uint64_t n, int W, double *out) -> int {
    std::vector<double> ts;
    for (int r = 0; r < reps + 1; ++r) {
      CKC(cudaStreamSynchronize(b.s));
      CKC(cudaEventRecord(b.e0, b.s));
      for (int w = 0; w < W; ++w)
        if (int e = mp_xfer(c, dst, src, n, &cfg, b.s)) return e;
      CKC(cudaEventRecord(b.e1, b.s));
      CKC(cudaEventSynchronize(b.e1));
      float ms = 0;
      CKC(cudaEventElapsedTime(&ms, b.e0, b.e1));
      if (r > 0) ts.push_back(ms * 1e-3);
    }
    *out = median(ts);
    return MP_OK;
  };
  auto timed_host = [&](const mp_config &cfg, uint64_t n, double *out) -> int {  // enqueue + wait-all
    std::vector<double> ts;
    for (int r = 0; r < reps + 1; ++r) {
      CKC(cudaStreamSynchronize(b.s));
      const auto t0 = clk::now();
      if (int e = mp_xfer(c, dst, src, n, &cfg, b.s)) return e;
      CKC(cudaStreamSynchronize(b.s));
      if (r > 0) ts.push_back(std::chrono::duration<double>(clk::now() - t0).count());
    }
    *out = median(ts);
    return MP_OK;
  };
  // C27: the host's submission time per call
  double h_sub = 0.0;
  {
    mp_config d4;
    std::memset(&d4, 0, sizeof(d4));
    d4.npaths = np;
    for (int j = 0; j < np; ++j) d4.path[j] = paths[j];
    d4.bytes[0] = 65536;
    d4.chunks[0] = 1;
    // the marginal host-clock cost of one more call in an OMB-style window (enqueue
    // W calls, wait for them): (t(64) − t(16)) / 48 — fixed costs (the first launch on
    // an idle stream, the wait) cancel.  64 KiB messages: their GPU time is below the
    // host's, and long enough for the next launch to overlap them (a 4 KiB kernel is
    // launch-bound on the GPU itself: ~2.9 µs per message vs ~2.0 µs from 64 KiB up)
    // Each t(W) is the mean over 50 consecutive windows, after 0.2 s of them: a
    // sustained window loop runs at the GPU's boost clock, isolated bursts do not (and
    // take ~2.9 µs per message instead of ~2.0).
    auto burst = [&](int W, double *out) -> int {
      std::vector<double> ts;
      const auto warm = clk::now();
      while (std::chrono::duration<double>(clk::now() - warm).count() < 0.2) {
        for (int w = 0; w < W; ++w)
          if (int e = mp_xfer(c, dst, src, 65536, &d4, b.s)) return e;
        CKC(cudaStreamSynchronize(b.s));
      }
      for (int r = 0; r < reps; ++r) {
        const auto t0 = clk::now();
        for (int it = 0; it < 50; ++it) {
          for (int w = 0; w < W; ++w)
            if (int e = mp_xfer(c, dst, src, 65536, &d4, b.s)) return e;
          CKC(cudaStreamSynchronize(b.s));
        }
        ts.push_back(std::chrono::duration<double>(clk::now() - t0).count() / 50);
      }
      *out = median(ts);
      return MP_OK;
    };
    double t16 = 0.0, t64 = 0.0;
    if ((st = burst(16, &t16)) || (st = burst(64, &t64))) return st;
    std::vector<double> hs{std::max(0.0, (t64 - t16) / 48.0)};
    CKC(cudaStreamSynchronize(b.s));
    if (st) return st;
    h_sub = median(hs);
  }
  struct Sample {
    int path;
    double t1, tw, pred, t1_host;
  };
  std::vector<Sample> smp;
  const uint64_t slot_lim = c->opts.slot_bytes ? c->opts.slot_bytes : c->slot_bytes;
  for (int i = 0; i < np && st == MP_OK; ++i)
    for (uint64_t n : sizes) {
      mp_config cfg;
      std::memset(&cfg, 0, sizeof(cfg));
      cfg.npaths = np;
      for (int j = 0; j < np; ++j) cfg.path[j] = paths[j];
      cfg.bytes[i] = n;
      cfg.chunks[0] = 1;
      if (i > 0) {
        uint64_t k = std::max<uint64_t>(8, (n + slot_lim - 1) / slot_lim);
        k = std::min<uint64_t>(k, std::max<uint64_t>(1, n / std::max<uint64_t>(1, c->opts.c_min)));
        cfg.chunks[i] = static_cast<uint32_t>(std::max<uint64_t>(1, k));
        if ((n + cfg.chunks[i] - 1) / cfg.chunks[i] > slot_lim) continue;
      }
      Sample sm{i, 0, 0, 0, 0};
      if ((st = mp_predict(c, 0, 0, n, &cfg, &sm.pred))) break;
      if ((st = timed(cfg, n, 1, &sm.t1))) break;
      if ((st = timed(cfg, n, window, &sm.tw))) break;
      if (i == 0 && (st = timed_host(cfg, n, &sm.t1_host))) break;
      smp.push_back(sm);
    }
  // κ: host legs alone and at once (reading C25)
  double kappa = 1.0;
  if (st == MP_OK && c->host_path) {
    uint8_t *hr = c->rings[c->n_loop_relays].data;
    double up = 0, down = 0;
    std::vector<double> n, t1, t2;
    if (!(st = time_copy(b, hr, src, hn, reps, &up, c->relay_ctas)) &&
        !(st = time_copy(b, dst, hr + ring_cap / 2, hn, reps, &down, c->relay_ctas)) &&
        !(st = sample_links_duplex(b, hr, src, dst, hr + ring_cap / 2, {hn}, reps, c->relay_ctas, true, &n, &t1,
                                   &t2)))
      kappa = std::min(1.0, 0.5 * (up / t1[0] + down / t2[0]));
  }
  cudaStreamSynchronize(b.s);
  cudaFree(src);
  cudaFree(dst);
  cudaFree(b.flush);
  cudaEventDestroy(b.e0);
  cudaEventDestroy(b.e1);
  cudaStreamDestroy(b.s);
  if (st) return st;
  int32_t derr = 0;
  CKC(cudaMemcpy(&derr, c->d_err, sizeof(derr), cudaMemcpyDeviceToHost));
  if (derr) return cfail(c, MP_ERR_TIMEOUT, "window calibration transfer timed out");
  if (smp.empty()) return cfail(c, MP_ERR_INVALID, "no calibration sample fits the staging rings");
  std::vector<int> sp;
  std::vector<double> s1, sw, spred;
  for (const Sample &sm : smp) {
    sp.push_back(sm.path);
    s1.push_back(sm.t1);
    sw.push_back(sm.tw);
    spred.push_back(sm.pred);
  }
  double h[MP_MAX_PATHS], tau = 0.0;
  if (int e = mp_fit_window(sp.data(), s1.data(), sw.data(), spred.data(), static_cast<int>(smp.size()), window, np,
                            h_sub, h, &tau))
    return cfail(c, e, "window fit failed");
  std::vector<double> sync;
  for (const Sample &sm : smp)
    if (sm.path == 0) sync.push_back(sm.t1_host - sm.t1);
  if (!sync.empty()) tau += std::max(0.0, median(sync));
  if (int e = mp_set_window_model(c, 0, 0, h, np, tau)) return e;
  if (int e = mp_set_submit_time(c, h_sub)) return e;
  if (int e = mp_set_host_duplex(c, c->rank, std::max(kappa, 1e-3))) return e;
  return MP_OK;
}

// Reading C28: the relay wake A of every relay rank r (multi-rank, collective, after
// the relay service is up, no traffic in flight).  Pair (s, d) = (r + 1, r + 2) mod W
// sends two relay-only messages of `bytes` (k = 1, above the eager limit) through r
// right after r's relay kernels have gone idle (linger + 1 ms of quiet).  The sender
// enqueues both first (its gate kernels wait on the device for the clear-to-send);
// after a barrier the receiver times recv 1 and recv 2 back to back on its stream,
// so no host skew enters.  Message 1 pays the relay's start (doorbell → service thread
// → kernel launch), message 2 finds the kernel lingering: t1 = O + max(T, A + k·s2),
// t2 = O + T (T = C3's time of the pair's model, O = per-message costs both pay), so
// when the wake binds (median(t1 − t2) > 1 µs) A = T − k·s2 + median(t1 − t2) (k = 1
// unless a slot is smaller than n: A = s1 + the median), else A = 0 (a wake that never
// binds changes no prediction).  Every
// GPU-staged path via r of every pair model and band takes wake = A_r;
// MPX_RELAY_WAKE_US overrides the probe.  calibrate_world re-runs it (its fresh models
// start at wake 0) when the relay service is up.
extern "C" int mp_calibrate_wake(mp_ctx *c, uint64_t bytes, int reps) {
  if (!c) return MP_ERR_INVALID;
  if (c->model_only) return cfail(c, MP_ERR_STATE, "model-only context");
  if (c->emulated) return cfail(c, MP_ERR_UNSUPPORTED, "calibration: not in an emulated world (no links to time)");
  const int W = c->world, me = c->rank;
  if (W < 3) return MP_OK;  // no relay ranks
  if (reps <= 0) reps = 7;
  if (bytes == 0) bytes = 2ull << 20;
  const uint64_t A = c->opts.align;
  bytes = std::max<uint64_t>(bytes, (c->eager_max / A + 1) * A);
  // chunks of at most a staging slot (k = 1 unless the slots are small)
  const uint64_t per = std::max<uint64_t>(A, (c->slot_bytes - A) / A * A);
  const uint32_t k = static_cast<uint32_t>((bytes + per - 1) / per);
  std::vector<double> wake(W, 0.0);
  if (const char *env = std::getenv("MPX_RELAY_WAKE_US")) {
    for (double &w : wake) w = std::max(0.0, std::atof(env) / 1e6);
  } else {
    if (!c->relay_svc) return cfail(c, MP_ERR_STATE, "mp_calibrate_wake: no relay service");
    const auto quiet = std::chrono::nanoseconds(world_relay_linger_ns(c)) + std::chrono::milliseconds(1);
    void *rbuf = nullptr, *src = nullptr;
    cudaStream_t st = nullptr;
    cudaEvent_t ev[3] = {nullptr, nullptr, nullptr};
    // every rank needs a probe buffer in its heap; a heap too small for one leaves
    // every wake at 0 (decided collectively: a rank that skips would strand its peers)
    int32_t no_room = mp_alloc(c, bytes, &rbuf) == MP_OK ? 0 : 1;
    c->last_error.clear();
    std::vector<int32_t> rooms(W);
    if (int e = world_allgather(c, &no_room, rooms.data(), sizeof(no_room))) return e;
    bool skip = false;
    for (int32_t v : rooms) skip = skip || v;
    // rc: a local failure — this rank stops probing but keeps joining every barrier, so
    // its peers are not stranded; brc: a failed barrier (the bootstrap is gone) — stop.
    int rc = MP_OK, brc = MP_OK;
    double mine = 0.0;  // this rank's result as the receiver of relay (me − 2) mod W
    if (!skip) {
      if (cudaMalloc(&src, bytes) != cudaSuccess || cudaMemset(src, 0x3c, bytes) != cudaSuccess ||
          cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) != cudaSuccess)
        rc = cfail(c, MP_ERR_CUDA, "mp_calibrate_wake: buffers");
      for (cudaEvent_t &e : ev)
        if (!rc && cudaEventCreate(&e) != cudaSuccess) rc = cfail(c, MP_ERR_CUDA, "mp_calibrate_wake: events");
      for (int r = 0; r < W && !brc; ++r) {
        const int s = (r + 1) % W, d = (r + 2) % W;
        const bool end = me == s || me == d;
        mp_config cfg{};
        mp_path_params prm[MP_MAX_PATHS];
        int np = 0, idx = -1;
        if (end && !rc) rc = mp_get_model(c, s, d, cfg.path, prm, &np, nullptr);
        for (int i = 0; i < np; ++i)
          if (cfg.path[i].kind == MP_PATH_GPU && cfg.path[i].via == r) idx = i;
        if (end && !rc && idx < 0)
          rc = cfail(c, MP_ERR_TOPOLOGY, "mp_calibrate_wake: pair has no path via relay " + std::to_string(r));
        if (me == s && !rc) {
          cfg.npaths = np;
          cfg.bytes[idx] = bytes;
          cfg.chunks[0] = 1;
          cfg.chunks[idx] = k;
        }
        std::vector<double> diffs;
        for (int i = 0; i < reps && !brc; ++i) {
          if ((brc = world_barrier(c))) break;
          std::this_thread::sleep_for(quiet);
          if (me == s)
            for (int j = 0; j < 2 && !rc; ++j) rc = mp_send(c, src, bytes, d, -1000 - j, &cfg, st);
          if ((brc = world_barrier(c))) break;
          if (me == d && !rc) {
            cudaEventRecord(ev[0], st);
            rc = mp_recv(c, rbuf, bytes, s, -1000, st);
            cudaEventRecord(ev[1], st);
            if (!rc) rc = mp_recv(c, rbuf, bytes, s, -1001, st);
            cudaEventRecord(ev[2], st);
          }
          if (end && !rc && cudaStreamSynchronize(st) != cudaSuccess)
            rc = cfail(c, MP_ERR_CUDA, "mp_calibrate_wake: stream");
          if (me == d && !rc) {
            float t1 = 0, t2 = 0;
            cudaEventElapsedTime(&t1, ev[0], ev[1]);
            cudaEventElapsedTime(&t2, ev[1], ev[2]);
            if (std::getenv("MPX_WAKE_DEBUG"))
              std::fprintf(stderr, "wake probe relay %d rep %d: t1 %.2f us t2 %.2f us (k %u)\n", r, i, t1 * 1e3,
                           t2 * 1e3, k);
            diffs.push_back((static_cast<double>(t1) - static_cast<double>(t2)) * 1e-3);
          }
        }
        if (!rc && me == d && !diffs.empty()) {
          // t1 − t2 = max(0, A + k·s2 − T) with T = C3's time of the pair's model (the
          // fixed per-message costs — clear-to-send, launches — cancel in the difference)
          const mp_path_params &q = prm[idx];
          const double m = static_cast<double>(bytes) / k;
          const double s1 = q.alpha + m / q.beta, s2 = q.eps + q.alpha2 + m / q.beta2;
          const double T = s1 + s2 + (k - 1) * std::max(s1, s2);
          const double delta = median(diffs);
          mine = delta > 1e-6 ? std::max(0.0, T - k * s2 + delta) : 0.0;
        }
      }
    }
    if (st) cudaStreamSynchronize(st);
    for (cudaEvent_t e : ev)
      if (e) cudaEventDestroy(e);
    if (st) cudaStreamDestroy(st);
    if (src) cudaFree(src);
    if (rbuf) mp_free(c, rbuf);
    if (brc) return brc;
    int32_t ok = rc ? 1 : 0;
    std::vector<int32_t> all_ok(W);
    if (int e = world_allgather(c, &ok, all_ok.data(), sizeof(ok))) return e;
    if (rc) return rc;
    for (int32_t v : all_ok)
      if (v) return cfail(c, MP_ERR_STATE, "wake calibration failed on another rank");
    std::vector<double> got(W);
    if (int e = world_allgather(c, &mine, got.data(), sizeof(double))) return e;
    for (int d = 0; d < W; ++d) wake[(d - 2 + W) % W] = got[d];  // rank d measured relay d − 2
  }
  auto apply = [&](PairModel &m) {
    for (PathModel &q : m.paths)
      if (q.kind == K_GPU && q.via >= 0 && q.via < W) q.wake = wake[q.via];
  };
  for (auto &kv : c->models) apply(kv.second);
  for (auto &kv : c->bands)
    for (auto &b : kv.second) apply(b.second);
  c->cache.clear();
  return world_barrier(c);
}

// The C24 estimator of mp_calibrate_window on given samples (pure host arithmetic).
// τ is a property of the window (idle-stream launch + the host wait), the same for
// every config: it is read off the direct path (path 0), which carries no
// staging-model error.  Per path, the steady per-message time s = (TW − T1)/(W − 1) =
// max(a, T1 − τ − a), read in the serve-bound branch: a = T1 − τ − s.
extern "C" int mp_fit_window(const int *path, const double *t1, const double *tw, const double *pred, int m,
                             int window, int npaths, double h_sub, double *h, double *tau) {
  if (!path || !t1 || !tw || !pred || !h || !tau || m < 1 || window < 2 || npaths < 1 || npaths > MP_MAX_PATHS)
    return MP_ERR_INVALID;
  std::vector<double> taus;
  for (int j = 0; j < m; ++j) {
    if (path[j] < 0 || path[j] >= npaths || !(t1[j] > 0.0) || !(tw[j] > 0.0)) return MP_ERR_INVALID;
    if (path[j] == 0) taus.push_back(t1[j] - pred[j]);
  }
  *tau = taus.empty() ? 0.0 : std::max(0.0, median(taus));
  for (int i = 0; i < npaths; ++i) {
    std::vector<double> as;
    for (int j = 0; j < m; ++j)
      if (path[j] == i) {
        const double steady = (tw[j] - t1[j]) / static_cast<double>(window - 1);
        if (!(steady > h_sub * (1.0 + 1e-6))) continue;  // submission-bound (C27): no information on a_i
        as.push_back(std::max(0.0, t1[j] - *tau - steady));
      }
    h[i] = as.empty() ? 0.0 : median(as);
  }
  return MP_OK;
}

extern "C" int mp_fit_hockney(const double *n, const double *t, int m, double *alpha, double *beta) {
  if (!n || !t || !alpha || !beta || m < 2) return MP_ERR_INVALID;
  for (int i = 0; i < m; ++i)
    if (!(t[i] > 0.0) || !(n[i] >= 0.0)) return MP_ERR_INVALID;
  const Fit f = fit_hockney(std::vector<double>(n, n + m), std::vector<double>(t, t + m));
  *alpha = f.alpha;
  *beta = f.beta;
  return MP_OK;
}

extern "C" int mp_fit_bands(const double *n, const double *t, int m, const double *edges, int nedges,
                            double *alpha, double *beta) {
  if (!n || !t || !edges || !alpha || !beta || m < 0 || nedges < 1 || edges[0] != 0.0) return MP_ERR_INVALID;
  for (int j = 1; j < nedges; ++j)
    if (!(edges[j] > edges[j - 1])) return MP_ERR_INVALID;
  for (int i = 0; i < m; ++i)
    if (!(t[i] > 0.0) || !(n[i] >= 0.0)) return MP_ERR_INVALID;
  std::vector<Fit> fits;
  if (!fit_bands_impl(std::vector<double>(n, n + m), std::vector<double>(t, t + m),
                      std::vector<double>(edges, edges + nedges), &fits))
    return MP_ERR_INVALID;
  for (int j = 0; j < nedges; ++j) {
    alpha[j] = fits[j].alpha;
    beta[j] = fits[j].beta;
  }
  return MP_OK;
}

extern "C" int mp_calibrate(mp_ctx *c, const uint64_t *sizes_in, int nsizes, int reps) {
  if (!c) return MP_ERR_INVALID;
  if (c->model_only) return cfail(c, MP_ERR_STATE, "model-only context");
  if (c->emulated) return cfail(c, MP_ERR_UNSUPPORTED, "calibration: not in an emulated world (no links to time)");
  if (reps <= 0) reps = 5;
  if (c->world != 1) {
    std::vector<uint64_t> sizes;
    if (sizes_in && nsizes > 0)
      sizes.assign(sizes_in, sizes_in + nsizes);
    else
      for (uint64_t s = 16ull << 20; s <= (1024ull << 20); s <<= 1) sizes.push_back(s);
    int32_t derr = 0;
    if (int s = calibrate_world(c, sizes, reps, std::vector<double>{0.0}, false)) return s;
    CKC(cudaMemcpy(&derr, c->d_err, sizeof(derr), cudaMemcpyDeviceToHost));
    if (derr) return cfail(c, MP_ERR_TIMEOUT, "calibration probe timed out");
    return MP_OK;
  }
  // Default sizes: the asymptotic range (C12).  A local HBM→HBM copy only shows its
  // steady-state rate once the working set exceeds the 126 MB L2, so the direct link
  // is fitted on 128 MiB .. 1 GiB; the ring legs on what the ring holds.
  std::vector<uint64_t> sizes;
  if (sizes_in && nsizes > 0)
    sizes.assign(sizes_in, sizes_in + nsizes);
  else
    for (uint64_t s = 16ull << 20; s <= (1024ull << 20); s <<= 1) sizes.push_back(s);
  const uint64_t big = *std::max_element(sizes.begin(), sizes.end());
  std::vector<uint64_t> direct_sizes;
  for (uint64_t s : sizes)
    if (s >= (128ull << 20)) direct_sizes.push_back(s);
  if (direct_sizes.size() < 2) direct_sizes = sizes;

  Bench b;
  b.c = c;
  CKC(cudaSetDevice(c->device));
  CKC(cudaStreamCreateWithFlags(&b.s, cudaStreamNonBlocking));
  CKC(cudaEventCreate(&b.e0));
  CKC(cudaEventCreate(&b.e1));
  void *src = nullptr, *dst = nullptr;
  CKC(cudaMalloc(&b.flush, b.flush_bytes));
  CKC(cudaMalloc(&src, big));
  CKC(cudaMalloc(&dst, big));
  CKC(cudaMemset(src, 0x5a, big));

  int st = MP_OK;
  Fit fd{}, f1{}, f2{}, fh1{}, fh2{};
  double eps_dev = 0, eps_host = 0;
  const uint64_t ring_cap = static_cast<uint64_t>(c->slots) * c->slot_bytes;
  do {
    if ((st = fit_link(b, dst, src, direct_sizes, big, reps, &fd))) break;
    if (c->n_loop_relays > 0) {
      uint8_t *ring = c->rings[0].data;
      if ((st = fit_link(b, ring, src, sizes, ring_cap, reps, &f1, c->relay_ctas))) break;
      if ((st = fit_link(b, dst, ring, sizes, ring_cap, reps, &f2, c->relay_ctas))) break;
      if ((st = time_pingpong(b, c->d_probe, false, 2000, &eps_dev))) break;
    }
    if (c->host_path) {
      uint8_t *hr = c->rings[c->n_loop_relays].data;
      std::vector<uint64_t> hs;
      for (uint64_t s : sizes)
        if (s <= std::min<uint64_t>(ring_cap / 2, 64ull << 20)) hs.push_back(s);
      if (hs.size() < 2) hs = {ring_cap / 8, ring_cap / 4};
      // On one GPU both host legs share its PCIe link (writes up, reads down at the
      // same time in the pipelined path): time them concurrently, so β and β' are
      // the full-duplex rates the staged path actually sees.
      if ((st = fit_links_duplex(b, hr, src, dst, hr + ring_cap / 2, hs, std::max(3, reps / 2), &fh1, &fh2,
                                 c->relay_ctas)))
        break;
      if ((st = time_pingpong(b, c->h_probe, true, 500, &eps_host))) break;
    }
  } while (false);

  cudaStreamSynchronize(b.s);
  cudaFree(src);
  cudaFree(dst);
  cudaFree(b.flush);
  cudaEventDestroy(b.e0);
  cudaEventDestroy(b.e1);
  cudaStreamDestroy(b.s);
  if (st) return st;
  int32_t derr = 0;
  CKC(cudaMemcpy(&derr, c->d_err, sizeof(derr), cudaMemcpyDeviceToHost));
  if (derr) return cfail(c, MP_ERR_TIMEOUT, "calibration probe timed out");

  // Install the loopback pair (0, 0): paths in A1 order.  Shared port = HBM:
  // a direct byte costs a read + a write (w = 2), a relay byte 4 (slot write + read
  // on top), a host byte 2 (src read, dst write; the slot is in host DRAM).
  mp_path paths[MP_MAX_PATHS];
  mp_path_params prm[MP_MAX_PATHS];
  int np = 0;
  paths[np] = mp_path{MP_PATH_DIRECT, -1};
  prm[np++] = mp_path_params{fd.alpha, fd.beta, 0, 0, 0, 1, 0, 2, 0};
  for (int r = 0; r < c->n_loop_relays; ++r) {
    paths[np] = mp_path{MP_PATH_GPU, r};
    prm[np++] = mp_path_params{f1.alpha, f1.beta, f2.alpha, f2.beta, std::max(eps_dev, 1e-8), 1, 0, 4, 0};
  }
  if (c->host_path) {
    paths[np] = mp_path{MP_PATH_HOST, -1};
    prm[np++] = mp_path_params{fh1.alpha, fh1.beta, fh2.alpha, fh2.beta, std::max(eps_host, 1e-8), 1, 0, 2, 0};
  }
  mp_port_params port{fd.alpha, 2.0 * fd.beta};
  if (int s = mp_set_model(c, 0, 0, paths, prm, np, &port)) return s;

  // φ (C4): "topology constants (in the form of c·f(n))", P:275 — the staged path alone
  // carries n bytes in k chunks over a grid of k; c = k_best / k* (Eq 14/15 with the
  // fitted α, β, ε), so Eq 19 reproduces the measured optimum at that size.
  double c_relay = 1.0, c_host = 1.0;
  if (c->n_loop_relays > 0) {
    const uint64_t n = std::min<uint64_t>(64ull << 20, static_cast<uint64_t>(c->slots) * c->slot_bytes);
    if (int s = fit_phi(c, 1, n, reps, &c_relay)) return s;
    for (int i = 1; i <= c->n_loop_relays; ++i) prm[i].c = c_relay;
  }
  if (c->host_path) {
    if (int s = fit_phi(c, np - 1, 16ull << 20, std::max(3, reps / 2), &c_host)) return s;
    prm[np - 1].c = c_host;
  }
  return mp_set_model(c, 0, 0, paths, prm, np, &port);
}
