// model.cpp — the paper's extended-Hockney model and Algorithm 1, host fp64.
//
// Sojoodi et al., SC-W '25, §3-§4.  Readings C1-C18: DESIGN.md §3.
// This is the product-side implementation behind mp_predict / mp_select; the
// test-side restatement lives in oracle/model.py and shares nothing with it.
#include "model.h"

#include <algorithm>
#include <cmath>
#include <limits>
#include <numeric>

namespace mpx {

namespace {

constexpr double kInf = std::numeric_limits<double>::infinity();

// Eq 13 case: case 1 iff β < β'; B200 mode breaks β = β' by α vs ε + α' (C3).
inline int bottleneck(const PathModel &p, int mode) {
  if (p.beta < p.beta2) return 1;
  if (mode == M_B200 && p.beta == p.beta2 && p.alpha > p.eps + p.alpha2) return 1;
  return 2;
}

// Staged path carrying x bytes in k chunks.  m = x/k (Eq 12);
// s1 = α + m/β, s2 = ε + α' + m/β'.  PAPER: Eq 13 (case 1 k·s1 + s2, case 2
// s1 + k·s2).  B200: s1 + s2 + (k−1)·max(s1, s2) (C3), and no earlier than the
// relay's start A plus k stage-2 services, A + k·s2 (C28).
inline double staged_time(const PathModel &p, double x, uint32_t k, int mode) {
  const double m = x / static_cast<double>(k);
  const double s1 = p.alpha + m / p.beta;
  const double s2 = p.eps + p.alpha2 + m / p.beta2;
  if (mode == M_B200)
    return std::max(s1 + s2 + static_cast<double>(k - 1) * std::max(s1, s2), p.wake + static_cast<double>(k) * s2);
  if (bottleneck(p, M_PAPER) == 1) return static_cast<double>(k) * s1 + s2;
  return s1 + static_cast<double>(k) * s2;
}

// Ω, Δ of the unpipelined model; direct Ω = 1/β, Δ = α.
inline void od_unpipelined(const PathModel &p, double *om, double *de) {
  if (p.kind == K_DIRECT) {
    *om = 1.0 / p.beta;
    *de = p.alpha;
  } else {
    *om = 1.0 / p.beta + 1.0 / p.beta2;
    *de = p.alpha + p.alpha2 + p.eps;
  }
}

// φ from the first-pass share x0 (Eq 19, two-pass reading C4).
inline double phi_of(const PathModel &p, double x0, int mode) {
  if (bottleneck(p, mode) == 1) return p.c * std::sqrt(p.alpha * p.beta2 / x0);
  return p.c * std::sqrt((p.eps + p.alpha2) * p.beta / x0);
}

// Ω, Δ of Eq 22.
inline void od_eq22(const PathModel &p, double phi, int mode, double *om, double *de) {
  if (bottleneck(p, mode) == 1) {
    *om = 1.0 / p.beta + phi / p.beta2;
    *de = p.eps + p.alpha2 + p.alpha / phi;
  } else {
    *om = phi / p.beta + 1.0 / p.beta2;
    *de = p.alpha + (p.eps + p.alpha2) / phi;
  }
}

// Eq 13 at a fixed integer k as an affine T = Ω x + Δ (pass 3, C18).
inline void od_fixed_k(const PathModel &p, uint32_t k, int mode, double *om, double *de) {
  if (p.kind == K_DIRECT) {
    *om = 1.0 / p.beta;
    *de = p.alpha;
    return;
  }
  const double kd = static_cast<double>(k);
  if (bottleneck(p, mode) == 1) {
    *om = 1.0 / p.beta + 1.0 / (kd * p.beta2);
    *de = kd * p.alpha + p.eps + p.alpha2;
  } else {
    *om = 1.0 / (kd * p.beta) + 1.0 / p.beta2;
    *de = p.alpha + kd * (p.eps + p.alpha2);
  }
}

// Eq 19.
inline double k_eq19(const PathModel &p, double x, double phi, int mode) {
  if (bottleneck(p, mode) == 1) return phi * x / (p.alpha * p.beta2);
  return phi * x / ((p.eps + p.alpha2) * p.beta);
}

// Alg 1 line 17 / P:318: accumulated issue latency of earlier active paths (C8).
void stagger_of(const PairModel &m, const std::vector<char> &act, const ModelOpts &o,
                std::vector<double> *st) {
  st->assign(m.paths.size(), 0.0);
  double acc = 0.0;
  for (size_t i = 0; i < m.paths.size(); ++i) {
    (*st)[i] = o.stagger ? acc : 0.0;
    if (act[i]) acc += (o.mode == M_PAPER) ? m.paths[i].alpha : m.paths[i].sigma;
  }
}

struct Level {
  std::vector<double> theta;
  double t = 0.0;
  std::vector<char> act;
};

// Eq 24 over the active set, dropping θ < 0 paths until none is left (C2).
Level level_paper(const PairModel &m, double n, const std::vector<double> &om,
                  const std::vector<double> &de, std::vector<char> act, const ModelOpts &o) {
  const size_t p = m.paths.size();
  std::vector<double> st;
  for (;;) {
    stagger_of(m, act, o, &st);
    double inv_sum = 0.0, delta_sum = 0.0;  // Alg 1 line 22
    for (size_t i = 0; i < p; ++i)
      if (act[i]) {
        inv_sum += 1.0 / om[i];
        delta_sum += (de[i] + st[i]) / om[i];
      }
    Level L;
    L.theta.assign(p, 0.0);
    bool any_neg = false;
    std::vector<char> next = act;
    for (size_t i = 0; i < p; ++i) {
      if (!act[i]) continue;
      const double d = de[i] + st[i];
      const double th = 1.0 / (om[i] * inv_sum) * (1.0 - d / n * inv_sum + delta_sum / n);
      L.theta[i] = th;
      if (th < 0.0) {
        any_neg = true;
        next[i] = 0;
      }
    }
    if (!any_neg) {
      L.t = (n + delta_sum) / inv_sum;
      L.act = act;
      return L;
    }
    act.swap(next);
  }
}

// B200 mode (C14): bytes deliverable by time T; fractional knapsack on the shared
// port, paths in ascending (w, index).
// *slope (if not null) receives d(total)/dT on T's linear piece: total is piecewise
// linear in T (a path contributes 1/Ω while it is below the port cap, the path the
// cap cuts (β_S − Σ_{earlier} w_j/Ω_j)/w, the paths after it 0).
double port_fill(const PairModel &m, double T, const std::vector<double> &om,
                 const std::vector<double> &de, const std::vector<char> &act,
                 const std::vector<size_t> &order, std::vector<double> *x, double *slope = nullptr) {
  const bool port = m.has_port();
  const bool port_open = port && T > m.port_alpha;
  double room = port ? std::max(0.0, T - m.port_alpha) * m.port_beta : kInf;
  double room_slope = port_open ? m.port_beta : 0.0;  // d(room)/dT while no path is cut
  bool cut = false;
  double total = 0.0, ds = 0.0;
  if (x) x->assign(m.paths.size(), 0.0);
  for (size_t i : order) {
    if (!act[i]) continue;
    double u = std::max(0.0, (T - de[i]) / om[i]);
    double du = u > 0.0 ? 1.0 / om[i] : 0.0;
    const double w = m.paths[i].w;
    if (w > 0.0 && port) {
      if (cut || room / w < u) {  // the port cap binds on this path
        u = cut ? 0.0 : room / w;
        du = cut ? 0.0 : room_slope / w;
        cut = true;
      }
      room -= w * u;
      room_slope -= w * du;
    }
    if (x) (*x)[i] = u;
    total += u;
    ds += du;
  }
  if (slope) *slope = ds;
  return total;
}

Level level_port(const PairModel &m, double n, const std::vector<double> &om,
                 const std::vector<double> &de, std::vector<char> act, const ModelOpts &o) {
  const size_t p = m.paths.size();
  std::vector<size_t> order(p);
  std::iota(order.begin(), order.end(), size_t{0});
  std::stable_sort(order.begin(), order.end(),
                   [&](size_t a, size_t b) { return m.paths[a].w < m.paths[b].w; });
  std::vector<double> st, ds(p), x;
  for (;;) {
    stagger_of(m, act, o, &st);
    for (size_t i = 0; i < p; ++i) ds[i] = de[i] + st[i];
    // smallest T with capacity(T) >= n: capacity is monotone and piecewise linear, so
    // a bracketed Newton step lands on the root of its piece (bisection as the
    // safeguard) — the same T as plain bisection, in a handful of evaluations.
    double lo = 0.0, hi = kInf;  // start: any one active path carrying everything
    for (size_t i = 0; i < p; ++i)
      if (act[i]) hi = std::min(hi, ds[i] + n * om[i]);
    if (!(hi > 1e-9) || !std::isfinite(hi)) hi = 1e-9;
    while (port_fill(m, hi, om, ds, act, order, nullptr) < n) {
      lo = hi;
      hi *= 2.0;
    }
    double T = hi;
    for (int it = 0; it < 400 && hi - lo > 4e-16 * hi; ++it) {
      double a = 0.0;
      const double c = port_fill(m, T, om, ds, act, order, nullptr, &a);
      if (c >= n)
        hi = T;
      else
        lo = T;
      if (c == n) break;
      double next = a > 0.0 ? T + (n - c) / a : 0.5 * (lo + hi);
      if (!(next > lo && next < hi)) next = 0.5 * (lo + hi);
      if (next == T) break;
      T = next;
    }
    port_fill(m, hi, om, ds, act, order, &x);
    bool changed = false;
    std::vector<char> next = act;
    for (size_t i = 0; i < p; ++i)
      if (act[i] && !(x[i] > 0.0)) {
        next[i] = 0;
        changed = true;
      }
    if (!changed) {
      Level L;
      L.theta.resize(p);
      for (size_t i = 0; i < p; ++i) L.theta[i] = x[i] / n;
      L.t = hi;
      L.act = act;
      return L;
    }
    act.swap(next);
  }
}

// dshift (NEXT f2, reading C24): the level solves use max(0, Δ_i − dshift_i).
Level solve(const PairModel &m, double n, const std::vector<double> &om,
            const std::vector<double> &de, const std::vector<char> &act, const ModelOpts &o,
            const double *dshift = nullptr) {
  if (dshift) {
    std::vector<double> ds(de.size());
    for (size_t i = 0; i < de.size(); ++i) ds[i] = std::max(0.0, de[i] - dshift[i]);
    return o.mode == M_B200 ? level_port(m, n, om, ds, act, o) : level_paper(m, n, om, ds, act, o);
  }
  return o.mode == M_B200 ? level_port(m, n, om, de, act, o) : level_paper(m, n, om, de, act, o);
}

// Alg 1 lines 23-28 (C7): floor non-direct shares to A, drop below C_min,
// leftover to the direct path.
void shares_of(uint64_t n, const Level &L, const ModelOpts &o, std::vector<uint64_t> *b) {
  const size_t p = L.theta.size();
  b->assign(p, 0);
  uint64_t sum = 0;
  for (size_t i = 1; i < p; ++i) {
    if (!L.act[i] || !(L.theta[i] > 0.0)) continue;
    const double units = std::floor(L.theta[i] * static_cast<double>(n) / static_cast<double>(o.align));
    uint64_t v = static_cast<uint64_t>(units) * o.align;
    if (v < o.c_min) v = 0;
    (*b)[i] = v;
    sum += v;
  }
  (*b)[0] = n - sum;
}

// C5 clamp: [⌈b/slot⌉, min(K_max, ⌊b/C_min⌋)], the slot bound winning.
uint32_t clamp_k(uint64_t k, uint64_t b, const ModelOpts &o) {
  const uint64_t hi = std::min<uint64_t>(o.k_max, std::max<uint64_t>(1, o.c_min ? b / o.c_min : b));
  k = std::min(k, hi);
  if (o.slot_bytes > 0) k = std::max<uint64_t>(k, (b + o.slot_bytes - 1) / o.slot_bytes);
  return static_cast<uint32_t>(std::max<uint64_t>(1, k));
}

// Reading C26 (B200 mode): the integer k in C5's clamp range minimising the exact
// pipeline time T(k) = max(k·s1 + s2, s1 + k·s2) (convex in k): the floor / ceiling of
// the minimiser of either piece (Eq 14, Eq 15) or of the stage crossover s1 = s2, or
// a bound of the range; ties to the smaller k.  C28: with a relay start A the third
// piece A + k·s2 (increasing in k) adds its crossovers with the other two.
uint32_t k_exact(const PathModel &p, double x, uint64_t b, const ModelOpts &o) {
  const uint32_t lo = clamp_k(1, b, o);
  const uint32_t hi = std::max(lo, clamp_k(1000000000ull, b, o));
  const double e = p.eps + p.alpha2;
  double reals[6] = {std::sqrt(x / (p.alpha * p.beta2)), std::sqrt(x / (p.beta * e)), -1.0, -1.0, -1.0, -1.0};
  if (p.alpha != e) reals[2] = x * (1.0 / p.beta2 - 1.0 / p.beta) / (p.alpha - e);
  if (p.wake > 0.0) {
    // A + k·e + x/β' = α + x/(kβ) + k·e + x/β'  ⇔  k = x / (β(A − α))
    if (p.wake > p.alpha) reals[3] = x / (p.beta * (p.wake - p.alpha));
    // A + k·e + x/β' = k·α + x/β + e + x/(kβ')  ⇔  (e − α)k² + (A − e + x/β' − x/β)k − x/β' = 0
    const double qa = e - p.alpha, qb = p.wake - e + x / p.beta2 - x / p.beta, qc = -x / p.beta2;
    if (qa == 0.0) {
      if (qb != 0.0) reals[4] = -qc / qb;
    } else {
      const double disc = qb * qb - 4.0 * qa * qc;
      if (disc >= 0.0) {
        reals[4] = (-qb + std::sqrt(disc)) / (2.0 * qa);
        reals[5] = (-qb - std::sqrt(disc)) / (2.0 * qa);
      }
    }
  }
  uint32_t cand[14] = {lo, hi, lo, lo, lo, lo, lo, lo, lo, lo, lo, lo, lo, lo};
  int nc = 2;
  for (double r : reals) {
    if (!(r > 0.0)) continue;
    for (double f : {std::floor(r), std::ceil(r)}) {
      const double c = std::min(static_cast<double>(hi), std::max(static_cast<double>(lo), f));
      cand[nc++] = static_cast<uint32_t>(c);
    }
  }
  uint32_t best = cand[0];
  double tb = staged_time(p, x, best, M_B200);
  for (int i = 1; i < nc; ++i) {
    const double t = staged_time(p, x, cand[i], M_B200);
    if (t < tb || (t == tb && cand[i] < best)) {  // ties to the smaller k
      tb = t;
      best = cand[i];
    }
  }
  return best;
}

// Reading C26: the affine piece of the exact pipeline time at k chunks binding at x
// (C28: the availability piece Ω = 1/β', Δ = A + k(ε + α') when it is the largest).
void piece_exact(const PathModel &p, double x, uint32_t k, double *om, double *de) {
  const double kd = static_cast<double>(k), m = x / kd;
  const double s1 = p.alpha + m / p.beta, s2 = p.eps + p.alpha2 + m / p.beta2;
  const double t12 = s1 + s2 + static_cast<double>(k - 1) * std::max(s1, s2);
  if (p.wake > 0.0 && p.wake + kd * s2 > t12) {
    *om = 1.0 / p.beta2;
    *de = p.wake + kd * (p.eps + p.alpha2);
  } else if (s1 >= s2) {
    *om = 1.0 / p.beta + 1.0 / (kd * p.beta2);
    *de = kd * p.alpha + p.eps + p.alpha2;
  } else {
    *om = 1.0 / (kd * p.beta) + 1.0 / p.beta2;
    *de = p.alpha + kd * (p.eps + p.alpha2);
  }
}

}  // namespace

bool PairModel::has_port() const { return port_beta > 0.0 && std::isfinite(port_beta); }

double k_star(const PathModel &p, double x, int mode) {
  if (bottleneck(p, mode) == 1) return std::sqrt(x / (p.alpha * p.beta2));
  return std::sqrt(x / (p.beta * (p.eps + p.alpha2)));
}

uint32_t k_from_real(double k_real) {
  // C5: smallest k >= 1 with k(k+1) >= k_real² (1e-12 relative slack for exact ties).
  const double target = k_real * k_real * (1.0 - 1e-12);
  uint64_t k = 1;
  if (!(target > 2.0)) return 1;
  if (!(target < 1e18)) return 0xffffffffu;  // clamped to K_max by the caller
  // start near sqrt(target) and settle exactly
  k = static_cast<uint64_t>(std::max(1.0, std::floor(std::sqrt(target)) - 1.0));
  while (k > 1 && static_cast<double>((k - 1) * k) >= target) --k;
  while (static_cast<double>(k * (k + 1)) < target) ++k;
  return static_cast<uint32_t>(std::min<uint64_t>(k, 0xffffffffu));
}

std::string validate_model(const PairModel &m) {
  if (m.paths.empty()) return "no paths";
  if (m.paths.size() > 16) return "more than MP_MAX_PATHS paths";
  if (m.paths[0].kind != K_DIRECT) return "paths[0] must be the direct path";
  for (size_t i = 0; i < m.paths.size(); ++i) {
    const PathModel &p = m.paths[i];
    if (p.kind < K_DIRECT || p.kind > K_HOST) return "bad path kind";
    if (i > 0 && p.kind == K_DIRECT) return "only paths[0] may be direct";
    if (!(p.beta > 0.0) || !std::isfinite(p.beta)) return "beta must be finite and > 0";
    if (!(p.alpha >= 0.0) || !std::isfinite(p.alpha)) return "alpha must be finite and >= 0";
    if (!(p.w >= 0.0) || !(p.sigma >= 0.0)) return "w and sigma must be >= 0";
    if (!(p.wake >= 0.0) || !std::isfinite(p.wake)) return "wake must be finite and >= 0";
    if (p.kind != K_DIRECT) {
      if (!(p.beta2 > 0.0) || !std::isfinite(p.beta2)) return "staged beta2 must be finite and > 0";
      if (!(p.alpha2 >= 0.0) || !(p.eps >= 0.0)) return "staged alpha2/eps must be >= 0";
      if (!(p.c > 0.0)) return "c must be > 0";
      // Eq 14/19 need α > 0 in case 1 (either mode may pick case 1) and ε + α' > 0 in case 2
      if (!(p.alpha > 0.0)) return "staged alpha must be > 0 (Eq 14)";
      if (!(p.eps + p.alpha2 > 0.0)) return "staged eps + alpha2 must be > 0 (Eq 15)";
    }
  }
  return "";
}

double predict(const PairModel &m, uint64_t n, const uint64_t *bytes, const uint32_t *chunks,
               const ModelOpts &o) {
  if (n == 0) return 0.0;
  const size_t p = m.paths.size();
  std::vector<char> act(p);
  for (size_t i = 0; i < p; ++i) act[i] = bytes[i] > 0;
  std::vector<double> st;
  stagger_of(m, act, o, &st);
  double t = 0.0;
  for (size_t i = 0; i < p; ++i) {
    if (!act[i]) continue;
    const PathModel &q = m.paths[i];
    const double b = static_cast<double>(bytes[i]);
    const double ti = (q.kind == K_DIRECT) ? q.alpha + b / q.beta           // Eq 6
                                           : staged_time(q, b, chunks[i], o.mode);  // Eq 13
    t = std::max(t, ti + st[i]);                                            // Eq 4
  }
  if (o.mode == M_B200 && m.has_port()) {
    double load = 0.0;
    for (size_t i = 0; i < p; ++i) load += m.paths[i].w * static_cast<double>(bytes[i]);
    if (load > 0.0) t = std::max(t, m.port_alpha + load / m.port_beta);
  }
  return t;
}

void select(const PairModel &m, uint64_t n, uint32_t mask, const ModelOpts &o, Selection *out,
            const double *dshift) {
  const size_t p = m.paths.size();
  out->bytes.assign(p, 0);
  out->chunks.assign(p, 0);
  out->theta.assign(p, 0.0);
  out->t_pred = out->t_level = 0.0;
  if (n == 0) return;
  const double nd = static_cast<double>(n);
  std::vector<char> act(p);
  for (size_t i = 0; i < p; ++i) act[i] = (i == 0) || mask == 0 || ((mask >> i) & 1u);

  // Pass 1: unpipelined Ω, Δ; Eq 11 / port level with the active set.
  std::vector<double> om(p), de(p);
  for (size_t i = 0; i < p; ++i) od_unpipelined(m.paths[i], &om[i], &de[i]);
  Level L0 = solve(m, nd, om, de, act, o, dshift);

  // Pass 2: φ from θ⁽⁰⁾, Eq 22, Eq 24.
  std::vector<double> phi(p, 0.0);
  for (size_t i = 0; i < p; ++i) {
    const PathModel &q = m.paths[i];
    if (q.kind == K_DIRECT || !L0.act[i]) {
      od_unpipelined(q, &om[i], &de[i]);
    } else {
      phi[i] = phi_of(q, L0.theta[i] * nd, o.mode);
      od_eq22(q, phi[i], o.mode, &om[i], &de[i]);
    }
  }
  std::vector<char> act1 = L0.act;
  act1[0] = 1;
  Level L = solve(m, nd, om, de, act1, o, dshift);

  shares_of(n, L, o, &out->bytes);
  out->chunks[0] = 1;
  for (size_t i = 1; i < p; ++i) {
    if (!out->bytes[i]) continue;
    const double kr = k_eq19(m.paths[i], L.theta[i] * nd, phi[i], o.mode);
    out->chunks[i] = clamp_k(k_from_real(kr), out->bytes[i], o);
  }

  const bool refine = o.refine >= 0 ? o.refine != 0 : o.mode == M_B200;
  if (refine && o.mode == M_B200) {  // pass 3, reading C26: exact-pipeline k and piece
    std::vector<char> act3(p);
    for (int round = 0; round < 2; ++round) {
      for (size_t i = 0; i < p; ++i) {
        const PathModel &q = m.paths[i];
        if (q.kind == K_DIRECT) {
          od_unpipelined(q, &om[i], &de[i]);
        } else if (out->bytes[i] == 0) {
          om[i] = 1.0;
          de[i] = 0.0;
        } else {
          const double x = static_cast<double>(out->bytes[i]);
          out->chunks[i] = k_exact(q, x, out->bytes[i], o);
          piece_exact(q, x, out->chunks[i], &om[i], &de[i]);
        }
        act3[i] = (i == 0) || out->bytes[i] > 0;
      }
      L = solve(m, nd, om, de, act3, o, dshift);
      shares_of(n, L, o, &out->bytes);
    }
    for (size_t i = 1; i < p; ++i)
      out->chunks[i] = out->bytes[i] ? k_exact(m.paths[i], static_cast<double>(out->bytes[i]), out->bytes[i], o) : 0;
    for (size_t i = 0; i < p; ++i) out->theta[i] = (i == 0 || out->bytes[i] > 0) ? L.theta[i] : 0.0;
    out->t_level = L.t;
    out->t_pred = predict(m, n, out->bytes.data(), out->chunks.data(), o);
    if (!dshift) {  // C26: the model decides between this split and the direct path alone
      std::vector<uint64_t> db(p, 0);
      std::vector<uint32_t> dk(p, 0);
      db[0] = n;
      dk[0] = 1;
      const double td = predict(m, n, db.data(), dk.data(), o);
      if (td < out->t_pred) {
        out->bytes = db;
        out->chunks = dk;
        out->theta.assign(p, 0.0);
        out->theta[0] = 1.0;
        out->t_pred = out->t_level = td;
      }
    }
    return;
  }
  if (refine) {  // pass 3 (C18), PAPER mode when asked for
    std::vector<char> act3(p);
    for (size_t i = 0; i < p; ++i) {
      od_fixed_k(m.paths[i], std::max<uint32_t>(1, out->chunks[i]), o.mode, &om[i], &de[i]);
      act3[i] = (i == 0) || out->bytes[i] > 0;
    }
    L = solve(m, nd, om, de, act3, o, dshift);
    std::vector<uint32_t> k_prev = out->chunks;
    shares_of(n, L, o, &out->bytes);
    for (size_t i = 1; i < p; ++i)
      out->chunks[i] = out->bytes[i] ? clamp_k(k_prev[i], out->bytes[i], o) : 0;
  }

  for (size_t i = 0; i < p; ++i)
    out->theta[i] = (i == 0 || out->bytes[i] > 0) ? L.theta[i] : 0.0;
  out->t_level = L.t;
  out->t_pred = predict(m, n, out->bytes.data(), out->chunks.data(), o);
}

// ------------------------------------------------------------------ NEXT f2 (C24)
// A window of w back-to-back messages with one config (PAPER.md Obs 2).  Path
// i's message = an issue phase a_i = min(h_i, α_i) that may overlap the previous
// message's serve phase, then the serve phase T_i − a_i: T_i^w = T_i + (w−1)·max(a_i,
// T_i − a_i).  The port is one more such pipeline with a_S = min(α_S, min a_i of the
// active paths through it).  T^w = τ + max(paths, port).  Reading C27: the host enqueues
// the messages h_sub apart, so the per-message step is max(a_i, T_i − a_i, h_sub).
// Reading C28: a relay's start A delays the window once (the relay then lingers); the
// selection spreads it over the window (A/w per message).

namespace {
inline double issue_part(const PathModel &p, const WindowModel &wm, size_t i) {
  const double h = i < wm.h.size() ? wm.h[i] : 0.0;
  return std::min(std::max(h, 0.0), p.alpha);
}
// C24, with C27's host submission: message j is released (j − 1)·h_sub after the first
inline double window_of(double t1, double a, uint32_t w, double h_sub) {
  return t1 + static_cast<double>(w - 1) * std::max(std::max(a, t1 - a), h_sub);
}
double port_issue(const PairModel &m, const WindowModel &wm, const std::vector<char> &act) {
  double a = kInf;
  for (size_t i = 0; i < m.paths.size(); ++i)
    if (act[i] && m.paths[i].w > 0.0) a = std::min(a, issue_part(m.paths[i], wm, i));
  return a == kInf ? 0.0 : std::min(m.port_alpha, a);
}
}  // namespace

double predict_window(const PairModel &m, const WindowModel &wm, uint64_t n, uint32_t w,
                      const uint64_t *bytes, const uint32_t *chunks, const ModelOpts &o) {
  if (n == 0) return 0.0;
  const size_t p = m.paths.size();
  std::vector<char> act(p);
  for (size_t i = 0; i < p; ++i) act[i] = bytes[i] > 0;
  std::vector<double> st;
  stagger_of(m, act, o, &st);
  double t = 0.0;
  for (size_t i = 0; i < p; ++i) {
    if (!act[i]) continue;
    const PathModel &q = m.paths[i];
    const double b = static_cast<double>(bytes[i]);
    if (q.kind == K_DIRECT || o.mode != M_B200 || q.wake <= 0.0) {
      const double ti = (q.kind == K_DIRECT) ? q.alpha + b / q.beta : staged_time(q, b, chunks[i], o.mode);
      t = std::max(t, window_of(ti + st[i], issue_part(q, wm, i), w, wm.submit));
    } else {
      // C28 in a window: the relay starts late once, then lingers through the window —
      // the steady pipeline of the wake-free message plus the first message's delay
      PathModel q0 = q;
      q0.wake = 0.0;
      const double t0 = staged_time(q0, b, chunks[i], o.mode);
      const double t1 = staged_time(q, b, chunks[i], o.mode);
      t = std::max(t, window_of(t0 + st[i], issue_part(q, wm, i), w, wm.submit) + (t1 - t0));
    }
  }
  if (o.mode == M_B200 && m.has_port()) {
    double load = 0.0;
    for (size_t i = 0; i < p; ++i) load += m.paths[i].w * static_cast<double>(bytes[i]);
    if (load > 0.0)
      t = std::max(t, window_of(m.port_alpha + load / m.port_beta, port_issue(m, wm, act), w, wm.submit));
  }
  return wm.tau + t;
}

void select_window(const PairModel &m, const WindowModel &wm, uint64_t n, uint32_t w, uint32_t mask,
                   const ModelOpts &o, Selection *out) {
  const size_t p = m.paths.size();
  const double f = 1.0 - 1.0 / static_cast<double>(w);
  std::vector<double> shift(p);
  std::vector<char> allowed(p);
  for (size_t i = 0; i < p; ++i) {
    shift[i] = f * issue_part(m.paths[i], wm, i);
    allowed[i] = (i == 0) || mask == 0 || ((mask >> i) & 1u);
  }
  PairModel mw = m;  // per-message port startup of the window
  if (m.has_port()) mw.port_alpha = m.port_alpha - f * port_issue(m, wm, allowed);
  for (PathModel &q : mw.paths) q.wake /= static_cast<double>(w);  // C28: one relay start per window
  select(mw, n, mask, o, out, shift.data());
  if (n == 0) return;
  out->t_pred = predict_window(m, wm, n, w, out->bytes.data(), out->chunks.data(), o);
  out->t_level = static_cast<double>(w) * out->t_level + wm.tau;
}

}  // namespace mpx

namespace mpx {

// Reading C19: MaxRate-style fair share for known concurrent flows
// ("if the communication pattern … can be known ahead of time, unused paths can
// be extracted"; MaxRate for contention on shared links).  Every link used by
// k flows gives each 1/k of its bandwidth; then every flow is selected on its own.
void select_flows(const std::vector<const PairModel *> &models, const std::vector<FlowSpec> &flows,
                  const ModelOpts &o, std::vector<Selection> *out, const std::vector<double> *kappa,
                  const std::vector<const WindowModel *> *windows) {
  const size_t F = flows.size();
  auto allowed = [&](size_t f, size_t i) {
    return i == 0 || flows[f].mask == 0 || ((flows[f].mask >> i) & 1u);
  };
  std::vector<int> k_out, k_in, endpoint, relay_users, host_out, host_in;
  auto grow = [](std::vector<int> &v, int g) {
    if (static_cast<int>(v.size()) <= g) v.resize(g + 1, 0);
  };
  int gmax = 0;
  for (size_t f = 0; f < F; ++f) {
    gmax = std::max(gmax, std::max(flows[f].src, flows[f].dst));
    for (const PathModel &p : models[f]->paths) gmax = std::max(gmax, p.via);
  }
  for (auto *v : {&k_out, &k_in, &endpoint, &relay_users, &host_out, &host_in}) grow(*v, gmax);
  for (size_t f = 0; f < F; ++f) {
    k_out[flows[f].src] += 1;
    k_in[flows[f].dst] += 1;
    endpoint[flows[f].src] = endpoint[flows[f].dst] = 1;
  }
  for (size_t f = 0; f < F; ++f) {
    const auto &paths = models[f]->paths;
    for (size_t i = 0; i < paths.size(); ++i) {
      if (!allowed(f, i)) continue;
      if (paths[i].kind == K_GPU && paths[i].via >= 0) relay_users[paths[i].via] += 1;
      if (paths[i].kind == K_HOST) {
        host_out[flows[f].src] += 1;
        host_in[flows[f].dst] += 1;
      }
    }
  }
  out->assign(F, Selection());
  for (size_t f = 0; f < F; ++f) {
    PairModel m = *models[f];
    const int s = flows[f].src, d = flows[f].dst;
    const double pdiv = std::max(k_out[s], k_in[d]);
    uint32_t mask = 0;
    for (size_t i = 0; i < m.paths.size(); ++i) {
      PathModel &p = m.paths[i];
      bool on = allowed(f, i);
      if (p.kind == K_DIRECT) {
        p.beta /= pdiv;
      } else if (p.kind == K_GPU) {
        if (p.via < 0 || endpoint[p.via]) {
          on = false;  // the relay is itself an endpoint: no spare NVLink capacity
        } else {
          const double div = std::max(1, relay_users[p.via]);
          p.beta /= div;
          p.beta2 /= div;
        }
      } else {
        p.beta /= std::max(1, host_out[s]);
        p.beta2 /= std::max(1, host_in[d]);
        // C25 (NEXT f2, Obs 5 P:379-385): a leg whose PCIe link also carries the other
        // direction runs at the duplex factor κ of that GPU; loopback legs are
        // calibrated duplex already.
        if (kappa && s != d) {
          auto kap = [&](int g) { return g < static_cast<int>(kappa->size()) ? (*kappa)[g] : 1.0; };
          if (host_in[s] > 0) p.beta *= kap(s);
          if (host_out[d] > 0) p.beta2 *= kap(d);
        }
      }
      if (on) mask |= 1u << i;
    }
    if (m.has_port()) m.port_beta /= pdiv;
    if (o.window > 1 && windows && (*windows)[f])  // C24: every flow sends a window
      select_window(m, *(*windows)[f], flows[f].bytes, o.window, mask | 1u, o, &(*out)[f]);
    else
      select(m, flows[f].bytes, mask | 1u, o, &(*out)[f]);
  }
}

}  // namespace mpx
