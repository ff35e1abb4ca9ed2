// model.h — host-side fp64 model evaluator and Algorithm 1 selector (internal).
//
// PAPER.md §3 (Eq 1-24) and §4 (Alg 1) under the readings of DESIGN.md §3.
// Independent of oracle/ (which is the test-side restatement); the two share no code.
#pragma once
#include <cstdint>
#include <string>
#include <vector>

namespace mpx {

enum { K_DIRECT = 0, K_GPU = 1, K_HOST = 2 };
enum { M_PAPER = 0, M_B200 = 1 };

struct PathModel {
  int kind = K_DIRECT;
  int via = -1;
  double alpha = 0, beta = 0, alpha2 = 0, beta2 = 0, eps = 0, c = 1, sigma = 0, w = 0;
  double wake = 0;  // B200 mode (C28): earliest start of stage 2 after the message starts [s]
};

struct PairModel {
  std::vector<PathModel> paths;  // paths[0] is the direct path
  double port_alpha = 0.0;
  double port_beta = 0.0;        // <= 0 or inf: no shared port
  bool has_port() const;
};

struct ModelOpts {
  int mode = M_PAPER;
  int stagger = 1;
  int refine = -1;
  uint64_t align = 256;
  uint64_t c_min = 65536;
  uint64_t k_max = 1024;
  uint64_t slot_bytes = 0;
  uint32_t window = 1;  // NEXT f2: the window mp_select assumes (C24)
};

struct Selection {
  std::vector<uint64_t> bytes;
  std::vector<uint32_t> chunks;
  std::vector<double> theta;
  double t_pred = 0.0;
  double t_level = 0.0;
};

// Returns an empty string when the pair model is valid, else the reason.
std::string validate_model(const PairModel &m);

// O2: predicted time of a config (bytes sum to n).
double predict(const PairModel &m, uint64_t n, const uint64_t *bytes, const uint32_t *chunks,
               const ModelOpts &o);

// O3: Algorithm 1.  mask bit i enables path i (bit 0 forced on).  dshift (NEXT f2,
// C24): per-path amounts subtracted from every Δ_i of the level solves (may be null).
void select(const PairModel &m, uint64_t n, uint32_t mask, const ModelOpts &o, Selection *out,
            const double *dshift = nullptr);

// NEXT f2 (reading C24): window parameters of a pair — h[i] the startup of path i a
// back-to-back successor overlaps (a_i = min(h_i, α_i); empty = 0), tau the fixed
// completion cost of a window [s].
struct WindowModel {
  std::vector<double> h;
  double tau = 0.0;
  double submit = 0.0;  // reading C27: host submission time per message (the context's)
};
// Time of w back-to-back messages of n bytes with one config (W1).
double predict_window(const PairModel &m, const WindowModel &wm, uint64_t n, uint32_t w,
                      const uint64_t *bytes, const uint32_t *chunks, const ModelOpts &o);
// Alg 1 on the window's per-message coefficients; t_pred = W1, t_level = w·level + τ.
void select_window(const PairModel &m, const WindowModel &wm, uint64_t n, uint32_t w, uint32_t mask,
                   const ModelOpts &o, Selection *out);

// The C5 integer rule (exposed for tests through the selector only).
uint32_t k_from_real(double k_real);

// NEXT f1 (reading C19): selection for a known set of concurrent flows with a
// MaxRate-style fair share of every NVLink / PCIe link among the flows using it.
struct FlowSpec {
  int src = 0, dst = 0;
  uint64_t bytes = 0;
  uint32_t mask = 0;  // path mask of the pair (0 = all)
};
// kappa (NEXT f2, reading C25): per-GPU host duplex factor (may be null = all 1).
// windows (NEXT f2, C24): per-flow window model, used when o.window > 1 (may be null).
void select_flows(const std::vector<const PairModel *> &models, const std::vector<FlowSpec> &flows,
                  const ModelOpts &o, std::vector<Selection> *out,
                  const std::vector<double> *kappa = nullptr,
                  const std::vector<const WindowModel *> *windows = nullptr);

// Eq 14 / Eq 15: the real optimal chunk count of a staged path
// carrying x bytes (used by the φ calibration).
double k_star(const PathModel &p, double x, int mode);

}  // namespace mpx
