/*
 * mp.h — C ABI of mpx, a B200-native implementation of the multi-path intra-node
 * GPU→GPU transfer of Sojoodi et al., "Accelerating Intra-Node GPU Communication:
 * A Performance Model for Multi-Path Transfers" (SC-W '25).  P:<line> cites
 * /root/reference/PAPER.md; C<n> cites the readings table in DESIGN.md §3.
 *
 * One message of n bytes from a source GPU to a destination GPU is split over
 * several intra-node paths at once: the direct NVLink/NVSwitch path,
 * two-hop relays staged through intermediate GPUs, and a pinned-host PCIe path.
 * The split θ and the per-path chunk counts k come from the paper's
 * extended-Hockney model (Eq 1-24) through Algorithm 1; the bytes are moved
 * by hand-written sm_100a kernels (SM-driven 128-bit stores into peer / pinned-host
 * memory, flag release/acquire handoff between pipeline stages).
 *
 * Conventions for every function below
 *   - returns an int status: MP_OK (0) or a negative MP_ERR_*; never aborts, never
 *     throws.  mp_strerror(status) names the code; mp_last_error(ctx) gives the last
 *     message recorded on ctx (library-owned string, valid until the next call).
 *   - pointers: "host" = CPU memory, "device" = CUDA device memory of the calling
 *     rank's GPU.  Buffers passed in are owned by the caller; the library keeps no
 *     reference after the call returns unless stated (stream-ordered work keeps
 *     using a buffer until that work completes on its stream).
 *   - units (C11): bytes, seconds, bytes/second.
 *   - a `stream` argument is a cudaStream_t passed as void* (NULL = legacy default
 *     stream).  Work is enqueued; completion is stream-ordered.
 *   - thread safety: a context may be used by one host thread at a time.
 */
#ifndef MPX_MP_H
#define MPX_MP_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MP_ABI_VERSION 5  /* 5: emulated world (mp_init_emulated, mp_emu_*; MP_INIT_EMULATED);
                             4: mp_path_params.wake (reading C28);
                             3: topology (mp_get/set_topology), fingerprinted parameter files;
                             2: NEXT f2 calls; mp_model_opts.window (was reserved) */
#define MP_MAX_PATHS 16

/* Status codes. */
enum {
  MP_OK = 0,
  MP_ERR_INVALID = -1,     /* bad argument (NULL, size mismatch, Σ shares != n, k out of range) */
  MP_ERR_CUDA = -2,        /* a CUDA runtime call failed (message in mp_last_error) */
  MP_ERR_TOPOLOGY = -3,    /* unknown rank / path not available between src and dst */
  MP_ERR_NOMEM = -4,       /* heap, ring or host allocation failed */
  MP_ERR_STATE = -5,       /* call not valid in this context state (e.g. model-only ctx) */
  MP_ERR_UNSUPPORTED = -6, /* feature not built / not supported on this system */
  MP_ERR_TIMEOUT = -7,     /* a device-side wait exceeded the timeout (sticky) */
  MP_ERR_MISMATCH = -8     /* send/recv size or tag mismatch detected on the device (sticky) */
};

/* Path kinds, P:107-111 (§3.1). */
enum { MP_PATH_DIRECT = 0, MP_PATH_GPU = 1, MP_PATH_HOST = 2 };

/* Model modes (C3, C8, C14, C18).
 * PAPER: Eq 13 with the printed case rule, stagger σ_j = α_j, no shared port.
 * B200 : exact two-stage pipeline time, calibrated stagger σ, one shared port
 *        (NVSwitch egress/ingress, or HBM in single-GPU loopback), integer-k pass 3. */
enum { MP_MODEL_PAPER = 0, MP_MODEL_B200 = 1 };

/* Init flags. */
enum {
  MP_INIT_MODEL_ONLY = 1,  /* no CUDA at all: model evaluator + selector only (CPU tests) */
  MP_INIT_NO_CALIBRATE = 2, /* do not measure α/β at init (use defaults / param file / mp_set_model) */
  MP_INIT_EMULATED = 4      /* set by mp_init_emulated only (mp_init rejects it otherwise) */
};

typedef struct mp_ctx mp_ctx;  /* opaque, library-owned */

/* One path between a (src, dst) pair.  via = relay rank for MP_PATH_GPU (in
 * single-GPU loopback: the index of an emulated relay ring), -1 otherwise. */
typedef struct mp_path {
  int32_t kind;
  int32_t via;
} mp_path;

/* Per-path model parameters — Table 1.  For a direct path only alpha,
 * beta (and sigma, w) are used (Eq 6: α' = ε = 0, 1/β' = 0). */
typedef struct mp_path_params {
  double alpha;   /* α_i  first-link startup latency [s] */
  double beta;    /* β_i  first-link bandwidth [B/s] */
  double alpha2;  /* α'_i second-link startup latency [s] (staged) */
  double beta2;   /* β'_i second-link bandwidth [B/s] (staged) */
  double eps;     /* ε_i  synchronisation overhead at the staging device [s] */
  double c;       /* multiplier of the topology constant φ_i (C4; 1 = Eq 14/15 at θ⁽⁰⁾) */
  double sigma;   /* issue latency counted by the stagger in B200 mode (C8) [s] */
  double w;       /* bytes of shared-port traffic per payload byte (C14) */
  double wake;    /* B200 mode (C28): earliest start of the second stage after the message
                     starts [s] — a relay rank's kernel launch through its doorbell thread;
                     0 = stage 2 ready at once.  T = max(C3's pipeline, wake + k·s2). */
} mp_path_params;

/* The shared port of B200 mode (C14): T >= alpha + Σ_i w_i b_i / beta.
 * beta <= 0 or +inf disables it. */
typedef struct mp_port_params {
  double alpha;
  double beta;
} mp_port_params;

/* Selector options (readings C5, C7, C8, C18). */
typedef struct mp_model_opts {
  int32_t mode;        /* MP_MODEL_PAPER | MP_MODEL_B200 */
  int32_t stagger;     /* 1: Alg 1 line 17 issue stagger; 0: off */
  int32_t refine;      /* pass 3 (C18): 1 on, 0 off, -1 = mode default (B200 on) */
  int32_t window;      /* NEXT f2 (C24): the window mp_select assumes — > 1 makes mp_select
                          (and so mp_send / mp_xfer with cfg = NULL) return
                          mp_select_window's config; 0 or 1 = per message (default) */
  uint64_t align;      /* A: share alignment and chunk unit, >= 1 (default 256) */
  uint64_t c_min;      /* smallest staged share and chunk (default 65536) */
  uint64_t k_max;      /* chunk-count cap (default 1024) */
  uint64_t slot_bytes; /* largest chunk a staging slot holds (0 = unlimited) */
} mp_model_opts;

/* Algorithm 1 output: shares[] and configs[] per path.  Caller-allocated.
 * bytes[] is authoritative and sums to n; theta[] is informational. */
typedef struct mp_config {
  int32_t npaths;
  int32_t reserved;
  mp_path path[MP_MAX_PATHS];
  double theta[MP_MAX_PATHS];
  uint64_t bytes[MP_MAX_PATHS];
  uint32_t chunks[MP_MAX_PATHS]; /* k_i >= 1 when bytes[i] > 0, else 0; direct k = 1 */
  double t_pred;                 /* O2 model time of this config [s] */
  double t_level;                /* linearised common finish time of the last level solve [s] */
} mp_config;

/* Bootstrap all-gather: every rank contributes `bytes` bytes at `in`; on return
 * `out` holds world*bytes bytes, rank-major.  Return 0 on success.  The library
 * calls it only inside mp_init/mp_finalize (collective calls). */
typedef int (*mp_allgather_fn)(void *user, const void *in, void *out, uint64_t bytes);

typedef struct mp_init_args {
  int32_t rank;          /* this process's rank, 0..world-1 */
  int32_t world;         /* number of ranks (one GPU each); 1 = single-GPU loopback */
  int32_t device;        /* local CUDA device ordinal */
  int32_t flags;         /* MP_INIT_* */
  int32_t n_loop_relays; /* loopback only: emulated relay rings (default 6 if < 0) */
  int32_t host_path;     /* 1: enable the pinned-host PCIe path (default 1 if < 0) */
  int32_t slots;         /* staging slots per ring (default 4 if <= 0) */
  int32_t relay_ctas;    /* CTAs per staged-path stage (default 16 if <= 0, max 32) */
  uint64_t heap_bytes;   /* symmetric receive heap per rank (default 2.25 GiB if 0) */
  uint64_t slot_bytes;   /* bytes per staging slot (default 32 MiB if 0) */
  double timeout_s;      /* device wait timeout (default 20 s if <= 0) */
  mp_allgather_fn allgather; /* required when world > 1 */
  void *allgather_user;
  const char *param_file;    /* optional: load model parameters (Step 2) */
} mp_init_args;

/* ---------------------------------------------------------------- lifetime */

/* Create a context — the paper's Steps 1-2 (parameters "extracted once per
 * system topology and stored on each compute node", loaded at start-up).  Collective
 * over all ranks when world > 1.  mp_init:
 *   - discovers the topology (mp_get_topology): every GPU's UUID, PCI location, NUMA
 *     node (sysfs), PCIe link and active NVLink links (NVML, loaded with dlopen; 0 =
 *     unknown), and per ordered pair of GPUs peer access, P2P performance rank and
 *     native atomics (cudaDeviceCanAccessPeer / cudaDeviceGetP2PAttribute where the
 *     peer GPU is visible in this process, else the outcome of the IPC mapping);
 *     a pair's relays (A1) are the ranks with peer access from the source and to the
 *     destination;
 *   - allocates the receive heap and control block, exchanges IPC handles, creates
 *     the shared pinned segments (relay doorbells, host rings) bound to their GPU's
 *     NUMA node (host-path quality depends on "PCIe configuration,
 *     and NUMA effects");
 *   - loads param_file if it exists (Step 2; refused with MP_ERR_TOPOLOGY when its
 *     topology fingerprint differs from this job's), and — unless
 *     MP_INIT_NO_CALIBRATE — calibrates α/β/ε of every path with the engine's own
 *     kernels (Step 1);
 *   - world >= 3: starts the relay service thread (launches a bounded relay kernel
 *     for each relayed message a sender announces; no kernel outlives its traffic,
 *     so device-wide synchronisation is allowed at any time).
 * With MP_INIT_MODEL_ONLY no CUDA call is made; world/rank still define the pairs
 * (topology unknown: every path assumed; mp_set_topology injects one).
 * Errors: MP_ERR_INVALID, MP_ERR_CUDA, MP_ERR_NOMEM, MP_ERR_TOPOLOGY (a peer's memory
 * cannot be mapped; a parameter file from another topology). */
int mp_init(mp_ctx **ctx, const mp_init_args *args);

/* Destroy a context (the end of the Step 5 engine's lifetime): waits for
 * outstanding work on this device (cudaDeviceSynchronize), stops the relay service (waits for
 * the relay kernels it launched), unmaps and frees everything.  Collective when
 * world > 1.  ctx may be NULL.  Returns MP_OK or the barrier's failure; MP_ERR_STATE
 * (and does nothing) for a context of an emulated world: mp_finalize_emulated tears
 * those down. */
int mp_finalize(mp_ctx *ctx);

/* ---------------------------------------------------------------- emulated world
 *
 * Every rank of a world as a context of THIS process on ONE GPU, for running the
 * multi-rank engine where there are fewer GPUs than ranks.  The engine's ranks wait on
 * one another on the device (the clear-to-send, the relay doorbells and ring flags,
 * the done counters of Step 5's pipelined chunks), so they must
 * never be separate launches sharing a GPU: nothing guarantees those launches run at
 * the same time.  Here every rank's kernels become CTA ranges of ONE cooperative
 * launch, co-resident by construction.
 *
 * mp_init_emulated: args->world (2..MP_MAX_PATHS) contexts, rank r in ctxs[r], all on
 * args->device, bootstrapped on one thread each through an in-process all-gather (the
 * same initialisation as a real job; peers' memory is addressed directly instead of
 * through CUDA IPC).  args->rank, ->allgather, ->allgather_user are ignored; no
 * calibration (MP_INIT_NO_CALIBRATE is implied: there are no links to time — set the
 * model with mp_set_model / mp_load_params).  Errors: as mp_init; on any error no
 * context is returned.
 * In an emulated world, mp_send / mp_recv (and mp_select, mp_alloc, every model
 * call) behave as in a real job except that they launch nothing: they record the
 * kernels' parameter blocks.  mp_register / mp_deregister (use mp_emu_register /
 * mp_emu_deregister), mp_alltoall / mp_allreduce (use mp_emu_alltoall /
 * mp_emu_allreduce) and the calibration calls return MP_ERR_UNSUPPORTED; mp_finalize
 * returns MP_ERR_STATE.
 *
 * mp_emu_run: ctxs = the world's n contexts in rank order.  Launches everything they
 * recorded since the last run as one cooperative grid on `stream` — per send its gate
 * and send CTAs, per receive its receive CTAs, the eager kernels, and per (relay rank,
 * sender) the relay kernel that rank's service thread would have launched, which reads
 * its doorbells on the device — then waits for the stream.  kernel_s (may be NULL):
 * the grid's device time [s] from CUDA events on `stream`.  Direct-path CTA groups
 * are shrunk (same bytes, fewer CTAs) so the grid fits the device's co-resident
 * capacity.  The recorded work must be one self-contained exchange: every recorded
 * send matched by a recorded receive, at most 64 rendezvous messages per ordered pair
 * (every receive posts its clear-to-send at once; mp_recv refuses a 65th with
 * MP_ERR_INVALID before recording it).  A refused run drops what was recorded and
 * leaves the pairs' sequence state inconsistent: create a new world.  Errors: MP_ERR_INVALID (not the whole world /
 * the fixed roles alone exceed one co-resident grid / a relay's doorbells not
 * consecutive), MP_ERR_CUDA, MP_ERR_TIMEOUT and MP_ERR_MISMATCH (any rank's device
 * error word; sticky as in a real job).
 *
 * mp_finalize_emulated: tears down all n contexts (one thread each) and the world. */
int mp_init_emulated(mp_ctx **ctxs, const mp_init_args *args);
/* mp_register / mp_deregister of every rank of an emulated world at once (each rank's
 * call runs on its own thread: the calls are collective): bufs[r], bytes[r] = rank r's
 * buffer (NULL / 0: none), its region id returned in ids[r]; rules and errors as
 * mp_register / mp_deregister (the first failing rank's status). */
int mp_emu_register(mp_ctx **ctxs, int n, void *const *bufs, const uint64_t *bytes, int *ids);
int mp_emu_deregister(mp_ctx **ctxs, int n, const int *ids);
int mp_emu_run(mp_ctx **ctxs, int n, void *stream, double *kernel_s);
int mp_finalize_emulated(mp_ctx **ctxs, int n);

/* ---------------------------------------------------------------- topology (Step 1) */

/* One GPU of the job.  0 / -1 = unknown (NVML or sysfs unavailable). */
typedef struct mp_gpu_info {
  char uuid[16];          /* cudaDeviceProp.uuid */
  int32_t device;         /* CUDA ordinal in the owning process */
  int32_t pci_domain, pci_bus, pci_device;
  int32_t numa_node;      /* NUMA node of the GPU's PCIe root (-1 unknown) */
  int32_t pcie_gen, pcie_width;  /* maximum PCIe link generation / width (NVML) */
  int32_t pcie_gen_cur;   /* current PCIe generation (power-managed; informational) */
  int32_t nvlinks;        /* active NVLink links (NVML) */
  int32_t sms;            /* streaming multiprocessors */
  int32_t reserved;
} mp_gpu_info;

/* The job's topology: gpu[r] is rank r's GPU; [s][d] matrices by rank. */
typedef struct mp_topology {
  int32_t world;
  int32_t reserved;
  uint64_t fingerprint;   /* FNV-1a of the GPUs (UUID, SMs, PCIe link, NVLinks, NUMA) and
                             the peer-access matrix; 0 = no topology known */
  mp_gpu_info gpu[MP_MAX_PATHS];
  int32_t peer_access[MP_MAX_PATHS][MP_MAX_PATHS];   /* 1: s can load/store d's memory */
  int32_t p2p_perf_rank[MP_MAX_PATHS][MP_MAX_PATHS]; /* cudaDevP2PAttrPerformanceRank */
  int32_t p2p_atomics[MP_MAX_PATHS][MP_MAX_PATHS];   /* cudaDevP2PAttrNativeAtomicSupported */
} mp_topology;

/* The topology found by mp_init (or injected).  A model-only context without one
 * reports fingerprint 0 and full peer access.  Host-only. */
int mp_get_topology(mp_ctx *ctx, mp_topology *out);

/* Inject a topology into a MODEL-ONLY context (tests, planning for another node):
 * in->world must equal the context's; the fingerprint is recomputed; every pair's
 * model returns to the default paths of that topology (relays need peer access from
 * the source and to the destination; a pair without peer access s -> d has no
 * direct path and is reported as MP_ERR_TOPOLOGY).  Errors: MP_ERR_STATE (not
 * model-only), MP_ERR_INVALID. */
int mp_set_topology(mp_ctx *ctx, const mp_topology *in);

const char *mp_strerror(int status);
const char *mp_last_error(mp_ctx *ctx);
int mp_abi_version(void);

/* ---------------------------------------------------------------- model (host, fp64) */

/* The default path list for (src, dst) in the order of reading A1: direct, GPU
 * relays by ascending rank (or loopback ring index), host.  out: MP_MAX_PATHS entries. */
int mp_paths(mp_ctx *ctx, int src, int dst, mp_path *out, int *npaths);

/* Install model parameters for the ordered pair (src, dst) (tests / parity /
 * Step 2 injection).  paths[i] and params[i] describe path i; paths[0] must be
 * MP_PATH_DIRECT.  port may be NULL (no shared port).  Invalidates the config
 * cache.  Errors: MP_ERR_INVALID (npaths out of range, β <= 0, staged α <= 0 with
 * β < β', staged ε + α' <= 0, ...). */
int mp_set_model(mp_ctx *ctx, int src, int dst, const mp_path *paths,
                 const mp_path_params *params, int npaths, const mp_port_params *port);
int mp_get_model(mp_ctx *ctx, int src, int dst, mp_path *paths, mp_path_params *params,
                 int *npaths, mp_port_params *port);

/* NEXT f4 size bands (P:360 Observation 4: the linear Hockney model
 * fitted on the asymptotic bandwidth is less accurate for small messages).  Reading
 * C20: a pair may carry several complete parameter sets; band j applies to messages
 * of n bytes with n_min_j <= n < n_min_{j+1}.  Band 0 (n_min = 0) is the model of
 * mp_set_model.  mp_predict, mp_select and mp_select_flows evaluate Eq 1-24 / Alg 1
 * unchanged with the parameters of n's band.
 * mp_set_model_band installs (or replaces, same n_min) band n_min > 0 of (src, dst):
 * params[npaths] in the order of the pair's paths (npaths must equal the pair's path
 * count; the path kinds are the base model's), port may be NULL (no shared port).
 * mp_set_model drops every band of the pair.  Invalidates the config cache.
 * Errors: MP_ERR_INVALID (n_min == 0, npaths mismatch, invalid parameters as in
 * mp_set_model), MP_ERR_TOPOLOGY.
 * mp_get_model_band reads band `band` (0 = base; ascending n_min): any output
 * pointer may be NULL; *nbands (if not NULL) receives the band count; band < 0
 * returns only the count.  Errors: MP_ERR_INVALID (band >= count). */
int mp_set_model_band(mp_ctx *ctx, int src, int dst, uint64_t n_min, const mp_path_params *params,
                      int npaths, const mp_port_params *port);
int mp_get_model_band(mp_ctx *ctx, int src, int dst, int band, uint64_t *n_min,
                      mp_path_params *params, int *npaths, mp_port_params *port, int *nbands);

/* Selector options for this context (invalidates the cache). */
int mp_set_options(mp_ctx *ctx, const mp_model_opts *opts);
int mp_get_options(mp_ctx *ctx, mp_model_opts *opts);

/* mp_predict — O2: modelled time of moving `bytes` from src to dst with
 * config `cfg` (Eq 6 direct, Eq 13 staged, + stagger, T = max_i T_i (Eq 4); B200
 * mode: exact pipeline and the shared port).  cfg->bytes must sum to `bytes`.
 * *seconds receives the time.  Host-only; no CUDA. */
int mp_predict(mp_ctx *ctx, int src, int dst, uint64_t bytes, const mp_config *cfg,
               double *seconds);

/* mp_select — Algorithm 1 without exhaustive search, reading O3: θ from
 * Eq 11 then Eq 24 with the two-pass φ (C4) and the active set (C2), k from Eq 19
 * (C5), shares floored to A with the leftover to the direct path (C7), optional
 * pass 3 (C18).  path_mask bit i enables path i of mp_paths() (bit 0, the direct
 * path, is always on; 0 = all paths).  The environment variable MPX_PATHS (read at
 * mp_init; e.g. "direct,host", "direct,gpu", "all") further restricts the path kinds
 * (P:312-313).  Results are cached (C10).  With mp_model_opts.window > 1 it returns
 * mp_select_window's config for that window (NEXT f2, C24).  Host-only. */
int mp_select(mp_ctx *ctx, int src, int dst, uint64_t bytes, uint32_t path_mask,
              mp_config *out);

/* One of several concurrent messages (NEXT f1). */
typedef struct mp_flow {
  int32_t src;
  int32_t dst;
  uint32_t path_mask;  /* as in mp_select (0 = all paths of the pair) */
  uint32_t reserved;
  uint64_t bytes;
} mp_flow;

/* mp_select_flows — contention-aware selection for a known set of concurrent flows
 * ("if the communication pattern … can be known ahead of time,
 * unused paths can be extracted", P:410 MaxRate for shared links).  Reading C19:
 * every link used by k of the flows gives each of them 1/k of its bandwidth — the
 * source egress / destination ingress (port and direct β) by max(k_out, k_in), a
 * relay's two legs by the number of flows that may use it (and a relay that is itself
 * an endpoint of a flow is excluded), the host legs by the flows sharing that PCIe
 * direction — then every flow is selected on its own (mp_select; with
 * mp_model_opts.window > 1, mp_select_window with the pair's window model, NEXT f2).
 * out: nflows configs, caller-allocated.  Not cached.  Host-only. */
int mp_select_flows(mp_ctx *ctx, int nflows, const mp_flow *flows, mp_config *out);

/* ---------------------------------------------------------------- NEXT f2: windows, BIBW */

/* Window model of the pair (src, dst) (PAPER.md Observation 2, P:358:
 * "larger window sizes allow for more concurrent transfers, reducing the impact of
 * latency"; OMB windows).  Reading C24: in a window of w
 * back-to-back messages with one config, path i's message is an issue phase
 * a_i = min(h[i], α_i) that may overlap the previous message, then a serve phase
 * T_i − a_i (T_i = the mp_predict path time), so T_i^w = T_i + (w−1)·max(a_i, T_i − a_i);
 * the shared port is one more such pipeline (a_S = min(α_S, min a_i of the active paths
 * through it)); the window adds a fixed completion cost tau (OMB's wait-all + ack):
 * T^w = tau + max(paths, port).  h[npaths] in seconds, in the order of mp_paths;
 * npaths must equal the pair's path count; h >= 0, tau >= 0 (defaults 0: h = 0 is the
 * paper's per-message model, T^w = w·T).  The window parameters apply to every size
 * band of the pair; mp_set_model with a different path count drops them.
 * Errors: MP_ERR_INVALID, MP_ERR_TOPOLOGY.  Host-only. */
int mp_set_window_model(mp_ctx *ctx, int src, int dst, const double *h, int npaths, double tau);
/* h (MP_MAX_PATHS entries), npaths and tau may each be NULL. */
int mp_get_window_model(mp_ctx *ctx, int src, int dst, double *h, int *npaths, double *tau);

/* mp_predict_window — T^w of C24 for `window` >= 1 messages of `bytes` each with config
 * cfg (validated as in mp_predict; window = 1 gives mp_predict + tau).  *seconds = the
 * whole window.  Errors as mp_predict; MP_ERR_INVALID for window = 0.  Host-only. */
int mp_predict_window(mp_ctx *ctx, int src, int dst, uint64_t bytes, uint32_t window,
                      const mp_config *cfg, double *seconds);

/* mp_select_window — Algorithm 1 for a window (reading C24): mp_select on the
 * window's per-message coefficients (every Δ_i − (1 − 1/w)·a_i, the port's
 * α_S − (1 − 1/w)·a_S).  out->t_pred = T^w of the result, out->t_level = w·(per-message
 * level) + tau.  window = 1 returns mp_select's config.  path_mask and MPX_PATHS as in
 * mp_select.  Not cached.  Host-only. */
int mp_select_window(mp_ctx *ctx, int src, int dst, uint64_t bytes, uint32_t window,
                     uint32_t path_mask, mp_config *out);

/* Host duplex factor κ of GPU `gpu` (rank; 0 <= gpu < MP_MAX_PATHS), reading C25
 * (PAPER.md Observation 5: "contention between the bidirectional transfers
 * along the host-staged path … the model should be extended to account for host-staged
 * contention, PCIe configuration").  In mp_select_flows, after C19's fair share, a flow
 * s -> d (s != d) runs its host up leg at κ_s·β if any flow's host down leg enters s,
 * and its down leg at κ_d·β' if any flow's host up leg leaves d.  Loopback flows
 * (s == d) are calibrated duplex and are not scaled.  kappa in (0, 1]; default 1.
 * Errors: MP_ERR_INVALID (kappa out of range), MP_ERR_TOPOLOGY (gpu out of range). */
int mp_set_host_duplex(mp_ctx *ctx, int gpu, double kappa);
int mp_get_host_duplex(mp_ctx *ctx, int gpu, double *kappa);

/* mp_calibrate_window — Step 1 for the C24/C25/C27 parameters of the loopback
 * pair (0, 0), timed as osu_bw times a window: the host clock around the
 * mp_xfer enqueues and the stream synchronisation that completes them.  First the host
 * submission time per call (C27; the marginal host-clock cost of one more 64 KiB
 * direct-only message in an OMB-style window, mp_set_submit_time).  Then, for every path alone (all bytes on it; staged
 * paths in >= 8 chunks) and every size (NULL/0 = 64 KiB, 1, 4, 16, 64 MiB), one message
 * on an idle stream (T1) and `window` (0 = 16) back-to-back messages (TW), median of
 * `reps` (0 = 7); tau = max(0, median(T1 − mp_predict) over the direct path's sizes),
 * h_i = median over the serve-bound sizes of max(0, T1 − tau − (TW − T1)/(window − 1))
 * (mp_fit_window with h_sub).  κ of
 * this GPU = the mean of (simplex / duplex time) of the two host legs at 64 MiB, each
 * leg moved by relay_ctas CTAs as in the engine.  Installs them with
 * mp_set_window_model / mp_set_host_duplex.  Parameters measured on B200: parity
 * unpinned (the paper prints none).  Errors: MP_ERR_STATE (model-only),
 * MP_ERR_UNSUPPORTED (world > 1), MP_ERR_INVALID, MP_ERR_CUDA, MP_ERR_TIMEOUT. */
int mp_calibrate_window(mp_ctx *ctx, const uint64_t *sizes, int nsizes, int window, int reps);

/* mp_calibrate_wake — reading C28: measure, per relay rank r, the time A_r
 * from a message's start to its relay kernel's start when r's relay service is idle
 * (doorbell → service thread → kernel launch), and install it as `wake` of every
 * GPU-staged path via r in every pair model and band.  Collective over the world
 * (world >= 3; a no-op below), after the relay service is up and with no traffic in
 * flight; mp_init calls it after Step 1 when it calibrates.  Probe: pair (r+1, r+2)
 * sends two relay-only messages of `bytes` (0 = 2 MiB; raised above the eager limit)
 * through r after linger + 1 ms of quiet, timed back to back on the receiver;
 * A_r = T − k·s2 + median(t1 − t2) over `reps` (0 = 7) with T, s2 of the pair's model
 * (k = 1: s1 + the median), or 0 when that difference is below 1 µs.  MPX_RELAY_WAKE_US (equal on every
 * rank) installs that value instead of probing.  Returns MP_ERR_STATE without a relay
 * service, MP_ERR_TOPOLOGY if a pair lacks the path via r. */
int mp_calibrate_wake(mp_ctx *ctx, uint64_t bytes, int reps);

/* mp_fit_window — the estimator of mp_calibrate_window on given samples (for parity):
 * sample j of path[j] (0 <= path < npaths; path 0 = direct) has T1 = t1[j] (one message
 * on an idle stream), TW = tw[j] (`window` >= 2 back-to-back messages) and the model's
 * time pred[j] of one message.  *tau = max(0, median over path-0 samples of
 * t1 − pred) (0 without one); h[i] = median over path i's samples of
 * max(0, t1 − tau − (tw − t1)/(window − 1)) (0 without one), skipping the samples whose
 * steady per-message time (tw − t1)/(window − 1) is <= h_sub·(1 + 1e-6) (submission-
 * bound, reading C27; h_sub = 0 keeps every sample); h has npaths entries.  Medians of
 * an even count take the upper middle value.  Errors: MP_ERR_INVALID. */
int mp_fit_window(const int *path, const double *t1, const double *tw, const double *pred, int m,
                  int window, int npaths, double h_sub, double *h, double *tau);

/* Host submission time per message (reading C27; NEXT f4 — P:360/P:375: small messages
 * behave differently; their windows are bound by the host's cost per call): the messages
 * of a window are enqueued h_sub seconds apart, so in mp_predict_window /
 * mp_select_window every path's (and the port's) per-message step is
 * max(a_i, T_i − a_i, h_sub).  One value per context (the caller's cost per mp_send /
 * mp_xfer call); mp_calibrate_window measures it from C; 0 by default.
 * Errors: MP_ERR_INVALID (negative or not finite). */
int mp_set_submit_time(mp_ctx *ctx, double seconds);
int mp_get_submit_time(mp_ctx *ctx, double *seconds);

/* ---------------------------------------------------------------- memory */

/* Allocate / free device memory from this rank's registered heap.  A buffer that
 * receives (mp_recv) must come from here, or from a region registered with
 * mp_register, when world > 1 (peers address it by heap offset, the analogue of UCX
 * cuda_ipc's cached IPC mappings).  256-B aligned. */
int mp_alloc(mp_ctx *ctx, uint64_t bytes, void **dptr);
int mp_free(mp_ctx *ctx, void *dptr);

/* The base address, valid in this process, of rank `rank`'s receive heap (its own
 * heap for rank == ctx's rank; the IPC mapping otherwise).  Lets a caller address a
 * peer's mp_alloc buffer by (base + offset), e.g. for one-sided copies or baselines.
 * Errors: MP_ERR_STATE (model-only), MP_ERR_TOPOLOGY (no such rank). */
int mp_peer_base(mp_ctx *ctx, int rank, void **base);

/* mp_register — make an arbitrary device buffer of this rank a receive target
 * (UCX cuda_ipc "caches IPC memory handles" so a user buffer is mapped once
 * and reused).  COLLECTIVE when world > 1: every rank calls it in the
 * same order (a rank with nothing to register passes buf = NULL, bytes = 0); every
 * rank exports the allocation holding its buffer (cudaIpcGetMemHandle of the base
 * found with cuMemGetAddressRange) and maps every peer's, so any rank may later act
 * as sender or relay for a message into it.  Mappings of one peer allocation are
 * shared between regions (reference-counted).  *id receives the region id, equal on
 * every rank (0 is the heap, never returned).  mp_recv into [buf, buf + bytes) then
 * needs no mp_alloc copy.  The buffer must stay allocated until mp_deregister.
 * world == 1: nothing to map; returns MP_OK with a local id.
 * No transfer may be in flight on any rank (the region table is rewritten).
 * Errors: MP_ERR_STATE (model-only), MP_ERR_NOMEM (region table full, 63 regions),
 * MP_ERR_UNSUPPORTED (the allocation cannot be exported, e.g. VMM / expandable
 * segments), MP_ERR_CUDA. */
int mp_register(mp_ctx *ctx, void *buf, uint64_t bytes, int *id);

/* mp_deregister — collective inverse of mp_register (same order on every rank). */
int mp_deregister(mp_ctx *ctx, int id);

/* ---------------------------------------------------------------- transfer */

/* Eager protocol (reading C23; NEXT f4's low-latency protocol): when
 * world > 1, a message of 1..1048576 bytes skips the rendezvous — one kernel per side,
 * the payload goes over the direct path into a slot the receiver owns (8 slots per
 * sender), and `cfg`'s split is not used.  Both sides classify by size alone; the
 * environment variable MPX_EAGER (equal on every rank, read at mp_init) sets the limit
 * in bytes (0 = off; at most 1 MiB). */
/* mp_send — Step 5 (the pipeline engine moves "the number of chunks and the
 * size of each chunk per path" the model chose) under MPI point-to-point semantics
 * (OMB's MPI_Isend / MPI_Irecv windows; matching FIFO per pair as in MPI).
 * Send `bytes` bytes at device pointer `buf` to rank dst with `tag`.  cfg = NULL
 * selects with mp_select(all paths); otherwise cfg->bytes/chunks/path are used as
 * given (validated: Σ bytes == n, 1 <= k <= max(1, ⌊b/A⌋), chunk <= slot_bytes,
 * paths available).  Stream-ordered: the send kernel waits on the device for the
 * matching mp_recv.  In single-GPU loopback (dst == rank == 0) the send is
 * recorded and the fused transfer is launched by the matching mp_recv.  Staged paths
 * share rings: a send whose relay or host ring was last used by a send on another
 * stream waits for that send first (ring positions follow call order). */
int mp_send(mp_ctx *ctx, const void *buf, uint64_t bytes, int dst, int tag,
            const mp_config *cfg, void *stream);

/* mp_recv — the receiving side of Step 5 with MPI semantics.
 * Receive `bytes` bytes from rank src with `tag` into device pointer `buf`
 * (heap memory or a registered region — mp_register — when world > 1).  Matching is FIFO per (src, dst); the tag and the
 * size must equal the sender's or the device raises MP_ERR_MISMATCH.  Work after
 * mp_recv on `stream` sees the whole message. */
int mp_recv(mp_ctx *ctx, void *buf, uint64_t bytes, int src, int tag, void *stream);

/* Single-process transfer src → dst on this GPU through every selected path
 * (loopback engine; the relay rings and the host ring stand in for the
 * intermediate GPUs and the host).  One fused kernel launch on `stream`.
 * cfg = NULL selects.  Used by calibration, the sweep and the benchmark. */
int mp_xfer(mp_ctx *ctx, void *dst, const void *src, uint64_t bytes, const mp_config *cfg,
            void *stream);

/* Block until all work this context enqueued has finished, then report any
 * sticky device error (MP_ERR_TIMEOUT / MP_ERR_MISMATCH).  A device-wide wait
 * (cudaDeviceSynchronize): it covers every stream the caller passed, including ones
 * destroyed since, and also waits for other work of this process on the device. */
int mp_sync(mp_ctx *ctx);

/* ---------------------------------------------------------------- calibration */

/* Step 1: measure α, β (per link) and ε (per staging device) with the
 * engine's own kernels, fit T(n) = α + n/β (C12) and install the model of every
 * pair plus the shared port.  sizes: byte counts to sweep (NULL = default 16 MiB ..
 * 1 GiB), reps: repeats per size (median).
 * world == 1: the loopback links (HBM copy, relay-ring legs, pinned-host legs).
 * world > 1: collective — every rank puts into its successor's heap over NVLink,
 * times its own host legs and a flag ping-pong through the successor's memory;
 * the measurements are all-gathered and every ordered pair's model is built from
 * them; each rank also times its two host legs at once against alone and every
 * rank's host duplex factor κ (reading C25) is installed (mp_set_host_duplex).
 * Requires empty receive heaps on every rank (call before mp_alloc), else
 * MP_ERR_STATE. */
int mp_calibrate(mp_ctx *ctx, const uint64_t *sizes, int nsizes, int reps);

/* NEXT f4 (P:360 Observation 4): Step 1 per size band (readings C20, C21).  Every
 * link is sampled over 4 KiB .. 1 GiB (capped by the rings / heap) with OMB-style
 * windows of back-to-back copies between the same buffers and fitted
 * per band (as mp_fit_bands); band 0 replaces the pair's model (mp_set_model), band
 * j >= 1 is installed with mp_set_model_band(edges[j]).  ε and, when the pair already
 * has a model, the φ multipliers c are kept (run mp_calibrate first).
 * edges[nedges]: band lower edges in bytes, edges[0] == 0, strictly increasing; NULL
 * = {0, 64 KiB, 256 KiB, 4, 8, 16, 32, 48, 64, 128 MiB}; sampled at powers of two from 4 KiB to
 * 1 GiB plus 6, 12, 24, 48, 96 MiB.  reps: windows per size (median).
 * Collective when world > 1 (same rules as mp_calibrate).
 * Errors: MP_ERR_STATE (model-only), MP_ERR_INVALID (bad edges), MP_ERR_CUDA. */
int mp_calibrate_bands(mp_ctx *ctx, const uint64_t *edges, int nedges, int reps);

/* Save / load the model parameters of every pair (Step 1/2: "once per system
 * topology and stored on each compute node").  The file carries the topology
 * fingerprint and one line per GPU (UUID, NVLinks, PCIe link, NUMA node); loading a
 * file whose fingerprint differs from the context's known topology fails with
 * MP_ERR_TOPOLOGY and installs nothing (a file without a fingerprint, or a context
 * without a topology, is accepted). */
int mp_save_params(mp_ctx *ctx, const char *path);
int mp_load_params(mp_ctx *ctx, const char *path);

/* Launch statistics: number of engine kernels launched by this context so far. */
int mp_stats(mp_ctx *ctx, uint64_t *kernel_launches);

/* ---------------------------------------------------------------- collectives (NEXT f3)
 *
 * PAPER.md §5.3: MPI_Alltoall and MPI_Allreduce as sequences of
 * model-driven multi-path P2P messages, without the host path (host staging
 * degrades bidirectional traffic).  Every P2P step of a collective is one
 * mp_send/mp_recv pair whose config comes from mp_select_flows over the step's
 * known pattern (all ranks send at once, reading C19).  Algorithms (reading C22):
 *   Alltoall : MP_ALGO_BRUCK (UCC's; ⌈log2 W⌉ steps, packed blocks) or
 *              MP_ALGO_PAIRWISE (W−1 steps, one block each).
 *   Allreduce: MP_ALGO_KNOMIAL (radix-2 K-nomial = recursive halving reduce-scatter +
 *              recursive doubling allgather; W a power of two) or
 *              MP_ALGO_RING (any W).
 *   MP_ALGO_AUTO: Bruck below 256 KiB per block, else pairwise; K-nomial when W is a
 *              power of two, else ring.
 * A schedule is data (mp_coll_plan): local copies before, P2P steps, local copies
 * after.  Buffers named in a plan: MP_BUF_SEND (the caller's send buffer),
 * MP_BUF_RECV (the caller's receive buffer), MP_BUF_TMP (library scratch, tmp_bytes).
 * A step sends the concatenation of its send segments to send_to and splits the
 * message it receives from recv_from over its recv segments, copying or — reduce = 1 —
 * adding elementwise. */
enum { MP_COLL_ALLTOALL = 0, MP_COLL_ALLREDUCE = 1 };
enum { MP_ALGO_AUTO = 0, MP_ALGO_BRUCK = 1, MP_ALGO_PAIRWISE = 2, MP_ALGO_KNOMIAL = 3, MP_ALGO_RING = 4 };
enum { MP_BUF_SEND = 0, MP_BUF_RECV = 1, MP_BUF_TMP = 2 };
enum { MP_DT_U8 = 0, MP_DT_I32 = 1, MP_DT_I64 = 2, MP_DT_F32 = 3, MP_DT_F64 = 4, MP_DT_BF16 = 5 };
enum { MP_OP_SUM = 0 };

#define MP_COLL_MAX_STEPS 64
#define MP_COLL_MAX_SEGS 512
#define MP_COLL_MAX_COPIES 64

typedef struct mp_coll_seg { int32_t buf; int32_t reserved; uint64_t off, len; } mp_coll_seg;
typedef struct mp_coll_copy { int32_t src_buf, dst_buf; uint64_t src_off, dst_off, len; } mp_coll_copy;
typedef struct mp_coll_step {
  int32_t send_to, recv_from;    /* ranks (never -1 in the algorithms above) */
  int32_t reduce, reserved;      /* 1: received data is added into the recv segments */
  uint32_t send_seg0, send_nseg; /* slice of mp_coll_plan.seg */
  uint32_t recv_seg0, recv_nseg;
  uint64_t bytes;                /* message bytes = Σ send lengths (the peer's Σ recv lengths) */
} mp_coll_step;
typedef struct mp_coll_plan {
  int32_t coll, algo, world, rank;
  uint64_t tmp_bytes;
  int32_t npre, nsteps, nsegs, npost;
  mp_coll_copy pre[MP_COLL_MAX_COPIES];
  mp_coll_step step[MP_COLL_MAX_STEPS];
  mp_coll_seg seg[MP_COLL_MAX_SEGS];
  mp_coll_copy post[MP_COLL_MAX_COPIES];
} mp_coll_plan;

/* Build rank `rank`'s plan of a collective over `world` ranks.  bytes: per destination
 * block for Alltoall (send and recv buffers hold world·bytes), the whole vector for
 * Allreduce (elem_size-byte elements; blocks split on element boundaries).  algo is
 * resolved (AUTO → the concrete algorithm, stored in out->algo).  Pure host function.
 * Errors: MP_ERR_INVALID (world < 1 or > 16, rank out of range, bytes not a multiple
 * of elem_size, K-nomial with W not a power of two, plan larger than the caps). */
int mp_coll_plan_build(int coll, int algo, int world, int rank, uint64_t bytes, uint32_t elem_size,
                       mp_coll_plan *out);

/* MPI_Alltoall over all ranks of ctx (collective; every rank calls it in the same
 * order): block s of rank r's send buffer (bytes_per_rank bytes at sendbuf + s·B)
 * lands at recvbuf + r·B on rank s.  Device buffers; recvbuf must come from mp_alloc
 * or mp_register when world > 1; sendbuf may be any device buffer.  Stream-ordered on
 * `stream` (the library forks internal send/receive streams from it and joins them
 * back).  world == 1: one local copy.  No P2P message of the caller may be in flight
 * between two ranks while a collective runs (matching is FIFO per pair).
 * Errors: as mp_send / mp_recv, MP_ERR_NOMEM (heap scratch). */
int mp_alltoall(mp_ctx *ctx, const void *sendbuf, void *recvbuf, uint64_t bytes_per_rank, int algo,
                void *stream);

/* MPI_Allreduce(op) of `count` elements of `dtype` (collective): recvbuf = Σ over ranks
 * of sendbuf, on every rank.  sendbuf == recvbuf is allowed (in place).  Integer sums
 * are exact (wrapping); floating-point sums are reassociated by the algorithm (bf16:
 * each addition in fp32, rounded to bf16).  Buffer rules as mp_alltoall.
 * Errors: MP_ERR_INVALID (dtype, op), as mp_alltoall. */
int mp_allreduce(mp_ctx *ctx, const void *sendbuf, void *recvbuf, uint64_t count, int dtype, int op,
                 int algo, void *stream);

/* The same two collectives over an emulated world (mp_init_emulated): ctxs = the
 * world's n contexts in rank order, sendbufs[r] / recvbufs[r] = rank r's buffers (rules
 * as above).  Every rank's plan runs in lock step on `stream`: every rank's pre copies;
 * per step, every rank's packing, then its send and receive as ONE cooperative grid
 * (mp_emu_run), then every rank's unpacking or reduction; every rank's post copies.
 * Returns once `stream` has finished.  Nothing else may be recorded on the world.
 * Errors: MP_ERR_INVALID (arguments, dtype, op, plan), MP_ERR_STATE (not an emulated
 * world), as mp_emu_run. */
int mp_emu_alltoall(mp_ctx **ctxs, int n, const void *const *sendbufs, void *const *recvbufs,
                    uint64_t bytes_per_rank, int algo, void *stream);
int mp_emu_allreduce(mp_ctx **ctxs, int n, const void *const *sendbufs, void *const *recvbufs,
                     uint64_t count, int dtype, int op, int algo, void *stream);

/* The Hockney fit of Step 1 (reading C12), exposed for parity tests: least squares of
 * T = α + n/β over m samples (n[i] bytes, t[i] seconds, host arrays), each residual
 * weighted by 1/t[i]² (relative error), subject to α >= 1e-7 s (Eq 14 needs α > 0:
 * when the free optimum violates it, α = 1e-7 and the slope is refitted for that α);
 * a non-positive slope falls back to β = n[m-1]/t[m-1].  m >= 2, else
 * MP_ERR_INVALID.  Pure host arithmetic, no context. */
int mp_fit_hockney(const double *n, const double *t, int m, double *alpha, double *beta);

/* The per-band Step-1 fit of reading C20 (NEXT f4), exposed for parity tests.
 * edges[nedges]: band lower edges in bytes, edges[0] == 0, strictly increasing.
 * Band j is fitted (as mp_fit_hockney) on the samples with edges[j] <= n[i] <=
 * edges[j+1] (both inclusive; the last band is unbounded above).  A band with fewer
 * than two samples takes the fit of the nearest band above it that has two, else of
 * the nearest below.  alpha[nedges], beta[nedges] receive the fits (host arrays).
 * Errors: MP_ERR_INVALID (bad edges, t <= 0, no band with two samples).  Pure host
 * arithmetic, no context. */
int mp_fit_bands(const double *n, const double *t, int m, const double *edges, int nedges,
                 double *alpha, double *beta);

#ifdef __cplusplus
}
#endif
#endif /* MPX_MP_H */
