// topo.cpp — topology discovery (Step 1's "once per system topology").
//
// PAPER.md §4 extracts the model parameters "once per system topology and stored on
// each compute node", and names what decides the host path's quality: "PCIe
// configuration, and NUMA effects".  mp_init therefore records, per
// GPU of the job: its UUID, PCI location, the NUMA node of its PCIe root (sysfs), its
// PCIe link (NVML: max generation / width, current generation), its active NVLink
// links (NVML) and SM count; per ordered pair of GPUs: peer access, the CUDA P2P
// performance rank and native-atomics support.  The paths of a pair (A1) follow from
// it (a relay r serves s → d only with peer access s → r and r → d), the pinned host
// segments are bound to their GPU's NUMA node, and a fingerprint of it keys the
// parameter file (mp_save_params / mp_load_params).  NVML is loaded with dlopen (no
// link-time dependency); anything it cannot report is 0 ("unknown").
#include <dlfcn.h>
#include <sys/syscall.h>
#include <unistd.h>

#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

#include "ctx.h"

namespace mpx {

namespace {

// The handful of NVML entry points used here (nvml.h types reduced to plain ints).
struct Nvml {
  bool ok = false;
  int (*init)() = nullptr;
  int (*by_pci)(const char *, void **) = nullptr;
  int (*link_state)(void *, unsigned, int *) = nullptr;
  int (*max_gen)(void *, unsigned *) = nullptr;
  int (*max_width)(void *, unsigned *) = nullptr;
  int (*cur_gen)(void *, unsigned *) = nullptr;
};

const Nvml &nvml() {
  static Nvml n = [] {
    Nvml m;
    void *h = dlopen("libnvidia-ml.so.1", RTLD_NOW | RTLD_LOCAL);
    if (!h) return m;
    m.init = reinterpret_cast<int (*)()>(dlsym(h, "nvmlInit_v2"));
    m.by_pci = reinterpret_cast<int (*)(const char *, void **)>(dlsym(h, "nvmlDeviceGetHandleByPciBusId_v2"));
    m.link_state = reinterpret_cast<int (*)(void *, unsigned, int *)>(dlsym(h, "nvmlDeviceGetNvLinkState"));
    m.max_gen = reinterpret_cast<int (*)(void *, unsigned *)>(dlsym(h, "nvmlDeviceGetMaxPcieLinkGeneration"));
    m.max_width = reinterpret_cast<int (*)(void *, unsigned *)>(dlsym(h, "nvmlDeviceGetMaxPcieLinkWidth"));
    m.cur_gen = reinterpret_cast<int (*)(void *, unsigned *)>(dlsym(h, "nvmlDeviceGetCurrPcieLinkGeneration"));
    m.ok = m.init && m.by_pci && m.init() == 0;
    return m;
  }();
  return n;
}

int sysfs_numa_node(int domain, int bus, int dev) {
  char path[128];
  std::snprintf(path, sizeof(path), "/sys/bus/pci/devices/%04x:%02x:%02x.0/numa_node", domain, bus, dev);
  FILE *f = std::fopen(path, "r");
  if (!f) return -1;
  int node = -1;
  if (std::fscanf(f, "%d", &node) != 1) node = -1;
  std::fclose(f);
  return node;
}

uint64_t fnv1a(uint64_t h, const void *p, size_t n) {
  const uint8_t *b = static_cast<const uint8_t *>(p);
  for (size_t i = 0; i < n; ++i) {
    h ^= b[i];
    h *= 0x100000001b3ull;
  }
  return h;
}

}  // namespace

// This process's GPU (c->device).
int topo_local(mp_ctx *c, mp_gpu_info *g) {
  std::memset(g, 0, sizeof(*g));
  cudaDeviceProp p;
  cudaError_t e = cudaGetDeviceProperties(&p, c->device);
  if (e != cudaSuccess) {
    c->last_error = std::string("cudaGetDeviceProperties: ") + cudaGetErrorString(e);
    return MP_ERR_CUDA;
  }
  std::memcpy(g->uuid, p.uuid.bytes, 16);
  g->device = c->device;
  g->pci_domain = p.pciDomainID;
  g->pci_bus = p.pciBusID;
  g->pci_device = p.pciDeviceID;
  g->sms = p.multiProcessorCount;
  g->numa_node = sysfs_numa_node(p.pciDomainID, p.pciBusID, p.pciDeviceID);
  const Nvml &n = nvml();
  if (n.ok) {
    char bdf[32];
    std::snprintf(bdf, sizeof(bdf), "%08X:%02X:%02X.0", p.pciDomainID, p.pciBusID, p.pciDeviceID);
    void *h = nullptr;
    if (n.by_pci(bdf, &h) == 0 && h) {
      unsigned v = 0;
      if (n.max_gen && n.max_gen(h, &v) == 0) g->pcie_gen = static_cast<int32_t>(v);
      if (n.max_width && n.max_width(h, &v) == 0) g->pcie_width = static_cast<int32_t>(v);
      if (n.cur_gen && n.cur_gen(h, &v) == 0) g->pcie_gen_cur = static_cast<int32_t>(v);
      if (n.link_state)
        for (unsigned l = 0; l < 18; ++l) {  // NVML_NVLINK_MAX_LINKS
          int st = 0;
          if (n.link_state(h, l, &st) == 0 && st == 1) g->nvlinks += 1;
        }
    }
  }
  return MP_OK;
}

// P2P attributes of (this process's device) → the device with `uuid`, if this process
// can see it (a job whose processes see every GPU); returns false otherwise.
static bool p2p_query(int my_dev, const char *uuid, int32_t *access, int32_t *perf, int32_t *atomics) {
  int n = 0;
  if (cudaGetDeviceCount(&n) != cudaSuccess) return false;
  for (int d = 0; d < n; ++d) {
    cudaDeviceProp p;
    if (cudaGetDeviceProperties(&p, d) != cudaSuccess) continue;
    if (std::memcmp(p.uuid.bytes, uuid, 16) != 0) continue;
    if (d == my_dev) {
      *access = 1;
      *perf = 0;
      *atomics = 1;
      return true;
    }
    int a = 0, r = 0, t = 0;
    cudaDeviceCanAccessPeer(&a, my_dev, d);
    cudaDeviceGetP2PAttribute(&r, cudaDevP2PAttrPerformanceRank, my_dev, d);
    cudaDeviceGetP2PAttribute(&t, cudaDevP2PAttrNativeAtomicSupported, my_dev, d);
    cudaGetLastError();
    *access = a;
    *perf = r;
    *atomics = t;
    return true;
  }
  return false;
}

// Fill c->topo for world == 1 (this GPU alone) or, collectively, for world > 1.
// mapped[r] = 1 when this rank could IPC-map rank r's memory (the evidence of peer
// access when r's GPU is not visible in this process).
int topo_discover(mp_ctx *c, const std::vector<mp_gpu_info> &gpus, const std::vector<int> &mapped) {
  mp_topology &T = c->topo;
  std::memset(&T, 0, sizeof(T));
  T.world = c->world;
  for (int r = 0; r < c->world; ++r) T.gpu[r] = gpus[r];
  struct Row {
    int32_t access[MP_MAX_PATHS], perf[MP_MAX_PATHS], atomics[MP_MAX_PATHS];
  } me;
  std::memset(&me, 0, sizeof(me));
  for (int r = 0; r < c->world; ++r) {
    int32_t a = 0, p = 0, t = 0;
    if (!p2p_query(c->device, gpus[r].uuid, &a, &p, &t)) {
      a = (r == c->rank || mapped[r]) ? 1 : 0;  // not visible here: the IPC mapping decides
      p = 0;
      t = 0;
    }
    me.access[r] = a;
    me.perf[r] = p;
    me.atomics[r] = t;
  }
  std::vector<Row> rows(c->world);
  if (c->world > 1) {
    if (int s = world_allgather(c, &me, rows.data(), sizeof(Row))) return s;
  } else {
    rows[0] = me;
  }
  for (int s = 0; s < c->world; ++s)
    for (int d = 0; d < c->world; ++d) {
      T.peer_access[s][d] = rows[s].access[d];
      T.p2p_perf_rank[s][d] = rows[s].perf[d];
      T.p2p_atomics[s][d] = rows[s].atomics[d];
    }
  T.fingerprint = topo_fingerprint(T);
  c->have_topo = true;
  return MP_OK;
}

// FNV-1a over what defines the paths and their speeds: the GPUs (UUID, SMs, PCIe link,
// NVLink count, NUMA node) and the peer-access matrix.  Process-local device ordinals
// and the current (power-managed) PCIe generation are excluded.
uint64_t topo_fingerprint(const mp_topology &T) {
  uint64_t h = 0xcbf29ce484222325ull;
  h = fnv1a(h, &T.world, sizeof(T.world));
  for (int r = 0; r < T.world && r < MP_MAX_PATHS; ++r) {
    const mp_gpu_info &g = T.gpu[r];
    h = fnv1a(h, g.uuid, sizeof(g.uuid));
    h = fnv1a(h, &g.sms, sizeof(g.sms));
    h = fnv1a(h, &g.pcie_gen, sizeof(g.pcie_gen));
    h = fnv1a(h, &g.pcie_width, sizeof(g.pcie_width));
    h = fnv1a(h, &g.nvlinks, sizeof(g.nvlinks));
    h = fnv1a(h, &g.numa_node, sizeof(g.numa_node));
    for (int d = 0; d < T.world && d < MP_MAX_PATHS; ++d) h = fnv1a(h, &T.peer_access[r][d], sizeof(int32_t));
  }
  return h ? h : 1;  // 0 means "no topology"
}

// Bind [p, p + n) to NUMA node `node` (preferred) before its pages are first touched,
// so pinned host rings sit next to the GPU that reads them.  No-op for node < 0.
void numa_prefer(void *p, size_t n, int node) {
  if (node < 0 || node >= 64) return;
  unsigned long mask = 1ul << node;
  const long MPOL_PREFERRED_ = 1;
  syscall(SYS_mbind, p, n, MPOL_PREFERRED_, &mask, 64ul, 0u);
}

}  // namespace mpx

// ---------------------------------------------------------------- ABI

using namespace mpx;

extern "C" int mp_get_topology(mp_ctx *c, mp_topology *out) {
  if (!c || !out) return MP_ERR_INVALID;
  if (!c->have_topo) {
    std::memset(out, 0, sizeof(*out));
    out->world = c->world;
    for (int s = 0; s < c->world; ++s)
      for (int d = 0; d < c->world; ++d) out->peer_access[s][d] = 1;  // unknown: all paths assumed
    return MP_OK;
  }
  *out = c->topo;
  return MP_OK;
}

extern "C" int mp_set_topology(mp_ctx *c, const mp_topology *in) {
  if (!c || !in) return MP_ERR_INVALID;
  if (!c->model_only) {
    c->last_error = "mp_set_topology: only a model-only context takes an injected topology";
    return MP_ERR_STATE;
  }
  if (in->world != c->world) {
    c->last_error = "mp_set_topology: world does not match the context";
    return MP_ERR_INVALID;
  }
  c->topo = *in;
  c->topo.fingerprint = topo_fingerprint(c->topo);
  c->have_topo = true;
  c->models.clear();  // the pairs' default paths follow the new topology
  c->bands.clear();
  c->windows.clear();
  c->cache.clear();
  return MP_OK;
}
