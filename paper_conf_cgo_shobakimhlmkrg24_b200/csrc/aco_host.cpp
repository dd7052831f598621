// aco_host.cpp -- host side of the C ABI (include/aco.h): validation and
// preprocessing of regions into the device arena (row a1 of SURVEY 8),
// the workspace plan, the launch sequence of L135-L139, and results.
//
// This is product code: it shares nothing with oracle/.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <atomic>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <new>
#include <thread>
#include <tuple>
#include <vector>

#include "aco_internal.h"

using namespace aco;

// Machine slots per device (c_mach[kMachSlots] in aco_kernels.cu): contexts
// with the same machine share a slot; a slot is rewritten only when no live
// context holds it (after a device synchronisation), so contexts with
// different machines can run on one device in any order.
namespace {
constexpr int kMaxDevices = 64;
struct MachineSlots {
  std::mutex mu;
  MachineDev m[kMaxDevices][kMachSlots]{};
  uint32_t refs[kMaxDevices][kMachSlots]{};
  bool written[kMaxDevices][kMachSlots]{};
  bool attrs[kMaxDevices]{};
};
MachineSlots &machine_slots() {
  static MachineSlots s;
  return s;
}
// Bind a machine to a slot of `device` (the current device); -1 on failure.
int acquire_machine_slot(int device, const MachineDev &m) {
  if (device < 0 || device >= kMaxDevices) return -1;
  MachineSlots &S = machine_slots();
  std::lock_guard<std::mutex> lk(S.mu);
  if (!S.attrs[device]) {
    if (init_kernel_attrs() != 0) return -1;
    S.attrs[device] = true;
  }
  for (uint32_t k = 0; k < kMachSlots; ++k)
    if (S.written[device][k] && std::memcmp(&S.m[device][k], &m, sizeof(m)) == 0) {
      S.refs[device][k]++;
      return (int)k;
    }
  for (uint32_t k = 0; k < kMachSlots; ++k)
    if (S.refs[device][k] == 0) {
      // kernels of a destroyed context may still read this slot
      if (S.written[device][k] && cudaDeviceSynchronize() != cudaSuccess) return -1;
      if (set_machine(k, m) != 0) return -1;
      S.m[device][k] = m;
      S.written[device][k] = true;
      S.refs[device][k] = 1;
      return (int)k;
    }
  return -1;  // more than kMachSlots distinct machines live on this device
}
void release_machine_slot(int device, int slot) {
  if (device < 0 || device >= kMaxDevices || slot < 0) return;
  MachineSlots &S = machine_slots();
  std::lock_guard<std::mutex> lk(S.mu);
  if (S.refs[device][slot]) S.refs[device][slot]--;
}
}  // namespace

// A planned run: launch classes, workspace offsets and the launch context.
struct Plan {
  std::vector<ClassLaunch> launches[3];
  uint32_t fin_smem[3] = {0, 0, 0};
  uint32_t init_smem = 0, p2_smem = 0, max_n = 0, n_upd = 0;
  uint32_t pass_mask = 0, iterations = 0;
  bool any_t32 = false, nc4 = false, timing = false, p2_done = false, stage_img = false, record = false;
  bool fused = false;  // the whole run in one k_fused launch (one block per region)
  uint32_t fused_threads = 0, fused_smem = 0, fused_wl = 0;  // fused_wl: lanes per lane-per-instruction ant (0: one thread per ant)
  uint64_t o_state = 0, o_rws = 0, o_upd = 0, o_gb2 = 0, o_gb2c = 0, o_keys = 0;
  LaunchCtx L{};
};

struct aco_ctx_s {
  int device = 0;
  Plan plan;
  bool planned = false;
  // plan cache: a run with the same parameters, workspace and loaded regions
  // as the previous one reuses its plan (launch classes, workspace layout and
  // the plan blob already in the workspace) -- ~11 ms of host time on C3
  bool cache_ok = false;
  bool cache_hit = false;  // the last make_plan reused the cached plan
  // CUDA graph of a whole aco_schedule_batch (every launch of both passes),
  // captured on the second run of a cached plan and replayed while the plan
  // stays cached (the launch-free iteration loop)
  cudaGraphExec_t gexec = nullptr;
  bool gexec_ok = false;
  uint64_t gexec_launches = 0;
  void drop_graph() {
    if (gexec) cudaGraphExecDestroy(gexec);
    gexec = nullptr;
    gexec_ok = false;
  }
  aco_params cache_params{};
  void *cache_ws = nullptr;
  size_t cache_ws_bytes = 0, cache_need = 0;
  uint32_t cache_ant_base = 0;
  bool cache_colony = false;
  const void *cache_dump[3] = {nullptr, nullptr, nullptr};
  MachineDev mach{};
  int mslot = -1;  // machine slot on `device` (acquire_machine_slot)
  // loaded batch
  uint32_t count = 0;
  std::vector<RegionDev> regions;  // host copy (offsets valid in the arena)
  std::vector<uint64_t> inst_off;  // prefix sums of n
  unsigned char *arena = nullptr;
  size_t arena_bytes = 0;
  // last run
  unsigned char *ws = nullptr;
  size_t ws_bytes = 0;
  void *stream = nullptr;
  RunCfg cfg{};
  uint64_t o_state = 0, o_rws = 0, o_gb2 = 0, o_gb2c = 0;
  bool have_run = false;
  uint64_t launches = 0;
  uint32_t *dump_cost = nullptr;
  uint64_t dump_len[3] = {0, 0, 0};  // elements of the dump buffers (costs, orders, cycles)
  uint16_t *dump_order = nullptr;
  uint32_t *dump_cycle = nullptr;
  std::vector<unsigned char> plan_blob;  // host staging of RegionWs + BlockItems
  std::vector<uint32_t> variants;        // construct variants of the last plan
  // ACO_FLAG_TIMING: event pairs per phase
  std::vector<cudaEvent_t> ev_pool;
  size_t ev_used = 0;
  std::vector<std::pair<size_t, size_t>> ev_pairs[3];
  uint64_t phase_launches[3] = {0, 0, 0};
  // pinned staging buffers for the H2D copies (arena, plan); an event per
  // buffer guards reuse while a previous async copy may still read it
  void *pin[2] = {nullptr, nullptr};
  size_t pin_bytes[2] = {0, 0};
  cudaEvent_t pin_ev[2] = {nullptr, nullptr};
  // internal streams for concurrent construct classes (fork / join per iteration)
  static constexpr int kStreams = 4;
  cudaStream_t side[kStreams] = {nullptr, nullptr, nullptr, nullptr};
  cudaEvent_t fork_ev = nullptr, join_ev[kStreams] = {nullptr, nullptr, nullptr, nullptr};
  // graph stream: the captured run is launched here, ordered after / before
  // the caller's stream by two events (the caller's stream may be the legacy
  // default stream, which cannot be captured)
  cudaStream_t gstream = nullptr;
  cudaEvent_t g_in = nullptr, g_out = nullptr;
  bool side_ok = false;
  bool make_side() {
    if (side_ok) return true;
    if (cudaStreamCreateWithFlags(&gstream, cudaStreamNonBlocking) != cudaSuccess) return false;
    if (cudaEventCreateWithFlags(&g_in, cudaEventDisableTiming) != cudaSuccess) return false;
    if (cudaEventCreateWithFlags(&g_out, cudaEventDisableTiming) != cudaSuccess) return false;
    for (int i = 0; i < kStreams; ++i) {
      if (cudaStreamCreateWithFlags(&side[i], cudaStreamNonBlocking) != cudaSuccess) return false;
      if (cudaEventCreateWithFlags(&join_ev[i], cudaEventDisableTiming) != cudaSuccess) return false;
    }
    if (cudaEventCreateWithFlags(&fork_ev, cudaEventDisableTiming) != cudaSuccess) return false;
    side_ok = true;
    return true;
  }
  ~aco_ctx_s() {
    drop_graph();
    release_machine_slot(device, mslot);
    for (int i = 0; i < kStreams; ++i) {
      if (side[i]) cudaStreamDestroy(side[i]);
      if (join_ev[i]) cudaEventDestroy(join_ev[i]);
    }
    if (fork_ev) cudaEventDestroy(fork_ev);
    if (gstream) cudaStreamDestroy(gstream);
    if (g_in) cudaEventDestroy(g_in);
    if (g_out) cudaEventDestroy(g_out);
    for (cudaEvent_t e : ev_pool) cudaEventDestroy(e);
    for (int i = 0; i < 2; ++i) {
      if (pin_ev[i]) cudaEventDestroy(pin_ev[i]);
      if (pin[i]) cudaFreeHost(pin[i]);
    }
  }
  // Copy `bytes` from host `src` to device `dst` through pinned staging slot k.
  // Pinned staging slot k with at least `bytes` (after its previous copy completed).
  aco_status pinned(int k, size_t bytes, unsigned char **out) {
    if (pin_ev[k]) {
      if (cudaEventSynchronize(pin_ev[k]) != cudaSuccess) return ACO_E_CUDA;
    } else if (cudaEventCreateWithFlags(&pin_ev[k], cudaEventDisableTiming) != cudaSuccess) {
      return ACO_E_CUDA;
    }
    if (pin_bytes[k] < bytes) {
      if (pin[k]) cudaFreeHost(pin[k]);
      pin[k] = nullptr;
      pin_bytes[k] = 0;
      const size_t want = bytes + bytes / 4;
      if (cudaMallocHost(&pin[k], want) != cudaSuccess) return ACO_E_CUDA;
      pin_bytes[k] = want;
    }
    *out = (unsigned char *)pin[k];
    return ACO_OK;
  }
  // H2D of the first `bytes` of pinned slot k (filled by the caller)
  aco_status pinned_h2d(int k, void *dst, size_t bytes, cudaStream_t s) {
    if (cudaMemcpyAsync(dst, pin[k], bytes, cudaMemcpyHostToDevice, s) != cudaSuccess) return ACO_E_CUDA;
    if (cudaEventRecord(pin_ev[k], s) != cudaSuccess) return ACO_E_CUDA;
    return ACO_OK;
  }
  aco_status staged_h2d(int k, void *dst, const void *src, size_t bytes, cudaStream_t s) {
    if (!bytes) return ACO_OK;
    unsigned char *p = nullptr;
    if (aco_status st = pinned(k, bytes, &p)) return st;
    std::memcpy(p, src, bytes);
    return pinned_h2d(k, dst, bytes, s);
  }
  cudaEvent_t next_event() {
    if (ev_used == ev_pool.size()) {
      cudaEvent_t e;
      if (cudaEventCreate(&e) != cudaSuccess) return nullptr;
      ev_pool.push_back(e);
    }
    return ev_pool[ev_used++];
  }
};

namespace {

struct Prepped {
  RegionDev rd{};
  std::vector<unsigned char> image;  // the block image (ImageLayout)
};

// Append array v to the image at a 16-byte aligned offset; returns the offset.
template <typename T>
uint32_t img_put(std::vector<unsigned char> &img, const std::vector<T> &v) {
  const uint64_t off = align16(img.size());
  img.resize(off + v.size() * sizeof(T), 0);
  if (!v.empty()) std::memcpy(img.data() + off, v.data(), v.size() * sizeof(T));
  return (uint32_t)off;
}

// Validation + preprocessing of one region.  Readings R31-R38.
aco_status prep_region(const aco_region_desc &d, const MachineDev &mach, Prepped &P) {
  const uint32_t n_classes = mach.n_classes;
  const uint32_t n = d.n_insts, E = d.n_edges, G = d.n_regs;
  if (n > ACO_MAX_INSTS || G > 16777215u) return ACO_E_TOO_LARGE;
  if (n > kMaxKernelInsts) return ACO_E_TOO_LARGE;
  if ((E && (!d.edge_src || !d.edge_dst || !d.edge_lat)) || (G && (!d.reg_class || !d.reg_flags)) ||
      !d.def_ptr || !d.use_ptr)
    return ACO_E_ARG;
  if (d.def_ptr[0] != 0 || d.use_ptr[0] != 0) return ACO_E_ARG;
  for (uint32_t j = 0; j < n; ++j)
    if (d.def_ptr[j + 1] < d.def_ptr[j] || d.use_ptr[j + 1] < d.use_ptr[j]) return ACO_E_ARG;
  if ((d.def_ptr[n] && !d.def_reg) || (d.use_ptr[n] && !d.use_reg)) return ACO_E_ARG;
  for (uint32_t g = 0; g < G; ++g)
    if (d.reg_class[g] >= n_classes || (d.reg_flags[g] & ~3u)) return ACO_E_ARG;
  // issue types (R42): < n_types on a multi-issue machine, else any type < 4
  const uint32_t n_types = mach.issue_width > 1 ? mach.n_types : 4u;
  if (d.inst_type)
    for (uint32_t j = 0; j < n; ++j)
      if (d.inst_type[j] >= n_types) return ACO_E_ARG;
  uint32_t max_lat = 0;
  for (uint32_t e = 0; e < E; ++e) {
    if (d.edge_src[e] >= n || d.edge_dst[e] >= n) return ACO_E_ARG;
    if (d.edge_lat[e] > ACO_MAX_LATENCY) return ACO_E_TOO_LARGE;
    if (d.edge_src[e] == d.edge_dst[e]) return ACO_E_DDG_CYCLE;
    max_lat = std::max(max_lat, d.edge_lat[e]);
  }
  for (uint32_t k = 0; k < d.def_ptr[n]; ++k)
    if (d.def_reg[k] >= G) return ACO_E_ARG;
  for (uint32_t k = 0; k < d.use_ptr[n]; ++k)
    if (d.use_reg[k] >= G) return ACO_E_ARG;
  // successor CSR (stable by input order) + duplicate check
  std::vector<uint32_t> sp(n + 1, 0), outs(E), lats(E), indeg(n, 0);
  for (uint32_t e = 0; e < E; ++e) sp[d.edge_src[e] + 1]++;
  for (uint32_t j = 0; j < n; ++j) sp[j + 1] += sp[j];
  {
    std::vector<uint32_t> fill(sp.begin(), sp.end() - 1);
    for (uint32_t e = 0; e < E; ++e) {
      const uint32_t s = d.edge_src[e];
      outs[fill[s]] = d.edge_dst[e];
      lats[fill[s]++] = d.edge_lat[e];
      indeg[d.edge_dst[e]]++;
    }
  }
  {
    std::vector<uint32_t> mark(n, 0xFFFFFFFFu);
    for (uint32_t j = 0; j < n; ++j)
      for (uint32_t q = sp[j]; q < sp[j + 1]; ++q) {
        if (mark[outs[q]] == j) return ACO_E_ARG;
        mark[outs[q]] = j;
      }
  }
  // topological order (Kahn), cycle detection
  std::vector<uint32_t> topo;
  topo.reserve(n);
  {
    std::vector<uint32_t> deg(indeg);
    for (uint32_t j = 0; j < n; ++j)
      if (!deg[j]) topo.push_back(j);
    for (size_t h = 0; h < topo.size(); ++h) {
      const uint32_t j = topo[h];
      for (uint32_t q = sp[j]; q < sp[j + 1]; ++q)
        if (--deg[outs[q]] == 0) topo.push_back(outs[q]);
    }
    if (topo.size() != n) return ACO_E_DDG_CYCLE;
  }
  // definitions
  std::vector<uint32_t> def_by(G, 0xFFFFFFFFu);
  for (uint32_t j = 0; j < n; ++j)
    for (uint32_t k = d.def_ptr[j]; k < d.def_ptr[j + 1]; ++k) {
      const uint32_t g = d.def_reg[k];
      if (def_by[g] != 0xFFFFFFFFu || (d.reg_flags[g] & kFlagLiveIn)) return ACO_E_DDG_MULTIDEF;
      def_by[g] = j;
    }
  // uses: de-duplicate per instruction (R33), check defining edges (R38)
  std::vector<uint32_t> uptr(n + 1, 0), ureg;
  std::vector<uint32_t> nuses(G, 0);
  {
    std::vector<uint32_t> seen(G, 0xFFFFFFFFu);
    std::vector<uint32_t> has_edge(n, 0xFFFFFFFFu);
    for (uint32_t j = 0; j < n; ++j) {
      for (uint32_t k = d.use_ptr[j]; k < d.use_ptr[j + 1]; ++k) {
        const uint32_t g = d.use_reg[k];
        if (seen[g] == j) continue;
        seen[g] = j;
        if (!(d.reg_flags[g] & kFlagLiveIn)) {
          const uint32_t p = def_by[g];
          if (p == 0xFFFFFFFFu) return ACO_E_ARG;
          bool found = false;
          for (uint32_t q = sp[p]; q < sp[p + 1] && !found; ++q) found = outs[q] == j;
          if (!found) return ACO_E_DDG_USE_NO_EDGE;
        }
        ureg.push_back(g);
        nuses[g]++;
      }
      uptr[j + 1] = (uint32_t)ureg.size();
    }
  }
  // device limits
  for (uint32_t j = 0; j < n; ++j)
    if (indeg[j] > ACO_MAX_INDEG || uptr[j + 1] - uptr[j] > 255u) return ACO_E_TOO_LARGE;
  for (uint32_t g = 0; g < G; ++g)
    if (nuses[g] > ACO_MAX_USES) return ACO_E_TOO_LARGE;
  if ((uint64_t)n * ((uint64_t)max_lat + 1) >= (1ull << 24)) return ACO_E_TOO_LARGE;
  // register categories (R14, R15): single-use / 2-use (partner check) /
  // >= 3 uses (u16 remaining-use counter); live-out registers never die
  std::vector<uint32_t> ctr(G, 0xFFFFFFFFu);
  uint32_t nctr = 0;
  for (uint32_t g = 0; g < G; ++g)
    if (nuses[g] >= 3 && !(d.reg_flags[g] & kFlagLiveOut)) ctr[g] = nctr++;
  if (nctr > 65535u) return ACO_E_TOO_LARGE;
  std::vector<uint32_t> user0(G, 0xFFFFFFFFu), user1(G, 0xFFFFFFFFu);
  for (uint32_t j = 0; j < n; ++j)
    for (uint32_t k = uptr[j]; k < uptr[j + 1]; ++k) {
      const uint32_t g = ureg[k];
      if (user0[g] == 0xFFFFFFFFu) user0[g] = j;
      else if (user1[g] == 0xFFFFFFFFu) user1[g] = j;
    }
  {
    uint32_t per_class[4] = {0, 0, 0, 0};
    for (uint32_t g = 0; g < G; ++g) per_class[d.reg_class[g]]++;
    for (uint32_t c = 0; c < 4; ++c)
      if (per_class[c] > 65535u) return ACO_E_TOO_LARGE;  // u16 live counters
  }
  // critical path heights (reverse topological relaxation)
  std::vector<uint32_t> cp(n, 0);
  for (size_t h = n; h-- > 0;) {
    const uint32_t j = topo[h];
    uint32_t v = 0;
    for (uint32_t q = sp[j]; q < sp[j + 1]; ++q) v = std::max(v, lats[q] + cp[outs[q]]);
    cp[j] = v;
  }
  uint32_t cp_max = 0;
  for (uint32_t j = 0; j < n; ++j) cp_max = std::max(cp_max, cp[j]);
  // per-instruction info + multi-use entries
  std::vector<uint32_t> info((size_t)n * 4, 0), muse;
  uint32_t L = 0, mc_max = 0;
  uint32_t lbvec[4] = {0, 0, 0, 0}, livein[4] = {0, 0, 0, 0}, liveout[4] = {0, 0, 0, 0};
  for (uint32_t g = 0; g < G; ++g) {
    if (d.reg_flags[g] & kFlagLiveIn) livein[d.reg_class[g]]++;
    if (d.reg_flags[g] & kFlagLiveOut) liveout[d.reg_class[g]]++;
  }
  for (uint32_t c = 0; c < 4; ++c) lbvec[c] = std::max(livein[c], n ? liveout[c] : 0u);
  for (uint32_t j = 0; j < n; ++j) {
    uint32_t defs[4] = {0, 0, 0, 0}, dead[4] = {0, 0, 0, 0}, sk[4] = {0, 0, 0, 0}, usec[4] = {0, 0, 0, 0};
    for (uint32_t k = d.def_ptr[j]; k < d.def_ptr[j + 1]; ++k) {
      const uint32_t g = d.def_reg[k], c = d.reg_class[g];
      defs[c]++;
      if (nuses[g] == 0 && !(d.reg_flags[g] & kFlagLiveOut)) dead[c]++;
    }
    const uint32_t mstart = (uint32_t)muse.size();
    uint32_t nonlo = 0;
    for (uint32_t k = uptr[j]; k < uptr[j + 1]; ++k) {
      const uint32_t g = ureg[k], c = d.reg_class[g];
      usec[c]++;
      if (d.reg_flags[g] & kFlagLiveOut) continue;
      nonlo++;
      if (nuses[g] == 1) {
        sk[c]++;
      } else if (nuses[g] == 2) {
        const uint32_t other = user0[g] == j ? user1[g] : user0[g];
        muse.push_back(other | (c << 16));
      } else {
        muse.push_back(ctr[g] | (c << 16) | kMuseCounter);
      }
    }
    L = std::max(L, nonlo);
    const uint32_t mcnt = (uint32_t)muse.size() - mstart;
    if (mcnt > 15u) return ACO_E_TOO_LARGE;  // 4-bit last-use counters
    {
      uint32_t mc[4] = {0, 0, 0, 0};
      for (uint32_t q = mstart; q < mstart + mcnt; ++q) mc[(muse[q] >> 16) & 3u]++;
      for (uint32_t c = 0; c < 4; ++c) mc_max = std::max(mc_max, mc[c]);
    }
    for (uint32_t c = 0; c < 4; ++c) {
      if (defs[c] > 255u || dead[c] > 255u || sk[c] > 255u) return ACO_E_TOO_LARGE;
      info[(size_t)j * 4 + 0] |= defs[c] << (8 * c);
      info[(size_t)j * 4 + 1] |= sk[c] << (8 * c);
      info[(size_t)j * 4 + 2] |= dead[c] << (8 * c);
      lbvec[c] = std::max(lbvec[c], std::max(defs[c], usec[c]));
    }
    if (mstart >= (1u << 24)) return ACO_E_TOO_LARGE;
    info[(size_t)j * 4 + 3] = (mstart << 8) | mcnt;
  }
  // heuristic tables (R4)
  const uint64_t km1 = (uint64_t)L * (cp_max + 1ull) + cp_max;
  const uint64_t d1 = km1 ? km1 : 1;
  std::vector<uint16_t> eta1((size_t)n * (L + 1)), eta2(n);
  for (uint32_t j = 0; j < n; ++j)
    for (uint32_t l = 0; l <= L; ++l) {
      const uint64_t key = (uint64_t)l * (cp_max + 1ull) + cp[j];
      eta1[(size_t)j * (L + 1) + l] = (uint16_t)(1 + key * 65534ull / d1);
    }
  for (uint32_t j = 0; j < n; ++j) eta2[j] = (uint16_t)(1 + (uint64_t)cp[j] * 65534ull / (cp_max ? cp_max : 1));
  // Row j of the device eta1 table is shifted by j's static kills (single-use
  // registers, always last uses): entry j*(L+1) + d = eta1(j, LUC = sk(j) + d),
  // so a candidate's score needs only its dynamic last-use count d.
  {
    std::vector<uint16_t> sh(eta1.size());
    for (uint32_t j = 0; j < n; ++j) {
      const uint32_t skw = info[(size_t)j * 4 + 1];
      const uint32_t skj = (skw & 0xFF) + ((skw >> 8) & 0xFF) + ((skw >> 16) & 0xFF) + (skw >> 24);
      for (uint32_t d = 0; d <= L; ++d)
        sh[(size_t)j * (L + 1) + d] = eta1[(size_t)j * (L + 1) + std::min(L, skj + d)];
    }
    eta1.swap(sh);
  }
  // pass-specific compact per-instruction records
  std::vector<uint32_t> ds((size_t)n * 4, 0);
  for (uint32_t j = 0; j < n; ++j) {
    ds[4 * j] = info[(size_t)j * 4 + 0];
    ds[4 * j + 1] = info[(size_t)j * 4 + 1];
  }
  // ds.z = eta2 | ready-time slot << 16: the instructions with an incoming
  // edge of latency > 1 get consecutive slots (lean pass-2 layout); the others
  // 0xFFFF (latency-ready as soon as their predecessors are placed)
  uint32_t nslot = 0;
  {
    static const bool all_slots = [] {  // A/B: every instruction owns a slot (the r01 lean layout)
      const char *e = getenv("ACO_SLOTS");
      return e && atoi(e) == 0;
    }();
    std::vector<uint8_t> need(n, all_slots ? 1 : 0);
    for (uint32_t q = 0; q < E; ++q)
      if (lats[q] > 1u) need[outs[q]] = 1;
    for (uint32_t j = 0; j < n; ++j) ds[4 * j + 2] = eta2[j] | ((need[j] ? nslot++ : 0xFFFFu) << 16);
  }
  // ds.w = issue type (R42, bits 0-3) | multi-use register count << 4 |
  // their start in the multi-use list << 8 (the lean pass-2 layout derives
  // the dynamic kills from them)
  for (uint32_t j = 0; j < n; ++j)
    ds[4 * j + 3] = (d.inst_type ? d.inst_type[j] : 0u) | ((info[(size_t)j * 4 + 3] & 0xFFu) << 4) |
                    (info[(size_t)j * 4 + 3] & ~0xFFu);
  // users of each counter register (to find the last remaining user)
  std::vector<uint32_t> cu_ptr(nctr + 1, 0), cu;
  for (uint32_t g = 0; g < G; ++g)
    if (ctr[g] != 0xFFFFFFFFu) cu_ptr[ctr[g] + 1] = nuses[g];
  for (uint32_t m = 0; m < nctr; ++m) cu_ptr[m + 1] += cu_ptr[m];
  cu.resize(cu_ptr[nctr]);
  {
    std::vector<uint32_t> fill(cu_ptr.begin(), cu_ptr.end() - 1);
    for (uint32_t j = 0; j < n; ++j)
      for (uint32_t k = uptr[j]; k < uptr[j + 1]; ++k) {
        const uint32_t g = ureg[k];
        if (ctr[g] != 0xFFFFFFFFu) cu[fill[ctr[g]]++] = j;
      }
  }
  // successor / predecessor lists
  std::vector<uint32_t> succ(E), pp(n + 1, 0), pred(E);
  for (uint32_t q = 0; q < E; ++q) succ[q] = outs[q] | (indeg[outs[q]] == 1 ? kSuccSingle : 0u) | (lats[q] << 16);
  for (uint32_t j = 0; j < n; ++j) pp[j + 1] = pp[j] + indeg[j];
  {
    std::vector<uint32_t> fill(pp.begin(), pp.end() - 1);
    for (uint32_t j = 0; j < n; ++j)
      for (uint32_t q = sp[j]; q < sp[j + 1]; ++q) pred[fill[outs[q]]++] = j | (lats[q] << 16);
  }
  // predecessor groups: per instruction, {bitset word, mask of its
  // predecessors in that word} (readiness test of pass 1 / compact pass 2)
  std::vector<uint32_t> pgp(n + 1, 0), pgv;
  pgv.reserve(2 * (size_t)E);
  std::vector<std::pair<uint32_t, uint32_t>> gr;  // (reused: one allocation per region)
  for (uint32_t v = 0; v < n; ++v) {
    gr.clear();
    for (uint32_t q = pp[v]; q < pp[v + 1]; ++q) {
      const uint32_t p = pred[q] & 0xFFFFu;
      bool found = false;
      for (auto &g : gr)
        if (g.first == p >> 5) {
          g.second |= 1u << (p & 31);
          found = true;
        }
      if (!found) gr.push_back({p >> 5, 1u << (p & 31)});
    }
    std::sort(gr.begin(), gr.end());
    for (auto &g : gr) {
      pgv.push_back(g.first);
      pgv.push_back(g.second);
    }
    pgp[v + 1] = (uint32_t)(pgv.size() / 2);
  }
  // the per-predecessor list is needed only by the u16/u32-cycle pass-2
  // layouts (ready time = max over predecessors at readiness)
  const bool compact = n_classes <= 2 && max_lat <= 511u && mc_max <= 7u;
  if (compact) {
    pred.clear();
    pp.assign(n + 1, 0);
  }
  // initial per-ant state
  const uint32_t nwr = (n + 31) / 32;
  std::vector<uint32_t> rb0(nwr, 0), rem0((nctr + 1) / 2, 0);
  for (uint32_t j = 0; j < n; ++j)
    if (!indeg[j]) rb0[j >> 5] |= 1u << (j & 31);
  for (uint32_t g = 0; g < G; ++g)
    if (ctr[g] != 0xFFFFFFFFu) rem0[ctr[g] >> 1] |= nuses[g] << (16 * (ctr[g] & 1));
  RegionDev &R = P.rd;
  std::memset(&R, 0, sizeof(R));
  std::vector<unsigned char> &img = P.image;
  img.clear();
  R.img.info = img_put(img, info);
  R.img.ds = img_put(img, ds);
  R.img.muse = img_put(img, muse);
  {  // kill tests of the multi-use entries on the per-ant state (lean pass 2):
     // a counter register (RB, SCH, then REM: word 2 nwr + m / 2, half m % 2)
     // is last-used at 1 remaining use; a 2-user register when its partner's
     // scheduled bit (SCH word nwr + p / 32) is set; word < 2 * 256 + 32768 fits 16 bits
    const uint32_t nwr0 = (n + 31) / 32;
    std::vector<uint32_t> mk(muse.size());
    for (size_t q = 0; q < muse.size(); ++q) {
      const uint32_t e = muse[q], c = (e >> 16) & 3u;
      if (e & kMuseCounter) {
        const uint32_t m = e & 0xFFFFu;
        mk[q] = (2 * nwr0 + (m >> 1)) | (((m & 1u) * 16) << 16) | kMkCounter | (c << 22);
      } else {
        const uint32_t pa = e & 0x1FFFu;
        mk[q] = (nwr0 + (pa >> 5)) | ((pa & 31u) << 16) | (c << 22);
      }
    }
    R.img.mk = img_put(img, mk);
  }
  R.img.cu_ptr = img_put(img, cu_ptr);
  R.img.cu = img_put(img, cu);
  R.img.eta1 = img_put(img, eta1);
  R.img.eta2 = img_put(img, eta2);
  R.img.succ_ptr = img_put(img, sp);
  R.img.succ = img_put(img, succ);
  R.img.pred_ptr = img_put(img, pp);
  R.img.pred = img_put(img, pred);
  R.img.rb0 = img_put(img, rb0);
  R.img.rem0 = img_put(img, rem0);
  R.img.pg_ptr = img_put(img, pgp);
  R.img.pg = img_put(img, pgv);
  img.resize(align16(img.size()) + 16, 0);
  R.img.bytes = (uint32_t)img.size();
  R.n = n;
  R.nwr = nwr;
  R.nremw = (nctr + 1) / 2;
  R.L = L;
  R.region_id = d.region_id;
  R.cp_max = cp_max;
  // LB_len = max(1 + CPmax, ceil(n / w), max_y ceil(n_y / min(slots_y, w))) (R30, R42)
  {
    const uint32_t w = std::max(1u, mach.issue_width);
    uint32_t l = (n + w - 1) / w;
    if (n) l = std::max(l, cp_max + 1);
    if (w > 1) {
      uint32_t ny[4] = {0, 0, 0, 0};
      for (uint32_t j = 0; j < n; ++j) ny[d.inst_type ? d.inst_type[j] : 0]++;
      for (uint32_t y = 0; y < 4; ++y) {
        const uint32_t s = std::min(w, (mach.type_slots >> (8 * y)) & 0xFFu);
        if (ny[y]) l = std::max(l, (ny[y] + s - 1) / s);
      }
    }
    R.lb_len = l;
  }
  R.max_cycle_bound = (uint32_t)std::min<uint64_t>(0xFFFFFFFFull, (uint64_t)n * (max_lat + 1ull) + 1);
  R.max_lat = max_lat;
  R.mc_max = mc_max;
  R.compact = compact ? 1u : 0u;
  R.nslot = nslot;
  for (uint32_t c = 0; c < 4; ++c) {
    R.livein[c] = livein[c];
    R.lbvec[c] = lbvec[c];
  }
  return ACO_OK;
}

aco_status cuda_status(cudaError_t e) { return e == cudaSuccess ? ACO_OK : ACO_E_CUDA; }

}  // namespace

extern "C" {

const char *aco_status_string(aco_status st) {
  switch (st) {
    case ACO_OK: return "ok";
    case ACO_E_ARG: return "invalid argument";
    case ACO_E_DDG_CYCLE: return "DDG has a cycle";
    case ACO_E_DDG_MULTIDEF: return "register defined more than once (or live-in defined)";
    case ACO_E_DDG_USE_NO_EDGE: return "use without a def->use edge";
    case ACO_E_TOO_LARGE: return "over a compiled limit";
    case ACO_E_WORKSPACE: return "buffer missing or too small";
    case ACO_E_CUDA: return "CUDA error";
    case ACO_E_STATE: return "call out of order";
    default: return "unknown status";
  }
}

aco_status aco_create(int device, const aco_machine *m, aco_ctx *out) {
  if (!m || !out || m->n_classes < 1 || m->n_classes > 4) return ACO_E_ARG;
  if (m->issue_width > 255u) return ACO_E_ARG;
  if (m->issue_width > 1) {  // R42
    if (m->n_types < 1 || m->n_types > 4) return ACO_E_ARG;
    for (uint32_t y = 0; y < m->n_types; ++y)
      if (m->type_slots[y] < 1 || m->type_slots[y] > 255u) return ACO_E_ARG;
  }
  for (uint32_t c = 0; c < m->n_classes; ++c)
    if (m->step_count[c] < 1 || m->step_count[c] > 16 || m->occ_max < m->step_count[c]) return ACO_E_ARG;
  aco_ctx ctx = new (std::nothrow) aco_ctx_s();
  if (!ctx) return ACO_E_ARG;
  ctx->device = device;
  ctx->mach.n_classes = m->n_classes;
  ctx->mach.occ_max = m->occ_max;
  for (int c = 0; c < 4; ++c) {
    ctx->mach.step_count[c] = m->step_count[c];
    for (int i = 0; i < 16; ++i) ctx->mach.step_max[c][i] = m->step_max[c][i];
    ctx->mach.perp_limit[c] = m->perp_limit[c];
  }
  ctx->mach.issue_width = std::max(1u, m->issue_width);
  ctx->mach.n_types = m->issue_width > 1 ? m->n_types : 1u;
  ctx->mach.type_slots = 0;
  if (m->issue_width > 1)
    for (uint32_t y = 0; y < m->n_types; ++y) ctx->mach.type_slots |= m->type_slots[y] << (8 * y);
  *out = ctx;  // no CUDA call here: the device is touched on first use
  return ACO_OK;
}

void aco_destroy(aco_ctx ctx) { delete ctx; }

aco_status aco_load_regions(aco_ctx ctx, const aco_region_desc *regions, uint32_t count, void *d_arena,
                            size_t arena_bytes, size_t *arena_needed, void *cuda_stream) {
  if (!ctx || (count && !regions)) return ACO_E_ARG;
  ctx->cache_ok = false;
  ctx->drop_graph();
  {  // unique region ids
    std::vector<uint32_t> ids(count);
    for (uint32_t i = 0; i < count; ++i) ids[i] = regions[i].region_id;
    std::sort(ids.begin(), ids.end());
    for (uint32_t i = 1; i < count; ++i)
      if (ids[i] == ids[i - 1]) return ACO_E_ARG;
  }
  // host preprocessing of the regions in parallel (independent per region)
  static const bool dbg_load = getenv("ACO_DEBUG_LOAD") != nullptr;
  const auto t_0 = std::chrono::steady_clock::now();
  std::vector<Prepped> P(count);
  std::vector<aco_status> stv(count, ACO_OK);
  {
    const uint32_t hw = std::max(1u, std::thread::hardware_concurrency());
    const uint32_t nt = std::min<uint32_t>(hw, std::max<uint32_t>(1, count / 16));
    std::atomic<uint32_t> next(0);
    auto work = [&]() {
      for (;;) {
        const uint32_t i = next.fetch_add(1);
        if (i >= count) break;
        stv[i] = prep_region(regions[i], ctx->mach, P[i]);
      }
    };
    std::vector<std::thread> th;
    for (uint32_t t = 1; t < nt; ++t) th.emplace_back(work);
    work();
    for (auto &t : th) t.join();
  }
  for (uint32_t i = 0; i < count; ++i)
    if (stv[i] != ACO_OK) return stv[i];
  const auto t_1 = std::chrono::steady_clock::now();
  // arena layout: RegionDev[count], then every image at a 16-byte aligned offset
  const size_t table = align16(sizeof(RegionDev) * (size_t)count + 16);
  size_t total = table;
  for (uint32_t i = 0; i < count; ++i) {
    P[i].rd.o_image = align16(total);
    total = P[i].rd.o_image + P[i].image.size();
  }
  const size_t need = align256(total);
  if (arena_needed) *arena_needed = need;
  if (!d_arena && getenv("ACO_DEBUG_PLAN")) {  // debug: keep host metadata for a sizing-only plan
    ctx->count = count;
    ctx->regions.resize(count);
    ctx->inst_off.assign(count + 1, 0);
    for (uint32_t i = 0; i < count; ++i) {
      ctx->regions[i] = P[i].rd;
      ctx->inst_off[i + 1] = ctx->inst_off[i] + P[i].rd.n;
    }
    ctx->arena = nullptr;
  }
  if (!d_arena) return ACO_OK;
  if (arena_bytes < need) return ACO_E_WORKSPACE;
  if (cudaSetDevice(ctx->device) != cudaSuccess) return ACO_E_CUDA;
  {  // assemble the arena directly in the pinned staging buffer (threads), one H2D
    unsigned char *pin = nullptr;
    if (aco_status st = ctx->pinned(0, total, &pin)) return st;
    std::memset(pin, 0, table);
    for (uint32_t i = 0; i < count; ++i) std::memcpy(pin + sizeof(RegionDev) * (size_t)i, &P[i].rd, sizeof(RegionDev));
    const uint32_t hw = std::max(1u, std::thread::hardware_concurrency());
    const uint32_t nt = std::min<uint32_t>(hw, std::max<uint32_t>(1, count / 64));
    auto fill = [&](uint32_t t) {
      for (uint32_t i = t; i < count; i += nt) {
        const size_t o = P[i].rd.o_image, e = i + 1 < count ? P[i + 1].rd.o_image : total;
        std::memcpy(pin + o, P[i].image.data(), P[i].image.size());
        std::memset(pin + o + P[i].image.size(), 0, e - o - P[i].image.size());  // (alignment padding)
      }
    };
    std::vector<std::thread> th;
    for (uint32_t t = 1; t < nt; ++t) th.emplace_back(fill, t);
    fill(0);
    for (auto &t : th) t.join();
    if (aco_status st = ctx->pinned_h2d(0, d_arena, total, (cudaStream_t)cuda_stream)) return st;
  }
  if (dbg_load) {
    const auto t_2 = std::chrono::steady_clock::now();
    fprintf(stderr, "[aco load] prep %.2f ms, arena assembly + H2D enqueue %.2f ms (%zu bytes)\n",
            std::chrono::duration<double, std::milli>(t_1 - t_0).count(),
            std::chrono::duration<double, std::milli>(t_2 - t_1).count(), total);
  }
  ctx->count = count;
  ctx->regions.resize(count);
  ctx->inst_off.assign(count + 1, 0);
  for (uint32_t i = 0; i < count; ++i) {
    ctx->regions[i] = P[i].rd;
    ctx->inst_off[i + 1] = ctx->inst_off[i] + P[i].rd.n;
  }
  ctx->arena = (unsigned char *)d_arena;
  ctx->arena_bytes = arena_bytes;
  ctx->have_run = false;
  ctx->planned = false;  // colony calls need a new aco_colony_begin
  return ACO_OK;
}

aco_status aco_set_dump(aco_ctx ctx, uint32_t *d_costs, uint64_t costs_len, uint16_t *d_orders,
                        uint64_t orders_len, uint32_t *d_cycles, uint64_t cycles_len) {
  if (!ctx) return ACO_E_ARG;
  ctx->dump_len[0] = d_costs ? costs_len : 0;
  ctx->dump_len[1] = d_orders ? orders_len : 0;
  ctx->dump_len[2] = d_cycles ? cycles_len : 0;
  ctx->dump_cost = d_costs;
  ctx->dump_order = d_orders;
  ctx->dump_cycle = d_cycles;
  return ACO_OK;
}

namespace {

// Launch shape of one region in one pass: ants per block, lanes per ant and
// whether tau is staged in shared memory.  Ants per block maximise resident
// ants per SM (shared memory is the usual limit); tau in smem is preferred
// unless it costs residency below 256 ants; lanes per ant are the smallest
// that give >= 16 resident warps per SM (latency hiding), within the
// register budget.
struct Shape {
  uint32_t apb, lanes, smem;
  bool ts;
  uint32_t resident = 0;  // resident threads per SM of this shape
  bool ig = false;        // image read through L1 instead of staged in shared memory
  uint32_t need = 0;      // dynamic shared memory the block actually needs (bytes, 128-aligned)
};

// Shared memory per SM and per-block reservation (sm_100: 228 KB per SM,
// at most 227 KB per block, 1 KB reserved by the system per resident block).
constexpr uint32_t kSmemSM = 228 * 1024, kBlockReserve = 1024;

// Dynamic shared memory of a launch whose blocks must fit k per SM: every
// class is keyed by k, so all its blocks reserve exactly this much.
uint32_t smem_for_k(uint32_t k) { return std::min(kSmemPerSM, (kSmemSM / k - kBlockReserve) & ~127u); }

// Launch shape of one region and pass.  Candidates: block = any multiple of
// 32 threads up to 512, lanes per ant L, tau staged or not; k = resident
// blocks per SM allowed by shared memory (smem_for_k), the register budget
// (max_threads) and the hardware (32).  Ranked by resident threads per SM
// capped at target_threads (latency hiding of the per-ant step chain), then
// fewer lanes per ant (less reduction overhead), then tau in shared memory,
// then more resident USEFUL ants (A ants of a region fill ceil(A/apb) blocks),
// then fewer blocks (one image copy per block).
// allow_ig: the image may instead be read through L1 (large regions; wide
// variants), which frees its shared memory for more resident ants; ranked
// after everything else, so it is taken only when it adds resident threads.
uint32_t lane_pow2(uint32_t words) {
  uint32_t l = 1;
  while (l < words && l < 32) l <<= 1;
  return l;
}

Shape pick_shape(uint32_t img, uint32_t tb, uint32_t W, uint32_t max_threads, bool allow_ts, bool lanes14,
                 uint32_t target_threads, uint32_t max_lanes, uint32_t A, uint32_t gsz, uint32_t coin_w,
                 bool allow_ig = false, uint32_t apb_mult = 1, uint32_t spread_cap = 0, uint32_t lane_pref = 1,
                 uint32_t max_block = kMaxBlockThreads) {
  Shape bests[2] = {Shape{0, 1, 0, false}, Shape{0, 1, 0, false}};
  for (int ig = 0; ig <= (allow_ig ? 1 : 0); ++ig) {
  Shape &best = bests[ig];
  uint64_t best_score = 0;
  for (int ts = 1; ts >= 0; --ts) {
    if (ts && (!allow_ts || ig)) continue;  // the image-through-L1 variants keep tau in global memory
    for (uint32_t L : {1u, 2u, 4u, 8u}) {
      if (lanes14 && L != 1 && L != 4) continue;
      if (spread_cap) {  // few ants in the whole batch: lanes ~ bitset words, small blocks
        const uint32_t lp = lanes14 ? (lane_pref >= 4 ? 4u : 1u) : lane_pref;
        if (L != lp) continue;
      } else if (L > max_lanes) {
        continue;
      }
      for (uint32_t threads : {32u, 64u, 96u, 128u, 192u, 256u, 384u, 512u}) {
        if (threads > max_block) break;  // (the kernel's launch bound)
        const uint32_t apb = threads / L;
        if (apb % apb_mult) continue;  // R45: whole ant groups per block
        if (spread_cap && apb > std::max(spread_cap, 32u / L)) break;
        const uint64_t bytes = (uint64_t)(ig ? 0u : img) + (ts ? tb : 0u) + (uint64_t)ant_stride(apb, L) * W * 4 +
                               (uint64_t)coin_groups(apb, gsz) * coin_w * 4;
        if (bytes > kSmemPerSM) break;
        uint32_t k = kSmemSM / ((uint32_t)bytes + kBlockReserve);
        k = std::min(k, max_threads / threads);
        k = std::min(k, 32u);
        while (k && smem_for_k(k) < bytes) --k;
        if (!k) continue;
        const uint64_t thr = std::min<uint64_t>((uint64_t)k * threads, target_threads);
        const uint64_t ants = std::min<uint64_t>((uint64_t)k * std::max(1u, A) / ((std::max(1u, A) + apb - 1) / apb), 4095);
        uint64_t score = (thr << 40) | ((uint64_t)(8 - L) << 32) | ((uint64_t)(ts ? 1 : 0) << 31) |
                         (ants << 12) | (uint64_t)(4095 - k);
        if (spread_cap) score = ((uint64_t)(ts ? 1 : 0) << 40) | ((uint64_t)apb << 20) | (uint64_t)(4095 - k);
        if (score > best_score) {  // strict: the staged image wins ties
          best_score = score;
          best = Shape{apb, L, smem_for_k(k), ts != 0, k * threads, ig != 0, ((uint32_t)bytes + 127u) & ~127u};
        }
      }
    }
  }
  }
  // Reading the image through L1 costs ~15 % per ant-step (measured, n = 300
  // and 450 pass 2); it pays only with >= 20 % more resident ants.
  if (bests[1].apb && (!bests[0].apb || 5ull * bests[1].resident >= 6ull * bests[0].resident)) return bests[1];
  return bests[0];
}

}  // namespace

namespace {

aco_status check_params(const aco_params *p) {
  if (p->pass < 1 || p->pass > 4 || p->cost_mode > 3 || p->group_size == 0 || p->stall_mod == 0 ||
      p->ws_weight > 1024u || p->heur_mix > 1u || p->rl_limit > 2u ||
      p->ants == 0 || p->tau_min > p->tau_max || p->tau_max > 65535u || p->tau0 > 65535u ||
      p->tau0 < p->tau_min || p->tau0 > p->tau_max || p->q0_t > (1ull << 32) || p->rho_q16 > 65536u ||
      p->iterations > 0x7FFFFFFFu)
    return ACO_E_ARG;
  return ACO_OK;
}

// Plan a run (launch classes, workspace layout), upload the plan blob and
// fill ctx->plan.  ants = this context's ants (ant ids ant_base ..).
aco_status make_plan(aco_ctx ctx, const aco_params *p, uint32_t ant_base, void *d_workspace, size_t ws_bytes,
                     size_t *ws_needed, void *cuda_stream, bool colony) {
  if (aco_status st = check_params(p)) return st;
  if (d_workspace && ctx->cache_ok && std::memcmp(p, &ctx->cache_params, sizeof(aco_params)) == 0 &&
      d_workspace == ctx->cache_ws && ws_bytes == ctx->cache_ws_bytes && ant_base == ctx->cache_ant_base &&
      colony == ctx->cache_colony && ctx->cache_dump[0] == ctx->dump_cost &&
      ctx->cache_dump[1] == ctx->dump_order && ctx->cache_dump[2] == ctx->dump_cycle) {
    Plan &P = ctx->plan;  // same run again: the plan and its blob in the workspace are current
    if (ws_needed) *ws_needed = ctx->cache_need;
    P.L.stream = cuda_stream;
    P.L.launches = 0;
    P.p2_done = false;  // per-run flags of the plan
    P.L.cfg.keys = nullptr;
    ctx->ev_used = 0;
    for (int ph = 0; ph < 3; ++ph) {
      ctx->ev_pairs[ph].clear();
      ctx->phase_launches[ph] = 0;
    }
    ctx->stream = cuda_stream;
    ctx->have_run = true;
    ctx->planned = true;
    ctx->cache_hit = true;
    return ACO_OK;
  }
  if (d_workspace) {  // (a sizing call leaves the cached plan intact)
    ctx->cache_ok = false;
    ctx->cache_hit = false;
    ctx->drop_graph();
  }
  if ((p->flags & ACO_FLAG_DUMP) && (!ctx->dump_cost || colony)) return ACO_E_ARG;
  if (p->flags & ACO_FLAG_DUMP) {  // the dump buffers must hold every (pass, iteration) slice
    const uint64_t sn = ctx->inst_off.empty() ? 0 : ctx->inst_off[ctx->count];
    const uint64_t slices = 2ull * p->iterations;
    if (ctx->dump_len[0] < slices * ctx->count * p->ants) return ACO_E_WORKSPACE;
    if (ctx->dump_order && ctx->dump_len[1] < slices * p->ants * sn) return ACO_E_WORKSPACE;
    if (ctx->dump_cycle && ctx->dump_len[2] < slices * p->ants * sn) return ACO_E_WORKSPACE;
  }
  // passes that run construct/finalize launches: pass 4 (weighted, R41) uses the pass-2 machinery
  const uint32_t pmask = p->pass == 4 ? 2u : p->pass;
  const uint32_t count = ctx->count, A = p->ants;
  // R45 (pass-1 ready-list limit): ant groups in lockstep inside one block;
  // not with the shared colony (a group would span ranks)
  const bool rl1 = p->rl_limit != 0 && (pmask & 1u);
  if (p->rl_limit && colony) return ACO_E_ARG;
  Plan saved = ctx->plan;  // a sizing call must not disturb a planned run
  Plan &P = ctx->plan;
  P = Plan();
  // ---- per-pass construct classes
  struct Cls {
    Shape sh;
    bool mask, t32, gs, wide = false, lean = false;
    uint32_t smem;
    std::vector<std::pair<uint64_t, uint32_t>> regs;  // (~work, region)
  };
  using Key = std::tuple<uint32_t, uint32_t, uint32_t, bool, bool, bool, bool, uint32_t, bool, bool, bool>;
  std::map<Key, Cls> classes;
  P.nc4 = ctx->mach.n_classes > 2;
  // launch-shape policy (tuning knobs; defaults measured on B200)
  uint32_t tgt_threads[2] = {384, 768}, max_lanes[2] = {8, 1};  // pass 1: 384 (C3 320/384/448/512: 615/615/625/625 ms)
  if (const char *e = getenv("ACO_TARGET_THREADS")) sscanf(e, "%u,%u", &tgt_threads[0], &tgt_threads[1]);
  if (const char *e = getenv("ACO_MAX_LANES")) sscanf(e, "%u,%u", &max_lanes[0], &max_lanes[1]);
  uint32_t max_lanes_w[2] = {max_lanes[0], max_lanes[1]};  // wide (large-region) classes
  uint32_t gs_min_threads[2] = {128, 64};  // measured: tools/probe_sizes.sh
  uint32_t gs_lanes[2] = {16, 16};
  // Spread mode: a batch with few ants in total (one region of 1,024 ants,
  // config 2; FIX10-A, config 1) cannot fill the SMs with large blocks, so
  // the ants are spread over >= 148 small blocks with lanes ~ bitset words
  // (the per-ant step latency, not issue slots, is then the bound).
  uint32_t spread_cap = 0;
  {
    const uint64_t total = (uint64_t)A * count;
    // measured: C2 75 -> 80 ms (the per-ant step latency, not the SM count,
    // bounds one region of 1,024 ants), so off unless asked for
    bool on = false;
    if (const char *e = getenv("ACO_SPREAD")) on = total < 148ull * 64 && atoi(e) != 0;
    if (on) spread_cap = (uint32_t)std::max<uint64_t>(1, (total + 147) / 148);
    if (const char *e = getenv("ACO_SPREAD_CAP")) spread_cap = on ? (uint32_t)atoi(e) : 0u;
  }
  // regions with at least this many instructions take the 4-wide candidate
  // scan (and, in pass 2, the lean layout), per pass.  Measured (r02s, ns per
  // ant-step at n = 130): pass 1 0.052 (1-wide) vs 0.056 (4-wide); pass 2
  // 0.077 vs 0.066
  uint32_t wide_n[2] = {kWideN, 120};
  if (const char *e = getenv("ACO_WIDE_N")) sscanf(e, "%u,%u", &wide_n[0], &wide_n[1]);
  bool smem_exact = true;  // classes reserve the shared memory they need (ACO_SMEM_EXACT)
  if (const char *e = getenv("ACO_SMEM_EXACT")) smem_exact = atoi(e) != 0;
  bool fill_sms = true;  // spread passes with fewer shared-memory blocks than SMs (below)
  if (const char *e = getenv("ACO_FILL")) fill_sms = atoi(e) != 0;
  uint32_t fill_img_max = 64 * 1024;
  uint32_t fill_lanes[2] = {0, 0};  // lanes per ant of spread shapes (0: the rule below)
  if (const char *e = getenv("ACO_FILL_LANES")) sscanf(e, "%u,%u", &fill_lanes[0], &fill_lanes[1]);
  if (const char *e = getenv("ACO_FILL_IMG")) fill_img_max = (uint32_t)atoi(e);
  uint32_t spread_lanes = 0;  // 0: lanes ~ bitset words
  if (const char *e = getenv("ACO_SPREAD_LANES")) spread_lanes = (uint32_t)atoi(e);
  uint32_t img_l1[2] = {0, 1};  // large regions may read the image through L1 (pass 2; pass 1 measured slower)
  if (const char *e = getenv("ACO_IMG_L1")) sscanf(e, "%u,%u", &img_l1[0], &img_l1[1]);
  bool lean_on = true;  // pass-2 lean layout for large regions
  if (const char *e = getenv("ACO_LEAN")) lean_on = atoi(e) != 0;
  uint32_t lean_gain = 0;  // % more resident ants the lean layout must reach (C3: 0 measured best)
  // pass-1 lean layout for large regions: off -- measured slower than the
  // stored last-use counts despite ~1.8x the resident ants (r02g: n = 450 /
  // 900 pass 1 0.174 / 0.314 -> 0.186 / 0.392 ns per ant-step; C5 1819 ->
  // 1911 ms; C3 710 -> 706 ms, noise); kept for A/B (ACO_LEAN1=1)
  bool lean1_on = false;
  if (const char *e = getenv("ACO_LEAN1")) lean1_on = atoi(e) != 0;
  uint32_t lean1_gain = 20;
  if (const char *e = getenv("ACO_LEAN1_GAIN")) lean1_gain = (uint32_t)atoi(e);
  if (const char *e = getenv("ACO_LEAN_GAIN")) lean_gain = (uint32_t)atoi(e);
  const bool gs_lanes_env = getenv("ACO_GS_LANES") != nullptr;
  // lane-per-instruction ants (one warp per ant, its state in registers;
  // aco_kernels.cu lpi_pass1/2) for regions of <= 128 instructions when the
  // whole batch has few ants, i.e. the per-ant step latency -- not issue
  // slots -- bounds the run (config 2: one region of 1,024 ants).
  // ACO_LPI: 0 off, 1 auto (default), 2 every eligible region (tests)
  uint32_t lpi_mode = 1;
  if (const char *e = getenv("ACO_LPI")) lpi_mode = (uint32_t)atoi(e);
  // ants (= warps) in the whole batch; measured crossover (tools/lpi_crossover.py,
  // profiles/r03_lpi_crossover.md): k regions of n = 30-128 with 1,024 ants
  // each, lane-per-instruction faster at 4,096 ants (n = 100: 6.4 vs 7.7 ms),
  // slower at 8,192 (11.2 vs 8.0 ms)
  uint64_t lpi_max_ants = 148ull * 32;
  if (const char *e = getenv("ACO_LPI_ANTS")) lpi_max_ants = strtoull(e, nullptr, 10);
  const bool lpi_batch = lpi_mode == 2 || (lpi_mode == 1 && (uint64_t)A * count <= lpi_max_ants);
  // huge regions (n > 1024): per-ant state in shared memory, image and tau
  // through L1/L2, 8 lanes per ant, 32-ant blocks, as many waves as needed.
  // Round 2 ran them on the global-state kernels: the first shared-state
  // version (every ant resident in one wave, 2 blocks reserving 113 KB each,
  // 64 registers) left L1 28 KB and spilled: C4 832 -> 1098 ms.  r03: the
  // blocks reserve exactly their state (L1 keeps ~120 KB for the image), 128
  // registers (launch bound ACO_HUGE_MINB = 1), waves allowed:
  // C4 842 -> 738 ms, C5 1927 -> 1813 ms (tools/gpu_r03e.sh, r03f.sh)
  bool huge_smem = true;
  if (const char *e = getenv("ACO_HUGE_SMEM")) huge_smem = atoi(e) != 0;
  // ... resident blocks per SM its kernels allow, several waves of ants
  // allowed, shared memory per SM capped (0: no cap), exact reservation, lanes
  uint32_t huge_k = 2, huge_waves = 1, huge_exact = 1, huge_lanes[2] = {8, 8};
  uint64_t huge_smem_max = 0;
  if (const char *e = getenv("ACO_HUGE_LANES")) sscanf(e, "%u,%u", &huge_lanes[0], &huge_lanes[1]);
  // In a batch with few ants in total (<= 148 x 512: config 5, not config 3)
  // regions above huge_min_n instructions take the huge-region kernels even
  // when a shared-memory shape exists: with few regions in flight the
  // standard blocks leave the SMs latency-starved (tools/gpu_r03s.sh / r03t.sh:
  // C5 1773 -> 1363 ms, its n = 500 row 155 -> 75 ms and n = 1,000 row
  // 602 -> 225 ms; forcing it on config 3 costs 690 -> 1104 ms)
  uint32_t huge_min_n = 400;
  if (const char *e = getenv("ACO_HUGE_MIN_N")) huge_min_n = (uint32_t)atoi(e);
  uint64_t huge_few_ants = 148ull * 512;
  if (const char *e = getenv("ACO_HUGE_FEW_ANTS")) huge_few_ants = strtoull(e, nullptr, 10);
  const bool huge_few = (uint64_t)A * count <= huge_few_ants;
  if (const char *e = getenv("ACO_HUGE_K")) huge_k = (uint32_t)atoi(e);
  if (const char *e = getenv("ACO_HUGE_WAVES")) huge_waves = (uint32_t)atoi(e);
  if (const char *e = getenv("ACO_HUGE_EXACT")) huge_exact = (uint32_t)atoi(e);
  if (const char *e = getenv("ACO_HUGE_SMEM_KB")) huge_smem_max = 1024ull * strtoull(e, nullptr, 10);
  uint32_t gs_wide[2] = {1, 1};  // 4-wide scan in the global-state kernels, per pass
  if (const char *e = getenv("ACO_GS_WIDE")) {
    if (sscanf(e, "%u,%u", &gs_wide[0], &gs_wide[1]) == 1) gs_wide[1] = gs_wide[0];
  }
  // ... with at most this many lanes per ant (pass 1, pass 2).  Measured
  // (r02d/h, ms per step): C5 (4 lanes) 1963 -> 1808; C4 (16 lanes) both
  // passes 855 -> 872, pass 1 only 894 -> 822 (pass 2 has ~5 ready
  // candidates per step at n = 2,000: a 4-wide batch rarely fills, and the
  // 64-register cap spills)
  uint32_t gs_wide_lanes[2] = {16, 8};
  if (const char *e = getenv("ACO_GS_WIDE_LANES")) {
    if (sscanf(e, "%u,%u", &gs_wide_lanes[0], &gs_wide_lanes[1]) == 1) gs_wide_lanes[1] = gs_wide_lanes[0];
  }
  if (const char *e = getenv("ACO_GS_LANES")) sscanf(e, "%u,%u", &gs_lanes[0], &gs_lanes[1]);
  if (const char *e = getenv("ACO_GS_MIN_THREADS")) sscanf(e, "%u,%u", &gs_min_threads[0], &gs_min_threads[1]);
  if (const char *e = getenv("ACO_MAX_LANES_WIDE")) sscanf(e, "%u,%u", &max_lanes_w[0], &max_lanes_w[1]);
  // registers of the construct kernels bound the resident threads per SM
  static uint32_t s_mt[16][2][3];
  static bool s_mt_ok[16];
  uint32_t mt[2][3];
  {
    const int dv = ctx->device >= 0 && ctx->device < 16 ? ctx->device : 0;
    if (!s_mt_ok[dv]) s_mt_ok[dv] = construct_max_threads(ctx->device, s_mt[dv]) == 0;
    if (s_mt_ok[dv]) std::memcpy(mt, s_mt[dv], sizeof(mt));
    else construct_max_threads(-2, mt);  // conservative defaults (no device: sizing only)
  }
  // Lanes per ant of the global-state (huge-region) kernels: enough lanes to
  // fill the SMs when few ants take that path (config 4: one region, 8,192
  // ants -> 16 lanes), fewer when many do (config 5: every n >= ~1,500 region
  // -> 4 lanes): ~148 x 1,024 threads in flight.  Measured (ms): C4 16/8/4
  // lanes 423/583/827, C5 2,961/2,529/2,328.
  uint64_t gs_ants[2] = {0, 0};  // ants of the regions that leave the shared-memory kernels, per pass
  {
    for (uint32_t r = 0; r < count; ++r) {
      const RegionDev &R = ctx->regions[r];
      if (R.n <= 600) continue;  // (host time: smaller regions always fit shared memory)
      const bool t32 = (P.nc4 ? R.max_cycle_bound > 65535u : (R.max_lat > 511u || R.mc_max > 7u));
      for (uint32_t pass = 1; pass <= 2; ++pass) {
        if (!(pmask & pass)) continue;
        const bool wide = R.n >= wide_n[pass - 1] && R.n <= 1024, rare = pass == 2 && (t32 || P.nc4);
        const uint32_t W = ant_words(pass, R.n, R.nwr, R.nremw, pass == 2 && t32, P.nc4);
        const Shape sh = pick_shape(R.img.bytes, tau_smem_bytes(R.n), W, mt[pass - 1][wide], !rare, rare,
                                    pass == 1 ? tgt_threads[0] : tgt_threads[1], (wide ? max_lanes_w : max_lanes)[pass - 1],
                                    A, p->group_size, coin_words(pass, R.n));
        if (sh.apb == 0 || sh.resident < gs_min_threads[pass - 1]) gs_ants[pass - 1] += A;
      }
    }
    for (int q = 0; q < 2 && !gs_lanes_env; ++q) {
      const uint64_t per = gs_ants[q] ? (148ull * 1024) / gs_ants[q] : 16;
      gs_lanes[q] = per >= 16 ? 16u : (per >= 8 ? 8u : 4u);
    }
  }
  std::vector<uint8_t> gs(count, 0);
  std::vector<uint32_t> gs_words(count, 0), scratch_words(count, 0);
  // Shape of one region in one pass (spread: ants-per-block cap with the
  // given lanes per ant, 0 = off).
  struct RegionPlan {
    Shape sh;
    bool g = false, lean = false, t32 = false, wide = false, on = false, huge = false, lpi = false;
    uint32_t W = 0;
  };
  auto plan_region = [&](uint32_t r, uint32_t pass, uint32_t spread, uint32_t lane_pref) {
    RegionPlan q;
    const RegionDev &R = ctx->regions[r];
    // pass-2 state variant: the compact layout (windowed u8 ready times) needs
    // latencies < 512, 2 classes and <= 7 multi-use registers per class and
    // instruction; otherwise u16 cycles (3-4 classes), or u32 when a
    // schedule may exceed 65535 cycles (or the compact layout does not apply)
    // (the general machine model, R42, runs in every layout but lean)
    const bool t32 = (P.nc4 ? R.max_cycle_bound > 65535u : (R.max_lat > 511u || R.mc_max > 7u));
    q.t32 = t32;
    const bool wide = R.n >= wide_n[pass - 1] && R.n <= 1024;
    q.wide = wide;
    // lean pass-2 layout (u8 ready times, kills derived at evaluation):
    // large regions, single issue, 2 classes, latencies < 128
    bool lean = pass == 2 && lean_on && wide && !t32 && !P.nc4 && ctx->mach.issue_width <= 1 && R.max_lat < 128u;
    uint32_t W = ant_words(pass, R.n, R.nwr, R.nremw, pass == 2 && t32, P.nc4);  // lean: decided below
    if (getenv("ACO_DEBUG_REGIONS"))
      fprintf(stderr, "[aco region] %u n %u pass %u img %u words %u nremw %u L %u\n", r, R.n, pass, R.img.bytes, W,
              R.nremw, R.L);
    if (lpi_batch && R.n >= 1 && R.n <= 128 && !P.nc4 && !p->heur_mix && !(rl1 && pass == 1) &&
        (pass == 1 || (ctx->mach.issue_width <= 1 && (uint64_t)R.max_cycle_bound + R.max_lat < 65536u))) {
      // (pass 2: single issue; ready times are u16 pairs in registers)
      // one warp per ant: ~148 blocks over the batch's ants (<= 8 warps each)
      const uint64_t tot = (uint64_t)A * count;
      uint32_t apb = (uint32_t)std::min<uint64_t>(kLpiMaxThreads / 32, std::max<uint64_t>(1, (tot + 147) / 148));
      apb = std::min(apb, std::max(1u, A));
      const uint64_t fixed = (uint64_t)ant_stride(apb, 32) * lpi_words(R.nremw) * 4 +
                             (uint64_t)coin_groups(apb, p->group_size) * coin_words(pass, R.n) * 4 + R.img.bytes;
      const bool ts = fixed + tau_smem_bytes(R.n) <= kSmemPerSM;
      const uint64_t bytes = fixed + (ts ? tau_smem_bytes(R.n) : 0u);
      if (bytes <= kSmemPerSM) {
        uint32_t k = std::min<uint32_t>(kSmemSM / ((uint32_t)bytes + kBlockReserve), 64u / apb);
        k = std::max(1u, std::min(k, 32u));
        while (k > 1 && smem_for_k(k) < bytes) --k;
        q.sh = Shape{apb, 32, smem_for_k(k), ts, k * apb * 32, false, ((uint32_t)bytes + 127u) & ~127u};
        q.lpi = true;
        q.W = lpi_words(R.nremw);
        q.wide = false;
        q.on = true;
        return q;
      }
    }
    const bool rare = pass == 2 && (t32 || P.nc4);  // variants compiled without tau staging, 1|4 lanes
    Shape sh = pick_shape(R.img.bytes, tau_smem_bytes(R.n), W, mt[pass - 1][wide], !rare, rare,
                          pass == 1 ? tgt_threads[0] : tgt_threads[1], (wide ? max_lanes_w : max_lanes)[pass - 1], A,
                          p->group_size, coin_words(pass, R.n) + (rl1 && pass == 1 ? 6u : 0u),
                          wide && !rare && img_l1[pass - 1], rl1 && pass == 1 ? p->group_size : 1u,
                          rl1 && pass == 1 ? 0u : spread, lane_pref);
    if (pass == 1 && lean1_on && wide && !q.t32) {
      // lean pass-1 layout (no stored last-use counts: derived from the
      // remaining-use counters and scheduled bits at evaluation, one lane per
      // ant): taken when it keeps >= lean1_gain % more ants resident
      const uint32_t Wl = ant_words(1, R.n, R.nwr, R.nremw, false, P.nc4, true);
      const Shape shl = pick_shape(R.img.bytes, tau_smem_bytes(R.n), Wl, mt[0][2], false, false, tgt_threads[0], 1, A,
                                   p->group_size, coin_words(1, R.n) + (rl1 ? 6u : 0u), img_l1[0] != 0,
                                   rl1 ? p->group_size : 1u, rl1 ? 0u : spread, 1u, kLeanMaxThreads);
      const uint64_t base_ants = sh.apb ? sh.resident / sh.lanes : 0;
      if (shl.apb && 100ull * shl.resident >= (100ull + lean1_gain) * base_ants) {
        sh = shl;
        W = Wl;
        lean = true;
      }
    }
    if (pass == 2 && lean && sh.lanes != 1) lean = false;  // (lean variants: one lane per ant)
    if (pass == 2 && lean) {
      // the lean layout costs per ant-step (kills derived at every
      // evaluation) and gains resident ants; on the mixed C3 batch it wins
      // whenever it fits at least as many ants (B200: 684 -> 645 ms/batch;
      // ACO_LEAN_GAIN = 20 / 50 %: 654 ms)
      const uint32_t Wl = ant_words(pass, R.n, R.nwr, R.nremw, false, P.nc4, true, R.nslot);
      const Shape shl = pick_shape(R.img.bytes, tau_smem_bytes(R.n), Wl, mt[1][2], false, false, tgt_threads[1], 1, A,
                                   p->group_size, coin_words(pass, R.n), img_l1[1] != 0, 1u, spread, 1u, kLeanMaxThreads);
      if (shl.apb && 100ull * shl.resident >= (100ull + lean_gain) * sh.resident) {
        sh = shl;
        W = Wl;
      } else {
        lean = false;
      }
    }
    // Huge regions whose image + state leave fewer than gs_min_threads
    // resident per SM are latency-starved in shared memory: the
    // global-state kernels (all ants resident, state through L1/L2) win
    // (measured: n = 2,000 pass 1, 1 warp/SM in smem, 9x slower).
    // (not for a spread shape: there few resident ants per SM is the point)
    if (sh.apb != 0 && !spread && sh.resident < gs_min_threads[pass - 1]) sh.apb = 0;
    const bool force_huge = huge_few && huge_min_n < 1024u && R.n > huge_min_n;
    const Shape sh_std = sh;
    if ((sh.apb == 0 || force_huge) && huge_smem && (R.n > 1024 || force_huge) && !t32 && !P.nc4 &&
        !(rl1 && pass == 1)) {
      // Huge regions with the per-ant state in SHARED memory, the image and
      // tau through L1, the global-state lane count and the 4-wide strided
      // scan; pass 2 in the lean layout when its latencies allow -- taken
      // when every ant of the path stays resident (one wave), else the
      // global-state kernels below
      const uint32_t gl = huge_lanes[pass - 1];
      const bool hl = pass == 2 && lean_on && R.max_lat < 128u && ctx->mach.issue_width <= 1;
      const uint32_t Wh = hl ? ant_words(2, R.n, R.nwr, R.nremw, false, false, true, R.nslot)
                             : ant_words(pass, R.n, R.nwr, R.nremw, false, false);
      const uint32_t maxb = kMaxBlockThreads;  // (huge variants: 512-thread bound, ACO_HUGE_MINB blocks per SM)
      const uint64_t need = std::max<uint64_t>(1, gs_ants[pass - 1]);
      for (uint32_t apb : {32u, 16u, 8u, 4u, 2u}) {
        const uint32_t thr = apb * gl;
        if (thr > maxb || thr < 32 || thr % 32) continue;
        const uint64_t bytes = (uint64_t)ant_stride(apb, gl) * Wh * 4 +
                               (uint64_t)coin_groups(apb, p->group_size) * coin_words(pass, R.n) * 4;
        if (bytes > kSmemPerSM) continue;
        uint32_t k = std::min<uint32_t>(kSmemSM / ((uint32_t)bytes + kBlockReserve), huge_k);  // (launch bound)
        k = std::min<uint32_t>(k, std::max<uint32_t>(1, 65536u / (thr * 128u)));  // (<= 128 registers per thread)
        while (k && smem_for_k(k) < bytes) --k;
        if (k && huge_smem_max && k * bytes > huge_smem_max) k = std::max<uint64_t>(1, huge_smem_max / bytes);
        if (!k || (!huge_waves && 148ull * k * apb < need)) continue;
        // (exact: the block reserves what it needs; the rest of the SM's
        // 256 KB stays L1 for the image and tau read through it)
        sh = Shape{apb, gl, smem_for_k(k), false, k * thr, true, huge_exact ? (((uint32_t)bytes + 127u) & ~127u) : 0u};
        q.huge = true;
        lean = hl;
        W = Wh;
        break;
      }
      if (!q.huge) sh = sh_std;
    }
    if (sh.apb == 0) {  // does not fit shared memory: global-state kernels
      // all ants are resident (state in the workspace); 16 lanes per ant
      // and 512-thread blocks measured best (tools/probe_gs_lanes.sh:
      // n = 2000, 8192 ants: 4 lanes x 64 ants 206 + 53 ms -> 45 + 34 ms
      // per 2 iterations), fewer ants per block when A is small
      uint32_t gl = gs_lanes[pass - 1];
      if (pass == 2 && (t32 || P.nc4)) gl = 4;  // the u16/u32-cycle GS variants have 4 lanes
      uint32_t gapb = std::min<uint64_t>(kMaxBlockThreads / gl, std::max<uint64_t>(8u, ((uint64_t)A * count / 148) & ~7ull));
      if (const char *e = getenv("ACO_GS_APB")) gapb = (uint32_t)atoi(e);
      while (gapb * gl > kMaxBlockThreads) gapb /= 2;
      sh = Shape{gapb, gl, 0, false};
      q.g = true;
      lean = false;
      W = ant_words(pass, R.n, R.nwr, R.nremw, pass == 2 && t32, P.nc4);
    }
    q.sh = sh;
    q.lean = lean;
    q.W = W;
    q.on = true;
    return q;
  };
  std::vector<RegionPlan> rp(2 * (size_t)count);
  for (uint32_t pass = 1; pass <= 2; ++pass) {
    if (!(pmask & pass)) continue;
    uint64_t blocks = 0, ants_smem = 0;
    for (uint32_t r = 0; r < count; ++r) {
      RegionPlan &q = rp[2 * r + pass - 1];
      q = plan_region(r, pass, spread_cap, spread_lanes ? spread_lanes : std::min(8u, lane_pow2(ctx->regions[r].nwr)));
      if (q.sh.apb == 0 && rl1 && pass == 1) {  // R45 needs a block-wide lockstep: shared-memory kernels only
        ctx->plan = saved;
        return ACO_E_ARG;
      }
      if (!q.g) {
        blocks += (A + q.sh.apb - 1) / q.sh.apb;
        ants_smem += A;
      }
    }
    // Fill the SMs in proportion to work: a region holding the share w_r of
    // the pass's work should spread its ants over >= 148 w_r blocks, else its
    // few large blocks run alone at the end of the pass while SMs idle (few
    // large regions: configs 2 and 5).  Such a region keeps its lanes per ant
    // and caps its ants per block (the ant step is latency-bound at this
    // scale: more SMs at fewer warps each); many-region batches (config 3)
    // are unaffected (w_r is tiny).
    if (fill_sms && !spread_cap && !(rl1 && pass == 1) && ants_smem) {
      double wtot = 0;
      for (uint32_t r = 0; r < count; ++r) wtot += (double)ctx->regions[r].n * (ctx->regions[r].n + 16.0);
      for (uint32_t r = 0; r < count; ++r) {
        RegionPlan &q = rp[2 * r + pass - 1];
        // (regions with a large image stay: staging it into more blocks costs
        // more than the extra SMs give -- C5 n = 1,000: 599 -> 643 ms)
        if (q.g || q.lpi || wtot <= 0 || ctx->regions[r].img.bytes > fill_img_max) continue;
        const double nr = ctx->regions[r].n;
        const uint32_t need = (uint32_t)std::ceil(148.0 * nr * (nr + 16.0) / wtot);
        const uint32_t have = (A + q.sh.apb - 1) / q.sh.apb;
        if (need <= have) continue;
        // lanes of a spread shape: pass 1 takes up to 4 lanes per bitset word
        // group (latency-bound at few ants per SM; C2: 72.6 -> 66.2 ms), pass 2
        // keeps the default pick's (more lanes measured slower: 76 / 83 ms)
        uint32_t fl = fill_lanes[pass - 1];
        if (!fl) fl = pass == 1 ? std::max(q.sh.lanes, std::min(4u, lane_pow2(ctx->regions[r].nwr))) : q.sh.lanes;
        const RegionPlan f = plan_region(r, pass, std::max(1u, (A + need - 1) / need), fl);
        if (!f.g && f.sh.apb && (A + f.sh.apb - 1) / f.sh.apb > have) q = f;
      }
    }
  }
  for (uint32_t r = 0; r < count; ++r) {
    const RegionDev &R = ctx->regions[r];
    P.max_n = std::max(P.max_n, R.n);
    for (uint32_t pass = 1; pass <= 2; ++pass) {
      const RegionPlan &q = rp[2 * r + pass - 1];
      P.any_t32 |= q.t32;
      if (!q.on) continue;
      Shape sh = q.sh;
      const bool g = q.g, t32 = q.t32, wide = q.wide, lean = q.lean;
      if (g) {
        gs[r] = 1;
        gs_words[r] = std::max(gs_words[r], (q.W + 3u) & ~3u);  // (ant-major rows padded to 16 B)
      }
      const bool mask = R.n <= 1024 && !g && !q.huge;  // (the huge-region variants scan strided words)
      if (g) sh.ig = false;
      // global-state kernels: 4-wide candidate scan over strided words (not in
      // the u32-cycle / 3-4 class instantiations), gs_wide_lanes above
      const bool gwide = g && gs_wide[pass - 1] && sh.lanes <= gs_wide_lanes[pass - 1] && !(pass == 2 && (t32 || P.nc4));
      const bool wk = (wide && mask) || gwide || q.huge;
      const bool ct32 = pass == 2 && t32 && !q.lpi;  // (lane-per-instruction ants keep u32 ready times in registers)
      const Key key(pass, sh.apb, sh.lanes, sh.ts, ct32, mask, g, sh.smem, wk, sh.ig, lean);
      Cls &c = classes[key];
      c.wide = wk;
      c.sh = sh;
      c.mask = mask;
      c.t32 = ct32;
      c.gs = g;
      c.lean = lean;
      // a class reserves what its largest block needs, not 1/k of the SM:
      // the unreserved shared memory becomes L1 (the driver picks the
      // smallest carveout that holds the resident blocks), which caches the
      // image and tau of the image-through-L1 and global-tau classes
      c.smem = std::max(c.smem, smem_exact && sh.need ? sh.need : sh.smem);
      c.regs.push_back({~(uint64_t)((uint64_t)R.n * (R.n + 16)), r});
    }
    P.p2_smem = std::max(P.p2_smem, 4 * R.n + 16);  // also k_post
  }
  // Replay (k_select) and greedy (k_init): one warp per region.  With many
  // regions the image is read through L1 and only the replay state is in
  // shared memory (many replays resident per SM); with few regions (a huge
  // region, config 4) the image is staged too (latency-bound serial replay).
  // Regions whose image + replay state exceed shared memory use the workspace.
  P.stage_img = count <= 2 * 148;
  std::vector<uint8_t> sgs(count, 0);
  for (uint32_t r = 0; r < count; ++r) {
    const RegionDev &R = ctx->regions[r];
    for (uint32_t pass = 1; pass <= 2; ++pass) {
      const uint32_t W = ant_words(pass, R.n, R.nwr, R.nremw, pass == 2 && P.any_t32, P.nc4);
      const uint32_t need_words = W + R.n + (R.n + 1) / 2 + 4;  // state + cycles + order
      const uint32_t fs = R.img.bytes + 4 * need_words + 64;
      if (fs > kSmemPerSM - 2048) sgs[r] = 1;  // replay scratch in the workspace too
      scratch_words[r] = std::max(scratch_words[r], need_words);
    }
  }
  for (uint32_t r = 0; r < count; ++r) {
    const RegionDev &R = ctx->regions[r];
    if (sgs[r]) continue;
    for (uint32_t pass = 1; pass <= 2; ++pass) {
      const uint32_t W = ant_words(pass, R.n, R.nwr, R.nremw, pass == 2 && P.any_t32, P.nc4);
      const uint32_t need_words = W + R.n + (R.n + 1) / 2 + 4;
      const uint32_t fs = R.img.bytes + 4 * need_words + 64;
      P.fin_smem[pass] = std::max(P.fin_smem[pass], P.stage_img ? fs : 4 * need_words + 64);
      if (pass == 1) P.init_smem = std::max(P.init_smem, fs);
    }
  }
  // ---- workspace layout
  uint64_t off = 0;
  P.o_state = off;
  off = align256(off + sizeof(RegionState) * (uint64_t)count);
  P.o_rws = off;
  off = align16(off + sizeof(RegionWs) * (uint64_t)count);
  const uint64_t o_items = off;
  uint64_t n_items = 0;
  std::vector<std::pair<Key, uint64_t>> class_item_off;
  for (auto &kv : classes) {
    class_item_off.push_back({kv.first, n_items});
    n_items += (uint64_t)kv.second.regs.size() * ((A + kv.second.sh.apb - 1) / kv.second.sh.apb);
  }
  off = align16(off + sizeof(BlockItem) * n_items);
  P.o_upd = off;
  uint64_t n_upd_max = 0;
  for (uint32_t r = 0; r < count; ++r) {
    const uint64_t n = ctx->regions[r].n;
    n_upd_max += ((((n + 1) * n + 7) / 8) + kUpdVec - 1) / kUpdVec;
  }
  off = align256(off + sizeof(UpdItem) * n_upd_max);
  const uint64_t sum_n = ctx->inst_off.empty() ? 0 : ctx->inst_off[count];
  const uint64_t o_gb1 = off;
  off = align256(off + 2 * sum_n + 16);
  P.o_gb2 = off;
  off = align256(off + 2 * sum_n + 16);
  P.o_gb2c = off;
  off = align256(off + 4 * sum_n + 16);
  const uint64_t o_heur = off;
  off = align256(off + 2 * sum_n + 16);
  const uint64_t o_next = off;
  off = align256(off + 2 * (sum_n + count) + 16);
  const uint64_t o_cost = off;
  off = align256(off + 4ull * A * count);
  const uint64_t n_grp = rl1 ? ((uint64_t)A + p->group_size - 1) / p->group_size : 0;
  const uint64_t o_rlk = off;  // R45: K per (ant group, step)
  off = align256(off + 2 * n_grp * sum_n + 16);
  // Record mode: every ant stores its schedule (step-major, coalesced) and
  // k_select copies the winner's instead of replaying it serially.  Measured
  // on B200 (ms per batch, replay -> record): C1 2.34 -> 1.80, C2 79.9 ->
  // 62.2, C3 674 -> 650, C4 500 -> 432, C5 3327 -> 3109; the writes (C3:
  // 2.9 GB per pass-2 iteration, coalesced) hide under the construction.
  uint64_t rec_mb = 16384;
  if (const char *e = getenv("ACO_RECORD_MB")) rec_mb = strtoull(e, nullptr, 10);
  const uint64_t rec_bytes = (uint64_t)A * sum_n * ((pmask & 2u) ? 6u : 2u) + 16ull * A * count;
  P.record = !colony && !(p->flags & ACO_FLAG_DUMP) && rec_bytes <= (rec_mb << 20);
  const uint64_t o_rec = off;
  if (P.record) off = align256(off + 2ull * A * sum_n + 16);
  const uint64_t o_recc = off;
  if (P.record && (pmask & 2u)) off = align256(off + 4ull * A * sum_n + 16);
  const uint64_t o_recp = off;
  if (P.record) off = align256(off + 16ull * A * count);
  P.o_keys = off;
  off = align256(off + 8ull * count);
  std::vector<RegionWs> rws(count);
  for (uint32_t r = 0; r < count; ++r) {
    const uint32_t n = ctx->regions[r].n;
    RegionWs &w = rws[r];
    std::memset(&w, 0, sizeof(w));
    w.tau_len = (uint32_t)(((uint64_t)(n + 1) * n + 7) & ~7ull);
    w.o_tau = off;
    off = align16(off + 2ull * w.tau_len);
    w.o_cost = o_cost + 4ull * A * r;
    w.o_gb1 = o_gb1 + 2 * ctx->inst_off[r];
    w.o_gb2 = P.o_gb2 + 2 * ctx->inst_off[r];
    w.o_gb2c = P.o_gb2c + 4 * ctx->inst_off[r];
    w.o_dump = (uint64_t)A * ctx->inst_off[r];
    w.o_next = o_next + 2 * (ctx->inst_off[r] + r);
    w.o_heur = o_heur + 2 * ctx->inst_off[r];
    w.o_rlk = o_rlk + 2 * n_grp * ctx->inst_off[r];
    w.o_rec = o_rec + 2ull * A * ctx->inst_off[r];
    w.o_recc = o_recc + 4ull * A * ctx->inst_off[r];
    w.o_recp = o_recp + 16ull * A * r;
    w.gs = sgs[r];  // k_init / k_select: image and replay state in the workspace
    if (gs[r]) {  // global-state construct kernels
      off = align256(off);
      w.o_gstate = off;
      off += 4ull * A * gs_words[r];
    }
    if (sgs[r]) {
      off = align256(off);
      w.o_scratch = off;
      off = align256(off + 4ull * scratch_words[r]);
    }
  }
  std::vector<UpdItem> upd;
  for (uint32_t r = 0; r < count; ++r)
    for (uint32_t v0 = 0; v0 < rws[r].tau_len / 8; v0 += kUpdVec) upd.push_back(UpdItem{r, v0});
  P.n_upd = (uint32_t)upd.size();
  const size_t need = align256(off);
  if (ws_needed) *ws_needed = need;
  const bool plan_only = !d_workspace;  // (debug: ACO_DEBUG_PLAN prints the plan)
  if (plan_only && !getenv("ACO_DEBUG_PLAN")) {
    ctx->plan = saved;
    return ACO_OK;
  }
  if (!plan_only) {
    if (!ctx->arena && ctx->count) return ACO_E_STATE;
    if (ws_bytes < need) {
      ctx->plan = saved;
      return ACO_E_WORKSPACE;
    }
    if (cudaSetDevice(ctx->device) != cudaSuccess) return ACO_E_CUDA;
    if (ctx->mslot < 0 && (ctx->mslot = acquire_machine_slot(ctx->device, ctx->mach)) < 0) return ACO_E_CUDA;
    if (!ctx->make_side()) return ACO_E_CUDA;
  }
  unsigned char *ws = (unsigned char *)d_workspace;
  // ---- host plan: RegionWs table + block items + update items, one H2D
  std::vector<unsigned char> &blob = ctx->plan_blob;
  blob.assign(P.o_upd - P.o_rws + sizeof(UpdItem) * upd.size(), 0);
  if (!upd.empty()) std::memcpy(blob.data() + (P.o_upd - P.o_rws), upd.data(), sizeof(UpdItem) * upd.size());
  std::memcpy(blob.data(), rws.data(), sizeof(RegionWs) * count);
  std::vector<uint64_t> class_work[3];
  {
    size_t ci = 0;
    for (auto &kv : classes) {
      Cls &c = kv.second;
      std::sort(c.regs.begin(), c.regs.end());
      const uint64_t base = class_item_off[ci++].second;
      BlockItem *items = (BlockItem *)(blob.data() + (o_items - P.o_rws)) + base;
      uint64_t k = 0;
      for (auto &pr : c.regs)
        for (uint32_t a0 = 0; a0 < A; a0 += c.sh.apb) items[k++] = BlockItem{pr.second, a0};
      ClassLaunch cl;
      cl.items = (const BlockItem *)(ws + o_items) + base;
      cl.n_blocks = (uint32_t)k;
      cl.ants_pb = c.sh.apb;
      cl.lanes = c.sh.lanes;
      cl.smem_bytes = c.smem;
      cl.max_n = c.mask ? 1024 : 65535;
      cl.tau_smem = c.sh.ts;
      cl.t32 = c.t32;
      cl.nc4 = P.nc4;
      cl.gs = c.gs;
      cl.wide = c.wide;
      cl.img_l1 = c.sh.ig;
      cl.lean = c.lean;
      P.launches[std::get<0>(kv.first)].push_back(cl);
      class_work[std::get<0>(kv.first)].push_back(0);
      for (auto &pr : c.regs) class_work[std::get<0>(kv.first)].back() += ~pr.first;
    }
  }
  for (int pass = 1; pass <= 2; ++pass) {  // biggest classes first (fork round-robin)
    std::vector<size_t> idx(P.launches[pass].size());
    for (size_t i = 0; i < idx.size(); ++i) idx[i] = i;
    std::sort(idx.begin(), idx.end(), [&](size_t a, size_t b) { return class_work[pass][a] > class_work[pass][b]; });
    std::vector<ClassLaunch> sorted;
    for (size_t i : idx) sorted.push_back(P.launches[pass][i]);
    P.launches[pass] = sorted;
    if (getenv("ACO_DEBUG_PLAN"))
      for (size_t i = 0; i < idx.size(); ++i)
        fprintf(stderr,
                "[aco plan] pass %d class %zu: blocks %u ants/blk %u lanes %u smem %u tau_smem %d t32 %d gs %d "
                "wide %d img_l1 %d lean %d work %.3g\n",
                pass, i, sorted[i].n_blocks, sorted[i].ants_pb, sorted[i].lanes, sorted[i].smem_bytes,
                (int)sorted[i].tau_smem, (int)sorted[i].t32, (int)sorted[i].gs, (int)sorted[i].wide,
                (int)sorted[i].img_l1, (int)sorted[i].lean,
                (double)class_work[pass][idx[i]]);
  }
  // Fused single-block run (k_fused): every region's ants fit one block and
  // its image, pheromone table, ant states and recorded schedules fit shared
  // memory; a batch with few ants in total (config 1), where the per-launch
  // latency of the multi-launch path dominates.  Word-mask scan, compact
  // pass-2 layout; not the shared colony nor the ready-list limit.
  {
    uint32_t fused_ants = 512;
    if (const char *e = getenv("ACO_FUSED_ANTS")) fused_ants = (uint32_t)atoi(e);
    bool ok = !colony && p->rl_limit == 0 && count > 0 && A <= 512 && (uint64_t)count * A <= fused_ants && !P.nc4;
    uint32_t smem = 0;
    for (uint32_t r = 0; r < count && ok; ++r) {
      const RegionDev &R = ctx->regions[r];
      ok = R.n <= 1024 && R.max_lat <= 511u && R.mc_max <= 7u;
      if (ok) smem = std::max(smem, fused_layout(R.n, R.nwr, R.nremw, R.img.bytes, A, p->group_size).bytes);
    }
    if (ok && smem <= kSmemPerSM) {
      P.fused = true;
      P.fused_threads = std::max(32u, (A + 31u) & ~31u);
      P.fused_smem = smem;
      P.fused_wl = 0;
      // lane-per-instruction ants inside the fused run (WL lanes per ant, the
      // smallest of 8 / 16 / 32 with n <= 4 WL; WL x A <= 512 threads): only
      // when forced (ACO_LPI=2 or ACO_FUSED_LPI=1) -- measured slower on
      // config 1 (0.641 -> 0.898 ms: with n = 10 a thread-per-ant step scans
      // ~3 candidates, less than the group's reductions and uniform commit)
      uint32_t nmax = 0;
      const bool fused_lpi = lpi_mode == 2 || (getenv("ACO_FUSED_LPI") && atoi(getenv("ACO_FUSED_LPI")) != 0);
      bool lok = fused_lpi && ctx->mach.issue_width <= 1 && !p->heur_mix;
      for (uint32_t r = 0; r < count; ++r) {
        const RegionDev &R = ctx->regions[r];
        nmax = std::max(nmax, R.n);
        lok = lok && (uint64_t)R.max_cycle_bound + R.max_lat < 65536u;
      }
      const uint32_t wl = nmax <= 32 ? 8u : (nmax <= 64 ? 16u : 32u);
      if (lok && nmax >= 1 && nmax <= 128 && (uint64_t)A * wl <= 512) {
        P.fused_wl = wl;
        P.fused_threads = std::max(32u, (A * wl + 31u) & ~31u);  // (whole warps: the select body is warp 0)
      }
    }
  }
  ctx->variants.clear();  // construct-kernel variants of this plan (aco_last_variants)
  if (P.fused) ctx->variants.push_back(kFusedVariant | (P.fused_wl ? kFusedLpi * (31 - __builtin_clz(P.fused_wl) - 2) : 0u));
  for (int pass = 1; pass <= 2 && !P.fused; ++pass)
    for (const ClassLaunch &cl : P.launches[pass]) {
      const uint32_t code = class_variant((uint32_t)pass, cl);
      if (std::find(ctx->variants.begin(), ctx->variants.end(), code) == ctx->variants.end())
        ctx->variants.push_back(code);
    }
  std::sort(ctx->variants.begin(), ctx->variants.end());
  if (plan_only) {
    ctx->plan = saved;
    return ACO_OK;
  }
  cudaStream_t s = (cudaStream_t)cuda_stream;
  if (aco_status hs = ctx->staged_h2d(1, ws + P.o_rws, blob.data(), blob.size(), s)) return hs;
  LaunchCtx &L = P.L;
  L.arena = ctx->arena;
  L.ws = ws;
  L.regions = (const RegionDev *)ctx->arena;
  L.state = (RegionState *)(ws + P.o_state);
  L.rws = (const RegionWs *)(ws + P.o_rws);
  L.dump_cost = ctx->dump_cost;
  L.dump_order = ctx->dump_order;
  L.dump_cycle = ctx->dump_cycle;
  RunCfg &cfg = L.cfg;
  std::memset(&cfg, 0, sizeof(cfg));
  cfg.seed = p->seed;
  cfg.q0_t = p->q0_t;
  cfg.ants = A;
  cfg.iterations = p->iterations;
  cfg.pass_mask = pmask;
  cfg.cost_mode = p->cost_mode;
  cfg.group_size = p->group_size;
  cfg.stall_mod = p->stall_mod;
  cfg.stall_rem = p->stall_rem;
  cfg.flags = p->flags;
  cfg.tau0 = p->tau0;
  cfg.rho_q16 = p->rho_q16;
  cfg.delta = p->delta;
  cfg.tau_min = p->tau_min;
  cfg.tau_max = p->tau_max;
  cfg.stop_no_improve = p->stop_no_improve;
  cfg.stop_at_lb = p->stop_at_lb;
  cfg.n_classes = ctx->mach.n_classes;
  cfg.count = count;
  cfg.ant_base = ant_base;
  cfg.weighted = p->pass == 4;
  cfg.ws_weight = p->ws_weight;
  cfg.pass2_gap = p->pass2_gap;
  cfg.revert_occ = p->revert_occ;
  cfg.revert_len = p->revert_len;
  cfg.heur_mix = p->heur_mix;
  cfg.stall_num = p->stall_num;
  cfg.rl_limit = p->rl_limit;
  cfg.mslot = (uint32_t)ctx->mslot;
  // global-state per-ant layout: [word][ant] (0) or ant-major (1); measured on
  // B200 (ms per step, r02b): C4 852 / 839, C5 1992 / 2027 -- within 2 %, [word][ant] kept
  cfg.gs_ant_major = 0;
  if (const char *e = getenv("ACO_GS_LAYOUT")) cfg.gs_ant_major = atoi(e) != 0;
  cfg.lazy_kills = 1;  // measured (r02j): C3 702 -> 695 ms, C5 and n = 200/450 neutral to -4 %
  if (const char *e = getenv("ACO_LAZY_KILLS")) cfg.lazy_kills = atoi(e) != 0;
  cfg.prune_cp = 0;
  if (const char *e = getenv("ACO_PRUNE_CP")) cfg.prune_cp = atoi(e) != 0;
  cfg.tau_prefetch = 0;
  if (const char *e = getenv("ACO_TAU_PREFETCH")) cfg.tau_prefetch = (uint32_t)strtoul(e, nullptr, 0);
  cfg.record = P.record ? 1u : 0u;
  cfg.stage_img = P.stage_img ? 1u : 0u;
  cfg.dump_slice = (uint64_t)A * sum_n;
  cfg.keys = nullptr;
  L.stream = cuda_stream;
  L.launches = 0;
  P.timing = (p->flags & ACO_FLAG_TIMING) != 0;
  P.pass_mask = pmask;
  P.iterations = p->iterations;
  ctx->ev_used = 0;
  for (int ph = 0; ph < 3; ++ph) {
    ctx->ev_pairs[ph].clear();
    ctx->phase_launches[ph] = 0;
  }
  ctx->ws = ws;
  ctx->ws_bytes = ws_bytes;
  ctx->stream = cuda_stream;
  ctx->cfg = cfg;
  ctx->o_state = P.o_state;
  ctx->o_rws = P.o_rws;
  ctx->o_gb2 = P.o_gb2;
  ctx->o_gb2c = P.o_gb2c;
  ctx->have_run = true;
  ctx->planned = true;
  ctx->cache_ok = !getenv("ACO_NO_PLAN_CACHE");
  ctx->cache_params = *p;
  ctx->cache_ws = d_workspace;
  ctx->cache_ws_bytes = ws_bytes;
  ctx->cache_need = need;
  ctx->cache_ant_base = ant_base;
  ctx->cache_colony = colony;
  ctx->cache_dump[0] = ctx->dump_cost;
  ctx->cache_dump[1] = ctx->dump_order;
  ctx->cache_dump[2] = ctx->dump_cycle;
  return ACO_OK;
}

// ---- phase runners (stream-ordered on the plan's stream)
struct Bracket {  // ACO_FLAG_TIMING: an event pair around a group of launches
  aco_ctx ctx;
  int ph;
  size_t e0;
  uint64_t l0;
  Bracket(aco_ctx c, int phase) : ctx(c), ph(phase), e0(0), l0(c->plan.L.launches) {
    if (!ctx->plan.timing) return;
    e0 = ctx->ev_used;
    if (cudaEvent_t e = ctx->next_event()) cudaEventRecord(e, (cudaStream_t)ctx->plan.L.stream);
  }
  ~Bracket() {
    ctx->phase_launches[ph] += ctx->plan.L.launches - l0;
    if (!ctx->plan.timing) return;
    const size_t e1 = ctx->ev_used;
    if (cudaEvent_t e = ctx->next_event()) cudaEventRecord(e, (cudaStream_t)ctx->plan.L.stream);
    ctx->ev_pairs[ph].push_back({e0, e1});
  }
};

int run_init(aco_ctx ctx) {
  Bracket b(ctx, 2);
  return launch_init(ctx->plan.L, ctx->plan.init_smem, ctx->plan.max_n);
}

int run_pass2_init(aco_ctx ctx) {
  Bracket b(ctx, 2);
  ctx->plan.p2_done = true;
  return launch_pass2_init(ctx->plan.L, ctx->plan.p2_smem, ctx->plan.max_n);
}

int run_post(aco_ctx ctx) {
  Bracket b(ctx, 2);
  return launch_post(ctx->plan.L, ctx->plan.p2_smem);
}

int run_construct(aco_ctx ctx, uint32_t pass, uint32_t it) {
  Plan &P = ctx->plan;
  LaunchCtx &L = P.L;
  Bracket b(ctx, 0);
  int err = 0;
  const std::vector<ClassLaunch> &cls = P.launches[pass];
  void *main = L.stream;
  cudaStream_t s = (cudaStream_t)main;
  if (cls.size() <= 1) {
    for (const ClassLaunch &cl : cls) err |= launch_construct(L, pass, it, cl);
  } else {  // fork: classes round-robin over the internal streams, join on the main stream
    static const int ks = [] {  // fork streams (A/B knob; 4 measured best, 8: C5 3109 -> 3996 ms)
      const char *e = getenv("ACO_STREAMS");
      const int v = e ? atoi(e) : aco_ctx_s::kStreams;
      return std::max(1, std::min(v, aco_ctx_s::kStreams));
    }();
    const int k = (int)std::min<size_t>(cls.size(), (size_t)ks);
    err |= cudaEventRecord(ctx->fork_ev, s) != cudaSuccess;
    for (int i = 0; i < k; ++i) err |= cudaStreamWaitEvent(ctx->side[i], ctx->fork_ev, 0) != cudaSuccess;
    for (size_t c = 0; c < cls.size(); ++c) {
      L.stream = ctx->side[c % k];
      err |= launch_construct(L, pass, it, cls[c]);
    }
    L.stream = main;
    for (int i = 0; i < k; ++i) {
      err |= cudaEventRecord(ctx->join_ev[i], ctx->side[i]) != cudaSuccess;
      err |= cudaStreamWaitEvent(s, ctx->join_ev[i], 0) != cudaSuccess;
    }
  }
  return err;
}

int run_finalize(aco_ctx ctx, uint32_t pass, uint32_t it, int64_t *keys) {
  Plan &P = ctx->plan;
  Bracket b(ctx, 1);
  P.L.cfg.keys = keys;
  // few regions with small tables: select + update + stop in one launch (ACO_FIN1=0: three launches)
  static const bool fin1_on = !getenv("ACO_FIN1") || atoi(getenv("ACO_FIN1")) != 0;
  const bool fin1 = fin1_on && P.L.cfg.count <= kFin1MaxRegions && P.max_n <= kFin1MaxN;
  const int err = launch_finalize(P.L, pass, it, P.fin_smem[pass], P.max_n, pass == 2 && P.any_t32, P.nc4,
                                  (const UpdItem *)(P.L.ws + P.o_upd), P.n_upd, fin1);
  P.L.cfg.keys = nullptr;
  return err;
}

}  // namespace

aco_status aco_schedule_batch(aco_ctx ctx, const aco_params *p, void *d_workspace, size_t ws_bytes,
                              size_t *ws_needed, void *cuda_stream) {
  if (!ctx || !p) return ACO_E_ARG;
  aco_status st = make_plan(ctx, p, 0, d_workspace, ws_bytes, ws_needed, cuda_stream, false);
  if (st != ACO_OK || !d_workspace) return st;
  cudaStream_t s = (cudaStream_t)cuda_stream;
  // Replay of the captured graph: the plan is cached (same parameters,
  // workspace, regions and dump buffers), so every launch and its arguments
  // are identical to the captured run's; the kernels take every data-dependent
  // decision (stop rules, active regions) on the device.
  static const bool graphs = [] {
    const char *e = getenv("ACO_GRAPH");
    return e ? atoi(e) != 0 : true;
  }();
  const bool use_graph = graphs && ctx->cache_hit && !ctx->plan.timing;
  // graph launch on the graph stream, ordered after and before the caller's stream
  auto launch_graph = [&]() {
    return cudaEventRecord(ctx->g_in, s) != cudaSuccess || cudaStreamWaitEvent(ctx->gstream, ctx->g_in, 0) != cudaSuccess ||
           cudaGraphLaunch(ctx->gexec, ctx->gstream) != cudaSuccess ||
           cudaEventRecord(ctx->g_out, ctx->gstream) != cudaSuccess || cudaStreamWaitEvent(s, ctx->g_out, 0) != cudaSuccess;
  };
  if (use_graph && ctx->gexec_ok) {
    ctx->launches = ctx->gexec_launches;
    return launch_graph() ? ACO_E_CUDA : ACO_OK;
  }
  if (ctx->plan.fused) {  // the whole run in one launch (no graph needed)
    Bracket b(ctx, 0);
    const int e = launch_fused(ctx->plan.L, ctx->plan.fused_threads, ctx->plan.fused_smem, ctx->plan.fused_wl);
    ctx->launches = ctx->plan.L.launches;
    return e ? ACO_E_CUDA : ACO_OK;
  }
  auto issue = [&]() {  // the launch sequence of L135-L139
    int e = run_init(ctx);
    for (uint32_t pass = 1; pass <= 2 && !e; ++pass) {
      if (pass == 2) e |= run_pass2_init(ctx);
      if (!(ctx->plan.pass_mask & pass)) continue;
      for (uint32_t it = 0; it < p->iterations && !e; ++it) {
        e |= run_construct(ctx, pass, it);
        e |= run_finalize(ctx, pass, it, nullptr);
      }
    }
    if (!e) e |= run_post(ctx);
    ctx->launches = ctx->plan.L.launches;
    return e;
  };
  if (use_graph && cudaStreamBeginCapture(ctx->gstream, cudaStreamCaptureModeThreadLocal) == cudaSuccess) {
    ctx->plan.L.stream = ctx->gstream;  // the launch sequence is recorded on the graph stream
    const int ce = issue();
    ctx->plan.L.stream = cuda_stream;
    cudaGraph_t g = nullptr;
    const bool ended = cudaStreamEndCapture(ctx->gstream, &g) == cudaSuccess && g;
    if (!ce && ended && cudaGraphInstantiate(&ctx->gexec, g, 0) == cudaSuccess) {
      ctx->gexec_ok = true;
      ctx->gexec_launches = ctx->launches;
    } else {
      ctx->drop_graph();
    }
    if (g) cudaGraphDestroy(g);
    cudaGetLastError();
    if (ctx->gexec_ok) return launch_graph() ? ACO_E_CUDA : ACO_OK;
    ctx->plan.L.launches = 0;  // capture failed: nothing ran, launch directly
  }
  return issue() ? ACO_E_CUDA : ACO_OK;
}

aco_status aco_colony_begin(aco_ctx ctx, const aco_params *p, uint32_t ant_base, void *d_workspace, size_t ws_bytes,
                            size_t *ws_needed, void *cuda_stream) {
  if (!ctx || !p) return ACO_E_ARG;
  if (p->flags & ACO_FLAG_DUMP) return ACO_E_ARG;
  aco_status st = make_plan(ctx, p, ant_base, d_workspace, ws_bytes, ws_needed, cuda_stream, true);
  if (st != ACO_OK || !d_workspace) return st;
  const int err = run_init(ctx);
  ctx->launches = ctx->plan.L.launches;
  return err ? ACO_E_CUDA : ACO_OK;
}

aco_status aco_colony_construct(aco_ctx ctx, uint32_t pass, uint32_t iter, int64_t *d_keys, void *cuda_stream) {
  if (!ctx || !d_keys || pass < 1 || pass > 2) return ACO_E_ARG;
  if (!ctx->planned) return ACO_E_STATE;
  Plan &P = ctx->plan;
  if (!(P.pass_mask & pass) || iter >= P.iterations) return ACO_E_ARG;
  P.L.stream = cuda_stream;
  int err = 0;
  if (pass == 2 && iter == 0) err |= run_pass2_init(ctx);
  err |= run_construct(ctx, pass, iter);
  err |= launch_local_keys(P.L, d_keys);
  ctx->launches = P.L.launches;
  return err ? ACO_E_CUDA : ACO_OK;
}

aco_status aco_colony_finalize(aco_ctx ctx, uint32_t pass, uint32_t iter, int64_t *d_keys, void *cuda_stream) {
  if (!ctx || !d_keys || pass < 1 || pass > 2) return ACO_E_ARG;
  if (!ctx->planned) return ACO_E_STATE;
  Plan &P = ctx->plan;
  if (!(P.pass_mask & pass) || iter >= P.iterations) return ACO_E_ARG;
  P.L.stream = cuda_stream;
  const int err = run_finalize(ctx, pass, iter, d_keys);
  ctx->launches = P.L.launches;
  return err ? ACO_E_CUDA : ACO_OK;
}

aco_status aco_colony_end(aco_ctx ctx, void *cuda_stream) {
  if (!ctx) return ACO_E_ARG;
  if (!ctx->planned) return ACO_E_STATE;
  Plan &P = ctx->plan;
  P.L.stream = cuda_stream;
  int err = 0;
  if (!P.p2_done) err |= run_pass2_init(ctx);  // ASAP timing of the pass-1 result
  err |= run_post(ctx);
  ctx->stream = cuda_stream;
  ctx->launches = P.L.launches;
  return err ? ACO_E_CUDA : ACO_OK;
}

aco_status aco_get_timing(aco_ctx ctx, double ms[3], uint64_t launches[3]) {
  if (!ctx || !ms || !launches) return ACO_E_ARG;
  if (!ctx->have_run) return ACO_E_STATE;
  if (cudaStreamSynchronize((cudaStream_t)ctx->stream) != cudaSuccess) return ACO_E_CUDA;
  for (int ph = 0; ph < 3; ++ph) {
    double t = 0;
    for (auto &pr : ctx->ev_pairs[ph]) {
      float f = 0;
      if (cudaEventElapsedTime(&f, ctx->ev_pool[pr.first], ctx->ev_pool[pr.second]) != cudaSuccess)
        return ACO_E_CUDA;
      t += f;
    }
    ms[ph] = t;
    launches[ph] = ctx->phase_launches[ph];
  }
  return ACO_OK;
}

aco_status aco_last_variants(aco_ctx ctx, uint32_t *codes, uint32_t cap, uint32_t *count) {
  if (!ctx || !count || (cap && !codes)) return ACO_E_ARG;
  *count = (uint32_t)ctx->variants.size();
  for (uint32_t i = 0; i < cap && i < ctx->variants.size(); ++i) codes[i] = ctx->variants[i];
  return ACO_OK;
}

aco_status aco_last_launch_count(aco_ctx ctx, uint64_t *launches) {
  if (!ctx || !launches) return ACO_E_ARG;
  *launches = ctx->launches;
  return ACO_OK;
}

aco_status aco_get_results(aco_ctx ctx, uint32_t first, uint32_t count, aco_result *out, uint32_t *orders,
                           uint32_t *cycles) {
  if (!ctx || (count && !out)) return ACO_E_ARG;
  if (!ctx->have_run) return ACO_E_STATE;
  if ((uint64_t)first + count > ctx->count) return ACO_E_ARG;
  if (cudaSetDevice(ctx->device) != cudaSuccess) return ACO_E_CUDA;
  cudaStream_t s = (cudaStream_t)ctx->stream;
  if (cudaStreamSynchronize(s) != cudaSuccess) return ACO_E_CUDA;
  if (!count) return ACO_OK;
  std::vector<RegionState> st(count);
  const uint64_t i0 = ctx->inst_off[first], i1 = ctx->inst_off[first + count];
  std::vector<uint16_t> o16(i1 - i0 + 1);
  std::vector<uint32_t> c32(i1 - i0 + 1);
  aco_status e = cuda_status(cudaMemcpy(st.data(), ctx->ws + ctx->o_state + sizeof(RegionState) * first,
                                        sizeof(RegionState) * count, cudaMemcpyDeviceToHost));
  if (e == ACO_OK && i1 > i0) {
    e = cuda_status(cudaMemcpy(o16.data(), ctx->ws + ctx->o_gb2 + 2 * i0, 2 * (i1 - i0), cudaMemcpyDeviceToHost));
    if (e == ACO_OK)
      e = cuda_status(cudaMemcpy(c32.data(), ctx->ws + ctx->o_gb2c + 4 * i0, 4 * (i1 - i0), cudaMemcpyDeviceToHost));
  }
  if (e != ACO_OK) return e;
  // host-side cost of the final PRP (R16) -- the machine tables
  auto aprp = [&](uint32_t c, uint32_t x) {
    for (uint32_t i = 0; i < ctx->mach.step_count[c]; ++i)
      if (x <= ctx->mach.step_max[c][i]) return ctx->mach.step_max[c][i];
    return x;
  };
  auto occ = [&](uint32_t c, uint32_t x) {
    for (uint32_t i = 0; i < ctx->mach.step_count[c]; ++i)
      if (x <= ctx->mach.step_max[c][i]) return ctx->mach.occ_max - i;
    return 0u;
  };
  for (uint32_t k = 0; k < count; ++k) {
    const RegionState &S = st[k];
    const RegionDev &R = ctx->regions[first + k];
    aco_result &o = out[k];
    std::memset(&o, 0, sizeof(o));
    o.n_insts = R.n;
    o.length = S.len2;
    uint32_t cost = 0;
    const uint32_t nc = ctx->mach.n_classes, mode = ctx->cfg.cost_mode;
    if (mode == ACO_COST_PRP_SUM) {
      for (uint32_t c = 0; c < nc; ++c) cost += S.prp2[c];
    } else if (mode == ACO_COST_APRP_SUM) {
      for (uint32_t c = 0; c < nc; ++c) cost += aprp(c, S.prp2[c]);
    } else if (mode == ACO_COST_OCC) {
      uint32_t m = ctx->mach.occ_max;
      for (uint32_t c = 0; c < nc; ++c) m = std::min(m, occ(c, S.prp2[c]));
      cost = ctx->mach.occ_max - m;
    } else {
      for (uint32_t c = 0; c < nc; ++c)
        cost += S.prp2[c] > ctx->mach.perp_limit[c] ? S.prp2[c] - ctx->mach.perp_limit[c] : 0;
    }
    o.cost_rp = cost;
    for (int c = 0; c < 4; ++c) {
      o.prp[c] = S.prp2[c];
      o.target[c] = S.target[c];
    }
    o.iters_run[0] = S.iters[0];
    o.iters_run[1] = S.iters[1];
    o.best_cost[0] = S.best[0];
    o.best_cost[1] = S.best[1];
    o.init_cost[0] = S.init[0];
    o.init_cost[1] = S.init[1];
    o.lb_cost = S.lb_cost;
    o.lb_len = R.lb_len;
    o.trace_hash = S.hash;
    o.policy = S.policy;
    o.heur_len = S.heur_len;
    o.ws_cost = ctx->cfg.weighted ? S.best[1] : 0u;
    o.ants_pruned = S.pruned;
    for (int c = 0; c < 4; ++c) o.heur_prp[c] = S.heur_prp[c];
  }
  for (uint64_t q = 0; q < i1 - i0; ++q) {
    if (orders) orders[q] = o16[q];
    if (cycles) cycles[q] = c32[q];
  }
  return ACO_OK;
}

}  // extern "C"
