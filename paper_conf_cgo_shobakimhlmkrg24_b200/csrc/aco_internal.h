// aco_internal.h -- device data layout of the B200 ACO scheduler (library
// internal; shared by aco_host.cpp and aco_kernels.cu only).
//
// Region statics live in the caller's ARENA (written once by
// aco_load_regions); run state lives in the caller's WORKSPACE (laid out by
// aco_schedule_batch).  All offsets are in BYTES from the buffer base.
#pragma once
#include <stdint.h>

#include "../../include/aco.h"

namespace aco {

constexpr uint32_t kInvalid = 0xFFFFFFFFu;  // R35
constexpr uint32_t kMaxKernelInsts = 8192;  // compiled limit of this version
constexpr uint32_t kFlagLiveIn = 1, kFlagLiveOut = 2;

// Per-region statics (arena).  Arrays are 16-byte aligned.
struct RegionDev {
  uint32_t n;        // instructions
  uint32_t nwr;      // words of an instruction bitset = ceil(n/32)
  uint32_t nmu;      // remaining-use counters (registers used >= 2 times, not live-out)
  uint32_t L;        // max LUC over instructions (rows of eta1 minus one)
  uint32_t region_id;
  uint32_t cp_max;
  uint32_t lb_len;   // max(n, 1 + CPmax) (R30)
  uint32_t ub_ready; // 1 + max #independent (L182), reporting only
  uint32_t livein[4];
  uint32_t lbvec[4]; // per-class PRP lower bound vector (R30)
  uint64_t o_succ_ptr;  // u32 [n+1]
  uint64_t o_succ;      // u32 [E]  v | lat << 16
  uint64_t o_info;      // uint4 [n] {defs c0..3 u8, dead defs u8x4, static kills u8x4, muse start<<8 | count}
  uint64_t o_muse;      // u32 [..] counter index | class << 16
  uint64_t o_rb0;       // u32 [nwr] roots bitset
  uint64_t o_cnt0;      // u32 [ceil(n/4)] packed u8 in-degrees
  uint64_t o_rem0;      // u32 [ceil(nmu/2)] packed u16 use counts
  uint64_t o_eta1;      // u16 [n * (L+1)] eta1(j, luc) at [j*(L+1) + luc]
  uint64_t o_eta2;      // u16 [n]
  uint64_t pad;
};

// Mutable per-region state (workspace).
struct RegionState {
  uint32_t active;       // the current pass still iterates
  uint32_t no_imp;       // iterations without improvement
  uint32_t iters[2];
  uint32_t best[2];      // pass-1 best cost, pass-2 best length
  uint32_t init[2];      // heuristic pass-1 cost, initial pass-2 length
  uint32_t prp1[4];      // PRP of the pass-1 global best
  uint32_t prp2[4];      // PRP of the pass-2 global best (final)
  uint32_t target[4];    // pass-2 target (R18)
  uint32_t prune_len;    // best completed length of the running iteration (R24)
  uint32_t lb_cost;
  uint64_t hash;         // FNV-1a trace
};

// Per-region workspace offsets (bytes from the workspace base).
struct RegionWs {
  uint64_t o_tau;    // u16 [(n+1)*n] padded to 8 elements
  uint64_t o_cost;   // u32 [ants]
  uint64_t o_gb1;    // u16 [n]  pass-1 global best order
  uint64_t o_gb2;    // u16 [n]  pass-2 global best order
  uint64_t o_gb2c;   // u32 [n]  pass-2 global best cycles (in order)
  uint64_t o_dump;   // element offset of this region in a dump (pass, iter) slice = ants * sum n_q
  uint32_t tau_len;  // (n+1)*n rounded up to a multiple of 8
  uint32_t pad;
};

// Constant run configuration.
struct RunCfg {
  uint64_t seed;
  uint64_t q0_t;
  uint32_t ants, iterations, pass_mask, cost_mode;
  uint32_t group_size, stall_mod, stall_rem, flags;
  uint32_t tau0, rho_q16, delta, tau_min, tau_max;
  uint32_t stop_no_improve, stop_at_lb, n_classes;
  uint32_t count;       // regions
  uint32_t pad;
  uint64_t dump_slice;  // elements per (pass, iter) order slice = ants * sum n
};

struct MachineDev {
  uint32_t n_classes, occ_max;
  uint32_t step_count[4];
  uint32_t step_max[4][16];
  uint32_t perp_limit[4];
};

// Construct-kernel work item: one block = ants [ant0, ant0 + blockDim) of a region.
struct BlockItem {
  uint32_t region;
  uint32_t ant0;
};

inline uint64_t align16(uint64_t x) { return (x + 15) & ~uint64_t(15); }
inline uint64_t align256(uint64_t x) { return (x + 255) & ~uint64_t(255); }

// Per-ant state words (u32) of a region for a pass, in the [word][ant] layout.
#ifdef __CUDACC__
#define ACO_HD __host__ __device__
#else
#define ACO_HD
#endif
ACO_HD inline uint32_t ant_words(uint32_t pass, uint32_t n, uint32_t nwr, uint32_t nmu) {
  uint32_t w = nwr + (nmu + 1) / 2;
  return pass == 1 ? w + (n + 3) / 4 : w + n;
}

// ---- launch interface implemented in aco_kernels.cu ----
struct LaunchCtx {
  const unsigned char *arena;
  unsigned char *ws;
  const RegionDev *regions;  // in arena
  RegionState *state;        // in ws
  const RegionWs *rws;       // in ws
  uint32_t *dump_cost;
  uint16_t *dump_order;
  uint32_t *dump_cycle;
  RunCfg cfg;
  void *stream;
  uint64_t launches;
};

struct ClassLaunch {
  const BlockItem *items;  // device pointer (in ws)
  uint32_t n_blocks;
  uint32_t ants_pb;
  uint32_t smem_bytes;
  uint32_t max_n;          // max n in the class (selects the mask variant)
};

int set_machine(const MachineDev &m);  // cudaMemcpyToSymbol; 0 on success
int launch_init(LaunchCtx &L, uint32_t smem, uint32_t max_n);
int launch_pass2_init(LaunchCtx &L, uint32_t smem, uint32_t max_n);
int launch_construct(LaunchCtx &L, uint32_t pass, uint32_t iter, const ClassLaunch &c);
int launch_finalize(LaunchCtx &L, uint32_t pass, uint32_t iter, uint32_t smem, uint32_t max_n);
int last_cuda_error();

}  // namespace aco
