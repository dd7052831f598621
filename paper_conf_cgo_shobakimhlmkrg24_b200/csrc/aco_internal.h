// aco_internal.h -- device data layout of the B200 ACO scheduler (library
// internal; shared by aco_host.cpp and aco_kernels.cu only).
//
// Region statics live in the caller's ARENA (written once by
// aco_load_regions) as one contiguous, 16-byte aligned BLOCK IMAGE per region
// whose internal layout is exactly what the kernels keep in shared memory;
// a block stages it with 16-byte copies.  Run state lives in the caller's
// WORKSPACE (laid out by aco_schedule_batch).  Offsets are in bytes.
#pragma once
#include <stdint.h>

#include "../../include/aco.h"

#ifdef __CUDACC__
#define ACO_HD __host__ __device__
#else
#define ACO_HD
#endif

namespace aco {

constexpr uint32_t kInvalid = 0xFFFFFFFFu;  // R35
constexpr uint32_t kMaxKernelInsts = 8191;  // ids use 13 bits in successor entries
constexpr uint32_t kFlagLiveIn = 1, kFlagLiveOut = 2;
constexpr uint32_t kSmemPerSM = 227 * 1024;  // max dynamic shared memory per block
constexpr uint32_t kMaxBlockThreads = 512;   // construct blocks (launch bounds)
// Lean variants: a 384-thread launch bound leaves the compiler up to 170
// registers (it takes ~150; at 512 it was capped at 128): measured (r02q) C3
// 692 -> 684 ms.  The planner caps lean blocks at this size.
#ifndef ACO_LEAN_LB
#define ACO_LEAN_LB 384
#endif
constexpr uint32_t kLeanMaxThreads = ACO_LEAN_LB;
// Regions with at least this many instructions use the 4-wide candidate scan
// (latency-bound: few ants fit an SM); smaller ones the 1-wide scan (issue-bound).
#ifndef ACO_WIDE_N
#define ACO_WIDE_N 160
#endif
constexpr uint32_t kWideN = ACO_WIDE_N;

// Successor entry: v (13 bits) | single-predecessor flag << 13 | latency << 16.
constexpr uint32_t kSuccSingle = 1u << 13;
// Multi-use register entry (uses of a register with >= 2 uses, not live-out):
//   bit 31 = 0: the register has exactly 2 users; bits 0..12 = the OTHER user
//   bit 31 = 1: >= 3 users; bits 0..15 = remaining-use counter index
//   bits 16..17 = register class
constexpr uint32_t kMuseCounter = 1u << 31;

// Offsets (bytes, relative to the image start) of the arrays of the block image.
struct ImageLayout {
  uint32_t info;      // uint4 [n] {defs u8x4, static kills u8x4, dead defs u8x4, muse start << 8 | count}
  uint32_t ds;        // uint4 [n] {defs u8x4, static kills u8x4, eta2, 0} (pass-2 candidates)
  uint32_t muse;      // u32 [nm]
  uint32_t cu_ptr;    // u32 [nctr+1]: users of each counter register
  uint32_t cu;        // u32 [..]
  uint32_t eta1;      // u16 [n * (L+1)]: eta1(j, sk(j) + d) at j*(L+1) + d, d = dynamic last uses (R4)
  uint32_t eta2;      // u16 [n]
  uint32_t succ_ptr;  // u32 [n+1]
  uint32_t succ;      // u32 [E]
  uint32_t pred_ptr;  // u32 [n+1]
  uint32_t pred;      // u32 [E]: p | latency << 16 (only for the u16/u32-cycle pass-2 layouts)
  uint32_t rb0;       // u32 [nwr]: roots bitset
  uint32_t rem0;      // u32 [nremw]: u16 use counts of >= 3-use registers
  uint32_t bytes;     // total, multiple of 16
  uint32_t pg_ptr;    // u32 [n+1]: predecessor groups of each instruction
  uint32_t pg;        // uint2 [..]: {bitset word, mask of the predecessors in that word}
  uint32_t mk;        // u32 [nm]: muse entry as a kill test on the per-ant state (lean layout):
                      //   word (bits 0-15, relative to the state base) | shift << 16 |
                      //   counter << 21 | class << 22; last use iff ((w >> shift) & (counter ? 0xFFFF : 1)) == 1
  uint32_t pad_img;
};
constexpr uint32_t kMkCounter = 1u << 21;

// Per-region statics (arena header array).
struct RegionDev {
  uint32_t n;        // instructions
  uint32_t nwr;      // words of an instruction bitset = ceil(n/32)
  uint32_t nremw;    // words of packed u16 counters = ceil(#counters / 2)
  uint32_t L;        // max LUC over instructions (rows of eta1 minus one)
  uint32_t region_id;
  uint32_t cp_max;
  uint32_t lb_len;   // max(n, 1 + CPmax) (R30)
  uint32_t max_cycle_bound;  // n * (max latency + 1): pass-2 cycles are below it
  uint32_t livein[4];
  uint32_t lbvec[4]; // per-class PRP lower bound vector (R30)
  uint32_t max_lat;  // largest edge latency
  uint32_t mc_max;   // max over instructions and classes of multi-use registers read
  uint32_t compact;  // pass 2 uses the compact layout (the image has no per-predecessor list)
  uint32_t nslot;    // instructions with an incoming edge of latency > 1 (lean pass-2 ready-time slots)
  uint64_t o_image;  // byte offset of the block image in the arena
  ImageLayout img;
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
  uint32_t pruned;       // pass-2 ants pruned (R24), summed over iterations; must follow prune_len
  uint32_t lb_cost;
  uint32_t len2;         // length of the pass-2 global best (pass 4: best[1] is the weighted cost)
  uint32_t policy;       // bit0 gap-filtered (R39), bit1 reverted (R40)
  uint32_t heur_len;     // the heuristic schedule's length (R40)
  uint32_t heur_prp[4];  // the heuristic schedule's PRP
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
  uint64_t o_next;   // u16 [n+1]: the iteration winner's successor of each row (0xFFFF: none)
  uint64_t o_gstate; // global-state regions: per-ant state [word][ant] (ants x words u32)
  uint64_t o_scratch;// global-state regions: replay scratch (words + cycles + order)
  uint64_t o_heur;   // u16 [n]  the heuristic (greedy pass-1) order, R40
  uint64_t o_rlk;    // u16 [ceil(ants/G)][n]: ready-list limit K per (ant group, step), R45 (rl_limit only)
  uint64_t o_rec;    // record mode: u16 [n][ants] every ant's order (step-major: coalesced stores)
  uint64_t o_recc;   // record mode: u32 [n][ants] pass-2 issue cycles
  uint64_t o_recp;   // record mode: uint4 [ants] {prp01, prp23, length, 0}
  uint32_t tau_len;  // (n+1)*n rounded up to a multiple of 8
  uint32_t gs;       // 1: the region's state does not fit shared memory (global-state kernels)
};

// Pheromone-update work item: vectors [v0, v0 + kUpdVec) of a region's table.
constexpr uint32_t kUpdVec = 2048;  // 16-byte vectors per block
struct UpdItem {
  uint32_t region;
  uint32_t v0;
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
  uint32_t ant_base;    // global id of this context's first ant (shared colony), else 0
  uint32_t weighted;    // pass 4: single weighted-sum pass on the pass-2 machinery (R41)
  uint32_t ws_weight;
  uint32_t pass2_gap, revert_occ, revert_len;  // compile policy (R39, R40)
  uint32_t heur_mix, stall_num;                // R43, R44
  uint32_t rl_limit;                           // R45: 0 off, 1 min, 2 mid
  uint32_t record;                             // ants record their schedules; k_select copies the winner's
  uint32_t stage_img;   // k_select stages the region image in shared memory (few regions)
  uint32_t mslot;       // machine slot (c_mach[mslot]) of this context
  uint32_t gs_ant_major;  // global-state kernels: per-ant state ant-major (1) or [word][ant] (0)
  uint32_t lazy_kills;    // lean pass 2: derive kills only for candidates where they decide
  uint32_t tau_prefetch;  // L1 prefetch of the next tau row: bit (pass-1) for smem-state kernels, bit 2 + (pass-1) for GS
  uint32_t prune_cp;      // R24 prune also with the critical-path bound of the scanned candidates
  uint64_t dump_slice;  // elements per (pass, iter) order slice = ants * sum n
  int64_t *keys;        // shared colony: per-region biased winner keys (NULL: local argmin)
};

struct MachineDev {
  uint32_t n_classes, occ_max;
  uint32_t step_count[4];
  uint32_t step_max[4][16];
  uint32_t perp_limit[4];
  uint32_t issue_width;  // >= 1 (R42)
  uint32_t type_slots;   // u8 x 4: issue slots per type (issue_width > 1)
  uint32_t n_types;
};

// Construct-kernel work item: one block = ants [ant0, ant0 + blockDim) of a region.
struct BlockItem {
  uint32_t region;
  uint32_t ant0;
};

inline uint64_t align16(uint64_t x) { return (x + 15) & ~uint64_t(15); }
inline uint64_t align256(uint64_t x) { return (x + 255) & ~uint64_t(255); }

// Per-ant state words (u32) of a region for a pass, [word][ant] interleave:
//   RB [nwr] ready set, SCH [nwr] scheduled set, REM [nremw] u16 counters, then
//   pass 1: DK [ceil(n/8)]  4-bit count of registers whose last remaining
//                           user is the instruction (dynamic part of LUC);
//                           none in the lean pass-1 layout (derived, dyn_kills)
//   pass 2, compact (2 classes, latencies < 512, <= 7 multi-use registers
//           per class and instruction):
//           X  [ceil(n/2)] u16: windowed ready time (10 bits) | last-use
//                           counts (2 classes x 3 bits) << 10
//   pass 2, lean (large regions, latencies < 128):
//           X8 [ceil(n/4)] u8 windowed ready time; last-use counts derived
//                           from REM / SCH at evaluation (dyn_kills)
//   pass 2, otherwise:
//           T  [ceil(n/2)] u16 (or [n] u32 if t32): issue cycle (placed) or
//                           ready time (ready instruction)
//           DK [ceil(n/4)] u8 = 2 classes x 4 bits (or [ceil(n/2)] u16 = 4
//                           classes x 4 bits if nc4): per-class last-use counts
ACO_HD inline uint32_t ant_words(uint32_t pass, uint32_t n, uint32_t nwr, uint32_t nremw, bool t32,
                                 bool nc4, bool lean = false, uint32_t nslot = 0xFFFFFFFFu) {
  const uint32_t w = 2 * nwr + nremw;
  if (pass == 1) return w + (lean ? 0u : (n + 7) / 8);  // lean pass 1: last-use counts derived, not stored
  if (lean) return w + ((nslot == 0xFFFFFFFFu ? n : nslot) + 3) / 4;  // lean: u8 ready-time slots (kills derived)
  if (!t32 && !nc4) return w + (n + 1) / 2;  // compact: u16 (windowed ready time | last uses)
  return w + (t32 ? n : (n + 1) / 2) + (nc4 ? (n + 1) / 2 : (n + 3) / 4);
}

// Lane-per-instruction ants (one warp per ant, state in registers): only the
// u16 remaining-use counters of >= 3-user registers are per-ant shared words.
ACO_HD inline uint32_t lpi_words(uint32_t nremw) { return nremw ? nremw : 1u; }
// The end of an iteration as one launch per region block (k_finalize1) for
// batches of at most this many regions of at most this many instructions.
constexpr uint32_t kFin1MaxRegions = 148, kFin1MaxN = 256;
constexpr uint32_t kLpiMaxThreads = 256;  // (8 ants per block: up to 255 registers per thread)

// Stride (in words) between consecutive state words of one ant in a block of
// apb ants x lg lanes.  stride = 32/lg (mod 32) makes the 32 lanes of a warp
// hit 32 distinct banks when lane l of every ant touches a word w = l (mod lg)
// (the split ready-bitset scan) and when only the group leaders touch
// arbitrary words (commit): bank = ant + (w mod lg) * 32/lg.
ACO_HD inline uint32_t ant_stride(uint32_t apb, uint32_t lg) {
  if (lg <= 1) return apb;
  const uint32_t m = 32 / lg;
  return ((apb + 31 - m) / 32) * 32 + m;
}

// Group-coin table of a construct block (R3): one bit per (step, group) for
// every exploit/explore group its apb consecutive ants span (group size g),
// pass 1 for the steps k < n, pass 2 for the cycles t < 32 * coin_words
// (later cycles draw their coin inline).
ACO_HD inline uint32_t coin_groups(uint32_t apb, uint32_t g) { return g >= apb ? 2u : (apb - 1) / g + 2u; }
ACO_HD inline uint32_t coin_words(uint32_t pass, uint32_t n) {
  return pass == 1 ? (n + 31) / 32 : (2 * n + 63) / 32;
}

// Bytes of the pheromone table as staged in shared memory.
ACO_HD inline uint32_t tau_smem_bytes(uint32_t n) { return (((n + 1) * n * 2) + 15) & ~15u; }

// Shared-memory layout of the fused single-block run (k_fused: all ants of a
// region in one block, every pass and iteration in one launch), offsets in
// bytes from the block's dynamic shared memory.
struct FusedLayout {
  uint32_t o_tau, o_state, o_reco, o_recc, o_costs, o_recp, o_ord, o_cyc, o_next, o_coins, bytes, words;
};
ACO_HD inline uint32_t round16(uint32_t x) { return (x + 15u) & ~15u; }
ACO_HD inline FusedLayout fused_layout(uint32_t n, uint32_t nwr, uint32_t nremw, uint32_t img_bytes, uint32_t ants,
                                       uint32_t group_size) {
  FusedLayout L;
  const uint32_t w1 = ant_words(1, n, nwr, nremw, false, false), w2 = ant_words(2, n, nwr, nremw, false, false);
  L.words = w1 > w2 ? w1 : w2;                         // per-ant state words (stride = ants)
  uint32_t off = round16(img_bytes);                   // the region's block image
  L.o_tau = off;   off += tau_smem_bytes(n);           // pheromone (n+1) x n u16
  L.o_state = off; off += round16(4u * L.words * ants);
  L.o_reco = off;  off += round16(2u * n * ants);      // every ant's order, [step][ant]
  L.o_recc = off;  off += round16(4u * (n * ants > n ? n * ants : n));  // pass-2 cycles (also ASAP scratch)
  L.o_costs = off; off += round16(4u * ants);
  L.o_recp = off;  off += 16u * ants;                  // {prp01, prp23, length, 0}
  L.o_ord = off;   off += round16(2u * n);             // the iteration winner's order / cycles
  L.o_cyc = off;   off += round16(4u * n);
  L.o_next = off;  off += round16(2u * (n + 1));       // its successor table (deposit links)
  L.o_coins = off; off += round16(4u * coin_groups(ants, group_size) * coin_words(2, n));  // group coins (R3)
  L.bytes = off;
  return L;
}
constexpr uint32_t kFusedVariant = 1u << 13;  // variant code of k_fused (aco_last_variants)
constexpr uint32_t kFusedLpi = 1u << 14;       // ... x 1 / 2 / 3: lane-per-instruction ants of 8 / 16 / 32 lanes

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
  uint32_t lanes;          // lanes per ant (1, 2, 4, 8): threads per block = ants_pb * lanes
  uint32_t smem_bytes;
  uint32_t max_n;          // max n in the class (selects the mask variant)
  bool tau_smem;           // stage tau in shared memory
  bool t32;                // u32 pass-2 cycle array
  bool nc4;                // 3-4 register classes (u16 last-use counts)
  bool gs;                 // per-ant state in global memory (huge regions)
  bool wide;               // 4-wide candidate scan (n >= kWideN: word-mask variant; global state: strided words)
  bool img_l1 = false;     // the block image is read through L1 (not staged): more ants per SM
  bool lean = false;       // lean per-ant layout: kills derived (pass 1: no last-use counts; pass 2: u8 ready times)
};

constexpr uint32_t kMachSlots = 8;  // distinct machine models resident per device
// Construct-kernel variant code (the template arguments of k_construct, see
// include/aco.h aco_last_variants): bit 0 4-wide scan, 1 global state, 2 3-4
// classes, 3 u32 cycles, 4 tau in smem, 5 word mask, 6-7 lanes (1,2,4,8),
// 8 pass-1, 9 lanes >= 16, 10 lanes 32, 11 image through L1, 12 lean.
ACO_HD constexpr uint32_t variant_code(uint32_t pass, uint32_t lg, bool m, bool ts, bool t3, bool n4, int gs, bool wd,
                                       bool lean = false) {
  return ((pass - 1) << 8) | ((lg == 1 ? 0u : lg == 2 ? 1u : lg == 4 ? 2u : 3u) << 6) | ((uint32_t)m << 5) |
         ((lg >= 16 ? 1u : 0u) << 9) | ((lg == 32 ? 1u : 0u) << 10) | ((gs == 2 ? 1u : 0u) << 11) |
         ((uint32_t)lean << 12) | ((uint32_t)ts << 4) | ((uint32_t)t3 << 3) | ((uint32_t)n4 << 2) |
         ((gs == 1 ? 1u : 0u) << 1) | (uint32_t)wd;
}
inline uint32_t class_variant(uint32_t pass, const ClassLaunch &c) {
  const bool mask = c.max_n <= 1024 && !c.gs;
  const bool rare = pass == 2 && (c.t32 || c.nc4) && !c.gs;
  return variant_code(pass, c.lanes, mask, c.tau_smem && !rare && !c.gs, pass == 2 && c.t32, pass == 2 && c.nc4,
                      c.gs ? 1 : (c.img_l1 ? 2 : 0), c.wide && (mask || c.gs || c.img_l1), c.lean);
}

int set_machine(uint32_t slot, const MachineDev &m);  // cudaMemcpyToSymbol into slot; 0 on success
int init_kernel_attrs();                              // shared-memory opt-in of every kernel (once per device)
// Resident threads per SM that the construct kernels' registers allow, per
// [pass-1][wide]; returns nonzero (and conservative defaults) without a device.
int construct_max_threads(int device, uint32_t out[2][3]);  // [pass-1][plain, wide, lean]
int launch_init(LaunchCtx &L, uint32_t smem, uint32_t max_n);
int launch_pass2_init(LaunchCtx &L, uint32_t smem, uint32_t max_n);
int launch_construct(LaunchCtx &L, uint32_t pass, uint32_t iter, const ClassLaunch &c);
int launch_finalize(LaunchCtx &L, uint32_t pass, uint32_t iter, uint32_t smem, uint32_t max_n, bool t32,
                    bool nc4, const UpdItem *upd, uint32_t n_upd, bool fin1);  // fin1: k_finalize1
int launch_local_keys(LaunchCtx &L, int64_t *keys);
int launch_post(LaunchCtx &L, uint32_t smem);
int launch_fused(LaunchCtx &L, uint32_t threads, uint32_t smem, uint32_t wl);  // the whole run, one block per region  // heuristic length + revert filter (R40)  // shared colony: per-region local argmin keys

// Biased winner key: (cost << 32 | global ant) XOR 2^63, so that a signed
// int64 MIN (NCCL / torch) orders keys like the unsigned (cost, ant) pair.
constexpr uint64_t kKeyBias = 1ull << 63;
int last_cuda_error();

}  // namespace aco
