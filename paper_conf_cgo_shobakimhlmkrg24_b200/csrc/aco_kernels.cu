// aco_kernels.cu -- sm_100a kernels of the ACO instruction scheduler.
//
// Mapping: ONE ANT PER THREAD (as the paper, L126), all
// ants of a block belong to one region.  Everything an ant touches per step
// is in SHARED MEMORY:
//   * the region's block image (per-instruction info, multi-use register
//     entries, eta tables, successor/predecessor lists) -- staged once per
//     block with 16-byte copies;
//   * the pheromone table when it fits (else read through L1 from the
//     workspace);
//   * the per-ant mutable state in a [word][ant] interleave (word w of ant a at
//     st[w * ants_per_block + a]): bank = lane, so the 32 data-dependent
//     accesses of a warp (each ant at its own instruction) never conflict.
// Exploit/explore is a coin per group of 64 ants (L198): a warp takes one
// branch in pass 1.  Candidates are scored four at a time so that their
// shared-memory loads overlap (ILP).
// Latency-bound batches (few ants in total: config 2) instead run
// lane-per-instruction ants (lpi_pass1/2): one warp per ant, every candidate
// on its own lane, the ant's state in registers.  Huge regions (n > 1024)
// keep the per-ant state in shared memory and read the image and tau through
// L1 (or, when even that does not fit, through L1/L2 from the workspace).
//
// Per pass and iteration (L135-L139):
//   k_construct : every ant builds a schedule and writes its cost (K1a); in
//                 record mode (the default) it also stores its order (and
//                 pass-2 cycles) step-major, coalesced across the ants
//   k_select    : per region: argmin over (cost, ant) (K1b); copy of the
//                 winner's recorded schedule -- or, in the shared colony and
//                 dump mode, a whole-warp replay of the winner from the same
//                 pheromone table and Philox counters; winner successor table;
//                 global-best epilogue (K1d)
//   k_update    : pheromone evaporate + deposit (K1c) over all tables
//   k_stop      : termination (K1d)
// Plus k_init (tau0, greedy heuristic schedule), k_pass2_init (target, ASAP
// of the pass-1 best, tau reset) and k_post (heuristic length, R40).
#include <cuda_runtime.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <stdint.h>

#include "aco_internal.h"


// Compile-time switches for A/B measurement (tools/ab_run.sh); the defaults
// are the product configuration.
#ifndef ACO_PREFETCH
#define ACO_PREFETCH 0
#endif
#ifndef ACO_BULK_STAGE  // k_construct stages image / tau with cp.async.bulk (else 16-byte copies by every thread)
#define ACO_BULK_STAGE 1
#endif
#ifndef ACO_BRANCHLESS1  // pass-1 4-wide evaluation without branches (measured faster)
#define ACO_BRANCHLESS1 1
#endif

namespace aco {

// Machine models (occupancy tables, issue width), one per slot: every context
// is bound to the slot holding its machine (aco_host.cpp: MachineSlots), so
// contexts with different machines can share a device (cfg.mslot).
__constant__ MachineDev c_mach[kMachSlots];

// ---------------------------------------------------------------- Philox
// Philox4x32-10 (Salmon et al., SC'11) -- R26.
__device__ __forceinline__ uint4 philox(uint32_t c0, uint32_t c1, uint32_t c2, uint32_t c3,
                                        uint64_t seed) {
  uint32_t k0 = (uint32_t)seed, k1 = (uint32_t)(seed >> 32);
#pragma unroll
  for (int i = 0; i < 10; ++i) {
    if (i) {
      k0 += 0x9E3779B9u;
      k1 += 0xBB67AE85u;
    }
    const uint32_t hi0 = __umulhi(0xD2511F53u, c0), lo0 = 0xD2511F53u * c0;
    const uint32_t hi1 = __umulhi(0xCD9E8D57u, c2), lo1 = 0xCD9E8D57u * c2;
    const uint32_t n0 = hi1 ^ c1 ^ k0, n2 = hi0 ^ c3 ^ k1;
    c0 = n0;
    c1 = lo1;
    c2 = n2;
    c3 = lo0;
  }
  return make_uint4(c0, c1, c2, c3);
}

// ---------------------------------------------------------------- costs (R16-R18)
__device__ __forceinline__ uint32_t occ_of(const MachineDev &M, uint32_t c, uint32_t x) {
  for (uint32_t i = 0; i < M.step_count[c]; ++i)
    if (x <= M.step_max[c][i]) return M.occ_max - i;
  return 0;
}
__device__ __forceinline__ uint32_t aprp_of(const MachineDev &M, uint32_t c, uint32_t x) {
  for (uint32_t i = 0; i < M.step_count[c]; ++i)
    if (x <= M.step_max[c][i]) return M.step_max[c][i];
  return x;
}
__device__ __noinline__ uint32_t cost_rp(uint32_t ms, uint32_t mode, uint32_t p0, uint32_t p1, uint32_t p2,
                                         uint32_t p3) {
  const MachineDev &c_mach = aco::c_mach[ms];
  const uint32_t prp[4] = {p0, p1, p2, p3};
  const uint32_t nc = c_mach.n_classes;
  uint32_t cost = 0;
  if (mode == ACO_COST_PRP_SUM) {
    for (uint32_t c = 0; c < nc; ++c) cost += prp[c];
  } else if (mode == ACO_COST_APRP_SUM) {
    for (uint32_t c = 0; c < nc; ++c) cost += aprp_of(c_mach, c, prp[c]);
  } else if (mode == ACO_COST_OCC) {
    uint32_t occ = c_mach.occ_max;
    for (uint32_t c = 0; c < nc; ++c) occ = min(occ, occ_of(c_mach, c, prp[c]));
    cost = c_mach.occ_max - occ;
  } else {
    for (uint32_t c = 0; c < nc; ++c)
      cost += prp[c] > c_mach.perp_limit[c] ? prp[c] - c_mach.perp_limit[c] : 0u;
  }
  return cost;
}
__device__ void target_of(uint32_t ms, uint32_t mode, const uint32_t best[4], uint32_t tgt[4]) {
  const MachineDev &c_mach = aco::c_mach[ms];
  const uint32_t nc = c_mach.n_classes;
  for (uint32_t c = 0; c < 4; ++c) tgt[c] = kInvalid;
  if (mode == ACO_COST_PRP_SUM) {
    for (uint32_t c = 0; c < nc; ++c) tgt[c] = best[c];
  } else if (mode == ACO_COST_APRP_SUM) {
    for (uint32_t c = 0; c < nc; ++c) tgt[c] = aprp_of(c_mach, c, best[c]);
  } else if (mode == ACO_COST_OCC) {
    uint32_t occ = c_mach.occ_max;
    for (uint32_t c = 0; c < nc; ++c) occ = min(occ, occ_of(c_mach, c, best[c]));
    if (occ > 0)
      for (uint32_t c = 0; c < nc; ++c) {
        const uint32_t idx = c_mach.occ_max - occ;
        const uint32_t cnt = c_mach.step_count[c];
        const uint32_t t = idx < cnt ? c_mach.step_max[c][idx] : c_mach.step_max[c][cnt - 1];
        tgt[c] = max(t, best[c]);
      }
  } else {
    for (uint32_t c = 0; c < nc; ++c) tgt[c] = max(best[c], c_mach.perp_limit[c]);
  }
}

// ---------------------------------------------------------------- statics view
struct SV {
  const uint4 *info;
  const uint4 *ds;
  const uint32_t *muse, *mk, *cu_ptr, *cu, *succ_ptr, *succ, *pred_ptr, *pred, *rb0, *rem0, *pg_ptr;
  const uint2 *pg;
  const uint16_t *eta1, *eta2;
  uint32_t n, nwr, nremw, region_id, L1, nslot, cpmax;
  uint32_t livein01, livein23;  // u16 x 2
};

__device__ __forceinline__ SV make_sv(const unsigned char *img, const RegionDev *rd) {
  SV V;
  V.info = (const uint4 *)(img + rd->img.info);
  V.ds = (const uint4 *)(img + rd->img.ds);
  V.muse = (const uint32_t *)(img + rd->img.muse);
  V.mk = (const uint32_t *)(img + rd->img.mk);
  V.cu_ptr = (const uint32_t *)(img + rd->img.cu_ptr);
  V.cu = (const uint32_t *)(img + rd->img.cu);
  V.eta1 = (const uint16_t *)(img + rd->img.eta1);
  V.eta2 = (const uint16_t *)(img + rd->img.eta2);
  V.succ_ptr = (const uint32_t *)(img + rd->img.succ_ptr);
  V.succ = (const uint32_t *)(img + rd->img.succ);
  V.pred_ptr = (const uint32_t *)(img + rd->img.pred_ptr);
  V.pred = (const uint32_t *)(img + rd->img.pred);
  V.pg_ptr = (const uint32_t *)(img + rd->img.pg_ptr);
  V.pg = (const uint2 *)(img + rd->img.pg);
  V.rb0 = (const uint32_t *)(img + rd->img.rb0);
  V.rem0 = (const uint32_t *)(img + rd->img.rem0);
  V.n = rd->n;
  V.nwr = rd->nwr;
  V.nremw = rd->nremw;
  V.nslot = rd->nslot;
  V.cpmax = rd->cp_max;
  V.region_id = rd->region_id;
  V.L1 = rd->L + 1;
  V.livein01 = (rd->livein[0] & 0xFFFFu) | (rd->livein[1] << 16);
  V.livein23 = (rd->livein[2] & 0xFFFFu) | (rd->livein[3] << 16);
  return V;
}

__device__ __forceinline__ uint32_t lo_pair(uint32_t w) { return __byte_perm(w, 0, 0x4140); }  // u8 b0,b1 -> u16x2
__device__ __forceinline__ uint32_t hi_pair(uint32_t w) { return __byte_perm(w, 0, 0x4342); }  // u8 b2,b3 -> u16x2

// Per-class comparisons of packed small counts (values < 2^15, no carry
// between lanes).  sm_100 has no native byte-SIMD compare / saturating add
// (each __vcmp*u4 / __vaddus4 is a chain of ~6 dependent LOP3/PRMT/IADD), so
// with <= 2 register classes the tests run on u16 x 2 lanes with a guard
// bit: all_le2(a, b) = every lane a_c <= b_c.
constexpr uint32_t kGuard2 = 0x80008000u;
__device__ __forceinline__ bool all_le2(uint32_t a2, uint32_t b2) {
  return (((b2 | kGuard2) - a2) & kGuard2) == kGuard2;
}
// some lane a_c < b_c
__device__ __forceinline__ bool any_lt2(uint32_t a2, uint32_t b2) {
  return ((((a2 | kGuard2) - b2) & kGuard2) != kGuard2);
}

// Per-ant state (stride S words between consecutive words of one ant).
struct St {
  uint32_t *RB, *SCH, *REM, *T, *DK;
  uint32_t S;
};

template <int PASS, bool T32, bool NC4, bool LEAN = false>
__device__ __forceinline__ St make_st(uint32_t *st, uint32_t S, const SV &V) {
  St A;
  A.S = S;
  A.RB = st;
  A.SCH = st + V.nwr * S;
  A.REM = A.SCH + V.nwr * S;
  A.T = A.REM + V.nremw * S;
  // pass 2, compact layout (!T32 && !NC4): one u16 per instruction in T,
  // ready time (windowed u8) | last-use counts << 8; DK aliases T
  A.DK = (PASS == 1 || (!T32 && !NC4)) ? A.T : A.T + (T32 ? V.n : (V.n + 1) / 2) * S;
  return A;
}

__device__ __forceinline__ uint32_t sch_bit(const St &A, uint32_t p) {
  return (A.SCH[(p >> 5) * A.S] >> (p & 31u)) & 1u;
}

// ---- last-use counts (DK): how many registers read by instruction j have j
// as their last unscheduled user (the dynamic part of kills_c(j), R14).
// pass 1: one 4-bit total per instruction
__device__ __forceinline__ uint32_t dk1_get(const St &A, uint32_t j) {
  return (A.DK[(j >> 3) * A.S] >> ((j & 7u) * 4)) & 0xFu;
}
// pass 2: 4 bits per class; returned as packed u8 x 4 per class
template <bool NC4>
__device__ __forceinline__ uint32_t dk2_get(const St &A, uint32_t j) {
  if (NC4) {
    uint32_t x = (A.DK[(j >> 1) * A.S] >> ((j & 1u) * 16)) & 0xFFFFu;
    x = (x | (x << 8)) & 0x00FF00FFu;
    return (x | (x << 4)) & 0x0F0F0F0Fu;
  }
  const uint32_t x = (A.DK[(j >> 2) * A.S] >> ((j & 3u) * 8)) & 0xFFu;
  return (x & 0xFu) | ((x & 0xF0u) << 4);
}
template <int PASS, bool T32, bool NC4>
__device__ __forceinline__ void dk_add(const St &A, uint32_t j, uint32_t c) {
  if (PASS == 1) {
    A.DK[(j >> 3) * A.S] += 1u << ((j & 7u) * 4);
  } else if (!T32 && !NC4) {  // compact: the high byte of j's u16
    A.T[(j >> 1) * A.S] += 1u << ((j & 1u) * 16 + 10 + 3 * c);
  } else if (NC4) {
    A.DK[(j >> 1) * A.S] += 1u << ((j & 1u) * 16 + 4 * c);
  } else {
    A.DK[(j >> 2) * A.S] += 1u << ((j & 3u) * 8 + 4 * c);
  }
}

template <bool T32>
__device__ __forceinline__ uint32_t t_get(const St &A, uint32_t j) {
  if (T32) return A.T[j * A.S];
  return (A.T[(j >> 1) * A.S] >> ((j & 1u) * 16)) & 0xFFFFu;
}
template <bool T32>
__device__ __forceinline__ void t_set(const St &A, uint32_t j, uint32_t v) {
  if (T32) {
    A.T[j * A.S] = v;
  } else {
    const uint32_t sh = (j & 1u) * 16;
    uint32_t *p = A.T + (j >> 1) * A.S;
    *p = (*p & ~(0xFFFFu << sh)) | (v << sh);
  }
}

// ---- pass-2 compact layout: x = u16 of instruction j = rt | dk0 << 10 |
// dk1 << 13, where rt (10 bits) = (ready time - B) for an unplaced
// instruction whose predecessors were placed (a push-style maximum of
// t_p + lat over placed predecessors; 0 for none), B is the ant's window base
// and dk_c (3 bits) the class-c last-use counts.  Invariant: t - B < kWin at
// every turn and latencies < kWin (host), so every stored rt <= 2 kWin - 2;
// when t - B reaches kWin (one jump moves t at most to B + 2 kWin - 2) the
// window slides by kWin (saturating: a clamped rt still reads as "ready now",
// which is all that matters for a value below t).  Host: the compact layout
// needs 2 classes, latencies < kWin and <= 7 multi-use registers per class
// and instruction.
constexpr uint32_t kWin = 512;
__device__ __forceinline__ uint32_t x_get(const St &A, uint32_t j) {
  return (A.T[(j >> 1) * A.S] >> ((j & 1u) * 16)) & 0xFFFFu;
}
__device__ __forceinline__ uint32_t x_dk(uint32_t x) {  // packed u8 x 4 per class
  return ((x >> 10) & 0x7u) | ((x & 0xE000u) >> 5);
}
__device__ __forceinline__ void x_push_rt(const St &A, uint32_t v, uint32_t rt) {
  uint32_t *p = A.T + (v >> 1) * A.S;
  const uint32_t sh = (v & 1u) * 16, w = *p, cur = (w >> sh) & 0x3FFu;
  if (rt > cur) *p = w + ((rt - cur) << sh);
}
// Slide both halves' 10-bit rt by kWin = 512, saturating at 0:
// rt >= 512 -> rt & 0x1FF, else 0 (rt < 1024).
__device__ __forceinline__ uint32_t x_slide2(uint32_t w) {
  return (w & 0xFC00FC00u) | (w & (((w >> 9) & 0x00010001u) * 0x1FFu));
}

// ---- pass-2 LEAN layout (large regions: more ants per SM): one u8 per
// instruction = ready time relative to the window base B (window kWin8 = 128,
// latencies < 128, so a stored value is <= 254), and NO stored last-use
// counts: the dynamic kills of a candidate are derived from its multi-use
// registers' remaining-use counters / partners' scheduled bits (dyn_kills).
constexpr uint32_t kWin8 = 128;
// Ready-time SLOTS (r02): only an instruction with an incoming edge of
// latency > 1 can be semi-ready (a latency-0/1 edge is met in the cycle after
// its source issues, i.e. by the time the instruction is in the ready set), so
// only those instructions own a u8 slot; ds.z >> 16 = slot, 0xFFFF = none
// (always latency-ready once its predecessors are placed).  Pushes skip
// latency <= 1 edges: they never decide "ready time <= t" (see commit).
constexpr uint32_t kNoSlot = 0xFFFFu;
__device__ __forceinline__ uint32_t r8_get(const St &A, uint32_t slot) {
  return slot == kNoSlot ? 0u : (A.T[(slot >> 2) * A.S] >> ((slot & 3u) * 8)) & 0xFFu;
}
__device__ __forceinline__ void r8_push(const St &A, uint32_t slot, uint32_t rt) {
  uint32_t *p = A.T + (slot >> 2) * A.S;
  *p = __vmaxu4(*p, rt << ((slot & 3u) * 8));  // byte-wise max (push-style ready time)
}
// kills_c(j) - static kills_c(j) as packed u8 x 4: registers read by j with >= 2
// users whose last unscheduled user j is (R14): a counter register with one
// remaining use, or a 2-user register whose partner is scheduled.
// dsw = ds.w of j (multi-use count << 4 | start << 8).
__device__ __forceinline__ uint32_t mk_last(const St &A, uint32_t e) {  // e: an mk entry (ImageLayout::mk)
  const uint32_t w = A.RB[(e & 0xFFFFu) * A.S];  // RB is the state base
  return ((w >> ((e >> 16) & 31u)) & ((e & kMkCounter) ? 0xFFFFu : 1u)) == 1u;
}
__device__ __forceinline__ uint32_t dyn_kills(const SV &V, const St &A, uint32_t dsw) {
  uint32_t K = 0;
  const uint32_t mc = (dsw >> 4) & 0xFu, m0 = dsw >> 8;
  for (uint32_t q = 0; q < mc; ++q) {
    const uint32_t e = V.mk[m0 + q];
    K += mk_last(A, e) << (8 * ((e >> 22) & 3u));
  }
  return K;
}
// dyn_kills of four candidates at once: level q of every candidate's
// multi-use list is fetched together (two dependent shared/L1 loads per
// level for all four, instead of four serial chains).  An exhausted list
// reads state word 0 (in bounds) and is masked out.
__device__ __forceinline__ void dyn_kills4w(const SV &V, const St &A, const uint32_t (&dsw)[4], uint32_t (&dk)[4]) {
  uint32_t mc[4], m0[4], mx = 0;
#pragma unroll
  for (int u = 0; u < 4; ++u) {
    mc[u] = (dsw[u] >> 4) & 0xFu;
    m0[u] = dsw[u] >> 8;
    dk[u] = 0;
    mx = ::max(mx, mc[u]);
  }
  for (uint32_t q = 0; q < mx; ++q) {
    uint32_t e[4], w[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) e[u] = q < mc[u] ? V.mk[m0[u] + q] : 0u;
#pragma unroll
    for (int u = 0; u < 4; ++u) w[u] = A.RB[(e[u] & 0xFFFFu) * A.S];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      const uint32_t last = ((w[u] >> ((e[u] >> 16) & 31u)) & ((e[u] & kMkCounter) ? 0xFFFFu : 1u)) == 1u;
      dk[u] += (q < mc[u] && last ? 1u : 0u) << (8 * ((e[u] >> 22) & 3u));
    }
  }
}
__device__ __forceinline__ void dyn_kills4(const SV &V, const St &A, const uint4 (&ds)[4], uint32_t (&dk)[4]) {
  const uint32_t dsw[4] = {ds[0].w, ds[1].w, ds[2].w, ds[3].w};
  dyn_kills4w(V, A, dsw, dk);
}

// ---- lane groups: LG consecutive lanes of a warp build one ant together.
// Lane l of a group scans the ready-bitset words w with w % LG == l; the group
// reduces with shuffles; lane 0 (the leader) performs every state update.
template <int LG>
struct Grp {
  uint32_t lane, mask;
  __device__ __forceinline__ Grp(uint32_t tid) {
    const uint32_t l = tid & 31u;
    lane = l & (LG - 1);
    mask = LG == 32 ? 0xFFFFFFFFu : (((1u << LG) - 1u) << (l - lane));
  }
  __device__ __forceinline__ bool leader() const { return lane == 0; }
  __device__ __forceinline__ uint32_t bcast(uint32_t v) const {
    return LG == 1 ? v : __shfl_sync(mask, v, 0, LG);
  }
  __device__ __forceinline__ uint32_t sum(uint32_t v) const {
#pragma unroll
    for (int o = LG / 2; o > 0; o >>= 1) v += __shfl_xor_sync(mask, v, o, LG);
    return v;
  }
  __device__ __forceinline__ uint32_t max(uint32_t v) const {
#pragma unroll
    for (int o = LG / 2; o > 0; o >>= 1) v = ::max(v, __shfl_xor_sync(mask, v, o, LG));
    return v;
  }
  __device__ __forceinline__ uint32_t min(uint32_t v) const {
#pragma unroll
    for (int o = LG / 2; o > 0; o >>= 1) v = ::min(v, __shfl_xor_sync(mask, v, o, LG));
    return v;
  }
  __device__ __forceinline__ unsigned long long max64(unsigned long long v) const {
#pragma unroll
    for (int o = LG / 2; o > 0; o >>= 1) v = ::max(v, __shfl_xor_sync(mask, v, o, LG));
    return v;
  }
  __device__ __forceinline__ unsigned long long sum64(unsigned long long v) const {
#pragma unroll
    for (int o = LG / 2; o > 0; o >>= 1) v += __shfl_xor_sync(mask, v, o, LG);
    return v;
  }
  __device__ __forceinline__ bool any(bool p) const {
    return LG == 1 ? p : (__ballot_sync(mask, p) & mask) != 0u;
  }
  __device__ __forceinline__ void sync() const {
    if (LG > 1) __syncwarp(mask);
  }
};

// Bits of a word-subset mask: words w with w % LG == lane (n <= 1024).
template <int LG>
__device__ __forceinline__ uint32_t lane_words(uint32_t lane) {
  return LG == 1 ? 0xFFFFFFFFu
                 : (LG == 2 ? 0x55555555u
                            : (LG == 4 ? 0x11111111u
                                       : (LG == 8 ? 0x01010101u : (LG == 16 ? 0x00010001u : 1u))))
                       << lane;
}

// Visit the set bits of the ready bitset in ascending order: all words
// (stride 1) or this lane's words (stride LG).  MASK: wmask has one bit per
// non-empty word (n <= 1024).
template <bool MASK, typename F>
__device__ __forceinline__ void scan_bits(const St &A, uint32_t nwr, uint32_t wmask, uint32_t first,
                                          uint32_t stride, uint32_t sub, F &&visit) {
  if (MASK) {
    uint32_t m = wmask & sub;
    while (m) {
      const uint32_t w = __ffs(m) - 1;
      m &= m - 1;
      uint32_t bits = A.RB[w * A.S];
      while (bits) {
        const uint32_t j = w * 32u + (__ffs(bits) - 1);
        bits &= bits - 1;
        if (visit(j)) return;
      }
    }
  } else {
    for (uint32_t w = first; w < nwr; w += stride) {
      uint32_t bits = A.RB[w * A.S];
      while (bits) {
        const uint32_t j = w * 32u + (__ffs(bits) - 1);
        bits &= bits - 1;
        if (visit(j)) return;
      }
    }
  }
}

// Batched scan (MASK variant, n <= 1024): visit(j[4], v[4]) receives the
// next four set bits of this lane's words in ascending order (v[u] = valid;
// an invalid slot repeats j[0], so its loads stay in bounds).  Extracting
// four candidates before touching their data lets a thread issue the four
// candidates' shared-memory / L2 loads back to back instead of one dependent
// chain per candidate (the step is latency-bound for large regions, where
// few ants fit on an SM).  wmask has exactly the non-empty words' bits, so
// one word fetch always refills an exhausted bits register.
template <typename F>
__device__ __forceinline__ void scan4(const St &A, uint32_t m, F &&visit) {
#if ACO_PREFETCH
  // the next non-empty word is fetched one word ahead (its load overlaps the
  // current word's candidates)
  uint32_t w = 0, bits = 0, nw = 0, nbits = 0;
  bool pend = m != 0u;
  if (pend) {
    nw = __ffs(m) - 1;
    m &= m - 1;
    nbits = A.RB[nw * A.S];
  }
  while (true) {
    uint32_t j[4];
    bool v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      if (!bits && pend) {
        w = nw;
        bits = nbits;
        pend = m != 0u;
        if (pend) {
          nw = __ffs(m) - 1;
          m &= m - 1;
          nbits = A.RB[nw * A.S];
        }
      }
      v[u] = bits != 0u;
      j[u] = v[u] ? w * 32u + (__ffs(bits) - 1) : j[0];
      bits &= bits - 1;
    }
    if (!v[0]) return;
    visit(j, v);
    if (!v[3] || (!bits && !pend)) return;
  }
#else
  uint32_t w = 0, bits = 0;
  while (true) {
    uint32_t j[4];
    bool v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      if (!bits && m) {
        w = __ffs(m) - 1;
        m &= m - 1;
        bits = A.RB[w * A.S];
      }
      v[u] = bits != 0u;
      j[u] = v[u] ? w * 32u + (__ffs(bits) - 1) : j[0];
      bits &= bits - 1;
    }
    if (!v[0]) return;
    visit(j, v);
    if (!v[3] || (!bits && !m)) return;
  }
#endif
}

// Batched scan without a word mask (huge regions, global-state kernels):
// this lane's words first, first + stride, ... < nwr, four set bits at a time
// in ascending order (same contract as scan4).
template <typename F>
__device__ __forceinline__ void scan4s(const St &A, uint32_t first, uint32_t stride, uint32_t nwr, F &&visit) {
  uint32_t w = 0, bits = 0, nw = first;
  while (true) {
    uint32_t j[4];
    bool v[4];
#pragma unroll
    for (int u = 0; u < 4; ++u) {
      while (!bits && nw < nwr) {
        w = nw;
        bits = A.RB[w * A.S];
        nw += stride;
      }
      v[u] = bits != 0u;
      j[u] = v[u] ? w * 32u + (__ffs(bits) - 1) : j[0];
      bits &= bits - 1;
    }
    if (!v[0]) return;
    visit(j, v);
    if (!v[3] || (!bits && nw >= nwr)) return;
  }
}
template <bool MASK, typename F>
__device__ __forceinline__ void scan4_any(const St &A, uint32_t m, uint32_t first, uint32_t stride, uint32_t nwr,
                                          F &&visit) {
  if constexpr (MASK) scan4(A, m, visit);
  else scan4s(A, first, stride, nwr, visit);
}

// Prefetch the pheromone row of the next step into L1 (the row of the
// instruction just placed; tau in global memory): one 128-byte line per lane
// and stride, issued right after the commit so the next scan's tau reads hit.
template <int LG>
__device__ __forceinline__ void tau_row_prefetch(const uint16_t *tau, uint32_t row, uint32_t n, const Grp<LG> &G) {
  const char *p = (const char *)(tau + (size_t)row * n);
  for (uint32_t b = G.lane * 128u; b < n * 2u; b += LG * 128u) asm volatile("prefetch.global.L1 [%0];" ::"l"(p + b));
}

struct AntOut {
  uint32_t cost;
  uint32_t prp01, prp23;
  uint32_t len;  // pass 2: schedule length (cost is the weighted cost in pass 4, R41)
};

// Optional stalls for ant group g (L202-L204; R23, R44).
__device__ __forceinline__ bool stall_group(const RunCfg &cfg, uint32_t g) {
  const uint32_t mod = cfg.stall_mod, rem = cfg.stall_rem % mod;
  return ((g % mod) + mod - rem) % mod < cfg.stall_num;
}
// Sum of the four u8 lanes (per-class last-use counts -> LUC).
__device__ __forceinline__ uint32_t sum_u8x4(uint32_t x) { return __dp4a(x, 0x01010101u, 0u); }

__device__ __forceinline__ uint32_t cost_of(uint32_t ms, uint32_t mode, uint32_t prp01, uint32_t prp23) {
  return cost_rp(ms, mode, prp01 & 0xFFFFu, prp01 >> 16, prp23 & 0xFFFFu, prp23 >> 16);
}

// Commit of instruction j at cycle t (both passes): scheduled / ready sets,
// the RP update (R14, R15), last-use bookkeeping of the registers j reads,
// and the successors that become ready (pass 2: with their ready times).
template <int PASS, bool MASK, bool T32, bool NC4, bool LEAN = false>
__device__ __forceinline__ void commit(const SV &V, const St &A, uint32_t j, uint32_t t, uint32_t &wmask,
                                       uint32_t &live01, uint32_t &live23, uint32_t &prp01,
                                       uint32_t &prp23, uint32_t B = 0) {
  constexpr bool CT = PASS == 2 && !T32 && !NC4;  // push-style ready times (compact or lean)
  {
    const uint32_t wi = j >> 5, bit = 1u << (j & 31u);
    const uint32_t nw = A.RB[wi * A.S] & ~bit;
    A.RB[wi * A.S] = nw;
    if (MASK && !nw) wmask &= ~(1u << wi);
    A.SCH[wi * A.S] |= bit;
  }
  if (PASS == 2 && !CT) t_set<T32>(A, j, t);
  const uint4 inf = V.info[j];
  uint32_t K = inf.y;  // static kills (single-use registers)
  {
    const uint32_t m0 = inf.w >> 8, mc = inf.w & 0xFFu;
    for (uint32_t q = 0; q < mc; ++q) {
      const uint32_t e = V.muse[m0 + q];
      const uint32_t c = (e >> 16) & 3u;
      if (e & kMuseCounter) {  // >= 3 users: remaining-use counter
        const uint32_t m = e & 0xFFFFu, sh = (m & 1u) * 16;
        uint32_t *p = A.REM + (m >> 1) * A.S;
        const uint32_t w = *p;
        *p = w - (1u << sh);
        const uint32_t left = (w >> sh) & 0xFFFFu;  // users left including j
        if (left == 1u) {
          K += 1u << (8 * c);  // j is the last user: the register dies here
        } else if (!LEAN && left == 2u) {  // one user remains: it becomes the last user
          for (uint32_t k = V.cu_ptr[m]; k < V.cu_ptr[m + 1]; ++k) {
            const uint32_t u = V.cu[k];
            if (!sch_bit(A, u)) {
              dk_add<PASS, T32, NC4>(A, u, c);
              break;
            }
          }
        }
      } else {  // 2 users: the partner
        const uint32_t p = e & 0x1FFFu;
        if (sch_bit(A, p)) K += 1u << (8 * c);
        else if (!LEAN) dk_add<PASS, T32, NC4>(A, p, c);
      }
    }
  }
  live01 = __vsub2(live01, lo_pair(K));
  live23 = __vsub2(live23, hi_pair(K));
  live01 = __vadd2(live01, lo_pair(inf.x));
  live23 = __vadd2(live23, hi_pair(inf.x));
  prp01 = __vmaxu2(prp01, live01);
  prp23 = __vmaxu2(prp23, live23);
  live01 = __vsub2(live01, lo_pair(inf.z));
  live23 = __vsub2(live23, hi_pair(inf.z));
  const uint32_t s0 = V.succ_ptr[j], s1 = V.succ_ptr[j + 1];
  for (uint32_t q = s0; q < s1; ++q) {
    const uint32_t e = V.succ[q];
    const uint32_t v = e & 0x1FFFu;
    bool ready = true;
    uint32_t rdy = t + (e >> 16);
    if (CT) {  // ready time = max over placed predecessors
      if (LEAN) {
        // (a latency <= 1 edge is met by the next cycle: no push; such a
        // successor of a slot-less instruction cannot occur)
        if ((e >> 16) > 1u) r8_push(A, V.ds[v].z >> 16, rdy - B);
      } else {
        x_push_rt(A, v, rdy - B);
      }
    }
    if (!(e & kSuccSingle) && (PASS == 1 || CT)) {
      // v is ready iff all its predecessors are placed: one scheduled-set
      // word per group of predecessors sharing a bitset word
      for (uint32_t k = V.pg_ptr[v]; k < V.pg_ptr[v + 1]; ++k) {
        const uint2 g = V.pg[k];
        if ((A.SCH[g.x * A.S] & g.y) != g.y) {
          ready = false;
          break;
        }
      }
    } else if (!(e & kSuccSingle)) {
      const uint32_t p0 = V.pred_ptr[v], p1 = V.pred_ptr[v + 1];
      if (PASS == 2 && !CT) rdy = 0;
      for (uint32_t k = p0; k < p1; ++k) {
        const uint32_t pe = V.pred[k];
        const uint32_t p = pe & 0xFFFFu;
        if (!sch_bit(A, p)) {
          ready = false;
          break;
        }
        if (PASS == 2 && !CT) rdy = max(rdy, t_get<T32>(A, p) + (pe >> 16));
      }
    }
    if (ready) {
      A.RB[(v >> 5) * A.S] |= 1u << (v & 31u);
      if (MASK) wmask |= 1u << (v >> 5);
      if (PASS == 2 && !CT) t_set<T32>(A, v, rdy);
    }
  }
}

// Initial per-ant state, written by the LG lanes of the ant's group (lane l
// takes words l, l + LG, ...); returns the non-empty-word mask (MASK) in
// every lane.
template <int PASS, bool MASK, bool T32, bool NC4, bool LEAN = false, int LG = 1>
__device__ __forceinline__ uint32_t init_state(const SV &V, const St &A, const Grp<LG> &G) {
  uint32_t wmask = 0;
  for (uint32_t w = G.lane; w < V.nwr; w += LG) {
    const uint32_t x = V.rb0[w];
    A.RB[w * A.S] = x;
    A.SCH[w * A.S] = 0;
    if (MASK && x) wmask |= 1u << w;
  }
  for (uint32_t w = G.lane; w < V.nremw; w += LG) A.REM[w * A.S] = V.rem0[w];
  const uint32_t n = V.n;
  const bool ct = PASS == 2 && !T32 && !NC4;
  const uint32_t tw = PASS == 1 ? 0 : (LEAN ? (V.nslot + 3) / 4 : (T32 ? n : (n + 1) / 2));
  const uint32_t dw = PASS == 1 ? (LEAN ? 0u : (n + 7) / 8) : (ct ? 0u : (NC4 ? (n + 1) / 2 : (n + 3) / 4));
  for (uint32_t w = G.lane; w < tw + dw; w += LG) A.T[w * A.S] = 0;  // T and DK are contiguous
  if (MASK && LG > 1) {
#pragma unroll
    for (int o = LG / 2; o > 0; o >>= 1) wmask |= __shfl_xor_sync(G.mask, wmask, o, LG);
  }
  G.sync();
  return wmask;
}

// Argmax key: highest score, ties to the lowest index (R1, R25).
__device__ __forceinline__ unsigned long long akey(uint32_t s, uint32_t j) {
  return ((unsigned long long)s << 32) | (0xFFFFFFFFu - j);
}

// ------------------------------------------------------------ pass-1 ant
// Ready-list size limit (L214; R45): the ants of one group of G consecutive
// ids (the paper's wavefront) run pass 1 in lockstep inside one block; at
// step k each ant considers only its first K ready instructions (ascending),
// K = the group's smallest ready-list size (mode 1) or the midpoint of the
// smallest and largest (mode 2).  buf: per-block shared counters, triple
// buffered by step (one barrier per step); out: K per step of the group
// (written by its first ant, read by the winner replay through `in`).
struct RL {
  uint32_t *buf;       // [3][ng][2] {min, max}; nullptr: no limit
  uint32_t gi, ng, mode;
  uint16_t *out;       // K per step of this ant's group, or nullptr
  const uint16_t *in;  // replay: the recorded K per step (no barriers)
};

// Block barrier for the lockstep steps: NOT the .aligned form of
// __syncthreads, because a warp may hold both live ants (in ant_pass1) and
// ghost lanes past the ant count (in k_construct's matching loop), which
// reach it from different code.
__device__ __forceinline__ void rl_barrier() { asm volatile("barrier.sync 0;" ::: "memory"); }

// Index of the K-th (1-based) set bit of the ready bitset in ascending order
// (the last candidate an ant may consider); n if there are fewer.
__device__ __forceinline__ uint32_t kth_ready(const St &A, uint32_t nwr, uint32_t K, uint32_t n) {
  for (uint32_t w = 0; w < nwr; ++w) {
    const uint32_t x = A.RB[w * A.S], c = __popc(x);
    if (K <= c) return w * 32u + __fns(x, 0, K);
    K -= c;
  }
  return n;
}
__device__ __forceinline__ uint32_t ready_count(const St &A, uint32_t nwr) {
  uint32_t c = 0;
  for (uint32_t w = 0; w < nwr; ++w) c += __popc(A.RB[w * A.S]);
  return c;
}

// RP pass (L108, L145; R19): latencies ignored, candidates = ready list,
// score tau[prev][j] * eta1(j, LUC(j)) (R1, R4).  The step index k is the
// Philox step (R26).  rec (leader, may be NULL) receives the order.  The
// result is valid in the leader lane.
template <int LG, bool MASK, bool WIDE = false, bool RLIM = false, bool LEAN = false>
__device__ __forceinline__ AntOut ant_pass1(const SV &V, const uint16_t *__restrict__ tau, const St &A,
                                            const Grp<LG> &G, const uint32_t ant, const uint32_t iter,
                                            const RunCfg &cfg, const bool greedy, uint16_t *rec,
                                            const uint32_t *coins = nullptr, const RL rl = RL{nullptr, 0, 0, 0, nullptr, nullptr},
                                            const uint32_t rec_stride = 1, const bool pf = false) {
  const uint32_t n = V.n, nwr = V.nwr, L1 = V.L1;
  constexpr bool limit = RLIM;  // R45 (rl.buf or rl.in set)
  uint32_t wmask = init_state<1, MASK, false, false, LEAN, LG>(V, A, G);
  uint32_t live01 = V.livein01, live23 = V.livein23, prp01 = live01, prp23 = live23;
  const uint32_t group = ant / cfg.group_size;
  const uint32_t sub = lane_words<LG>(G.lane);
  constexpr bool wide = WIDE;  // 4-wide scan (word mask or strided words)
  // R43: odd groups are guided by the ILP heuristic (CP, eta2) instead
  const bool mix = !greedy && cfg.heur_mix && (group & 1u);
  uint32_t prev = n;
  for (uint32_t k = 0; k < n; ++k) {
    bool exploit = greedy;
    if (!greedy) {
      if (coins) {  // the block's precomputed group coins (R3)
        exploit = (coins[k >> 5] >> (k & 31u)) & 1u;
      } else {
        const uint4 g = philox(k, 0x80000000u | group, iter, V.region_id, cfg.seed);
        exploit = (uint64_t)g.x < cfg.q0_t;
      }
    }
    const uint16_t *trow = tau + prev * n;
    // R45: the last candidate index this ant may consider at step k
    uint32_t jmax = n;
    if constexpr (limit) {
      uint32_t K;
      if (rl.in) {
        K = rl.in[k];
      } else {
        uint32_t *slot = rl.buf + ((k % 3u) * rl.ng + rl.gi) * 2u;
        if (G.leader()) {
          const uint32_t c = ready_count(A, nwr);
          atomicMin(slot, c);
          atomicMax(slot + 1, c);
        }
        if (threadIdx.x == 0) {  // reset the buffer of step k + 1 (last read at step k - 2)
          uint32_t *nb = rl.buf + ((k + 1u) % 3u) * rl.ng * 2u;
          for (uint32_t g = 0; g < rl.ng; ++g) {
            nb[2 * g] = 0xFFFFFFFFu;
            nb[2 * g + 1] = 0u;
          }
        }
        rl_barrier();
        const uint32_t lo = slot[0], hi = slot[1];
        K = rl.mode == 1 ? lo : (lo + hi) / 2u;
        if (rl.out && G.leader()) rl.out[k] = (uint16_t)K;
      }
      if (G.leader()) jmax = kth_ready(A, nwr, K, n);
      jmax = G.bcast(jmax);
    }
    // score(j) = tau[prev][j] * eta1(j, sk(j) + d(j)) (R1, R4)
    // (lean layout: the dynamic last-use count is derived from the state, R14)
    auto score = [&](uint32_t j) -> uint32_t {
      if (mix) return (uint32_t)trow[j] * (V.ds[j].z & 0xFFFFu);
      const uint32_t d = LEAN ? sum_u8x4(dyn_kills(V, A, V.ds[j].w)) : dk1_get(A, j);
      return (uint32_t)trow[j] * (uint32_t)V.eta1[j * L1 + d];
    };
    // Lane-local argmax in ascending order: strict '>' keeps the lowest
    // index among equal scores; bs1 = best score + 1 (0 = no candidate; a
    // score is < 2^32 - 1, so +1 cannot wrap).
    uint32_t bs1 = 0, bj = 0;
    unsigned long long sum = 0;
    if constexpr (wide) {
      scan4_any<MASK>(A, wmask & sub, G.lane, LG, nwr, [&](const uint32_t(&j)[4], const bool(&v0)[4]) {
        uint32_t tv[4], dk[4];
        bool v[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          v[u] = v0[u] && (!limit || j[u] <= jmax);  // R45
          tv[u] = trow[j[u]];
          if constexpr (!LEAN) dk[u] = A.DK[(j[u] >> 3) * A.S];
        }
        if constexpr (LEAN) {  // dynamic last-use counts from the state (four candidates at once)
          uint32_t dsw[4];
#pragma unroll
          for (int u = 0; u < 4; ++u) dsw[u] = V.ds[j[u]].w;
          dyn_kills4w(V, A, dsw, dk);
#pragma unroll
          for (int u = 0; u < 4; ++u) dk[u] = mix ? (V.ds[j[u]].z & 0xFFFFu) : V.eta1[j[u] * L1 + sum_u8x4(dk[u])];
        } else {
#pragma unroll
          for (int u = 0; u < 4; ++u)
            dk[u] = mix ? (V.ds[j[u]].z & 0xFFFFu) : V.eta1[j[u] * L1 + ((dk[u] >> ((j[u] & 7u) * 4)) & 0xFu)];
        }
#if ACO_BRANCHLESS1
        // branch-free: the four candidates' chains interleave (ILP)
        uint32_t sc[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) sc[u] = v[u] ? tv[u] * dk[u] + 1u : 0u;  // score + 1, 0 = none
#pragma unroll
        for (int u = 0; u < 4; ++u) {  // ascending: strict keeps the lowest index
          const bool b = sc[u] > bs1;
          bs1 = b ? sc[u] : bs1;
          bj = b ? j[u] : bj;
        }
        if (!exploit) {
          uint32_t s01 = (sc[0] ? sc[0] - 1u : 0u), s23 = (sc[2] ? sc[2] - 1u : 0u);
          const uint64_t a = (uint64_t)s01 + (sc[1] ? sc[1] - 1u : 0u);
          const uint64_t b = (uint64_t)s23 + (sc[3] ? sc[3] - 1u : 0u);
          sum += a + b;
        }
#else
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          const uint32_t sc = tv[u] * dk[u];
          if (v[u]) {
            if (sc + 1u > bs1) {
              bs1 = sc + 1u;
              bj = j[u];
            }
            if (!exploit) sum += sc;
          }
        }
#endif
      });
    } else {
      scan_bits<MASK>(A, nwr, wmask, G.lane, LG, sub, [&](uint32_t j) {
        if (limit && j > jmax) return true;  // R45: ascending, nothing further is allowed
        const uint32_t sc = score(j);
        if (sc + 1u > bs1) {
          bs1 = sc + 1u;
          bj = j;
        }
        if (!exploit) sum += sc;
        return false;
      });
    }
    uint32_t jstar;
    if (LG == 1) {
      jstar = bj;
    } else {
      const unsigned long long best = G.max64(bs1 ? akey(bs1 - 1u, bj) : 0ull);
      jstar = 0xFFFFFFFFu - (uint32_t)best;
    }
    if (!exploit) {  // roulette (R27): the leader scans every candidate in ascending order
      sum = G.sum64(sum);
      if (G.leader()) {
        const uint4 x = philox(k, ant, iter, V.region_id, cfg.seed);
        const uint64_t r = __umul64hi(((uint64_t)x.y << 32) | x.x, sum);
        uint64_t pre = 0;
        scan_bits<MASK>(A, nwr, wmask, 0, 1, 0xFFFFFFFFu, [&](uint32_t j) {
          pre += score(j);  // (j <= jmax: the prefix exceeds r within the allowed candidates)
          if (pre > r) {
            jstar = j;
            return true;
          }
          return false;
        });
      }
      jstar = G.bcast(jstar);
    }
    if (G.leader()) {
      commit<1, MASK, false, false, LEAN>(V, A, jstar, 0, wmask, live01, live23, prp01, prp23);
      if (rec) rec[(size_t)k * rec_stride] = (uint16_t)jstar;
    }
    wmask = G.bcast(wmask);
    G.sync();
    prev = jstar;
    if (pf) tau_row_prefetch<LG>(tau, prev, n, G);
  }
  AntOut o;
  o.prp01 = prp01;
  o.prp23 = prp23;
  o.len = 0;
  o.cost = G.leader() ? cost_of(cfg.mslot, cfg.cost_mode, prp01, prp23) : 0u;
  return o;
}

// ------------------------------------------------------------ pass-2 ant
// ILP pass (L108, L118, L147-L164, L200-L206; R19-R24).  t is the cycle;
// stalls skip ahead without drawing.  rec_o / rec_c (leader, may be NULL)
// receive the order and the cycles.  Valid in the leader lane.
// General machine model (L64; R42; not the lean layout): the ant stays in
// cycle t until issue_width instructions were placed; a latency-met
// instruction whose slot (width / type) is full counts as semi-ready with
// ready time t + 1; the Philox step is t * issue_width + used.
// Weighted single pass (pass 4, R41): no target, cost = length + W * cost_rp.
template <int LG, bool MASK, bool T32, bool NC4, bool WIDE = false, bool LEAN = false>
__device__ __forceinline__ AntOut ant_pass2(const SV &V, const uint16_t *__restrict__ tau, const St &A,
                                            const Grp<LG> &G, const uint32_t ant, const uint32_t iter,
                                            const RunCfg &cfg, const uint32_t tgt[4], uint32_t *prune_len,
                                            const bool prune, uint16_t *rec_o, uint32_t *rec_c,
                                            const uint32_t *coins = nullptr, uint32_t coin_t = 0,
                                            const uint32_t rec_stride = 1, const bool pf = false) {
  const uint32_t n = V.n, nwr = V.nwr, L1 = V.L1;
  uint32_t wmask = init_state<2, MASK, T32, NC4, LEAN, LG>(V, A, G);
  uint32_t live01 = V.livein01, live23 = V.livein23, prp01 = live01, prp23 = live23;
  const uint32_t group = ant / cfg.group_size;
  const bool stall_en = stall_group(cfg, group);      // R23, R44
  const bool mix = cfg.heur_mix && (group & 1u);      // R43: odd groups use eta1 (LUC, CP)
  const uint32_t c2 = 0x80000000u | iter;
  const uint32_t sub = lane_words<LG>(G.lane);
  constexpr bool wide = WIDE;  // 4-wide scan (word mask or strided words)
  constexpr bool CT = !T32 && !NC4;  // compact layout (x_get)
  // general machine model (R42): runtime, only in the u32-cycle variants
  // (every layout but lean: the lean ready-time slots assume a placement
  // ends its cycle, so lean is planned for single issue only)
  const uint32_t w = LEAN ? 1u : c_mach[cfg.mslot].issue_width;
  const bool mi = w > 1u;
  const uint32_t slots = c_mach[cfg.mslot].type_slots;  // u8 x 4
  uint32_t used = 0, used_t = 0;              // placed in cycle t: total, per type (u8 x 4)
  uint32_t t = 0, placed = 0, kopt = 0, prev = n, turn = 0, B = 0;
  // ready time and per-class last-use counts of instruction j (LEAN: the
  // counts come from dyn_kills once ds is loaded)
  auto rd_dk = [&](uint32_t j, uint32_t &rd, uint32_t &dk) {
    if constexpr (LEAN) {  // (the ready time needs ds.z: lean_rd below)
      rd = 0;
      dk = 0;
      (void)j;
    } else if constexpr (CT) {
      const uint32_t x = x_get(A, j);
      rd = B + (x & 0x3FFu);
      dk = x_dk(x);
    } else {
      rd = t_get<T32>(A, j);
      dk = dk2_get<NC4>(A, j);
    }
  };
  auto lean_rd = [&](uint32_t dsz) -> uint32_t { return B + r8_get(A, dsz >> 16); };
  // R24 with a critical-path bound: an unplaced instruction j with ready time
  // rd is issued at >= max(rd, t) and its longest successor chain needs CP(j)
  // more cycles, so length >= max(rd, t) + CP(j) + 1.  CP(j) >= the floor of
  // (eta2(j) - 1) CPmax / 65534 (eta2 = 1 + floor(CP 65534 / CPmax), R4).
  const bool pcp = prune && cfg.prune_cp;
  uint32_t cp_run = 0;
  auto cp_floor = [&](uint32_t dsz) -> uint32_t {
    return (uint32_t)(((uint64_t)((dsz & 0xFFFFu) - 1u) * V.cpmax) / 65534u);
  };
  const bool lazy = LEAN && cfg.lazy_kills && !stall_en && !mix;  // (lean: kills only where they decide)
  // heuristic of a feasible candidate: eta2 (CP), or eta1 (LUC, CP) for mixed odd groups
  auto eta_of = [&](uint32_t j, uint32_t e2, uint32_t dk) -> uint32_t {
    return mix ? (uint32_t)V.eta1[j * L1 + sum_u8x4(dk)] : e2;
  };
  AntOut o;
  o.prp01 = o.prp23 = 0;
  o.len = kInvalid;
  while (placed < n) {
    if (LEAN && t - B >= kWin8) {  // slide the u8 window: saturating byte subtract
      for (uint32_t q = G.lane; q < (V.nslot + 3) / 4; q += LG) A.T[q * A.S] = __vsubus4(A.T[q * A.S], 0x80808080u);
      B += kWin8;
      G.sync();
    } else if (!LEAN && CT && t - B >= kWin) {  // slide the ready-time window (t - B <= 2 kWin - 2 here)
      for (uint32_t q = G.lane; q < (n + 1) / 2; q += LG) A.T[q * A.S] = x_slide2(A.T[q * A.S]);
      B += kWin;
      G.sync();
    }
    if (prune && ((++turn & 7u) == 0u)) {  // R24: winner-invariant prune
      uint32_t bl = 0;
      if (G.leader()) bl = *(volatile uint32_t *)prune_len;
      bl = G.bcast(bl);
      uint32_t lbf = mi ? t + (n - placed + used + w - 1) / w : t + (n - placed);
      if (pcp) lbf = ::max(lbf, G.max(cp_run) + 1u);
      if (lbf > bl) {
        if (G.leader()) atomicAdd(prune_len + 1, 1u);  // RegionState::pruned follows prune_len
        o.cost = kInvalid;
        return o;
      }
    }
    const uint32_t step = mi ? t * w + used : t;  // Philox step (R26, R42)
    // free issue slots per type this cycle (0xFF per byte = free), R42
    const uint32_t avail = mi ? (used < w ? __vcmpltu4(used_t, slots) : 0u) : 0xFFFFFFFFu;
    // slack_c = target_c - live_c, saturated to a byte (R21); live <= target always
    uint32_t slack = 0;
    {
      const uint32_t lv[4] = {live01 & 0xFFFFu, live01 >> 16, live23 & 0xFFFFu, live23 >> 16};
#pragma unroll
      for (int c = 0; c < 4; ++c) slack |= ::min(tgt[c] - lv[c], 255u) << (8 * c);
    }
    const uint32_t slack2 = lo_pair(slack);  // classes 0, 1 as u16 x 2 (<= 2 classes: !NC4)
    const uint16_t *trow = tau + prev * n;
    uint32_t counts = 0, min_s = 0xFFFFFFFFu;  // counts = |R| | |F| << 16
    bool f_not_inc = false, s_dec = false, any_s = false;
    uint32_t bs1 = 0, bj = 0;  // lane-local best score + 1 (0 = none) and its index
    unsigned long long sum = 0;
    // the roulette sum is needed unless this step's group coin is a known exploit
    const bool need_sum = !(step < coin_t && ((coins[step >> 5] >> (step & 31u)) & 1u));
    auto eval = [&](uint32_t j, uint32_t rdy, const uint4 &ds, uint32_t dk, uint32_t tv) {
      const uint32_t K = ds.y + dk;                   // kills per class (R14)
      const bool lat_ok = rdy <= t;
      if (pcp) cp_run = ::max(cp_run, ::max(rdy, t) + cp_floor(ds.z));
      if (lat_ok && (!mi || ((avail >> (8 * (ds.w & 0xFu))) & 1u))) {
        counts += 1u;
        // feasible: defs_c <= slack_c + kills_c in every class (R21)
        const bool feas = NC4 ? __vcmpgtu4(ds.x, __vaddus4(slack, K)) == 0u
                              : all_le2(lo_pair(ds.x), slack2 + lo_pair(K));
        if (feas) {
          const uint32_t s = tv * eta_of(j, ds.z & 0xFFFFu, dk);
          counts += 1u << 16;
          // max_c Delta_c <= 0
          f_not_inc |= NC4 ? __vcmpgtu4(ds.x, K) == 0u : all_le2(lo_pair(ds.x), lo_pair(K));
          if (s + 1u > bs1) {  // ascending: strict keeps the lowest index (R1, R25)
            bs1 = s + 1u;
            bj = j;
          }
          if (need_sum) sum += s;
        }
      } else {
        any_s = true;
        min_s = ::min(min_s, lat_ok ? t + 1u : rdy);        // slot-blocked: next cycle (R42)
        // min_c Delta_c < 0
        s_dec |= NC4 ? __vcmpltu4(ds.x, K) != 0u : any_lt2(lo_pair(ds.x), lo_pair(K));
      }
    };
    if constexpr (wide) {
      scan4_any<MASK>(A, wmask & sub, G.lane, LG, nwr, [&](const uint32_t(&j)[4], const bool(&v)[4]) {
        uint32_t rd[4], dk[4], tv[4];
        uint4 ds[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) {
          rd_dk(j[u], rd[u], dk[u]);
          ds[u] = V.ds[j[u]];                         // defs, static kills, eta2 | slot, type
          tv[u] = trow[j[u]];
        }
        if constexpr (LEAN) {
#pragma unroll
          for (int u = 0; u < 4; ++u) rd[u] = lean_rd(ds[u].z);
          if (lazy) {
            // kills decide nothing for a candidate of an ant that may not stall
            // (nor mixes heuristics) unless it is latency-ready and some class
            // has more defs than slack: its K is skipped (dk = 0; exact)
            uint32_t dsw[4];
#pragma unroll
            for (int u = 0; u < 4; ++u)
              dsw[u] = (v[u] && rd[u] <= t && !all_le2(lo_pair(ds[u].x), slack2)) ? ds[u].w : (ds[u].w & ~0xF0u);
            dyn_kills4w(V, A, dsw, dk);
          } else {
            dyn_kills4(V, A, ds, dk);
          }
        }
#pragma unroll
        for (int u = 0; u < 4; ++u)
          if (v[u]) eval(j[u], rd[u], ds[u], dk[u], tv[u]);
      });
    } else {
      scan_bits<MASK>(A, nwr, wmask, G.lane, LG, sub, [&](uint32_t j) {
        uint32_t rd, dk;
        rd_dk(j, rd, dk);
        const uint4 ds = V.ds[j];
        if (LEAN) {
          rd = lean_rd(ds.z);
          dk = dyn_kills(V, A, ds.w);
        }
        eval(j, rd, ds, dk, trow[j]);
        return false;
      });
    }
    counts = G.sum(counts);
    min_s = G.min(min_s);
    if (need_sum) sum = G.sum64(sum);
    any_s = G.any(any_s);
    const bool all_f_inc = !G.any(f_not_inc);
    const bool some_s_dec = G.any(s_dec);
    const uint32_t nr = counts & 0xFFFFu, nf = counts >> 16;
    if (nr == 0) {  // necessary stall (L153): skip ahead to the next ready time
      t = min_s;
      used = used_t = 0;
      continue;
    }
    if (nf == 0) {
      if (stall_en && any_s) {  // forced optional stall (L155, R22)
        kopt += min_s - t;
        t = min_s;
        used = used_t = 0;
        continue;
      }
      o.cost = kInvalid;  // the ant is terminated (L149)
      return o;
    }
    uint4 x = make_uint4(0, 0, 0, 0);
    bool have_x = false;
    if (stall_en && any_s && all_f_inc && some_s_dec) {  // discretionary stall (L157-L164)
      x = philox(step, ant, c2, V.region_id, cfg.seed);
      have_x = true;
      const uint32_t thr = (kopt + 1 >= 32) ? 0u : (0xFFFFFFFFu >> (kopt + 1));
      if (x.z < thr) {
        ++kopt;
        ++t;
        used = used_t = 0;
        continue;
      }
    }
    bool exploit;
    if (step < coin_t) {  // the block's precomputed group coins (R3)
      exploit = (coins[step >> 5] >> (step & 31u)) & 1u;
    } else {
      const uint4 g = philox(step, 0x80000000u | group, c2, V.region_id, cfg.seed);
      exploit = (uint64_t)g.x < cfg.q0_t;
    }
    uint32_t jstar = bj;
    if (LG > 1) jstar = 0xFFFFFFFFu - (uint32_t)G.max64(bs1 ? akey(bs1 - 1u, bj) : 0ull);
    if (!exploit) {  // explore: roulette over F (R27), leader in ascending order
      if (G.leader()) {
        if (!have_x) x = philox(step, ant, c2, V.region_id, cfg.seed);
        const uint64_t r = __umul64hi(((uint64_t)x.y << 32) | x.x, sum);
        uint64_t pre = 0;
        scan_bits<MASK>(A, nwr, wmask, 0, 1, 0xFFFFFFFFu, [&](uint32_t j) {
          uint32_t rd, dk;
          rd_dk(j, rd, dk);
          const uint4 ds = V.ds[j];
          if (LEAN) rd = lean_rd(ds.z);
          if (rd > t) return false;
          if (LEAN) dk = dyn_kills(V, A, ds.w);
          if (mi && !((avail >> (8 * (ds.w & 0xFu))) & 1u)) return false;
          if (NC4 ? __vcmpgtu4(ds.x, __vaddus4(slack, ds.y + dk)) != 0u
                  : !all_le2(lo_pair(ds.x), slack2 + lo_pair(ds.y + dk)))
            return false;
          pre += (uint32_t)trow[j] * eta_of(j, ds.z & 0xFFFFu, dk);
          if (pre > r) {
            jstar = j;
            return true;
          }
          return false;
        });
      }
      jstar = G.bcast(jstar);
    }
    if (G.leader()) {
      commit<2, MASK, T32, NC4, LEAN>(V, A, jstar, t, wmask, live01, live23, prp01, prp23, B);
      if (rec_o) {
        rec_o[(size_t)placed * rec_stride] = (uint16_t)jstar;
        rec_c[(size_t)placed * rec_stride] = t;
      }
    }
    wmask = G.bcast(wmask);
    live01 = G.bcast(live01);
    live23 = G.bcast(live23);
    G.sync();
    ++placed;
    prev = jstar;
    if (pf) tau_row_prefetch<LG>(tau, prev, n, G);
    if (mi) {  // R42: the cycle is complete after issue_width placements
      ++used;
      used_t += 1u << (8 * (V.ds[jstar].w & 0xFu));
      if (used == w) {
        ++t;
        used = used_t = 0;
      }
    } else {
      ++t;
    }
  }
  const uint32_t len = t + (used ? 1u : 0u);  // last issue cycle + 1 (R20)
  if (prune && G.leader()) atomicMin(prune_len, len);
  o.prp01 = prp01;
  o.prp23 = prp23;
  o.len = len;
  o.cost = len;
  if (cfg.weighted && G.leader()) o.cost = len + cfg.ws_weight * cost_of(cfg.mslot, cfg.cost_mode, prp01, prp23);  // R41
  return o;
}

// ------------------------------------------------- lane-per-instruction ants
// Latency-bound batches (few ants in total, config 2: one region of 1,024
// ants leaves ~1 warp per SM): ONE WARP PER ANT, lane l owns instructions
// j = 32 q + l (q < Q, n <= 32 Q).  The ant's mutable state lives in
// registers -- ready bits, counts of unplaced predecessors, dynamic last-use
// counts per class (R14), pass-2 ready times; the scheduled set is a
// warp-uniform bitset -- so a step evaluates every candidate at once (one
// lane each), selects with warp reductions (redux.sync max / min; the
// roulette's ascending prefix with a shuffle scan) and commits with
// warp-uniform control flow in which the owner lanes update their registers.
// Only the remaining-use counters of >= 3-user registers stay in shared
// memory.  The per-ant step chain drops from ~600 dependent warp
// instructions (one ant per lane group, state in shared memory) to ~100.
// Same decisions in the same order with the same arithmetic and Philox
// counters as ant_pass1 / ant_pass2 (R1-R27): bit-exact with them and the
// oracle.  Single issue, <= 2 register classes, no R43 / R45 (host planner).
constexpr uint32_t kFull = 0xFFFFFFFFu;

// The lanes of one ant: WL = 32 (a warp, k_construct) or 8 / 16 (a fused
// single-block run of a small region, k_fused): lane l of the group owns
// instructions j = WL q + l; mask = the group's lanes for the .sync
// collectives (redux / ballot / shuffle with width WL).
template <int WL>
struct LpiGrp {
  uint32_t lane, base, mask;
  __device__ __forceinline__ LpiGrp() {
    const uint32_t l = threadIdx.x & 31u;
    lane = l & (WL - 1);
    base = l - lane;
    mask = WL == 32 ? kFull : (((1u << WL) - 1u) << base);
  }
  __device__ __forceinline__ uint32_t ballot(bool p) const {  // the group's bits, lane 0 = bit 0
    return WL == 32 ? __ballot_sync(kFull, p) : (__ballot_sync(mask, p) >> base) & ((1u << WL) - 1u);
  }
};

// The mutable per-lane state is packed into scalars (no register arrays
// updated under a runtime index: nvcc would move those to local memory).
struct LpiAnt {
  uint32_t rdy;             // bit q: j_q is in the ready set RB (predecessors placed, not scheduled)
  uint32_t npl;             // u8 x 4: predecessors of j_q not yet placed (n <= 128: in-degree < 255)
  uint32_t dkA, dkB;        // dynamic last-use counts (R14), u8 per class (2 classes): j_0, j_1 | j_2, j_3
  uint32_t rtA, rtB;        // pass 2: ready times u16 x 2 (max over placed predecessors of t_p + latency)
  uint32_t s0, s1, s2, s3;  // scheduled set, words 0-3 (warp-uniform)
};
__device__ __forceinline__ uint32_t lpi_sch(const LpiAnt &X, uint32_t w) {
  return w == 0 ? X.s0 : (w == 1 ? X.s1 : (w == 2 ? X.s2 : X.s3));
}
// (q is a constant after unrolling)
__device__ __forceinline__ uint32_t lpi_dk(const LpiAnt &X, uint32_t q) {  // u8 x 4 per class (classes 0, 1)
  return ((q < 2 ? X.dkA : X.dkB) >> (16 * (q & 1))) & 0xFFFFu;
}
__device__ __forceinline__ uint32_t lpi_rt(const LpiAnt &X, uint32_t q) {
  return ((q < 2 ? X.rtA : X.rtB) >> (16 * (q & 1))) & 0xFFFFu;
}

template <int WL, int Q>
__device__ __forceinline__ void lpi_init(const SV &V, uint32_t *rem, uint32_t S, const LpiGrp<WL> &G, LpiAnt &X) {
  for (uint32_t w = G.lane; w < V.nremw; w += WL) rem[w * S] = V.rem0[w];
  X.rdy = 0;
  X.npl = 0xFFFFFFFFu;  // (lanes past n never become ready)
  X.dkA = X.dkB = X.rtA = X.rtB = 0;
  X.s0 = X.s1 = X.s2 = X.s3 = 0;
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const uint32_t j = (uint32_t)WL * q + G.lane;
    if (j < V.n) {
      uint32_t c = 0;
      for (uint32_t k = V.pg_ptr[j]; k < V.pg_ptr[j + 1]; ++k) c += __popc(V.pg[k].y);
      if (!c) X.rdy |= 1u << q;
      X.npl = (X.npl & ~(0xFFu << (8 * q))) | (c << (8 * q));
    }
  }
  __syncwarp(G.mask);
}

// Commit of instruction j at cycle t (the warp-uniform counterpart of
// commit()): scheduled / ready sets, RP update (R14, R15), last-use
// bookkeeping of the registers j reads (the new last user's owner lane bumps
// its count; dirty: its q bits), successors' readiness and (pass 2) ready times.
template <int PASS, int WL, int Q>
__device__ __forceinline__ void lpi_commit(const SV &V, uint32_t *rem, uint32_t S, const LpiGrp<WL> &G, LpiAnt &X,
                                           uint32_t j, uint32_t t, uint32_t &live01, uint32_t &live23,
                                           uint32_t &prp01, uint32_t &prp23, uint32_t &dirty) {
  const uint32_t qj = j >> 5, bj = 1u << (j & 31u);  // (the scheduled set's word and bit)
  X.s0 |= qj == 0 ? bj : 0u;
  if (Q > 1) X.s1 |= qj == 1 ? bj : 0u;
  if (Q > 2) {
    X.s2 |= qj == 2 ? bj : 0u;
    X.s3 |= qj == 3 ? bj : 0u;
  }
  if (G.lane == j % WL) X.rdy &= ~(1u << (j / WL));
  const uint4 inf = V.info[j];
  uint32_t K = inf.y;  // static kills (single-use registers)
  const uint32_t m0 = inf.w >> 8, mc = inf.w & 0xFFu;
  for (uint32_t q = 0; q < mc; ++q) {
    const uint32_t e = V.muse[m0 + q];
    const uint32_t c = (e >> 16) & 3u;
    uint32_t u = kInvalid;  // the instruction that becomes the register's last user
    if (e & kMuseCounter) {  // >= 3 users: remaining-use counter
      const uint32_t m = e & 0xFFFFu, sh = (m & 1u) * 16;
      uint32_t *p = rem + (m >> 1) * S;
      const uint32_t w = *p;
      const uint32_t left = (w >> sh) & 0xFFFFu;  // users left including j
      __syncwarp(G.mask);
      if (G.lane == 0) *p = w - (1u << sh);
      __syncwarp(G.mask);
      if (left == 1u) {
        K += 1u << (8 * c);
      } else if (left == 2u) {  // the first unscheduled user (in the list's order) remains
        const uint32_t k0 = V.cu_ptr[m], k1 = V.cu_ptr[m + 1];
        for (uint32_t b = k0; b < k1; b += WL) {
          const uint32_t kk = b + G.lane;
          const uint32_t x = kk < k1 ? V.cu[kk] : 0u;
          const bool un = kk < k1 && !((lpi_sch(X, x >> 5) >> (x & 31u)) & 1u);
          const uint32_t bal = G.ballot(un);
          if (bal) {
            u = __shfl_sync(G.mask, x, __ffs(bal) - 1, WL);
            break;
          }
        }
      }
    } else {  // 2 users: the partner
      const uint32_t pa = e & 0x1FFFu;
      if ((lpi_sch(X, pa >> 5) >> (pa & 31u)) & 1u) K += 1u << (8 * c);
      else u = pa;
    }
    if (u != kInvalid && G.lane == u % WL) {
      const uint32_t qu = u / WL, bump = 1u << (8 * c + 16 * (qu & 1u));
      if (qu < 2) X.dkA += bump;
      else X.dkB += bump;
      dirty |= 1u << qu;
    }
  }
  live01 = __vsub2(live01, lo_pair(K));
  live23 = __vsub2(live23, hi_pair(K));
  live01 = __vadd2(live01, lo_pair(inf.x));
  live23 = __vadd2(live23, hi_pair(inf.x));
  prp01 = __vmaxu2(prp01, live01);
  prp23 = __vmaxu2(prp23, live23);
  live01 = __vsub2(live01, lo_pair(inf.z));
  live23 = __vsub2(live23, hi_pair(inf.z));
  const uint32_t s0 = V.succ_ptr[j], s1 = V.succ_ptr[j + 1];
  for (uint32_t q = s0; q < s1; ++q) {
    const uint32_t e = V.succ[q];
    const uint32_t v = e & 0x1FFFu;
    if (G.lane == v % WL) {
      const uint32_t qv = v / WL;
      if (PASS == 2) {  // ready time = max over placed predecessors (t + latency < 2^16: host)
        const uint32_t r = (t + (e >> 16)) << (16 * (qv & 1u));
        if (qv < 2) X.rtA = __vmaxu2(X.rtA, r);
        else X.rtB = __vmaxu2(X.rtB, r);
      }
      X.npl -= 1u << (8 * qv);
      if (((X.npl >> (8 * qv)) & 0xFFu) == 0u) X.rdy |= 1u << qv;
    }
  }
}

// Roulette over the lanes' candidates (R27): the first candidate in
// ascending j = 32 q + lane whose inclusive prefix of scores exceeds
// r = floor(R64 * sum / 2^64).  Scores are scanned as 16-bit halves (no
// carries within a 32-lane chunk).  Returns kInvalid if none exceeds r.
template <int WL, int Q>
__device__ __forceinline__ uint32_t lpi_roulette(const uint32_t (&sc)[Q], uint32_t valid, const LpiGrp<WL> &G,
                                                 uint64_t r64) {
  uint32_t plo[Q], phi[Q];
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const uint32_t s = ((valid >> q) & 1u) ? sc[q] : 0u;
    plo[q] = s & 0xFFFFu;
    phi[q] = s >> 16;
  }
#pragma unroll
  for (int o = 1; o < WL; o <<= 1) {
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const uint32_t a = __shfl_up_sync(G.mask, plo[q], o, WL), b = __shfl_up_sync(G.mask, phi[q], o, WL);
      if (G.lane >= (uint32_t)o) {
        plo[q] += a;
        phi[q] += b;
      }
    }
  }
  uint64_t pre[Q], base = 0;
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    pre[q] = base + ((uint64_t)phi[q] << 16) + plo[q];
    base += ((uint64_t)__shfl_sync(G.mask, phi[q], WL - 1, WL) << 16) + __shfl_sync(G.mask, plo[q], WL - 1, WL);
  }
  const uint64_t r = __umul64hi(r64, base);
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const uint32_t b = G.ballot(((valid >> q) & 1u) && pre[q] > r);
    if (b) return (uint32_t)WL * q + (__ffs(b) - 1);
  }
  return kInvalid;
}

// Warp argmax over (key desc, j asc): key = score + 1 of a candidate, 0 = none.
template <int WL, int Q>
__device__ __forceinline__ uint32_t lpi_argmax(const uint32_t (&key)[Q], const LpiGrp<WL> &G) {
  uint32_t bk = 0, bq = 0;
#pragma unroll
  for (int q = 0; q < Q; ++q)
    if (key[q] > bk) {  // ascending q: strict keeps the lane's lowest j
      bk = key[q];
      bq = q;
    }
  const uint32_t mx = __reduce_max_sync(G.mask, bk);
  return __reduce_min_sync(G.mask, (bk == mx && mx) ? (uint32_t)WL * bq + G.lane : kInvalid);
}

// RP pass, one ant per warp (as ant_pass1: R1, R4, R19, R25-R27).
template <int WL, int Q>
__device__ __forceinline__ AntOut lpi_pass1(const SV &V, const uint16_t *__restrict__ tau, uint32_t *rem, uint32_t S,
                                            const uint32_t ant, const uint32_t iter, const RunCfg &cfg, uint16_t *rec,
                                            const uint32_t *coins, const uint32_t rec_stride) {
  const LpiGrp<WL> G;
  const uint32_t n = V.n, L1 = V.L1;
  LpiAnt X;
  lpi_init<WL, Q>(V, rem, S, G, X);
  uint32_t e1[Q];  // eta1(j, sk(j) + d(j)) at the current d (R4)
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const uint32_t j = ::min((uint32_t)WL * q + G.lane, n - 1);
    e1[q] = V.eta1[j * L1];
  }
  uint32_t live01 = V.livein01, live23 = V.livein23, prp01 = live01, prp23 = live23;
  uint32_t prev = n;
  for (uint32_t k = 0; k < n; ++k) {
    const bool exploit = (coins[k >> 5] >> (k & 31u)) & 1u;  // group coin (R3)
    const uint16_t *trow = tau + prev * n;
    uint32_t sc[Q], key[Q];
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const uint32_t j = ::min((uint32_t)WL * q + G.lane, n - 1);
      sc[q] = (uint32_t)trow[j] * e1[q];
      key[q] = ((X.rdy >> q) & 1u) ? sc[q] + 1u : 0u;
    }
    uint32_t jstar = lpi_argmax<WL, Q>(key, G);
    if (!exploit) {
      const uint4 x = philox(k, ant, iter, V.region_id, cfg.seed);
      const uint32_t jr = lpi_roulette<WL, Q>(sc, X.rdy, G, ((uint64_t)x.y << 32) | x.x);
      if (jr != kInvalid) jstar = jr;
    }
    uint32_t dirty = 0;
    lpi_commit<1, WL, Q>(V, rem, S, G, X, jstar, 0, live01, live23, prp01, prp23, dirty);
    if (dirty) {
#pragma unroll
      for (int q = 0; q < Q; ++q)
        if ((dirty >> q) & 1u) e1[q] = V.eta1[((uint32_t)WL * q + G.lane) * L1 + sum_u8x4(lpi_dk(X, q))];
    }
    if (rec && G.lane == 0) rec[(size_t)k * rec_stride] = (uint16_t)jstar;
    prev = jstar;
  }
  AntOut o;
  o.prp01 = prp01;
  o.prp23 = prp23;
  o.len = 0;
  o.cost = cost_of(cfg.mslot, cfg.cost_mode, prp01, prp23);
  return o;
}

// ILP pass, one ant per warp (as ant_pass2 on the single-issue machine:
// R19-R24, R41; stalls, the RP-feasible set, the prune).
template <int WL, int Q>
__device__ __forceinline__ AntOut lpi_pass2(const SV &V, const uint16_t *__restrict__ tau, uint32_t *rem, uint32_t S,
                                            const uint32_t ant, const uint32_t iter, const RunCfg &cfg,
                                            const uint32_t tgt[4], uint32_t *prune_len, const bool prune,
                                            uint16_t *rec_o, uint32_t *rec_c, const uint32_t *coins,
                                            const uint32_t coin_t, const uint32_t rec_stride) {
  const LpiGrp<WL> G;
  const uint32_t n = V.n;
  LpiAnt X;
  lpi_init<WL, Q>(V, rem, S, G, X);
  uint32_t dx2[Q], dy[Q], e2[Q], K2[Q];  // defs (u16 x 2), static kills (u8 x 4), eta2, kills (u16 x 2)
  uint32_t fnim = 0, sdm = 0;  // bit q: max_c Delta_c <= 0 / min_c Delta_c < 0 for j_q (change only with its kills)
  auto kill_tests = [&](int q) {
    K2[q] = lo_pair(dy[q] + lpi_dk(X, q));  // kills per class (R14)
    fnim = (fnim & ~(1u << q)) | ((all_le2(dx2[q], K2[q]) ? 1u : 0u) << q);
    sdm = (sdm & ~(1u << q)) | ((any_lt2(dx2[q], K2[q]) ? 1u : 0u) << q);
  };
#pragma unroll
  for (int q = 0; q < Q; ++q) {
    const uint4 ds = V.ds[::min((uint32_t)WL * q + G.lane, n - 1)];
    dx2[q] = lo_pair(ds.x);
    dy[q] = ds.y;
    e2[q] = ds.z & 0xFFFFu;
    kill_tests(q);
  }
  uint32_t live01 = V.livein01, live23 = V.livein23, prp01 = live01, prp23 = live23;
  const uint32_t group = ant / cfg.group_size;
  const bool stall_en = stall_group(cfg, group);  // R23, R44
  const uint32_t c2 = 0x80000000u | iter;
  uint32_t t = 0, placed = 0, kopt = 0, prev = n, turn = 0;
  AntOut o;
  o.prp01 = o.prp23 = 0;
  o.len = kInvalid;
  while (placed < n) {
    if (prune && ((++turn & 7u) == 0u)) {  // R24: winner-invariant prune
      uint32_t bl = 0;
      if (G.lane == 0) bl = *(volatile uint32_t *)prune_len;
      bl = __shfl_sync(G.mask, bl, 0, WL);
      if (t + (n - placed) > bl) {
        if (G.lane == 0) atomicAdd(prune_len + 1, 1u);
        o.cost = kInvalid;
        return o;
      }
    }
    // slack_c = target_c - live_c saturated to a byte (R21), classes 0 and 1 as u16 x 2
    const uint32_t slack2 = ::min(tgt[0] - (live01 & 0xFFFFu), 255u) | (::min(tgt[1] - (live01 >> 16), 255u) << 16);
    const uint16_t *trow = tau + prev * n;
    uint32_t sc[Q], key[Q], lat = 0, feas = 0, semi = 0, mins = kInvalid;
#pragma unroll
    for (int q = 0; q < Q; ++q) {
      const bool inr = (X.rdy >> q) & 1u;
      const uint32_t rtq = lpi_rt(X, q);
      const bool l = inr && rtq <= t;
      const bool s = inr && rtq > t;
      const bool f = l && all_le2(dx2[q], slack2 + K2[q]);  // defs_c <= slack_c + kills_c (R21)
      sc[q] = (uint32_t)trow[::min((uint32_t)WL * q + G.lane, n - 1)] * e2[q];
      key[q] = f ? sc[q] + 1u : 0u;
      if (s) mins = ::min(mins, rtq);
      lat |= (uint32_t)l << q;
      feas |= (uint32_t)f << q;
      semi |= (uint32_t)s << q;
    }
    const bool fni = (feas & fnim) != 0u;   // a feasible candidate with max_c Delta_c <= 0
    const bool sdec = (semi & sdm) != 0u;   // a semi-ready one with min_c Delta_c < 0
    const uint32_t min_s = __reduce_min_sync(G.mask, mins);
    if (!__any_sync(G.mask, lat != 0u)) {  // necessary stall (L153): skip to the next ready time
      t = min_s;
      continue;
    }
    const bool any_s = __any_sync(G.mask, semi != 0u);
    if (!__any_sync(G.mask, feas != 0u)) {
      if (stall_en && any_s) {  // forced optional stall (L155, R22)
        kopt += min_s - t;
        t = min_s;
        continue;
      }
      o.cost = kInvalid;  // the ant is terminated (L149)
      return o;
    }
    uint4 x = make_uint4(0, 0, 0, 0);
    bool have_x = false;
    if (stall_en && any_s && !__any_sync(G.mask, fni) && __any_sync(G.mask, sdec)) {  // discretionary (L157-L164)
      x = philox(t, ant, c2, V.region_id, cfg.seed);
      have_x = true;
      const uint32_t thr = (kopt + 1 >= 32) ? 0u : (0xFFFFFFFFu >> (kopt + 1));
      if (x.z < thr) {
        ++kopt;
        ++t;
        continue;
      }
    }
    bool exploit;
    if (t < coin_t) {
      exploit = (coins[t >> 5] >> (t & 31u)) & 1u;
    } else {
      const uint4 g = philox(t, 0x80000000u | group, c2, V.region_id, cfg.seed);
      exploit = (uint64_t)g.x < cfg.q0_t;
    }
    uint32_t jstar = lpi_argmax<WL, Q>(key, G);
    if (!exploit) {
      if (!have_x) x = philox(t, ant, c2, V.region_id, cfg.seed);
      const uint32_t jr = lpi_roulette<WL, Q>(sc, feas, G, ((uint64_t)x.y << 32) | x.x);
      if (jr != kInvalid) jstar = jr;
    }
    uint32_t dirty = 0;
    lpi_commit<2, WL, Q>(V, rem, S, G, X, jstar, t, live01, live23, prp01, prp23, dirty);
    if (dirty) {
#pragma unroll
      for (int q = 0; q < Q; ++q)
        if ((dirty >> q) & 1u) kill_tests(q);
    }
    if (rec_o && G.lane == 0) {
      rec_o[(size_t)placed * rec_stride] = (uint16_t)jstar;
      rec_c[(size_t)placed * rec_stride] = t;
    }
    ++placed;
    prev = jstar;
    ++t;
  }
  if (prune && G.lane == 0) atomicMin(prune_len, t);
  o.prp01 = prp01;
  o.prp23 = prp23;
  o.len = t;
  o.cost = t;
  if (cfg.weighted) o.cost = t + cfg.ws_weight * cost_of(cfg.mslot, cfg.cost_mode, prp01, prp23);  // R41
  return o;
}

// ------------------------------------------------------------ kernels
struct KArgs {
  const unsigned char *arena;
  unsigned char *ws;
  const RegionDev *regions;
  RegionState *state;
  const RegionWs *rws;
  uint32_t *dump_cost;
  uint16_t *dump_order;
  uint32_t *dump_cycle;
  RunCfg cfg;
};

// Stage the region's block image (and tau) into shared memory.
__device__ __forceinline__ void stage(uint4 *dst, const uint4 *src, uint32_t bytes) {
  for (uint32_t i = threadIdx.x; i < bytes / 16; i += blockDim.x) dst[i] = src[i];
}
// ... by one warp (the select body, also run by warp 0 of k_finalize1's block)
__device__ __forceinline__ void stage_warp(uint4 *dst, const uint4 *src, uint32_t bytes) {
  for (uint32_t i = threadIdx.x & 31u; i < bytes / 16; i += 32) dst[i] = src[i];
}

// Bulk-async staging (sm_90+ bulk-copy / TMA engine, cp.async.bulk with an
// mbarrier transaction count).  Sources, destinations and sizes are 16-byte
// aligned multiples (block images and tau tables are padded to 16 bytes).
constexpr uint32_t kBulkChunk = 32768;
__device__ __forceinline__ void bulk_arm(uint32_t mbar, uint32_t bytes) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(mbar) : "memory");
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(mbar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_copy(void *dst, const void *src, uint32_t bytes, uint32_t mbar) {
  const uint32_t d = (uint32_t)__cvta_generic_to_shared(dst);
  for (uint32_t off = 0; off < bytes; off += kBulkChunk) {
    const uint32_t b = ::min(kBulkChunk, bytes - off);
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(d + off),
                 "l"((const char *)src + off), "r"(b), "r"(mbar)
                 : "memory");
  }
}
__device__ __forceinline__ void bulk_wait_inval(uint32_t mbar) {
  asm volatile(
      "{\n .reg .pred p;\n WAIT_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n @!p bra WAIT_%=;\n}" ::"r"(mbar)
      : "memory");
  asm volatile("mbarrier.inval.shared::cta.b64 [%0];" ::"r"(mbar) : "memory");
}

// Launch bounds: the 1-wide variants keep <= 64 registers (2 x 512 threads per
// SM); the 4-wide ones (large regions, few ants per SM by shared memory) may
// use up to 128.
// GS: 0 = image and per-ant state in shared memory; 1 = huge region, both
// through L1/L2 (state in the workspace); 2 = image read through L1 (it is
// small next to the state of large regions), per-ant state (and tau when
// staged) in shared memory: more ants resident per SM.
// LEAN: pass-2 lean per-ant layout (u8 ready times, dynamic kills).
template <int PASS, int LG, bool MASK, bool TAU_SMEM, bool T32, bool NC4, int GS, bool WIDE, bool LEAN = false>
#ifndef ACO_NARROW_MINB  // min blocks per SM of the 1-wide variants (2: <= 64 registers)
#define ACO_NARROW_MINB 2
#endif
#ifndef ACO_HUGE_MINB  // min blocks per SM of the huge shared-state variants (1: up to 128 registers)
#define ACO_HUGE_MINB 1
#endif
// (huge regions with shared-memory state, !MASK && GS == 2: two blocks per SM,
// every ant of config 4 resident)
// (LG == 32: lane-per-instruction ants, one warp each: latency-bound
// batches with few warps per SM, registers unconstrained)
__global__ void __launch_bounds__(LG == 32 ? kLpiMaxThreads : ((LEAN && MASK) ? kLeanMaxThreads : kMaxBlockThreads),
                                  LG == 32 ? 1 : ((WIDE && GS != 1) ? ((MASK || GS != 2) ? 1 : ACO_HUGE_MINB) : ACO_NARROW_MINB))
    k_construct(KArgs A, const BlockItem *__restrict__ items, uint32_t iter) {
  const BlockItem bi = items[blockIdx.x];
  RegionState &rs = A.state[bi.region];
  if (!rs.active) return;  // block-uniform
  const RegionDev *rd = A.regions + bi.region;
  const RegionWs &W = A.rws[bi.region];
  extern __shared__ uint4 smem4[];
  unsigned char *smem = (unsigned char *)smem4;
  const uint32_t local = threadIdx.x / LG;  // ant within the block
  const uint32_t ai = bi.ant0 + local;      // ant within this context's share of the region
  const uint32_t ant = A.cfg.ant_base + ai; // global ant id (Philox key, groups, winner key)
  const uint16_t *tau = (const uint16_t *)(A.ws + W.o_tau);
  const unsigned char *img = A.arena + rd->o_image;
  uint32_t *stbase;
  uint32_t stride;
  const uint32_t *coins = nullptr;
  uint32_t coin_t = 0;
  RL rl{nullptr, 0, 0, A.cfg.rl_limit, nullptr, nullptr};
  if (GS == 1) {  // huge region: statics through L1/L2, per-ant state in the workspace
    if (ai >= A.cfg.ants) return;
    if (A.cfg.gs_ant_major) {  // ant-major: the lanes of one ant read consecutive words (coalesced scan)
      const uint32_t wpa = (ant_words(PASS, rd->n, rd->nwr, rd->nremw, T32, NC4) + 3u) & ~3u;
      stbase = (uint32_t *)(A.ws + W.o_gstate) + (size_t)ai * wpa;
      stride = 1;
    } else {  // word-major [word][ant]
      stbase = (uint32_t *)(A.ws + W.o_gstate) + ai;
      stride = A.cfg.ants;
    }
  } else {
    const uint32_t img_bytes = GS == 0 ? rd->img.bytes : 0u;
    const uint32_t tb = TAU_SMEM ? tau_smem_bytes(rd->n) : 0u;
    uint32_t state_off = img_bytes + tb;
#if ACO_BULK_STAGE
    // image and tau by the bulk-copy (TMA) engine: thread 0 arms an mbarrier
    // (in the first per-ant state words, unused until the ants initialise
    // them) with the byte count and issues 1-D bulk copies; the block builds
    // its coin table meanwhile; thread 0 waits, then the block barrier
    const uint32_t mbar = (uint32_t)__cvta_generic_to_shared(smem + state_off);
    if (threadIdx.x == 0 && img_bytes + tb) {
      bulk_arm(mbar, img_bytes + tb);
      if (GS == 0) bulk_copy(smem, img, img_bytes, mbar);
      if (TAU_SMEM) bulk_copy(smem + img_bytes, A.ws + W.o_tau, tb, mbar);
    }
#else
    if (GS == 0) stage(smem4, (const uint4 *)img, img_bytes);
    if (TAU_SMEM) stage((uint4 *)(smem + img_bytes), (const uint4 *)(A.ws + W.o_tau), tb);
#endif
    if (TAU_SMEM) tau = (const uint16_t *)(smem + img_bytes);
    const uint32_t apb = blockDim.x / LG;
    stride = ant_stride(apb, LG);
    // Group coins (R3) of every (step, group) of this block, one warp per
    // 32 steps of a group (ballot), instead of one Philox per ant-step.
    {
      const uint32_t gsz = A.cfg.group_size, abase = A.cfg.ant_base + bi.ant0, g0 = abase / gsz;
      const uint32_t ng = (abase + apb - 1) / gsz - g0 + 1, cw = coin_words(PASS, rd->n);
      uint32_t *cz = (uint32_t *)(smem + state_off) +
                     stride * (LG == 32 ? lpi_words(rd->nremw)
                                        : ant_words(PASS, rd->n, rd->nwr, rd->nremw, T32, NC4, LEAN, rd->nslot));
      const uint32_t lane = threadIdx.x & 31u, c2 = PASS == 1 ? iter : (0x80000000u | iter);
      for (uint32_t task = threadIdx.x >> 5; task < ng * cw; task += blockDim.x >> 5) {
        const uint32_t gi = task / cw, k = (task - gi * cw) * 32 + lane;
        const uint4 x = philox(k, 0x80000000u | (g0 + gi), c2, rd->region_id, A.cfg.seed);
        const uint32_t word = __ballot_sync(0xFFFFFFFFu, (uint64_t)x.x < A.cfg.q0_t);
        if (lane == 0) cz[task] = word;
      }
      coins = cz + (ant / gsz - g0) * cw;
      coin_t = PASS == 1 ? 0xFFFFFFFFu : cw * 32;
      if (PASS == 1 && A.cfg.rl_limit) {  // R45: group min/max counters after the coin table
        rl.buf = cz + ng * cw;
        rl.gi = ant / gsz - g0;
        rl.ng = ng;
        for (uint32_t i = threadIdx.x; i < 3 * ng; i += blockDim.x) {
          rl.buf[2 * i] = 0xFFFFFFFFu;
          rl.buf[2 * i + 1] = 0u;
        }
        if (ai < A.cfg.ants && ai % gsz == 0) rl.out = (uint16_t *)(A.ws + W.o_rlk) + (size_t)(ai / gsz) * rd->n;
      }
    }
#if ACO_BULK_STAGE
    if (threadIdx.x == 0 && img_bytes + tb) bulk_wait_inval(mbar);
#endif
    __syncthreads();
    if (ai >= A.cfg.ants) {  // whole lane group
      if (PASS == 1 && rl.buf)  // the block's lockstep steps need every thread at the barrier (R45)
        for (uint32_t k = 0; k < rd->n; ++k) rl_barrier();
      return;
    }
    if (GS == 0) img = smem;
    stbase = (uint32_t *)(smem + state_off) + local;
  }
  const Grp<LG> G(threadIdx.x);
  const SV V = make_sv(img, rd);
  // tau rows read from global memory: prefetch the next step's row into L1
  const bool pf = !TAU_SMEM && (A.cfg.tau_prefetch & (1u << (PASS - 1 + (GS == 1 ? 2 : 0))));
  const bool dump = (A.cfg.flags & ACO_FLAG_DUMP) != 0;
  AntOut o;
  if constexpr (LG == 32) {  // lane-per-instruction ant (n <= 128): only its >= 3-user counters in stbase
    static_assert(MASK && !T32 && !NC4 && GS == 0 && !WIDE && !LEAN, "LPI variants");
    const uint32_t qn = (V.n + 31) / 32;
    if constexpr (PASS == 1) {
      uint16_t *rec = nullptr;
      uint32_t rs1 = 1;
      if (dump && A.dump_order) {
        rec = A.dump_order + (size_t)iter * A.cfg.dump_slice + W.o_dump + (size_t)ai * V.n;
      } else if (A.cfg.record) {
        rec = (uint16_t *)(A.ws + W.o_rec) + ai;
        rs1 = A.cfg.ants;
      }
      if (qn <= 1) o = lpi_pass1<32, 1>(V, tau, stbase, stride, ant, iter, A.cfg, rec, coins, rs1);
      else if (qn <= 2) o = lpi_pass1<32, 2>(V, tau, stbase, stride, ant, iter, A.cfg, rec, coins, rs1);
      else o = lpi_pass1<32, 4>(V, tau, stbase, stride, ant, iter, A.cfg, rec, coins, rs1);
    } else {
      uint32_t tgt[4];
#pragma unroll
      for (int c = 0; c < 4; ++c) tgt[c] = rs.target[c];
      const bool prune = !dump && !(A.cfg.flags & ACO_FLAG_NO_PRUNE) && !A.cfg.keys && !A.cfg.weighted;
      uint16_t *rec_o = nullptr;
      uint32_t *rec_c = nullptr;
      if (dump && A.dump_order && A.dump_cycle) {
        const size_t base =
            ((size_t)A.cfg.iterations + iter) * A.cfg.dump_slice + W.o_dump + (size_t)ai * V.n;
        rec_o = A.dump_order + base;
        rec_c = A.dump_cycle + base;
      }
      uint32_t rs2 = 1;
      if (!rec_o && A.cfg.record) {
        rec_o = (uint16_t *)(A.ws + W.o_rec) + ai;
        rec_c = (uint32_t *)(A.ws + W.o_recc) + ai;
        rs2 = A.cfg.ants;
      }
      if (qn <= 1)
        o = lpi_pass2<32, 1>(V, tau, stbase, stride, ant, iter, A.cfg, tgt, &rs.prune_len, prune, rec_o, rec_c, coins,
                         coin_t, rs2);
      else if (qn <= 2)
        o = lpi_pass2<32, 2>(V, tau, stbase, stride, ant, iter, A.cfg, tgt, &rs.prune_len, prune, rec_o, rec_c, coins,
                         coin_t, rs2);
      else
        o = lpi_pass2<32, 4>(V, tau, stbase, stride, ant, iter, A.cfg, tgt, &rs.prune_len, prune, rec_o, rec_c, coins,
                         coin_t, rs2);
    }
  } else if constexpr (PASS == 1) {
    const St S = make_st<PASS, T32, NC4, LEAN>(stbase, stride, V);
    uint16_t *rec = nullptr;
    uint32_t rs1 = 1;
    if (dump && A.dump_order) {
      rec = A.dump_order + (size_t)iter * A.cfg.dump_slice + W.o_dump + (size_t)ai * V.n;
    } else if (A.cfg.record) {
      rec = (uint16_t *)(A.ws + W.o_rec) + ai;
      rs1 = A.cfg.ants;
    }
    if (rl.buf)
      o = ant_pass1<LG, MASK, WIDE, true, LEAN>(V, tau, S, G, ant, iter, A.cfg, false, rec, coins, rl, rs1, pf);
    else
      o = ant_pass1<LG, MASK, WIDE, false, LEAN>(V, tau, S, G, ant, iter, A.cfg, false, rec, coins, rl, rs1, pf);
  } else {
    const St S = make_st<PASS, T32, NC4, LEAN>(stbase, stride, V);
    uint32_t tgt[4];
#pragma unroll
    for (int c = 0; c < 4; ++c) tgt[c] = rs.target[c];
    const bool prune = !dump && !(A.cfg.flags & ACO_FLAG_NO_PRUNE) && !A.cfg.keys && !A.cfg.weighted;
    uint16_t *rec_o = nullptr;
    uint32_t *rec_c = nullptr;
    if (dump && A.dump_order && A.dump_cycle) {
      const size_t base =
          ((size_t)A.cfg.iterations + iter) * A.cfg.dump_slice + W.o_dump + (size_t)ai * V.n;
      rec_o = A.dump_order + base;
      rec_c = A.dump_cycle + base;
    }
    uint32_t rs2 = 1;
    if (!rec_o && A.cfg.record) {
      rec_o = (uint16_t *)(A.ws + W.o_rec) + ai;
      rec_c = (uint32_t *)(A.ws + W.o_recc) + ai;
      rs2 = A.cfg.ants;
    }
    o = ant_pass2<LG, MASK, T32, NC4, WIDE, LEAN>(V, tau, S, G, ant, iter, A.cfg, tgt, &rs.prune_len, prune, rec_o,
                                      rec_c, coins, coin_t, rs2, pf);
  }
  if (G.leader()) {
    uint32_t *costs = (uint32_t *)(A.ws + W.o_cost);
    costs[ai] = o.cost;
    if (A.cfg.record) ((uint4 *)(A.ws + W.o_recp))[ai] = make_uint4(o.prp01, o.prp23, o.len, 0u);
    if (dump && A.dump_cost)
      A.dump_cost[(((size_t)(PASS - 1) * A.cfg.iterations + iter) * A.cfg.count + bi.region) * A.cfg.ants + ai] =
          o.cost;
  }
}

__device__ __forceinline__ uint64_t fnv_u32(uint64_t h, uint32_t v) {
#pragma unroll
  for (int b = 0; b < 4; ++b) {
    h ^= (v >> (8 * b)) & 0xFFu;
    h *= 0x100000001b3ull;
  }
  return h;
}

__device__ __forceinline__ uint32_t no_improve_limit(const RunCfg &cfg, uint32_t n) {
  if (cfg.stop_no_improve != 0xFFFFFFFFu) return cfg.stop_no_improve;
  return n < 50 ? 1u : (n < 100 ? 2u : 3u);  // L226
}

// Fill tau with tau0 (16-byte stores).
__device__ void tau_fill(uint16_t *tau, uint32_t len, uint32_t tau0) {
  uint4 *t4 = (uint4 *)tau;
  const uint32_t v = tau0 | (tau0 << 16);
  const uint4 q = make_uint4(v, v, v, v);
  for (uint32_t i = threadIdx.x; i < len / 8; i += blockDim.x) t4[i] = q;
}

// Evaporate + deposit + clamp (R6-R9) over all active regions' tables, 8
// entries per 16-byte access.  One block = kUpdVec vectors of one region;
// next[i] = the winner's successor of row i (0xFFFF: no deposit).
__device__ __forceinline__ void update_vecs(const KArgs &A, uint32_t region, uint32_t v0, uint32_t v1, uint32_t tid,
                                            uint32_t nthr) {
  const RegionDev *rd = A.regions + region;
  const RegionWs &W = A.rws[region];
  const uint32_t n = rd->n;
  const uint32_t total = (n + 1) * n;
  const uint16_t *next = (const uint16_t *)(A.ws + W.o_next);
  uint4 *t4 = (uint4 *)(A.ws + W.o_tau);
  const uint32_t vend = min(v1, W.tau_len / 8);
  const uint32_t rho = A.cfg.rho_q16, dl = A.cfg.delta, lo = A.cfg.tau_min, hi = A.cfg.tau_max;
  for (uint32_t v = v0 + tid; v < vend; v += nthr) {
    const uint4 q = t4[v];
    uint32_t w[4] = {q.x, q.y, q.z, q.w};
    const uint32_t e0 = v * 8;
    uint32_t i = e0 / n, j = e0 - i * n;
    uint32_t nx = i <= n ? next[i] : 0xFFFFu;
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      if (e0 + u < total) {
        const uint32_t sh = (u & 1) * 16;
        uint32_t x = (w[u >> 1] >> sh) & 0xFFFFu;
        x = (x * rho) >> 16;
        if (nx == j) x += dl;
        x = min(max(x, lo), hi);
        w[u >> 1] = (w[u >> 1] & ~(0xFFFFu << sh)) | (x << sh);
        if (++j == n) {
          j = 0;
          ++i;
          nx = i <= n ? next[i] : 0xFFFFu;
        }
      }
    }
    t4[v] = make_uint4(w[0], w[1], w[2], w[3]);
  }
}
__global__ void __launch_bounds__(256) k_update(KArgs A, const UpdItem *__restrict__ items) {
  const UpdItem it = items[blockIdx.x];
  if (!A.state[it.region].active) return;  // the pass ended: tau is not used again
  update_vecs(A, it.region, it.v0, it.v0 + kUpdVec, threadIdx.x, blockDim.x);
}

// Per-region initialisation: tau0, the greedy pass-1 heuristic schedule
// (R28: the q0 = 1 ant on a uniform tau), LB check (L251).
// The greedy heuristic schedule (warp 0 as one 32-lane group, scratch state
// stw) and the region state at the start of a run.  tau is uniform (tau0).
template <bool MASK>
__device__ __forceinline__ void init_greedy(const KArgs &A, const RegionDev *rd, const RegionWs &W, RegionState &rs,
                                            const unsigned char *img, const uint16_t *tau, uint32_t *stw) {
  if (threadIdx.x >= 32) return;
  const SV V = make_sv(img, rd);
  const St S = make_st<1, false, false>(stw, 1, V);
  uint16_t *gb1 = (uint16_t *)(A.ws + W.o_gb1);
  const Grp<32> G32(threadIdx.x);
  AntOut o = ant_pass1<32, MASK>(V, tau, S, G32, 0, 0, A.cfg, true, gb1);
  __syncwarp();
  uint16_t *heur = (uint16_t *)(A.ws + W.o_heur);  // the heuristic order, kept for R40
  for (uint32_t k = threadIdx.x; k < rd->n; k += 32) heur[k] = gb1[k];
  if (threadIdx.x == 0) {
    rs.lb_cost = cost_rp(A.cfg.mslot, A.cfg.cost_mode, rd->lbvec[0], rd->lbvec[1], rd->lbvec[2], rd->lbvec[3]);
    rs.init[0] = rs.best[0] = o.cost;
    const uint32_t prp[4] = {o.prp01 & 0xFFFFu, o.prp01 >> 16, o.prp23 & 0xFFFFu, o.prp23 >> 16};
    for (int c = 0; c < 4; ++c) rs.prp1[c] = rs.prp2[c] = rs.heur_prp[c] = prp[c];
    rs.policy = 0;
    rs.heur_len = 0;
    rs.iters[0] = rs.iters[1] = 0;
    rs.no_imp = 0;
    rs.prune_len = kInvalid;
    rs.pruned = 0;
    rs.hash = 0xcbf29ce484222325ull;
    rs.active = (A.cfg.pass_mask & 1u) && A.cfg.iterations > 0 && !(A.cfg.stop_at_lb && o.cost == rs.lb_cost);
  }
}

// Per-region initialisation: tau0, the greedy pass-1 heuristic schedule
// (R28: the q0 = 1 ant on a uniform tau), LB check (L251).
template <bool MASK, bool GS>
__device__ __forceinline__ void init_body(const KArgs &A, unsigned char *smem) {
  const uint32_t r = blockIdx.x;
  const RegionDev *rd = A.regions + r;
  const RegionWs &W = A.rws[r];
  RegionState &rs = A.state[r];
  uint16_t *tau = (uint16_t *)(A.ws + W.o_tau);
  const unsigned char *img = A.arena + rd->o_image;
  uint32_t *stw = (uint32_t *)(A.ws + W.o_scratch);
  if (!GS) {
    stage((uint4 *)smem, (const uint4 *)img, rd->img.bytes);
    img = smem;
    stw = (uint32_t *)(smem + rd->img.bytes);
  }
  tau_fill(tau, W.tau_len, A.cfg.tau0);
  __syncthreads();
  init_greedy<MASK>(A, rd, W, rs, img, tau, stw);
}

template <bool MASK>
__global__ void __launch_bounds__(128) k_init(KArgs A) {
  extern __shared__ uint4 smem4[];
  if (A.rws[blockIdx.x].gs) init_body<false, true>(A, (unsigned char *)smem4);
  else if (A.regions[blockIdx.x].n <= 1024) init_body<true, false>(A, (unsigned char *)smem4);
  else init_body<false, false>(A, (unsigned char *)smem4);
  (void)MASK;
}

// ASAP timing of an order (R29) on the general machine model (R42): in-order
// issue, c_k = max(c_{k-1}, ready time), moved to c_{k-1} + 1 when cycle
// c_{k-1} has no free slot (width or the instruction's type).  One thread;
// rdyv[n] is zeroed scratch.  Returns the length.
__device__ uint32_t asap_order(const MachineDev &M, const SV &V, const uint16_t *order, uint16_t *out_o,
                               uint32_t *out_c, uint32_t *rdyv) {
  const uint32_t n = V.n, w = M.issue_width;
  uint32_t t = 0, used = 0, used_t = 0;
  for (uint32_t k = 0; k < n; ++k) {
    const uint32_t j = order[k], y = V.ds[j].w & 0xFu;
    uint32_t c = k == 0 ? rdyv[j] : max(t, rdyv[j]);
    if (k > 0 && c == t && (used >= w || ((used_t >> (8 * y)) & 0xFFu) >= ((M.type_slots >> (8 * y)) & 0xFFu)))
      c = t + 1;
    if (k == 0 || c != t) used = used_t = 0;
    t = c;
    ++used;
    used_t += 1u << (8 * y);
    if (out_o) out_o[k] = (uint16_t)j;
    if (out_c) out_c[k] = t;
    for (uint32_t q = V.succ_ptr[j]; q < V.succ_ptr[j + 1]; ++q) {
      const uint32_t e = V.succ[q];
      const uint32_t v = e & 0x1FFFu;
      rdyv[v] = max(rdyv[v], t + (e >> 16));
    }
  }
  return n ? t + 1 : 0;
}

// Pass transition (L147; R13, R18, R29): target from the pass-1 best, the
// initial pass-2 schedule = ASAP(pass-1 best order), tau reset, the cycle-gap
// filter (R39).  Weighted pass (R41): no target, weighted initial cost.
// (block-wide: every thread of the block calls it)
__device__ __forceinline__ void pass2_init_body(const KArgs &A, const RegionDev *rd, const RegionWs &W, RegionState &rs,
                                                const unsigned char *img, uint16_t *tau, uint32_t *rdyv) {
  const uint32_t n = rd->n;
  tau_fill(tau, W.tau_len, A.cfg.tau0);
  for (uint32_t i = threadIdx.x; i < n; i += blockDim.x) rdyv[i] = 0;
  __syncthreads();
  if (threadIdx.x == 0) {
    const SV V = make_sv(img, rd);
    const uint16_t *gb1 = (const uint16_t *)(A.ws + W.o_gb1);
    uint16_t *gb2 = (uint16_t *)(A.ws + W.o_gb2);
    uint32_t *gb2c = (uint32_t *)(A.ws + W.o_gb2c);
    const uint32_t len = asap_order(c_mach[A.cfg.mslot], V, gb1, gb2, gb2c, rdyv);
    for (int c = 0; c < 4; ++c) rs.prp2[c] = rs.prp1[c];
    rs.len2 = len;
    uint32_t tgt[4];
    uint32_t best = len, lb = rd->lb_len;
    if (A.cfg.weighted) {  // R41: cost = length + W * cost_rp, no RP target
      for (int c = 0; c < 4; ++c) tgt[c] = kInvalid;
      best = len + A.cfg.ws_weight * cost_rp(A.cfg.mslot, A.cfg.cost_mode, rs.prp1[0], rs.prp1[1], rs.prp1[2], rs.prp1[3]);
      lb = rd->lb_len + A.cfg.ws_weight * rs.lb_cost;
    } else {
      target_of(A.cfg.mslot, A.cfg.cost_mode, rs.prp1, tgt);
    }
    rs.init[1] = rs.best[1] = best;
    for (int c = 0; c < 4; ++c) rs.target[c] = tgt[c];
    rs.no_imp = 0;
    rs.prune_len = kInvalid;
    // R39: pass 2 only if the input schedule is >= pass2_gap cycles above LB_len
    const bool gap_cut = !A.cfg.weighted && (A.cfg.pass_mask & 2u) && A.cfg.pass2_gap > 0 &&
                         len < rd->lb_len + A.cfg.pass2_gap;
    if (gap_cut) rs.policy |= 1u;
    rs.active = (A.cfg.pass_mask & 2u) && A.cfg.iterations > 0 && !gap_cut && !(A.cfg.stop_at_lb && best == lb);
  }
}

__global__ void __launch_bounds__(128) k_pass2_init(KArgs A) {
  const uint32_t r = blockIdx.x;
  const RegionDev *rd = A.regions + r;
  const RegionWs &W = A.rws[r];
  extern __shared__ uint32_t rdyv[];  // rdy[n]
  pass2_init_body(A, rd, W, A.state[r], A.arena + rd->o_image, (uint16_t *)(A.ws + W.o_tau), rdyv);
}

// After the last pass (L366; R40): the heuristic schedule's length, and the
// revert filter -- report the heuristic schedule when the result gained at
// least revert_occ occupancy but is more than revert_len cycles longer.
// (thread 0 works; rdyv must be zeroed by the caller)
__device__ __forceinline__ void post_body(const KArgs &A, const RegionDev *rd, const RegionWs &W, RegionState &rs,
                                          const unsigned char *img, uint32_t *rdyv) {
  const uint32_t n = rd->n;
  const SV V = make_sv(img, rd);
  const uint16_t *heur = (const uint16_t *)(A.ws + W.o_heur);
  const MachineDev &M = c_mach[A.cfg.mslot];
  const uint32_t hlen = asap_order(M, V, heur, nullptr, nullptr, rdyv);
  rs.heur_len = hlen;
  if (A.cfg.revert_occ == 0) return;
  uint32_t of = M.occ_max, oh = M.occ_max;
  for (uint32_t c = 0; c < M.n_classes; ++c) {
    of = min(of, occ_of(M, c, rs.prp2[c]));
    oh = min(oh, occ_of(M, c, rs.heur_prp[c]));
  }
  if (of >= oh + A.cfg.revert_occ && (uint64_t)rs.len2 > (uint64_t)hlen + A.cfg.revert_len) {
    for (uint32_t i = 0; i < n; ++i) rdyv[i] = 0;
    asap_order(M, V, heur, (uint16_t *)(A.ws + W.o_gb2), (uint32_t *)(A.ws + W.o_gb2c), rdyv);
    for (int c = 0; c < 4; ++c) rs.prp2[c] = rs.heur_prp[c];
    rs.len2 = hlen;
    rs.policy |= 2u;
  }
}

__global__ void __launch_bounds__(32) k_post(KArgs A) {
  const uint32_t r = blockIdx.x;
  const RegionDev *rd = A.regions + r;
  extern __shared__ uint32_t rdyv[];  // rdy[n]
  for (uint32_t i = threadIdx.x; i < rd->n; i += blockDim.x) rdyv[i] = 0;
  __syncwarp();
  if (threadIdx.x == 0) post_body(A, rd, A.rws[r], A.state[r], A.arena + rd->o_image, rdyv);
}

// The iteration winner's successor table (pheromone deposit links, R8-R9)
// and the global-best epilogue (L139; R11): one warp.
template <int PASS>
__device__ __forceinline__ void epilogue_body(const KArgs &A, uint32_t iter, RegionState &rs, const RegionWs &W,
                                              uint32_t n, bool have, uint32_t wcost, uint32_t want, const uint16_t *ord,
                                              const uint32_t *cyc, uint16_t *next, const uint32_t *s_prp,
                                              uint32_t &s_flag) {
  for (uint32_t i = threadIdx.x; i <= n; i += 32) next[i] = 0xFFFFu;
  __syncwarp();
  if (have) {
    for (uint32_t k = threadIdx.x; k + 1 < n; k += 32) next[ord[k]] = ord[k + 1];
    if (threadIdx.x == 0 && n) next[n] = ord[0];
  }
  // ---- epilogue (first thread, L139)
  if (threadIdx.x == 0) {
    rs.hash = fnv_u32(fnv_u32(fnv_u32(fnv_u32(rs.hash, PASS == 2 && A.cfg.weighted ? 4u : PASS), iter),
                              have ? wcost : kInvalid),
                      have ? want : kInvalid);
    const bool improved = have && wcost < rs.best[PASS - 1];  // strict (R11)
    s_flag = improved;
    if (improved) {
      rs.best[PASS - 1] = wcost;
      rs.no_imp = 0;
      uint32_t *prp = PASS == 1 ? rs.prp1 : rs.prp2;
      prp[0] = s_prp[0] & 0xFFFFu;
      prp[1] = s_prp[0] >> 16;
      prp[2] = s_prp[1] & 0xFFFFu;
      prp[3] = s_prp[1] >> 16;
      if (PASS == 2) rs.len2 = s_prp[2];
    } else {
      rs.no_imp++;
    }
    rs.iters[PASS - 1] = iter + 1;
    rs.prune_len = kInvalid;
  }
  __syncwarp();
  if (s_flag) {
    if (PASS == 1) {
      uint16_t *gb1 = (uint16_t *)(A.ws + W.o_gb1);
      for (uint32_t k = threadIdx.x; k < n; k += 32) gb1[k] = ord[k];
    } else {
      uint16_t *gb2 = (uint16_t *)(A.ws + W.o_gb2);
      uint32_t *gb2c = (uint32_t *)(A.ws + W.o_gb2c);
      for (uint32_t k = threadIdx.x; k < n; k += 32) {
        gb2[k] = ord[k];
        gb2c[k] = cyc[k];
      }
    }
  }
}

// End of an iteration for one region (L137-L139), one warp: argmin over
// (cost, ant) (R10) -- or the shared colony's allreduced key -- replay of the
// winner by the whole warp to recover its order, the winner's successor
// table for the pheromone update, and the epilogue.
template <int PASS, bool MASK, bool T32, bool NC4, bool GS>
__device__ __forceinline__ void select_body(const KArgs &A, uint32_t iter, unsigned char *smem,
                                            uint32_t *s_prp, uint32_t &s_flag) {
  const uint32_t r = blockIdx.x;
  RegionState &rs = A.state[r];
  const RegionDev *rd = A.regions + r;
  const RegionWs &W = A.rws[r];
  const uint32_t n = rd->n;
  const uint16_t *tau = (const uint16_t *)(A.ws + W.o_tau);
  const uint32_t *costs = (const uint32_t *)(A.ws + W.o_cost);
  const unsigned char *img = A.arena + rd->o_image;
  uint32_t *stw = (uint32_t *)(A.ws + W.o_scratch);
  if (!GS) {
    // the replay is one warp per region: with many regions the image is read
    // through L1 (no per-block staging) and only the replay state lives in
    // shared memory, so many replays are resident per SM; with few regions
    // the image is staged as well (latency-bound serial replay)
    if (A.cfg.stage_img) {
      stage_warp((uint4 *)smem, (const uint4 *)img, rd->img.bytes);
      img = smem;
      stw = (uint32_t *)(smem + rd->img.bytes);
      __syncwarp();
    } else {
      stw = (uint32_t *)smem;
    }
  }
  unsigned long long best = ~0ull;
  if (A.cfg.keys) {
    best = (unsigned long long)A.cfg.keys[r] ^ kKeyBias;
  } else {
    for (uint32_t a = threadIdx.x; a < A.cfg.ants; a += 32)
      best = min(best, ((unsigned long long)costs[a] << 32) | (A.cfg.ant_base + a));
#pragma unroll
    for (int off = 16; off; off >>= 1) best = min(best, __shfl_xor_sync(0xFFFFFFFFu, best, off));
  }
  const uint32_t wcost = (uint32_t)(best >> 32), want = (uint32_t)best;
  const bool have = wcost != kInvalid;
  // state: [ant state | cycle u32[n] | order u16[n]]
  const SV V = make_sv(img, rd);
  uint32_t *cyc = stw + ant_words(PASS, n, rd->nwr, rd->nremw, T32, NC4);
  uint16_t *ord = (uint16_t *)(cyc + n);
  __syncwarp();
  if (have && A.cfg.record && !A.cfg.keys) {  // the winner recorded its schedule: copy it
    const uint32_t wl = want - A.cfg.ant_base, na = A.cfg.ants;
    const uint16_t *ro = (const uint16_t *)(A.ws + W.o_rec) + wl;
    const uint32_t *rc = (const uint32_t *)(A.ws + W.o_recc) + wl;
    for (uint32_t k = threadIdx.x; k < n; k += 32) {
      ord[k] = ro[(size_t)k * na];
      if (PASS == 2) cyc[k] = rc[(size_t)k * na];
    }
    if (threadIdx.x == 0) {
      const uint4 q = ((const uint4 *)(A.ws + W.o_recp))[wl];
      s_prp[0] = q.x;
      s_prp[1] = q.y;
      s_prp[2] = q.z;
    }
  } else if (have) {  // the whole warp replays the winner as one 32-lane group
    const St S = make_st<PASS, T32, NC4>(stw, 1, V);
    const Grp<32> G32(threadIdx.x);
    AntOut o;
    if constexpr (PASS == 1) {
      RL rl{nullptr, 0, 0, A.cfg.rl_limit, nullptr, nullptr};
      if (A.cfg.rl_limit)  // R45: the winner's group limits as recorded by the construct kernel
        rl.in = (const uint16_t *)(A.ws + W.o_rlk) + (size_t)((want - A.cfg.ant_base) / A.cfg.group_size) * n;
      if (rl.in) o = ant_pass1<32, MASK, false, true>(V, tau, S, G32, want, iter, A.cfg, false, ord, nullptr, rl);
      else o = ant_pass1<32, MASK>(V, tau, S, G32, want, iter, A.cfg, false, ord, nullptr, rl);
    } else {
      uint32_t tgt[4];
      for (int c = 0; c < 4; ++c) tgt[c] = rs.target[c];
      o = ant_pass2<32, MASK, T32, NC4>(V, tau, S, G32, want, iter, A.cfg, tgt, nullptr, false, ord, cyc);
    }
    if (threadIdx.x == 0) {
      s_prp[0] = o.prp01;
      s_prp[1] = o.prp23;
      s_prp[2] = o.len;
    }
  }
  __syncwarp();
  epilogue_body<PASS>(A, iter, rs, W, n, have, wcost, want, ord, cyc, (uint16_t *)(A.ws + W.o_next), s_prp, s_flag);
}

template <int PASS, bool MASK, bool T32, bool NC4>
__global__ void __launch_bounds__(32) k_select(KArgs A, uint32_t iter) {
  if (!A.state[blockIdx.x].active) return;
  extern __shared__ uint4 smem4[];
  __shared__ uint32_t s_prp[3], s_flag;
  // a batch with some u32-cycle regions launches the T32 variant; its compact
  // regions replay with the compact layout (their image has no predecessor list)
  const bool ct = PASS == 2 && T32 && !NC4 && A.regions[blockIdx.x].compact;
  if (A.rws[blockIdx.x].gs) {
    if (ct) select_body<PASS, false, false, false, true>(A, iter, (unsigned char *)smem4, s_prp, s_flag);
    else select_body<PASS, false, T32, NC4, true>(A, iter, (unsigned char *)smem4, s_prp, s_flag);
  } else if (A.regions[blockIdx.x].n <= 1024) {  // word-mask scan per region (MASK: n <= 1024)
    if (ct) select_body<PASS, true, false, false, false>(A, iter, (unsigned char *)smem4, s_prp, s_flag);
    else select_body<PASS, true, T32, NC4, false>(A, iter, (unsigned char *)smem4, s_prp, s_flag);
  } else {
    if (ct) select_body<PASS, false, false, false, false>(A, iter, (unsigned char *)smem4, s_prp, s_flag);
    else select_body<PASS, false, T32, NC4, false>(A, iter, (unsigned char *)smem4, s_prp, s_flag);
  }
  (void)MASK;
}

// Shared colony: per-region local argmin over this context's ants, written as
// a biased key for a signed int64 MIN allreduce across ranks.
__global__ void __launch_bounds__(32) k_local_keys(KArgs A, int64_t *keys) {
  const uint32_t r = blockIdx.x;
  const uint32_t *costs = (const uint32_t *)(A.ws + A.rws[r].o_cost);
  unsigned long long best = ~0ull;
  for (uint32_t a = threadIdx.x; a < A.cfg.ants; a += 32)
    best = min(best, ((unsigned long long)costs[a] << 32) | (A.cfg.ant_base + a));
#pragma unroll
  for (int off = 16; off; off >>= 1) best = min(best, __shfl_xor_sync(0xFFFFFFFFu, best, off));
  if (threadIdx.x == 0) keys[r] = (int64_t)(best ^ kKeyBias);
}

// Termination (L110, L139, L226; R12), after the pheromone update.
__device__ __forceinline__ void stop_body(const KArgs &A, uint32_t r, uint32_t pass) {
  RegionState &rs = A.state[r];
  if (!rs.active) return;
  const RegionDev *rd = A.regions + r;
  const uint32_t lim = no_improve_limit(A.cfg, rd->n);
  const uint32_t lb = pass == 1 ? rs.lb_cost : rd->lb_len + (A.cfg.weighted ? A.cfg.ws_weight * rs.lb_cost : 0u);
  if ((A.cfg.stop_at_lb && rs.best[pass - 1] == lb) || (lim > 0 && rs.no_imp >= lim) ||
      rs.iters[pass - 1] >= A.cfg.iterations)
    rs.active = 0;
}
__global__ void k_stop(KArgs A, uint32_t pass) {
  const uint32_t r = blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= A.cfg.count) return;
  stop_body(A, r, pass);
}

// Few regions with small tables (config 2): the end of an iteration in ONE
// launch, one block per region -- select (warp 0: argmin, winner copy or
// replay, epilogue), the block's evaporate + deposit over the region's table,
// the termination test: the bodies of k_select, k_update and k_stop in their
// per-region order (regions are independent), two launches fewer per
// iteration.
template <int PASS, bool MASK, bool T32, bool NC4>
__global__ void __launch_bounds__(256) k_finalize1(KArgs A, uint32_t iter) {
  const uint32_t r = blockIdx.x;
  if (!A.state[r].active) return;  // block-uniform
  extern __shared__ uint4 smem4[];
  __shared__ uint32_t s_prp[3], s_flag;
  if (threadIdx.x < 32) {
    const bool ct = PASS == 2 && T32 && !NC4 && A.regions[r].compact;
    if (A.rws[r].gs) {
      if (ct) select_body<PASS, false, false, false, true>(A, iter, (unsigned char *)smem4, s_prp, s_flag);
      else select_body<PASS, false, T32, NC4, true>(A, iter, (unsigned char *)smem4, s_prp, s_flag);
    } else if (ct) {
      select_body<PASS, MASK, false, false, false>(A, iter, (unsigned char *)smem4, s_prp, s_flag);
    } else {
      select_body<PASS, MASK, T32, NC4, false>(A, iter, (unsigned char *)smem4, s_prp, s_flag);
    }
  }
  __syncthreads();
  update_vecs(A, r, 0, A.rws[r].tau_len / 8, threadIdx.x, blockDim.x);
  __syncthreads();
  if (threadIdx.x == 0) stop_body(A, r, PASS);
}

// ------------------------------------------------------------ fused run
// The whole two-pass ACO of one region in ONE block (the
// paper's cooperative kernel runs construct -> reduce -> update -> epilogue
// in one launch).  Used for batches whose ants all fit one block per region
// (config 1): image, pheromone table, every ant's state and its recorded
// schedule stay in shared memory across the iterations; block barriers
// replace the kernel boundaries of the multi-launch path, so the sequence of
// states -- and every result -- is that of the launches it replaces (the
// same device functions run in the same order).  One ant per thread
// (word-mask scan, compact pass-2 layout, group coins drawn inline).
// FW: 4-wide candidate scan (off by default: the small regions of a fused run
// have too few candidates per step to fill a batch of four).
// WL > 0: every ant is a group of WL lanes (lane-per-instruction ants,
// lpi_pass1/2; n <= 4 WL); else one thread per ant.
template <bool FW, int WL = 0>
__global__ void __launch_bounds__(512, 1) k_fused(KArgs A) {
  const uint32_t r = blockIdx.x;
  const RegionDev *rd = A.regions + r;
  const RegionWs &W = A.rws[r];
  // the region state lives in shared memory for the whole run (its serial
  // epilogue updates stay on chip) and is written back at the end
  __shared__ RegionState srs;
  RegionState &rs = srs;
  extern __shared__ uint4 smem4[];
  unsigned char *smem = (unsigned char *)smem4;
  __shared__ uint32_t s_prp[3], s_flag, s_active;
  const uint32_t n = rd->n, na = A.cfg.ants, tid = threadIdx.x;
  for (uint32_t i = tid; i < sizeof(RegionState) / 4; i += blockDim.x) ((uint32_t *)&srs)[i] = 0;
  const FusedLayout F = fused_layout(n, rd->nwr, rd->nremw, rd->img.bytes, na, A.cfg.group_size);
  stage(smem4, (const uint4 *)(A.arena + rd->o_image), rd->img.bytes);
  const unsigned char *img = smem;
  uint16_t *tau = (uint16_t *)(smem + F.o_tau);
  uint32_t *st = (uint32_t *)(smem + F.o_state);
  uint16_t *rec_o = (uint16_t *)(smem + F.o_reco);
  uint32_t *rec_c = (uint32_t *)(smem + F.o_recc);
  uint32_t *costs = (uint32_t *)(smem + F.o_costs);
  uint4 *recp = (uint4 *)(smem + F.o_recp);
  uint16_t *ord = (uint16_t *)(smem + F.o_ord);
  uint32_t *cyc = (uint32_t *)(smem + F.o_cyc);
  uint16_t *next = (uint16_t *)(smem + F.o_next);
  uint32_t *coins = (uint32_t *)(smem + F.o_coins);
  tau_fill(tau, W.tau_len, A.cfg.tau0);
  __syncthreads();
  init_greedy<true>(A, rd, W, rs, img, tau, st);  // (k_init)
  __syncthreads();
  const SV V = make_sv(img, rd);
  const bool dump = (A.cfg.flags & ACO_FLAG_DUMP) != 0;
  for (uint32_t pass = 1; pass <= 2; ++pass) {
    if (pass == 2) {  // (k_pass2_init)
      pass2_init_body(A, rd, W, rs, img, tau, rec_c);
      __syncthreads();
    }
    if (!(A.cfg.pass_mask & pass)) continue;
    for (uint32_t it = 0; it < A.cfg.iterations; ++it) {
      if (tid == 0) s_active = rs.active;
      __syncthreads();
      if (!s_active) break;  // block-uniform
      // group coins (R3) of every (step, group) of this iteration, one warp per
      // 32 steps of a group (ballot), as k_construct precomputes them
      const uint32_t gsz = A.cfg.group_size, g0 = A.cfg.ant_base / gsz;
      const uint32_t ng = (A.cfg.ant_base + na - 1) / gsz - g0 + 1, cw = coin_words(pass, n);
      {
        const uint32_t lane = tid & 31u, c2 = pass == 1 ? it : (0x80000000u | it);
        for (uint32_t task = tid >> 5; task < ng * cw; task += blockDim.x >> 5) {
          const uint32_t gi = task / cw, k = (task - gi * cw) * 32 + lane;
          const uint4 x = philox(k, 0x80000000u | (g0 + gi), c2, rd->region_id, A.cfg.seed);
          const uint32_t word = __ballot_sync(0xFFFFFFFFu, (uint64_t)x.x < A.cfg.q0_t);
          if (lane == 0) coins[task] = word;
        }
      }
      __syncthreads();
      const uint32_t ai = WL ? tid / WL : tid;  // the ant of this thread
      if (ai < na) {  // (k_construct) ant ai
        const Grp<1> G(tid);
        const uint32_t ant = A.cfg.ant_base + ai;
        AntOut o;
        if constexpr (WL > 0) {
          const uint32_t qn = (n + WL - 1) / WL;
          const uint32_t *cz = coins + (ant / gsz - g0) * cw;
          if (pass == 1) {
            if (qn <= 1) o = lpi_pass1<WL, 1>(V, tau, st + ai, na, ant, it, A.cfg, rec_o + ai, cz, na);
            else if (qn <= 2) o = lpi_pass1<WL, 2>(V, tau, st + ai, na, ant, it, A.cfg, rec_o + ai, cz, na);
            else o = lpi_pass1<WL, 4>(V, tau, st + ai, na, ant, it, A.cfg, rec_o + ai, cz, na);
          } else {
            uint32_t tgt[4];
#pragma unroll
            for (int c = 0; c < 4; ++c) tgt[c] = rs.target[c];
            const bool prune = !dump && !(A.cfg.flags & ACO_FLAG_NO_PRUNE) && !A.cfg.keys && !A.cfg.weighted;
            if (qn <= 1)
              o = lpi_pass2<WL, 1>(V, tau, st + ai, na, ant, it, A.cfg, tgt, &rs.prune_len, prune, rec_o + ai,
                                   rec_c + ai, cz, cw * 32, na);
            else if (qn <= 2)
              o = lpi_pass2<WL, 2>(V, tau, st + ai, na, ant, it, A.cfg, tgt, &rs.prune_len, prune, rec_o + ai,
                                   rec_c + ai, cz, cw * 32, na);
            else
              o = lpi_pass2<WL, 4>(V, tau, st + ai, na, ant, it, A.cfg, tgt, &rs.prune_len, prune, rec_o + ai,
                                   rec_c + ai, cz, cw * 32, na);
          }
        } else if (pass == 1) {
          const St S = make_st<1, false, false>(st + tid, na, V);
          o = ant_pass1<1, true, FW>(V, tau, S, G, ant, it, A.cfg, false, rec_o + tid, coins + (ant / gsz - g0) * cw,
                                 RL{nullptr, 0, 0, 0, nullptr, nullptr}, na);
        } else {
          const St S = make_st<2, false, false>(st + tid, na, V);
          uint32_t tgt[4];
#pragma unroll
          for (int c = 0; c < 4; ++c) tgt[c] = rs.target[c];
          const bool prune = !dump && !(A.cfg.flags & ACO_FLAG_NO_PRUNE) && !A.cfg.keys && !A.cfg.weighted;
          o = ant_pass2<1, true, false, false, FW>(V, tau, S, G, ant, it, A.cfg, tgt, &rs.prune_len, prune, rec_o + tid,
                                               rec_c + tid, coins + (ant / gsz - g0) * cw, cw * 32, na);
        }
        if (!WL || tid % WL == 0) {  // (the group's lane 0 recorded the schedule)
          costs[ai] = o.cost;
          recp[ai] = make_uint4(o.prp01, o.prp23, o.len, 0u);
          if (dump && A.dump_cost) {
            A.dump_cost[(((size_t)(pass - 1) * A.cfg.iterations + it) * A.cfg.count + r) * na + ai] = o.cost;
            const size_t base =
                ((size_t)(pass - 1) * A.cfg.iterations + it) * A.cfg.dump_slice + W.o_dump + (size_t)ai * n;
            if (A.dump_order && o.cost != kInvalid)
              for (uint32_t k = 0; k < n; ++k) A.dump_order[base + k] = rec_o[k * na + ai];
            if (A.dump_cycle && pass == 2 && o.cost != kInvalid)
              for (uint32_t k = 0; k < n; ++k) A.dump_cycle[base + k] = rec_c[k * na + ai];
          }
        }
      }
      __syncthreads();
      if (tid < 32) {  // (k_select) argmin over (cost, ant), copy of the winner's schedule, epilogue
        unsigned long long best = ~0ull;
        for (uint32_t a = tid; a < na; a += 32)
          best = min(best, ((unsigned long long)costs[a] << 32) | (A.cfg.ant_base + a));
#pragma unroll
        for (int off = 16; off; off >>= 1) best = min(best, __shfl_xor_sync(0xFFFFFFFFu, best, off));
        const uint32_t wcost = (uint32_t)(best >> 32), want = (uint32_t)best;
        const bool have = wcost != kInvalid;
        if (have) {
          const uint32_t wl = want - A.cfg.ant_base;
          for (uint32_t k = tid; k < n; k += 32) {
            ord[k] = rec_o[k * na + wl];
            if (pass == 2) cyc[k] = rec_c[k * na + wl];
          }
          if (tid == 0) {
            const uint4 q = recp[wl];
            s_prp[0] = q.x;
            s_prp[1] = q.y;
            s_prp[2] = q.z;
          }
        }
        __syncwarp();
        if (pass == 1) epilogue_body<1>(A, it, rs, W, n, have, wcost, want, ord, cyc, next, s_prp, s_flag);
        else epilogue_body<2>(A, it, rs, W, n, have, wcost, want, ord, cyc, next, s_prp, s_flag);
      }
      __syncthreads();
      {  // (k_update) evaporate + deposit + clamp, R6-R9
        const uint32_t rho = A.cfg.rho_q16, dl = A.cfg.delta, lo = A.cfg.tau_min, hi = A.cfg.tau_max;
        for (uint32_t e = tid; e < (n + 1) * n; e += blockDim.x) {
          const uint32_t i = e / n, j = e - i * n;
          uint32_t x = ((uint32_t)tau[e] * rho) >> 16;
          if (next[i] == j) x += dl;
          tau[e] = (uint16_t)min(max(x, lo), hi);
        }
      }
      if (tid == 0) {  // (k_stop) termination, R12
        const uint32_t lim = no_improve_limit(A.cfg, n);
        const uint32_t lb = pass == 1 ? rs.lb_cost : rd->lb_len + (A.cfg.weighted ? A.cfg.ws_weight * rs.lb_cost : 0u);
        if ((A.cfg.stop_at_lb && rs.best[pass - 1] == lb) || (lim > 0 && rs.no_imp >= lim) ||
            rs.iters[pass - 1] >= A.cfg.iterations)
          rs.active = 0;
      }
      __syncthreads();
    }
  }
  for (uint32_t i = tid; i < n; i += blockDim.x) rec_c[i] = 0;  // (k_post)
  __syncthreads();
  if (tid == 0) post_body(A, rd, W, rs, img, rec_c);
  __syncthreads();
  for (uint32_t i = tid; i < sizeof(RegionState) / 4; i += blockDim.x)
    ((uint32_t *)(A.state + r))[i] = ((const uint32_t *)&srs)[i];
}

// ------------------------------------------------------------ launchers
static KArgs kargs(const LaunchCtx &L) {
  KArgs a;
  a.arena = L.arena;
  a.ws = L.ws;
  a.regions = L.regions;
  a.state = L.state;
  a.rws = L.rws;
  a.dump_cost = L.dump_cost;
  a.dump_order = L.dump_order;
  a.dump_cycle = L.dump_cycle;
  a.cfg = L.cfg;
  return a;
}

// ACO_SYNC_DEBUG=1: synchronise after every launch and name the failing one
// (debugging aid; compute-sanitizer is not available on every pool).
static int check(const char *tag = "", uint32_t code = 0) {
  static const bool sync_debug = getenv("ACO_SYNC_DEBUG") != nullptr;
  cudaError_t e = cudaGetLastError();
  if (sync_debug && e == cudaSuccess) {
    e = cudaDeviceSynchronize();
    if (e != cudaSuccess) fprintf(stderr, "[aco sync] %s (variant %u): %s\n", tag, code, cudaGetErrorString(e));
  }
  return e == cudaSuccess ? 0 : (int)e;
}

int last_cuda_error() { return check(); }

// ---- construct-kernel variants: one table of every instantiation, used for
// the shared-memory opt-in, the register limits the planner needs and the
// launch dispatch (a class launch looks its kernel up by variant code).
using ConstructFn = void (*)(KArgs, const BlockItem *, uint32_t);

template <int P, int LG, bool M, bool TS, bool T3, bool N4, int GS, bool WD, typename F, bool LN = false>
static void reg1(F &f) {
  f(&k_construct<P, LG, M, TS, T3, N4, GS, WD, LN>, variant_code(P, LG, M, TS, T3, N4, GS, WD, LN));
}
template <int P, int LG, bool M, bool TS, bool T3, bool N4, typename F>
static void reg_w(F &f) {  // the 4-wide scan exists only with the word mask (n <= 1024)
  reg1<P, LG, M, TS, T3, N4, false, false>(f);
  if constexpr (M) reg1<P, LG, M, TS, T3, N4, false, true>(f);
}
template <int LG, typename F>
static void reg_lg(F &f) {
  reg1<1, LG, true, false, false, false, 2, true>(f);  // large regions, image through L1
  reg1<2, LG, true, false, false, false, 2, true>(f);
  if constexpr (LG == 1) {  // lean layouts (large regions), image staged or through L1
    reg1<2, 1, true, false, false, false, 0, true, F, true>(f);
    reg1<2, 1, true, false, false, false, 2, true, F, true>(f);
    reg1<1, 1, true, false, false, false, 0, true, F, true>(f);
    reg1<1, 1, true, false, false, false, 2, true, F, true>(f);
  }
  reg_w<1, LG, true, true, false, false>(f);
  reg_w<1, LG, true, false, false, false>(f);
  reg_w<1, LG, false, true, false, false>(f);
  reg_w<1, LG, false, false, false, false>(f);
  reg_w<2, LG, true, true, false, false>(f);
  reg_w<2, LG, true, false, false, false>(f);
  reg_w<2, LG, false, true, false, false>(f);
  reg_w<2, LG, false, false, false, false>(f);
}
template <int LG, bool M, typename F>
static void reg_rare(F &f) {  // pass 2 with u32 cycles and/or 3-4 classes: tau in global memory, 1 or 4 lanes
  reg_w<2, LG, M, false, true, false>(f);
  reg_w<2, LG, M, false, false, true>(f);
  reg_w<2, LG, M, false, true, true>(f);
}
template <int LG, typename F>
static void reg_huge(F &f) {
  reg1<1, LG, false, false, false, false, 2, true>(f);
  reg1<2, LG, false, false, false, false, 2, true>(f);
  reg1<2, LG, false, false, false, false, 2, true, F, true>(f);
}
template <typename F>
static void for_each_construct(F &&f) {
  // lane-per-instruction ants (one warp per ant, n <= 128), tau staged or not
  reg1<1, 32, true, true, false, false, 0, false>(f);
  reg1<1, 32, true, false, false, false, 0, false>(f);
  reg1<2, 32, true, true, false, false, 0, false>(f);
  reg1<2, 32, true, false, false, false, 0, false>(f);
  reg_lg<1>(f);
  reg_lg<2>(f);
  reg_lg<4>(f);
  reg_lg<8>(f);
  reg_rare<1, true>(f);
  reg_rare<1, false>(f);
  reg_rare<4, true>(f);
  reg_rare<4, false>(f);
  // huge regions: per-ant state in the workspace, 4 / 8 / 16 lanes per ant,
  // 1-wide or 4-wide candidate scan (strided words, scan4s)
  reg1<1, 4, false, false, false, false, 1, false>(f);
  reg1<2, 4, false, false, false, false, 1, false>(f);
  reg1<1, 8, false, false, false, false, 1, false>(f);
  reg1<2, 8, false, false, false, false, 1, false>(f);
  reg1<1, 16, false, false, false, false, 1, false>(f);
  reg1<2, 16, false, false, false, false, 1, false>(f);
  reg1<1, 4, false, false, false, false, 1, true>(f);
  reg1<2, 4, false, false, false, false, 1, true>(f);
  reg1<1, 8, false, false, false, false, 1, true>(f);
  reg1<2, 8, false, false, false, false, 1, true>(f);
  reg1<1, 16, false, false, false, false, 1, true>(f);
  reg1<2, 16, false, false, false, false, 1, true>(f);
  reg1<2, 4, false, false, true, false, 1, false>(f);
  reg1<2, 4, false, false, false, true, 1, false>(f);
  reg1<2, 4, false, false, true, true, 1, false>(f);
  // huge regions with the per-ant state in shared memory, image and tau
  // through L1 (GS = 2, no word mask), 4-wide strided scan; pass 2 compact or lean
  reg_huge<4>(f);
  reg_huge<8>(f);
  reg_huge<16>(f);
}

static ConstructFn g_construct[8192];
static bool g_table_ready = false;
static void build_table() {
  if (g_table_ready) return;
  for_each_construct([](ConstructFn f, uint32_t code) { g_construct[code] = f; });
  g_table_ready = true;
}

// Resident threads per SM the registers of the construct kernels allow, per
// (pass, plain | wide | lean); conservative defaults when no device is visible.
int construct_max_threads(int device, uint32_t out[2][3]) {
  out[0][0] = out[1][0] = 1024;
  out[0][1] = out[1][1] = 512;
  out[0][2] = out[1][2] = 512;
  int cur = -1;
  if (cudaGetDevice(&cur) != cudaSuccess || (device >= 0 && cur != device && cudaSetDevice(device) != cudaSuccess)) {
    cudaGetLastError();
    return 1;
  }
  uint32_t regs[2][3] = {{0, 0, 0}, {0, 0, 0}};
  bool ok = true;
  for_each_construct([&](ConstructFn f, uint32_t code) {
    cudaFuncAttributes fa;
    if (cudaFuncGetAttributes(&fa, f) != cudaSuccess) {
      ok = false;
      return;
    }
    if (code & (1u << 10)) return;  // (lane-per-instruction variants: planned separately)
    const uint32_t p = (code >> 8) & 1u, w = ((code >> 12) & 1u) ? 2u : (code & 1u);
    regs[p][w] = std::max(regs[p][w], (uint32_t)fa.numRegs);
  });
  if (!ok) {
    cudaGetLastError();
    return 1;
  }
  for (int p = 0; p < 2; ++p)
    for (int w = 0; w < 3; ++w) {
      const uint32_t r8 = std::max(8u, (regs[p][w] + 7u) & ~7u);  // allocation unit: 8 registers per thread
      const uint32_t warps = std::min(64u, 65536u / (32u * r8));
      out[p][w] = warps * 32u;
    }
  return 0;
}

// Opt every kernel into the largest dynamic shared memory it can use (the
// per-block maximum minus its static shared memory, rounded down to 1 KB).
static int g_attr_err = 0;
template <typename K>
static void big_smem(K kernel) {
  cudaFuncAttributes fa;
  if (cudaFuncGetAttributes(&fa, kernel) != cudaSuccess) {
    g_attr_err = 1;
    return;
  }
  const int dyn = (int)((kSmemPerSM - (uint32_t)fa.sharedSizeBytes) & ~1023u);
  if (cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, dyn) != cudaSuccess)
    g_attr_err = 1;
}

int set_machine(uint32_t slot, const MachineDev &m) {
  if (slot >= kMachSlots) return 1;
  if (cudaMemcpyToSymbol(c_mach, &m, sizeof(m), sizeof(m) * slot) != cudaSuccess) return 1;
  return check(__func__);
}

int init_kernel_attrs() {
  g_attr_err = 0;
  big_smem(k_init<true>);
  big_smem(k_init<false>);
  big_smem(k_pass2_init);
  big_smem(k_finalize1<1, true, false, false>);
  big_smem(k_finalize1<2, true, false, false>);
  big_smem(k_finalize1<2, true, true, false>);
  big_smem(k_finalize1<2, true, false, true>);
  big_smem(k_finalize1<2, true, true, true>);
  big_smem(k_post);
  big_smem(k_fused<false>);
  big_smem(k_fused<false, 8>);
  big_smem(k_fused<false, 16>);
  big_smem(k_fused<false, 32>);
  big_smem(k_fused<true>);
#define ACO_SEL(M) big_smem(k_select<1, M, false, false>); big_smem(k_select<2, M, false, false>); \
  big_smem(k_select<2, M, true, false>); big_smem(k_select<2, M, false, true>); big_smem(k_select<2, M, true, true>);
  ACO_SEL(true) ACO_SEL(false)
#undef ACO_SEL
  for_each_construct([](ConstructFn f, uint32_t) { big_smem(f); });
  const int e = check();
  return e ? e : g_attr_err;
}

int launch_init(LaunchCtx &L, uint32_t smem, uint32_t max_n) {
  if (!L.cfg.count) return 0;
  cudaStream_t s = (cudaStream_t)L.stream;
  if (max_n <= 1024)
    k_init<true><<<L.cfg.count, 128, smem, s>>>(kargs(L));
  else
    k_init<false><<<L.cfg.count, 128, smem, s>>>(kargs(L));
  L.launches++;
  return check(__func__);
}

int launch_pass2_init(LaunchCtx &L, uint32_t smem, uint32_t max_n) {
  (void)max_n;
  if (!L.cfg.count) return 0;
  k_pass2_init<<<L.cfg.count, 128, smem, (cudaStream_t)L.stream>>>(kargs(L));
  L.launches++;
  return check(__func__);
}

int launch_construct(LaunchCtx &L, uint32_t pass, uint32_t iter, const ClassLaunch &c) {
  if (!c.n_blocks) return 0;
  build_table();
  const uint32_t lg = c.lanes;
  const uint32_t code = class_variant(pass, c);
  const ConstructFn f = g_construct[code];
  if (!f) return (int)cudaErrorInvalidDeviceFunction;
  f<<<c.n_blocks, c.ants_pb * lg, c.smem_bytes, (cudaStream_t)L.stream>>>(kargs(L), c.items, iter);
  L.launches++;
  return check("k_construct", code);
}

template <bool M>
static void sel(uint32_t pass, bool t32, bool nc4, uint32_t grid, uint32_t smem, cudaStream_t s, const KArgs &a,
                uint32_t iter) {
  if (pass == 1) k_select<1, M, false, false><<<grid, 32, smem, s>>>(a, iter);
  else if (!t32 && !nc4) k_select<2, M, false, false><<<grid, 32, smem, s>>>(a, iter);
  else if (t32 && !nc4) k_select<2, M, true, false><<<grid, 32, smem, s>>>(a, iter);
  else if (!t32 && nc4) k_select<2, M, false, true><<<grid, 32, smem, s>>>(a, iter);
  else k_select<2, M, true, true><<<grid, 32, smem, s>>>(a, iter);
}

int launch_finalize(LaunchCtx &L, uint32_t pass, uint32_t iter, uint32_t smem, uint32_t max_n, bool t32,
                    bool nc4, const UpdItem *upd, uint32_t n_upd, bool fin1) {
  if (!L.cfg.count) return 0;
  cudaStream_t s = (cudaStream_t)L.stream;
  KArgs a = kargs(L);
  if (fin1) {  // few small regions: one launch (k_finalize1)
    if (pass == 1) k_finalize1<1, true, false, false><<<L.cfg.count, 256, smem, s>>>(a, iter);
    else if (!t32 && !nc4) k_finalize1<2, true, false, false><<<L.cfg.count, 256, smem, s>>>(a, iter);
    else if (t32 && !nc4) k_finalize1<2, true, true, false><<<L.cfg.count, 256, smem, s>>>(a, iter);
    else if (!t32 && nc4) k_finalize1<2, true, false, true><<<L.cfg.count, 256, smem, s>>>(a, iter);
    else k_finalize1<2, true, true, true><<<L.cfg.count, 256, smem, s>>>(a, iter);
    L.launches += 1;
    return check("k_finalize1", pass);
  }
  if (max_n <= 1024) sel<true>(pass, t32, nc4, L.cfg.count, smem, s, a, iter);
  else sel<false>(pass, t32, nc4, L.cfg.count, smem, s, a, iter);
  if (n_upd) k_update<<<n_upd, 256, 0, s>>>(a, upd);
  k_stop<<<(L.cfg.count + 255) / 256, 256, 0, s>>>(a, pass);
  L.launches += 2 + (n_upd ? 1 : 0);
  return check("k_select/k_update/k_stop", pass);
}

int launch_post(LaunchCtx &L, uint32_t smem) {
  if (!L.cfg.count) return 0;
  k_post<<<L.cfg.count, 32, smem, (cudaStream_t)L.stream>>>(kargs(L));
  L.launches++;
  return check(__func__);
}

int launch_fused(LaunchCtx &L, uint32_t threads, uint32_t smem, uint32_t wl) {
  if (!L.cfg.count) return 0;
  if (wl) {  // lane-per-instruction ants of wl lanes
    if (wl == 8) k_fused<false, 8><<<L.cfg.count, threads, smem, (cudaStream_t)L.stream>>>(kargs(L));
    else if (wl == 16) k_fused<false, 16><<<L.cfg.count, threads, smem, (cudaStream_t)L.stream>>>(kargs(L));
    else k_fused<false, 32><<<L.cfg.count, threads, smem, (cudaStream_t)L.stream>>>(kargs(L));
    L.launches++;
    return check(__func__);
  }
  static const int fw = [] {  // (measured, C1: 1-wide 0.654 ms, 4-wide 0.702 ms: few candidates per step)
    const char *e = getenv("ACO_FUSED_WIDE");
    return e ? atoi(e) : 0;
  }();
  if (fw) k_fused<true><<<L.cfg.count, threads, smem, (cudaStream_t)L.stream>>>(kargs(L));
  else k_fused<false><<<L.cfg.count, threads, smem, (cudaStream_t)L.stream>>>(kargs(L));
  L.launches++;
  return check(__func__);
}

int launch_local_keys(LaunchCtx &L, int64_t *keys) {
  if (!L.cfg.count) return 0;
  k_local_keys<<<L.cfg.count, 32, 0, (cudaStream_t)L.stream>>>(kargs(L), keys);
  L.launches++;
  return check(__func__);
}

}  // namespace aco
