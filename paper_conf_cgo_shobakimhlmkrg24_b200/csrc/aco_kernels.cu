// aco_kernels.cu -- sm_100a kernels of the ACO instruction scheduler.
//
// Mapping: ONE ANT PER THREAD, as in the paper (L126),
// but with every per-ant mutable array in SHARED MEMORY in a [word][ant]
// interleave (word w of ant a at smem[w * ants_per_block + a]) so that the
// data-dependent gathers of 32 ants of a warp (each at its own instruction)
// always hit 32 distinct banks: conflict-free regardless of which
// instruction each ant touches.  Region statics are read-only and shared by
// all ants of a block (L1/L2 via the read-only path).  Exploit/explore is a
// coin per group of 64 ants (L198), so a warp (32 ants) takes one branch.
//
// Kernels per pass and iteration (L135-L139):
//   k_construct  : every ant builds a schedule, writes its cost (K1a)
//   k_finalize   : per region: argmin over (cost, ant) (K1b), replay of the
//                  winner to recover its order (no per-ant order is ever
//                  stored), pheromone evaporate+deposit (K1c), global-best
//                  epilogue and termination flags (K1d).
// Plus k_init (tau0, the greedy heuristic schedule) and k_pass2_init
// (target, ASAP of the pass-1 best, tau reset).
#include <cuda_runtime.h>
#include <stdint.h>

#include "aco_internal.h"

namespace aco {

__constant__ MachineDev c_mach;

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
__device__ __forceinline__ uint32_t occ_of(uint32_t c, uint32_t x) {
  for (uint32_t i = 0; i < c_mach.step_count[c]; ++i)
    if (x <= c_mach.step_max[c][i]) return c_mach.occ_max - i;
  return 0;
}
__device__ __forceinline__ uint32_t aprp_of(uint32_t c, uint32_t x) {
  for (uint32_t i = 0; i < c_mach.step_count[c]; ++i)
    if (x <= c_mach.step_max[c][i]) return c_mach.step_max[c][i];
  return x;
}
__device__ uint32_t cost_rp(uint32_t mode, const uint32_t prp[4]) {
  const uint32_t nc = c_mach.n_classes;
  uint32_t cost = 0;
  if (mode == ACO_COST_PRP_SUM) {
    for (uint32_t c = 0; c < nc; ++c) cost += prp[c];
  } else if (mode == ACO_COST_APRP_SUM) {
    for (uint32_t c = 0; c < nc; ++c) cost += aprp_of(c, prp[c]);
  } else if (mode == ACO_COST_OCC) {
    uint32_t occ = c_mach.occ_max;
    for (uint32_t c = 0; c < nc; ++c) occ = min(occ, occ_of(c, prp[c]));
    cost = c_mach.occ_max - occ;
  } else {
    for (uint32_t c = 0; c < nc; ++c)
      cost += prp[c] > c_mach.perp_limit[c] ? prp[c] - c_mach.perp_limit[c] : 0u;
  }
  return cost;
}
__device__ void target_of(uint32_t mode, const uint32_t best[4], uint32_t tgt[4]) {
  const uint32_t nc = c_mach.n_classes;
  for (uint32_t c = 0; c < 4; ++c) tgt[c] = kInvalid;
  if (mode == ACO_COST_PRP_SUM) {
    for (uint32_t c = 0; c < nc; ++c) tgt[c] = best[c];
  } else if (mode == ACO_COST_APRP_SUM) {
    for (uint32_t c = 0; c < nc; ++c) tgt[c] = aprp_of(c, best[c]);
  } else if (mode == ACO_COST_OCC) {
    uint32_t occ = c_mach.occ_max;
    for (uint32_t c = 0; c < nc; ++c) occ = min(occ, occ_of(c, best[c]));
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

// ---------------------------------------------------------------- region view
struct RV {
  uint32_t n, nwr, nmu, Lp1, region_id;
  const uint32_t *succ_ptr, *succ, *muse, *rb0, *cnt0, *rem0;
  const uint4 *info;
  const uint16_t *eta1, *eta2;
  uint32_t livein[4];
};

__device__ __forceinline__ RV make_rv(const unsigned char *arena, const RegionDev *rd) {
  RV R;
  R.n = rd->n;
  R.nwr = rd->nwr;
  R.nmu = rd->nmu;
  R.Lp1 = rd->L + 1;
  R.region_id = rd->region_id;
  R.succ_ptr = (const uint32_t *)(arena + rd->o_succ_ptr);
  R.succ = (const uint32_t *)(arena + rd->o_succ);
  R.info = (const uint4 *)(arena + rd->o_info);
  R.muse = (const uint32_t *)(arena + rd->o_muse);
  R.rb0 = (const uint32_t *)(arena + rd->o_rb0);
  R.cnt0 = (const uint32_t *)(arena + rd->o_cnt0);
  R.rem0 = (const uint32_t *)(arena + rd->o_rem0);
  R.eta1 = (const uint16_t *)(arena + rd->o_eta1);
  R.eta2 = (const uint16_t *)(arena + rd->o_eta2);
  for (int c = 0; c < 4; ++c) R.livein[c] = rd->livein[c];
  return R;
}

__device__ __forceinline__ uint32_t byte_of(uint32_t w, uint32_t c) { return (w >> (8 * c)) & 0xFFu; }
__device__ __forceinline__ uint32_t byte_sum(uint32_t w) { return (w * 0x01010101u) >> 24; }

// remaining-use counter m (u16 packed two per word)
__device__ __forceinline__ uint32_t rem_get(const uint32_t *REM, uint32_t S, uint32_t m) {
  return (REM[(m >> 1) * S] >> ((m & 1u) * 16)) & 0xFFFFu;
}

// Iterate set bits of the ant's instruction bitset in ascending order (R25).
// MASK: a register holds one bit per non-empty bitset word (n <= 1024).
#define ACO_FOR_EACH_BIT(MASK, wmask, RB, S, nwr, J, BODY)                  \
  {                                                                         \
    uint32_t _m = (wmask);                                                  \
    uint32_t _w = 0;                                                        \
    bool _stop = false;                                                     \
    while (!_stop) {                                                        \
      if (MASK) {                                                           \
        if (!_m) break;                                                     \
        _w = __ffs(_m) - 1;                                                 \
        _m &= _m - 1;                                                       \
      } else if (_w >= (nwr)) {                                             \
        break;                                                              \
      }                                                                     \
      uint32_t _bits = (RB)[_w * (S)];                                      \
      while (_bits) {                                                       \
        const uint32_t J = _w * 32u + (__ffs(_bits) - 1);                   \
        _bits &= _bits - 1;                                                 \
        BODY                                                                \
      }                                                                     \
      if (!MASK) ++_w;                                                      \
    }                                                                       \
  }
#define ACO_BREAK_SCAN \
  {                    \
    _stop = true;      \
    break;             \
  }

struct AntOut {
  uint32_t cost;
  uint32_t prp[4];
};

// ------------------------------------------------------------ pass-1 ant
// RP pass (L108, L145; R19): latencies ignored, candidates = ready list,
// eta1 = LUC-then-CP (R4), score tau[prev][j] * eta1 (R1).  One step per
// instruction; the step index k is the Philox step (R26).
template <bool MASK, bool REC>
__device__ __forceinline__ AntOut ant_pass1(const RV &R, const uint16_t *__restrict__ tau,
                                            uint32_t *st, const uint32_t S, const uint32_t ant,
                                            const uint32_t iter, const RunCfg &cfg, const bool greedy,
                                            uint16_t *rec) {
  const uint32_t n = R.n, nwr = R.nwr;
  uint32_t *RB = st;
  uint32_t *CNT = st + nwr * S;
  uint32_t *REM = CNT + ((n + 3) >> 2) * S;
  uint32_t wmask = 0;
  for (uint32_t w = 0; w < nwr; ++w) {
    const uint32_t x = __ldg(R.rb0 + w);
    RB[w * S] = x;
    if (MASK && x) wmask |= 1u << w;
  }
  for (uint32_t w = 0; w < ((n + 3) >> 2); ++w) CNT[w * S] = __ldg(R.cnt0 + w);
  for (uint32_t w = 0; w < ((R.nmu + 1) >> 1); ++w) REM[w * S] = __ldg(R.rem0 + w);
  uint32_t live[4], prp[4];
#pragma unroll
  for (int c = 0; c < 4; ++c) live[c] = prp[c] = R.livein[c];
  const uint32_t group = ant / cfg.group_size;
  uint32_t prev = n;
  for (uint32_t k = 0; k < n; ++k) {
    bool exploit = greedy;
    if (!greedy) {
      const uint4 g = philox(k, 0x80000000u | group, iter, R.region_id, cfg.seed);
      exploit = (uint64_t)g.x < cfg.q0_t;
    }
    const uint16_t *trow = tau + (size_t)prev * n;
    uint32_t best_s = 0, best_j = 0;
    uint64_t sum = 0;
#define ACO_SCORE1(J, OUT)                                                   \
  uint32_t OUT;                                                              \
  {                                                                          \
    const uint4 inf = __ldg(R.info + J);                                     \
    uint32_t luc = byte_sum(inf.z);                                          \
    const uint32_t m0 = inf.w >> 8, mc = inf.w & 0xFFu;                      \
    for (uint32_t q = 0; q < mc; ++q) {                                      \
      const uint32_t mm = __ldg(R.muse + m0 + q) & 0xFFFFu;                  \
      luc += rem_get(REM, S, mm) == 1u;                                      \
    }                                                                        \
    OUT = (uint32_t)__ldg(trow + J) * (uint32_t)__ldg(R.eta1 + J * R.Lp1 + luc); \
  }
    ACO_FOR_EACH_BIT(MASK, wmask, RB, S, nwr, j, {
      ACO_SCORE1(j, s)
      if (exploit) {
        if (s > best_s) {
          best_s = s;
          best_j = j;
        }
      } else {
        sum += s;
      }
    })
    if (!exploit) {
      const uint4 x = philox(k, ant, iter, R.region_id, cfg.seed);
      const uint64_t r = __umul64hi(((uint64_t)x.y << 32) | x.x, sum);
      uint64_t pre = 0;
      ACO_FOR_EACH_BIT(MASK, wmask, RB, S, nwr, j, {
        ACO_SCORE1(j, s)
        pre += s;
        if (pre > r) {
          best_j = j;
          ACO_BREAK_SCAN
        }
      })
    }
#undef ACO_SCORE1
    // ---- commit best_j: RP update (R14, R15), successors, order
    const uint32_t j = best_j;
    {
      const uint32_t wi = j >> 5;
      const uint32_t nw = RB[wi * S] & ~(1u << (j & 31u));
      RB[wi * S] = nw;
      if (MASK && !nw) wmask &= ~(1u << wi);
    }
    const uint4 inf = __ldg(R.info + j);
#pragma unroll
    for (int c = 0; c < 4; ++c) live[c] -= byte_of(inf.z, c);
    {
      const uint32_t m0 = inf.w >> 8, mc = inf.w & 0xFFu;
      for (uint32_t q = 0; q < mc; ++q) {
        const uint32_t e = __ldg(R.muse + m0 + q);
        const uint32_t mm = e & 0xFFFFu, cls = e >> 16;
        const uint32_t sh = (mm & 1u) * 16;
        const uint32_t word = REM[(mm >> 1) * S];
        REM[(mm >> 1) * S] = word - (1u << sh);
        if (((word >> sh) & 0xFFFFu) == 1u) {
#pragma unroll
          for (int c = 0; c < 4; ++c) live[c] -= (cls == (uint32_t)c);
        }
      }
    }
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      live[c] += byte_of(inf.x, c);
      prp[c] = max(prp[c], live[c]);
      live[c] -= byte_of(inf.y, c);
    }
    {
      const uint32_t s0 = __ldg(R.succ_ptr + j), s1 = __ldg(R.succ_ptr + j + 1);
      for (uint32_t q = s0; q < s1; ++q) {
        const uint32_t v = __ldg(R.succ + q) & 0xFFFFu;
        const uint32_t sh = (v & 3u) * 8;
        const uint32_t word = CNT[(v >> 2) * S] - (1u << sh);
        CNT[(v >> 2) * S] = word;
        if (((word >> sh) & 0xFFu) == 0u) {
          RB[(v >> 5) * S] |= 1u << (v & 31u);
          if (MASK) wmask |= 1u << (v >> 5);
        }
      }
    }
    if (REC) rec[k] = (uint16_t)j;
    prev = j;
  }
  AntOut o;
#pragma unroll
  for (int c = 0; c < 4; ++c) o.prp[c] = prp[c];
  o.cost = cost_rp(cfg.cost_mode, prp);
  return o;
}

// ------------------------------------------------------------ pass-2 ant
// ILP pass (L108, L118, L147-L164, L200-L206; R19-R24).  t is the cycle and
// the Philox step; stalls skip ahead without drawing.
template <bool MASK, bool REC>
__device__ __forceinline__ AntOut ant_pass2(const RV &R, const uint16_t *__restrict__ tau,
                                            uint32_t *st, const uint32_t S, const uint32_t ant,
                                            const uint32_t iter, const RunCfg &cfg,
                                            const uint32_t tgt[4], uint32_t *prune_len, const bool prune,
                                            uint16_t *rec_o, uint32_t *rec_c) {
  const uint32_t n = R.n, nwr = R.nwr;
  uint32_t *RB = st;             // avail bitset: all preds placed, not placed
  uint32_t *RC = st + nwr * S;   // per instruction: ready time << 8 | preds left
  uint32_t *REM = RC + n * S;
  uint32_t wmask = 0;
  for (uint32_t w = 0; w < nwr; ++w) {
    const uint32_t x = __ldg(R.rb0 + w);
    RB[w * S] = x;
    if (MASK && x) wmask |= 1u << w;
  }
  for (uint32_t w = 0; w < ((n + 3) >> 2); ++w) {
    const uint32_t x = __ldg(R.cnt0 + w);
#pragma unroll
    for (uint32_t b = 0; b < 4; ++b)
      if (w * 4 + b < n) RC[(w * 4 + b) * S] = byte_of(x, b);
  }
  for (uint32_t w = 0; w < ((R.nmu + 1) >> 1); ++w) REM[w * S] = __ldg(R.rem0 + w);
  uint32_t live[4], prp[4];
#pragma unroll
  for (int c = 0; c < 4; ++c) live[c] = prp[c] = R.livein[c];
  const uint32_t group = ant / cfg.group_size;
  const bool stall_en = (group % cfg.stall_mod) == cfg.stall_rem;  // R23
  const uint32_t c2 = 0x80000000u | iter;
  uint32_t t = 0, placed = 0, kopt = 0, prev = n, turn = 0;
  AntOut o;
  while (placed < n) {
    if (prune && ((++turn & 7u) == 0u)) {  // R24: winner-invariant prune
      const uint32_t bl = *(volatile uint32_t *)prune_len;
      if (t + (n - placed) > bl) {
        o.cost = kInvalid;
        return o;
      }
    }
    const uint16_t *trow = tau + (size_t)prev * n;
    uint32_t nr = 0, nf = 0, ns = 0, min_s = 0xFFFFFFFFu;
    bool all_f_inc = true, some_s_dec = false;
    uint32_t best_s = 0, best_j = 0;
    uint64_t sum = 0;
    // Delta_c(j) = defs_c - kills_c at the current state; feasible iff
    // live_c + Delta_c <= target_c for every class (R21).
#define ACO_DELTA(J, D)                                                       \
  int D[4];                                                                   \
  {                                                                           \
    const uint4 inf = __ldg(R.info + J);                                      \
    _Pragma("unroll") for (int c = 0; c < 4; ++c) D[c] =                      \
        (int)byte_of(inf.x, c) - (int)byte_of(inf.z, c);                      \
    const uint32_t m0 = inf.w >> 8, mc = inf.w & 0xFFu;                       \
    for (uint32_t q = 0; q < mc; ++q) {                                       \
      const uint32_t e = __ldg(R.muse + m0 + q);                              \
      if (rem_get(REM, S, e & 0xFFFFu) == 1u) {                               \
        const uint32_t cls = e >> 16;                                         \
        _Pragma("unroll") for (int c = 0; c < 4; ++c) D[c] -= (cls == (uint32_t)c); \
      }                                                                       \
    }                                                                         \
  }
#define ACO_FEASIBLE(D, OK)                                                   \
  bool OK = true;                                                             \
  _Pragma("unroll") for (int c = 0; c < 4; ++c) OK =                          \
      OK && ((uint32_t)((int)live[c] + D[c]) <= tgt[c]);
    ACO_FOR_EACH_BIT(MASK, wmask, RB, S, nwr, j, {
      const uint32_t rdy = RC[j * S] >> 8;
      if (rdy <= t) {
        ++nr;
        ACO_DELTA(j, d)
        ACO_FEASIBLE(d, ok)
        if (ok) {
          ++nf;
          const uint32_t s = (uint32_t)__ldg(trow + j) * (uint32_t)__ldg(R.eta2 + j);
          if (s > best_s) {
            best_s = s;
            best_j = j;
          }
          sum += s;
          if (stall_en) {
            int mx = d[0];
            _Pragma("unroll") for (int c = 1; c < 4; ++c) mx = max(mx, d[c]);
            if (!(mx > 0)) all_f_inc = false;
          }
        }
      } else {
        ++ns;
        min_s = min(min_s, rdy);
        if (stall_en && !some_s_dec) {
          ACO_DELTA(j, d)
          int mn = d[0];
          _Pragma("unroll") for (int c = 1; c < 4; ++c) mn = min(mn, d[c]);
          if (mn < 0) some_s_dec = true;
        }
      }
    })
    if (nr == 0) {  // necessary stall (L153): skip ahead
      t = min_s;
      continue;
    }
    if (nf == 0) {
      if (stall_en && ns > 0) {  // forced optional stall (L155, R22)
        kopt += min_s - t;
        t = min_s;
        continue;
      }
      o.cost = kInvalid;  // the ant is terminated (L149)
      return o;
    }
    uint4 x = make_uint4(0, 0, 0, 0);
    bool have_x = false;
    if (stall_en && ns > 0 && all_f_inc && some_s_dec) {  // discretionary stall (L157-L164)
      x = philox(t, ant, c2, R.region_id, cfg.seed);
      have_x = true;
      const uint32_t thr = (kopt + 1 >= 32) ? 0u : (0xFFFFFFFFu >> (kopt + 1));
      if (x.z < thr) {
        ++kopt;
        ++t;
        continue;
      }
    }
    const uint4 g = philox(t, 0x80000000u | group, c2, R.region_id, cfg.seed);
    if (!((uint64_t)g.x < cfg.q0_t)) {  // explore: roulette over F (R27)
      if (!have_x) x = philox(t, ant, c2, R.region_id, cfg.seed);
      const uint64_t r = __umul64hi(((uint64_t)x.y << 32) | x.x, sum);
      uint64_t pre = 0;
      ACO_FOR_EACH_BIT(MASK, wmask, RB, S, nwr, j, {
        if ((RC[j * S] >> 8) <= t) {
          ACO_DELTA(j, d)
          ACO_FEASIBLE(d, ok)
          if (ok) {
            pre += (uint32_t)__ldg(trow + j) * (uint32_t)__ldg(R.eta2 + j);
            if (pre > r) {
              best_j = j;
              ACO_BREAK_SCAN
            }
          }
        }
      })
    }
#undef ACO_DELTA
#undef ACO_FEASIBLE
    // ---- commit best_j at cycle t
    const uint32_t j = best_j;
    {
      const uint32_t wi = j >> 5;
      const uint32_t nw = RB[wi * S] & ~(1u << (j & 31u));
      RB[wi * S] = nw;
      if (MASK && !nw) wmask &= ~(1u << wi);
    }
    const uint4 inf = __ldg(R.info + j);
#pragma unroll
    for (int c = 0; c < 4; ++c) live[c] -= byte_of(inf.z, c);
    {
      const uint32_t m0 = inf.w >> 8, mc = inf.w & 0xFFu;
      for (uint32_t q = 0; q < mc; ++q) {
        const uint32_t e = __ldg(R.muse + m0 + q);
        const uint32_t mm = e & 0xFFFFu, cls = e >> 16;
        const uint32_t sh = (mm & 1u) * 16;
        const uint32_t word = REM[(mm >> 1) * S];
        REM[(mm >> 1) * S] = word - (1u << sh);
        if (((word >> sh) & 0xFFFFu) == 1u) {
#pragma unroll
          for (int c = 0; c < 4; ++c) live[c] -= (cls == (uint32_t)c);
        }
      }
    }
#pragma unroll
    for (int c = 0; c < 4; ++c) {
      live[c] += byte_of(inf.x, c);
      prp[c] = max(prp[c], live[c]);
      live[c] -= byte_of(inf.y, c);
    }
    {
      const uint32_t s0 = __ldg(R.succ_ptr + j), s1 = __ldg(R.succ_ptr + j + 1);
      for (uint32_t q = s0; q < s1; ++q) {
        const uint32_t e = __ldg(R.succ + q);
        const uint32_t v = e & 0xFFFFu, lat = e >> 16;
        const uint32_t w = RC[v * S];
        const uint32_t rdy = max(w >> 8, t + lat);
        const uint32_t cnt = (w & 0xFFu) - 1u;
        RC[v * S] = (rdy << 8) | cnt;
        if (cnt == 0u) {
          RB[(v >> 5) * S] |= 1u << (v & 31u);
          if (MASK) wmask |= 1u << (v >> 5);
        }
      }
    }
    if (REC) {
      rec_o[placed] = (uint16_t)j;
      rec_c[placed] = t;
    }
    ++placed;
    prev = j;
    ++t;
  }
  if (prune) atomicMin(prune_len, t);
#pragma unroll
  for (int c = 0; c < 4; ++c) o.prp[c] = prp[c];
  o.cost = t;  // length = last issue cycle + 1 (R20)
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

template <int PASS, bool MASK, bool DUMP>
__global__ void __launch_bounds__(256) k_construct(KArgs A, const BlockItem *__restrict__ items,
                                                   uint32_t iter) {
  const BlockItem it = items[blockIdx.x];
  RegionState &rs = A.state[it.region];
  if (!rs.active) return;
  const uint32_t ant = it.ant0 + threadIdx.x;
  if (ant >= A.cfg.ants) return;
  const RV R = make_rv(A.arena, A.regions + it.region);
  const RegionWs &W = A.rws[it.region];
  const uint16_t *tau = (const uint16_t *)(A.ws + W.o_tau);
  extern __shared__ uint32_t smem[];
  uint32_t *st = smem + threadIdx.x;
  const uint32_t S = blockDim.x;
  AntOut o;
  if (PASS == 1) {
    uint16_t *rec = nullptr;
    if (DUMP && A.dump_order)
      rec = A.dump_order + (size_t)iter * A.cfg.dump_slice + W.o_dump + (size_t)ant * R.n;
    o = ant_pass1<MASK, DUMP>(R, tau, st, S, ant, iter, A.cfg, false, rec);
  } else {
    uint32_t tgt[4];
#pragma unroll
    for (int c = 0; c < 4; ++c) tgt[c] = rs.target[c];
    uint16_t *rec_o = nullptr;
    uint32_t *rec_c = nullptr;
    uint16_t scratch_o[1];
    uint32_t scratch_c[1];
    if (DUMP) {
      const size_t base = ((size_t)A.cfg.iterations + iter) * A.cfg.dump_slice + W.o_dump + (size_t)ant * R.n;
      rec_o = A.dump_order ? A.dump_order + base : scratch_o;
      rec_c = A.dump_cycle ? A.dump_cycle + base : scratch_c;
      if (!A.dump_order || !A.dump_cycle) rec_o = nullptr;
    }
    const bool prune = !DUMP && !(A.cfg.flags & ACO_FLAG_NO_PRUNE);
    if (DUMP && rec_o)
      o = ant_pass2<MASK, true>(R, tau, st, S, ant, iter, A.cfg, tgt, &rs.prune_len, prune, rec_o, rec_c);
    else
      o = ant_pass2<MASK, false>(R, tau, st, S, ant, iter, A.cfg, tgt, &rs.prune_len, prune, nullptr,
                                 nullptr);
  }
  uint32_t *costs = (uint32_t *)(A.ws + W.o_cost);
  costs[ant] = o.cost;
  if (DUMP && A.dump_cost)
    A.dump_cost[(((size_t)(PASS - 1) * A.cfg.iterations + iter) * A.cfg.count + it.region) * A.cfg.ants + ant] =
        o.cost;
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

// Evaporate + deposit + clamp over the (n+1) x n table (R6-R9), 8 entries
// per 16-byte access; next[i] = the winner's successor of i (0xFFFF: none).
__device__ void tau_update(uint16_t *tau, uint32_t n, uint32_t len, const uint16_t *next,
                           const RunCfg &cfg) {
  const uint32_t total = (n + 1) * n;
  uint4 *t4 = (uint4 *)tau;
  for (uint32_t v = threadIdx.x; v < len / 8; v += blockDim.x) {
    uint4 q = t4[v];
    uint32_t w[4] = {q.x, q.y, q.z, q.w};
    const uint32_t e0 = v * 8;
    uint32_t i = e0 / n, j = e0 - i * n;
    uint32_t nx = i <= n ? next[i] : 0xFFFFu;
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const uint32_t e = e0 + u;
      if (e < total) {
        const uint32_t sh = (u & 1) * 16;
        uint32_t x = (w[u >> 1] >> sh) & 0xFFFFu;
        x = (x * cfg.rho_q16) >> 16;
        if (nx == j) x += cfg.delta;
        x = min(max(x, cfg.tau_min), cfg.tau_max);
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

// Per-region initialisation: tau0, the greedy pass-1 heuristic schedule
// (R28: the q0 = 1 ant on a uniform tau), LB check (L251).
template <bool MASK>
__global__ void __launch_bounds__(128) k_init(KArgs A) {
  const uint32_t r = blockIdx.x;
  const RV R = make_rv(A.arena, A.regions + r);
  const RegionWs &W = A.rws[r];
  RegionState &rs = A.state[r];
  uint16_t *tau = (uint16_t *)(A.ws + W.o_tau);
  extern __shared__ uint32_t smem[];
  tau_fill(tau, W.tau_len, A.cfg.tau0);
  __syncthreads();
  if (threadIdx.x == 0) {
    uint16_t *gb1 = (uint16_t *)(A.ws + W.o_gb1);
    AntOut o = ant_pass1<MASK, true>(R, tau, smem, 1, 0, 0, A.cfg, true, gb1);
    const RegionDev *rd = A.regions + r;
    uint32_t lbv[4];
    for (int c = 0; c < 4; ++c) lbv[c] = rd->lbvec[c];
    rs.lb_cost = cost_rp(A.cfg.cost_mode, lbv);
    rs.init[0] = rs.best[0] = o.cost;
    for (int c = 0; c < 4; ++c) rs.prp1[c] = rs.prp2[c] = o.prp[c];
    rs.iters[0] = rs.iters[1] = 0;
    rs.no_imp = 0;
    rs.prune_len = kInvalid;
    rs.hash = 0xcbf29ce484222325ull;
    rs.active = (A.cfg.pass_mask & 1u) && A.cfg.iterations > 0 &&
                !(A.cfg.stop_at_lb && o.cost == rs.lb_cost);
  }
}

// Pass transition (L147; R13, R18, R29): target from the pass-1 best, the
// initial pass-2 schedule = ASAP(pass-1 best order), tau reset.
__global__ void __launch_bounds__(128) k_pass2_init(KArgs A) {
  const uint32_t r = blockIdx.x;
  const RV R = make_rv(A.arena, A.regions + r);
  const RegionWs &W = A.rws[r];
  RegionState &rs = A.state[r];
  uint16_t *tau = (uint16_t *)(A.ws + W.o_tau);
  extern __shared__ uint32_t smem[];  // rdy[n]
  tau_fill(tau, W.tau_len, A.cfg.tau0);
  for (uint32_t i = threadIdx.x; i < R.n; i += blockDim.x) smem[i] = 0;
  __syncthreads();
  if (threadIdx.x == 0) {
    const uint16_t *gb1 = (const uint16_t *)(A.ws + W.o_gb1);
    uint16_t *gb2 = (uint16_t *)(A.ws + W.o_gb2);
    uint32_t *gb2c = (uint32_t *)(A.ws + W.o_gb2c);
    uint32_t t = 0;
    bool first = true;
    for (uint32_t k = 0; k < R.n; ++k) {
      const uint32_t j = gb1[k];
      t = first ? smem[j] : max(t + 1, smem[j]);
      first = false;
      gb2[k] = (uint16_t)j;
      gb2c[k] = t;
      const uint32_t s0 = __ldg(R.succ_ptr + j), s1 = __ldg(R.succ_ptr + j + 1);
      for (uint32_t q = s0; q < s1; ++q) {
        const uint32_t e = __ldg(R.succ + q);
        const uint32_t v = e & 0xFFFFu;
        smem[v] = max(smem[v], t + (e >> 16));
      }
    }
    const uint32_t len = R.n ? t + 1 : 0;
    rs.init[1] = rs.best[1] = len;
    for (int c = 0; c < 4; ++c) rs.prp2[c] = rs.prp1[c];
    uint32_t tgt[4];
    target_of(A.cfg.cost_mode, rs.prp1, tgt);
    for (int c = 0; c < 4; ++c) rs.target[c] = tgt[c];
    rs.no_imp = 0;
    rs.prune_len = kInvalid;
    const uint32_t lb_len = A.regions[r].lb_len;
    rs.active = (A.cfg.pass_mask & 2u) && A.cfg.iterations > 0 && !(A.cfg.stop_at_lb && len == lb_len);
  }
}

// End of an iteration for one region (L137-L139).
template <int PASS, bool MASK>
__global__ void __launch_bounds__(256) k_finalize(KArgs A, uint32_t iter) {
  const uint32_t r = blockIdx.x;
  RegionState &rs = A.state[r];
  if (!rs.active) return;
  const RV R = make_rv(A.arena, A.regions + r);
  const RegionWs &W = A.rws[r];
  const uint32_t n = R.n;
  uint16_t *tau = (uint16_t *)(A.ws + W.o_tau);
  const uint32_t *costs = (const uint32_t *)(A.ws + W.o_cost);
  extern __shared__ uint32_t smem[];
  __shared__ unsigned long long s_red[8];
  __shared__ uint32_t s_flag;
  // ---- argmin over (cost, ant) (R10): packed u64 keys, warp shuffles
  unsigned long long best = ~0ull;
  for (uint32_t a = threadIdx.x; a < A.cfg.ants; a += blockDim.x)
    best = min(best, ((unsigned long long)costs[a] << 32) | a);
#pragma unroll
  for (int off = 16; off; off >>= 1) best = min(best, __shfl_xor_sync(0xFFFFFFFFu, best, off));
  if ((threadIdx.x & 31) == 0) s_red[threadIdx.x >> 5] = best;
  __syncthreads();
  if (threadIdx.x == 0) {
    for (uint32_t w = 1; w < blockDim.x / 32; ++w) best = min(best, s_red[w]);
    s_red[0] = best;
  }
  __syncthreads();
  best = s_red[0];
  const uint32_t wcost = (uint32_t)(best >> 32), want = (uint32_t)best;
  const bool have = wcost != kInvalid;
  // smem: [ant state | order u16[n] | cycle u32[n] | next u16[n+1]]
  const uint32_t words = ant_words(PASS, n, R.nwr, R.nmu);
  uint32_t *cyc = smem + words;
  uint16_t *ord = (uint16_t *)(cyc + n);
  uint16_t *next = ord + ((n + 1) & ~1u);
  // ---- replay the winner (deterministic: same tau, same Philox counters)
  if (have && threadIdx.x == 0) {
    AntOut o;
    if (PASS == 1) {
      o = ant_pass1<MASK, true>(R, tau, smem, 1, want, iter, A.cfg, false, ord);
    } else {
      uint32_t tgt[4];
      for (int c = 0; c < 4; ++c) tgt[c] = rs.target[c];
      o = ant_pass2<MASK, true>(R, tau, smem, 1, want, iter, A.cfg, tgt, nullptr, false, ord, cyc);
    }
    s_red[1] = o.prp[0] | ((unsigned long long)o.prp[1] << 32);
    s_red[2] = o.prp[2] | ((unsigned long long)o.prp[3] << 32);
  }
  __syncthreads();
  for (uint32_t i = threadIdx.x; i <= n; i += blockDim.x) next[i] = 0xFFFFu;
  __syncthreads();
  if (have) {
    for (uint32_t k = threadIdx.x; k + 1 < n; k += blockDim.x) next[ord[k]] = ord[k + 1];
    if (threadIdx.x == 0 && n) next[n] = ord[0];
  }
  __syncthreads();
  if (n) tau_update(tau, n, W.tau_len, next, A.cfg);
  // ---- epilogue (first thread, L139)
  if (threadIdx.x == 0) {
    rs.hash = fnv_u32(fnv_u32(fnv_u32(fnv_u32(rs.hash, PASS), iter), have ? wcost : kInvalid),
                      have ? want : kInvalid);
    const bool improved = have && wcost < rs.best[PASS - 1];  // strict (R11)
    s_flag = improved;
    if (improved) {
      rs.best[PASS - 1] = wcost;
      rs.no_imp = 0;
      uint32_t *prp = PASS == 1 ? rs.prp1 : rs.prp2;
      prp[0] = (uint32_t)s_red[1];
      prp[1] = (uint32_t)(s_red[1] >> 32);
      prp[2] = (uint32_t)s_red[2];
      prp[3] = (uint32_t)(s_red[2] >> 32);
    } else {
      rs.no_imp++;
    }
    rs.iters[PASS - 1] = iter + 1;
    const uint32_t lim = no_improve_limit(A.cfg, n);
    const uint32_t lb = PASS == 1 ? rs.lb_cost : A.regions[r].lb_len;
    if ((A.cfg.stop_at_lb && rs.best[PASS - 1] == lb) || (lim > 0 && rs.no_imp >= lim) ||
        iter + 1 >= A.cfg.iterations)
      rs.active = 0;
    rs.prune_len = kInvalid;
  }
  __syncthreads();
  if (s_flag) {
    if (PASS == 1) {
      uint16_t *gb1 = (uint16_t *)(A.ws + W.o_gb1);
      for (uint32_t k = threadIdx.x; k < n; k += blockDim.x) gb1[k] = ord[k];
    } else {
      uint16_t *gb2 = (uint16_t *)(A.ws + W.o_gb2);
      uint32_t *gb2c = (uint32_t *)(A.ws + W.o_gb2c);
      for (uint32_t k = threadIdx.x; k < n; k += blockDim.x) {
        gb2[k] = ord[k];
        gb2c[k] = cyc[k];
      }
    }
  }
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

static int check() {
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? 0 : (int)e;
}

int last_cuda_error() { return check(); }

int set_machine(const MachineDev &m) {
  if (cudaMemcpyToSymbol(c_mach, &m, sizeof(m)) != cudaSuccess) return 1;
  // allow large dynamic shared memory for every kernel variant
  const int big = 227 * 1024;
  cudaFuncSetAttribute(k_init<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaFuncSetAttribute(k_init<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaFuncSetAttribute(k_pass2_init, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaFuncSetAttribute(k_finalize<1, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaFuncSetAttribute(k_finalize<1, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaFuncSetAttribute(k_finalize<2, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  cudaFuncSetAttribute(k_finalize<2, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
#define ACO_ATTR(P, M, D) \
  cudaFuncSetAttribute(k_construct<P, M, D>, cudaFuncAttributeMaxDynamicSharedMemorySize, big);
  ACO_ATTR(1, true, false) ACO_ATTR(1, false, false) ACO_ATTR(1, true, true) ACO_ATTR(1, false, true)
  ACO_ATTR(2, true, false) ACO_ATTR(2, false, false) ACO_ATTR(2, true, true) ACO_ATTR(2, false, true)
#undef ACO_ATTR
  return check();
}

int launch_init(LaunchCtx &L, uint32_t smem, uint32_t max_n) {
  if (!L.cfg.count) return 0;
  cudaStream_t s = (cudaStream_t)L.stream;
  if (max_n <= 1024)
    k_init<true><<<L.cfg.count, 128, smem, s>>>(kargs(L));
  else
    k_init<false><<<L.cfg.count, 128, smem, s>>>(kargs(L));
  L.launches++;
  return check();
}

int launch_pass2_init(LaunchCtx &L, uint32_t smem, uint32_t max_n) {
  (void)max_n;
  if (!L.cfg.count) return 0;
  k_pass2_init<<<L.cfg.count, 128, smem, (cudaStream_t)L.stream>>>(kargs(L));
  L.launches++;
  return check();
}

int launch_construct(LaunchCtx &L, uint32_t pass, uint32_t iter, const ClassLaunch &c) {
  if (!c.n_blocks) return 0;
  cudaStream_t s = (cudaStream_t)L.stream;
  const bool mask = c.max_n <= 1024;
  const bool dump = (L.cfg.flags & ACO_FLAG_DUMP) != 0;
  KArgs a = kargs(L);
#define ACO_LAUNCH(P, M, D) k_construct<P, M, D><<<c.n_blocks, c.ants_pb, c.smem_bytes, s>>>(a, c.items, iter)
  if (pass == 1) {
    if (mask) {
      if (dump) ACO_LAUNCH(1, true, true); else ACO_LAUNCH(1, true, false);
    } else {
      if (dump) ACO_LAUNCH(1, false, true); else ACO_LAUNCH(1, false, false);
    }
  } else {
    if (mask) {
      if (dump) ACO_LAUNCH(2, true, true); else ACO_LAUNCH(2, true, false);
    } else {
      if (dump) ACO_LAUNCH(2, false, true); else ACO_LAUNCH(2, false, false);
    }
  }
#undef ACO_LAUNCH
  L.launches++;
  return check();
}

int launch_finalize(LaunchCtx &L, uint32_t pass, uint32_t iter, uint32_t smem, uint32_t max_n) {
  if (!L.cfg.count) return 0;
  cudaStream_t s = (cudaStream_t)L.stream;
  const bool mask = max_n <= 1024;
  KArgs a = kargs(L);
  if (pass == 1) {
    if (mask) k_finalize<1, true><<<L.cfg.count, 256, smem, s>>>(a, iter);
    else k_finalize<1, false><<<L.cfg.count, 256, smem, s>>>(a, iter);
  } else {
    if (mask) k_finalize<2, true><<<L.cfg.count, 256, smem, s>>>(a, iter);
    else k_finalize<2, false><<<L.cfg.count, 256, smem, s>>>(a, iter);
  }
  L.launches++;
  return check();
}

}  // namespace aco
