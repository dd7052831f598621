/*
 * aco_oracle.c -- plain, slow, sequential CPU oracle for ACO-based
 * register-pressure-aware instruction scheduling.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load this code.  It
 * shares no code, header, table or constant generator with the CUDA path.
 *
 * Source: Shobaki et al., "Instruction Scheduling for the GPU on the GPU",
 * CGO 2024 -- /root/reference/PAPER.md ("L<n>" = line n).  The paper defers
 * the selection, deposit and decay formulas to its ref. [11] (L114, L116,
 * L120); every point it leaves open is fixed by a reading R<k> in DESIGN.md
 * section 3 and cited where it is used below.
 *
 * Everything is integer arithmetic (R36): pheromone tau is u16 in units of
 * 2^-12, heuristic eta is in [1, 65535], a score tau*eta fits in u32, sums
 * are u64 and the roulette draw uses a 128-bit product.
 *
 * Parity status of every function is listed in DESIGN.md section 4 (pins).
 */
#include "aco_oracle.h"

#include <pthread.h>
#include <stdlib.h>
#include <string.h>

#define ROOT_ROW(n) (n) /* the extra pheromone row for the first pick (R5) */
#define INVALID_COST 0xFFFFFFFFu /* R35 */
#define FLAG_LIVE_IN 1u
#define FLAG_LIVE_OUT 2u

/* ------------------------------------------------------------------------ */
/* Philox4x32-10, R26 (Random123; Salmon et al. SC'11).                      */
/* ------------------------------------------------------------------------ */
void orc_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]) {
  uint32_t c0 = ctr[0], c1 = ctr[1], c2 = ctr[2], c3 = ctr[3];
  uint32_t k0 = key[0], k1 = key[1];
  for (int round = 0; round < 10; ++round) {
    if (round > 0) {
      k0 += 0x9E3779B9u;
      k1 += 0xBB67AE85u;
    }
    uint64_t p0 = (uint64_t)0xD2511F53u * c0;
    uint64_t p1 = (uint64_t)0xCD9E8D57u * c2;
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    uint32_t n0 = hi1 ^ c1 ^ k0;
    uint32_t n1 = lo1;
    uint32_t n2 = hi0 ^ c3 ^ k1;
    uint32_t n3 = lo0;
    c0 = n0; c1 = n1; c2 = n2; c3 = n3;
  }
  out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* Counter layout (R26): ant draw   = (step, ant, (pass-1)<<31 | iter, region)
 *                       group coin = (step, 0x80000000 | group, ..., region) */
static void draw_ant(uint64_t seed, uint32_t region, uint32_t pass, uint32_t iter,
                     uint32_t ant, uint32_t step, uint32_t out[4]) {
  uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
  uint32_t ctr[4] = {step, ant, ((pass - 1u) << 31) | iter, region};
  orc_philox4x32_10(ctr, key, out);
}

static uint32_t draw_group_coin(uint64_t seed, uint32_t region, uint32_t pass, uint32_t iter,
                                uint32_t group, uint32_t step) {
  uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32)};
  uint32_t ctr[4] = {step, 0x80000000u | group, ((pass - 1u) << 31) | iter, region};
  uint32_t out[4];
  orc_philox4x32_10(ctr, key, out);
  return out[0];
}

/* ------------------------------------------------------------------------ */
/* Region model: DDG (L62) + Def/Use sets (L66).                             */
/* ------------------------------------------------------------------------ */
typedef struct {
  uint32_t n, n_regs, n_classes;
  const orc_region *src;
  /* successor / predecessor adjacency, built from the edge list */
  uint32_t *succ_ptr, *succ, *succ_lat;
  uint32_t *pred_ptr, *pred, *pred_lat;
  uint32_t *indeg;
  uint32_t *nuses;    /* number of instructions using each register */
  uint32_t *def_by;   /* defining instruction or UINT32_MAX */
  uint32_t *cp;       /* critical-path height, R4 */
  uint32_t cp_max;
  uint32_t max_luc;   /* max over j of #{r in Use(j): not LIVE_OUT}, R4 */
  uint32_t livein[4]; /* live-in registers per class */
} model;

static void model_free(model *m) {
  free(m->succ_ptr); free(m->succ); free(m->succ_lat);
  free(m->pred_ptr); free(m->pred); free(m->pred_lat);
  free(m->indeg); free(m->nuses); free(m->def_by); free(m->cp);
  memset(m, 0, sizeof(*m));
}

/* Validation (R31-R34, R37, R38). Returns ORC_OK or a negative code. */
int orc_validate(const orc_region *r, uint32_t n_classes) {
  uint32_t n = r->n_insts;
  if (n_classes < 1 || n_classes > 4) return ORC_E_ARG;
  if (n > 65535u || r->n_regs > 16777215u) return ORC_E_TOO_LARGE;
  if (r->def_ptr[0] != 0 || r->use_ptr[0] != 0) return ORC_E_ARG;
  for (uint32_t j = 0; j < n; ++j)
    if (r->def_ptr[j + 1] < r->def_ptr[j] || r->use_ptr[j + 1] < r->use_ptr[j]) return ORC_E_ARG;
  for (uint32_t g = 0; g < r->n_regs; ++g)
    if (r->reg_class[g] >= n_classes || (r->reg_flags[g] & ~3u)) return ORC_E_ARG;
  for (uint32_t e = 0; e < r->n_edges; ++e) {
    if (r->edge_src[e] >= n || r->edge_dst[e] >= n) return ORC_E_ARG;
    if (r->edge_lat[e] > 65535u) return ORC_E_TOO_LARGE;
    if (r->edge_src[e] == r->edge_dst[e]) return ORC_E_DDG_CYCLE;
  }
  for (uint32_t j = 0; j < n; ++j) {
    for (uint32_t k = r->def_ptr[j]; k < r->def_ptr[j + 1]; ++k)
      if (r->def_reg[k] >= r->n_regs) return ORC_E_ARG;
    for (uint32_t k = r->use_ptr[j]; k < r->use_ptr[j + 1]; ++k)
      if (r->use_reg[k] >= r->n_regs) return ORC_E_ARG;
  }
  /* duplicate edges are rejected (R37): check with a per-source marker */
  uint32_t *mark = malloc(sizeof(uint32_t) * (n ? n : 1));
  uint32_t *deg = calloc(n + 1, sizeof(uint32_t));
  for (uint32_t j = 0; j < n; ++j) mark[j] = UINT32_MAX;
  int st = ORC_OK;
  for (uint32_t e = 0; e < r->n_edges; ++e) deg[r->edge_src[e]]++;
  /* bucket edges by source */
  uint32_t *ptr = calloc(n + 1, sizeof(uint32_t));
  for (uint32_t j = 0; j < n; ++j) ptr[j + 1] = ptr[j] + deg[j];
  uint32_t *fill = calloc(n + 1, sizeof(uint32_t));
  uint32_t *dst = malloc(sizeof(uint32_t) * (r->n_edges ? r->n_edges : 1));
  for (uint32_t e = 0; e < r->n_edges; ++e) {
    uint32_t s = r->edge_src[e];
    dst[ptr[s] + fill[s]++] = r->edge_dst[e];
  }
  for (uint32_t j = 0; j < n && st == ORC_OK; ++j)
    for (uint32_t k = ptr[j]; k < ptr[j + 1]; ++k) {
      if (mark[dst[k]] == j) { st = ORC_E_ARG; break; }
      mark[dst[k]] = j;
    }
  /* acyclicity: Kahn's algorithm (R31) */
  if (st == ORC_OK) {
    uint32_t *indeg = calloc(n + 1, sizeof(uint32_t));
    uint32_t *queue = malloc(sizeof(uint32_t) * (n ? n : 1));
    for (uint32_t e = 0; e < r->n_edges; ++e) indeg[r->edge_dst[e]]++;
    uint32_t head = 0, tail = 0;
    for (uint32_t j = 0; j < n; ++j) if (indeg[j] == 0) queue[tail++] = j;
    while (head < tail) {
      uint32_t j = queue[head++];
      for (uint32_t k = ptr[j]; k < ptr[j + 1]; ++k)
        if (--indeg[dst[k]] == 0) queue[tail++] = dst[k];
    }
    if (tail != n) st = ORC_E_DDG_CYCLE;
    free(indeg); free(queue);
  }
  /* single definition, no definition of a live-in register (R34) */
  uint32_t *def_by = NULL;
  if (st == ORC_OK) {
    def_by = malloc(sizeof(uint32_t) * (r->n_regs ? r->n_regs : 1));
    for (uint32_t g = 0; g < r->n_regs; ++g) def_by[g] = UINT32_MAX;
    for (uint32_t j = 0; j < n && st == ORC_OK; ++j)
      for (uint32_t k = r->def_ptr[j]; k < r->def_ptr[j + 1]; ++k) {
        uint32_t g = r->def_reg[k];
        if (def_by[g] != UINT32_MAX || (r->reg_flags[g] & FLAG_LIVE_IN)) { st = ORC_E_DDG_MULTIDEF; break; }
        def_by[g] = j;
      }
  }
  /* every use is of a live-in register or of a register defined by a direct
   * predecessor (R38) */
  if (st == ORC_OK) {
    for (uint32_t j = 0; j < n && st == ORC_OK; ++j)
      for (uint32_t k = r->use_ptr[j]; k < r->use_ptr[j + 1]; ++k) {
        uint32_t g = r->use_reg[k];
        if (r->reg_flags[g] & FLAG_LIVE_IN) continue;
        uint32_t d = def_by[g];
        if (d == UINT32_MAX) { st = ORC_E_ARG; break; }
        int found = 0;
        for (uint32_t q = ptr[d]; q < ptr[d + 1]; ++q) if (dst[q] == j) found = 1;
        if (!found) { st = ORC_E_DDG_USE_NO_EDGE; break; }
      }
  }
  free(def_by); free(mark); free(deg); free(ptr); free(fill); free(dst);
  return st;
}

/* Is register g used by instruction j?  Use is a set (R33): duplicates in the
 * input list count once. */
static int first_occurrence(const orc_region *r, uint32_t j, uint32_t k) {
  for (uint32_t q = r->use_ptr[j]; q < k; ++q)
    if (r->use_reg[q] == r->use_reg[k]) return 0;
  return 1;
}

/* General machine model (L64; R42).  issue_width <= 1: single issue, any
 * type (R32).  Otherwise at most issue_width instructions per cycle and at
 * most type_slots[y] of type y. */
static uint32_t m_width(const orc_machine *m) { return m->issue_width > 1 ? m->issue_width : 1u; }
static uint32_t m_slots(const orc_machine *m, uint32_t y) {
  if (m->issue_width <= 1) return 1u;
  return m->type_slots[y];
}
static uint32_t itype(const orc_region *r, uint32_t j) { return r->inst_type ? r->inst_type[j] : 0u; }

/* The machine model and instruction types are consistent (R42). */
static int machine_check(const orc_region *r, const orc_machine *m) {
  if (m->issue_width > 1) {
    if (m->n_types < 1 || m->n_types > 4) return ORC_E_ARG;
    for (uint32_t y = 0; y < m->n_types; ++y)
      if (m->type_slots[y] < 1) return ORC_E_ARG;
  }
  uint32_t nt = m->issue_width > 1 ? m->n_types : 4u;
  if (r->inst_type)
    for (uint32_t j = 0; j < r->n_insts; ++j)
      if (r->inst_type[j] >= nt) return ORC_E_ARG;
  return ORC_OK;
}

static int model_build(model *m, const orc_region *r, uint32_t n_classes) {
  memset(m, 0, sizeof(*m));
  int st = orc_validate(r, n_classes);
  if (st != ORC_OK) return st;
  uint32_t n = r->n_insts;
  m->n = n; m->n_regs = r->n_regs; m->n_classes = n_classes; m->src = r;
  m->succ_ptr = calloc(n + 1, sizeof(uint32_t));
  m->pred_ptr = calloc(n + 1, sizeof(uint32_t));
  m->succ = malloc(sizeof(uint32_t) * (r->n_edges + 1));
  m->succ_lat = malloc(sizeof(uint32_t) * (r->n_edges + 1));
  m->pred = malloc(sizeof(uint32_t) * (r->n_edges + 1));
  m->pred_lat = malloc(sizeof(uint32_t) * (r->n_edges + 1));
  m->indeg = calloc(n + 1, sizeof(uint32_t));
  m->nuses = calloc(r->n_regs + 1, sizeof(uint32_t));
  m->def_by = malloc(sizeof(uint32_t) * (r->n_regs + 1));
  m->cp = calloc(n + 1, sizeof(uint32_t));
  for (uint32_t e = 0; e < r->n_edges; ++e) {
    m->succ_ptr[r->edge_src[e] + 1]++;
    m->pred_ptr[r->edge_dst[e] + 1]++;
  }
  for (uint32_t j = 0; j < n; ++j) {
    m->succ_ptr[j + 1] += m->succ_ptr[j];
    m->pred_ptr[j + 1] += m->pred_ptr[j];
  }
  uint32_t *fs = calloc(n + 1, sizeof(uint32_t)), *fp = calloc(n + 1, sizeof(uint32_t));
  /* successor lists keep the input edge order; nothing depends on it */
  for (uint32_t e = 0; e < r->n_edges; ++e) {
    uint32_t s = r->edge_src[e], d = r->edge_dst[e];
    m->succ[m->succ_ptr[s] + fs[s]] = d;
    m->succ_lat[m->succ_ptr[s] + fs[s]++] = r->edge_lat[e];
    m->pred[m->pred_ptr[d] + fp[d]] = s;
    m->pred_lat[m->pred_ptr[d] + fp[d]++] = r->edge_lat[e];
    m->indeg[d]++;
  }
  free(fs); free(fp);
  for (uint32_t g = 0; g < r->n_regs; ++g) m->def_by[g] = UINT32_MAX;
  for (uint32_t j = 0; j < n; ++j) {
    for (uint32_t k = r->def_ptr[j]; k < r->def_ptr[j + 1]; ++k) m->def_by[r->def_reg[k]] = j;
    for (uint32_t k = r->use_ptr[j]; k < r->use_ptr[j + 1]; ++k)
      if (first_occurrence(r, j, k)) m->nuses[r->use_reg[k]]++;
  }
  for (uint32_t g = 0; g < r->n_regs; ++g)
    if (r->reg_flags[g] & FLAG_LIVE_IN) m->livein[r->reg_class[g]]++;
  orc_critical_path(r, m->cp);
  m->cp_max = 0;
  for (uint32_t j = 0; j < n; ++j) if (m->cp[j] > m->cp_max) m->cp_max = m->cp[j];
  m->max_luc = 0;
  for (uint32_t j = 0; j < n; ++j) {
    uint32_t c = 0;
    for (uint32_t k = r->use_ptr[j]; k < r->use_ptr[j + 1]; ++k)
      if (first_occurrence(r, j, k) && !(r->reg_flags[r->use_reg[k]] & FLAG_LIVE_OUT)) c++;
    if (c > m->max_luc) m->max_luc = c;
  }
  return ORC_OK;
}

/* CP(j) = max over edges j->s of lat(j,s) + CP(s); 0 for sinks (R4, [1]).
 * Computed by repeated relaxation in reverse topological order. */
int orc_critical_path(const orc_region *r, uint32_t *cp) {
  uint32_t n = r->n_insts;
  uint32_t *outdeg = calloc(n + 1, sizeof(uint32_t));
  uint32_t *order = malloc(sizeof(uint32_t) * (n + 1));
  uint32_t *indeg = calloc(n + 1, sizeof(uint32_t));
  for (uint32_t e = 0; e < r->n_edges; ++e) indeg[r->edge_dst[e]]++;
  /* topological order by Kahn (plain O(n*E)) */
  uint32_t cnt = 0;
  char *done = calloc(n + 1, 1);
  while (cnt < n) {
    int progressed = 0;
    for (uint32_t j = 0; j < n; ++j) {
      if (done[j] || indeg[j]) continue;
      done[j] = 1; order[cnt++] = j; progressed = 1;
      for (uint32_t e = 0; e < r->n_edges; ++e)
        if (r->edge_src[e] == j) indeg[r->edge_dst[e]]--;
    }
    if (!progressed) break;
  }
  for (uint32_t j = 0; j < n; ++j) cp[j] = 0;
  for (uint32_t q = cnt; q-- > 0;) {
    uint32_t j = order[q];
    for (uint32_t e = 0; e < r->n_edges; ++e)
      if (r->edge_src[e] == j) {
        uint32_t v = r->edge_lat[e] + cp[r->edge_dst[e]];
        if (v > cp[j]) cp[j] = v;
      }
  }
  free(outdeg); free(order); free(indeg); free(done);
  return cnt == n ? ORC_OK : ORC_E_DDG_CYCLE;
}

/* ------------------------------------------------------------------------ */
/* Register-pressure simulator (L66, L70; R14, R15).                         */
/* ------------------------------------------------------------------------ */
typedef struct {
  uint32_t *rem;     /* remaining (unscheduled) users of each register */
  uint32_t live[4];  /* live registers per class */
  uint32_t prp[4];   /* peak so far per class */
} rp_state;

static void rp_init(const model *m, rp_state *s) {
  for (uint32_t g = 0; g < m->n_regs; ++g) s->rem[g] = m->nuses[g];
  for (uint32_t c = 0; c < 4; ++c) {
    s->live[c] = m->livein[c]; /* live-in registers are live at entry (R15) */
    s->prp[c] = s->live[c];    /* and the entry point counts for the peak */
  }
}

/* kills_c(j): registers of class c whose last remaining use is j and that
 * are not live-out (R14). */
static uint32_t rp_kills(const model *m, const rp_state *s, uint32_t j, uint32_t c) {
  const orc_region *r = m->src;
  uint32_t k_c = 0;
  for (uint32_t k = r->use_ptr[j]; k < r->use_ptr[j + 1]; ++k) {
    if (!first_occurrence(r, j, k)) continue;
    uint32_t g = r->use_reg[k];
    if (r->reg_class[g] == c && s->rem[g] == 1 && !(r->reg_flags[g] & FLAG_LIVE_OUT)) k_c++;
  }
  return k_c;
}

static uint32_t rp_defs(const model *m, uint32_t j, uint32_t c) {
  const orc_region *r = m->src;
  uint32_t d = 0;
  for (uint32_t k = r->def_ptr[j]; k < r->def_ptr[j + 1]; ++k)
    if (r->reg_class[r->def_reg[k]] == c) d++;
  return d;
}

/* Delta_c(j) = |Def_c(j)| - kills_c(j): the change of live_c at j's peak point. */
static int64_t rp_delta(const model *m, const rp_state *s, uint32_t j, uint32_t c) {
  return (int64_t)rp_defs(m, j, c) - (int64_t)rp_kills(m, s, j, c);
}

/* issue(j): 1 kill last uses, 2 add defs, 3 update peaks, 4 drop dead defs (R14, R15). */
static void rp_issue(const model *m, rp_state *s, uint32_t j) {
  const orc_region *r = m->src;
  for (uint32_t k = r->use_ptr[j]; k < r->use_ptr[j + 1]; ++k) {
    if (!first_occurrence(r, j, k)) continue;
    uint32_t g = r->use_reg[k];
    s->rem[g]--;
    if (s->rem[g] == 0 && !(r->reg_flags[g] & FLAG_LIVE_OUT)) s->live[r->reg_class[g]]--;
  }
  for (uint32_t k = r->def_ptr[j]; k < r->def_ptr[j + 1]; ++k)
    s->live[r->reg_class[r->def_reg[k]]]++;
  for (uint32_t c = 0; c < 4; ++c)
    if (s->live[c] > s->prp[c]) s->prp[c] = s->live[c];
  for (uint32_t k = r->def_ptr[j]; k < r->def_ptr[j + 1]; ++k) {
    uint32_t g = r->def_reg[k];
    if (m->nuses[g] == 0 && !(r->reg_flags[g] & FLAG_LIVE_OUT)) s->live[r->reg_class[g]]--;
  }
}

/* LUC(j) = sum_c kills_c(j) (Last-Use-Count heuristic [61], L122). */
static uint32_t rp_luc(const model *m, const rp_state *s, uint32_t j) {
  uint32_t t = 0;
  for (uint32_t c = 0; c < m->n_classes; ++c) t += rp_kills(m, s, j, c);
  return t;
}

int orc_prp_of_order(const orc_region *r, uint32_t n_classes, const uint32_t *order, uint32_t *prp) {
  model m;
  int st = model_build(&m, r, n_classes);
  if (st != ORC_OK) return st;
  rp_state s;
  s.rem = calloc(m.n_regs + 1, sizeof(uint32_t));
  rp_init(&m, &s);
  for (uint32_t k = 0; k < m.n; ++k) rp_issue(&m, &s, order[k]);
  for (uint32_t c = 0; c < 4; ++c) prp[c] = s.prp[c];
  free(s.rem);
  model_free(&m);
  return ORC_OK;
}

/* ASAP timing of an order on the single-issue machine (L64; R20, R29):
 * c_0 = 0, c_k = max(c_{k-1} + 1, max_{p in preds(o_k)} c_p + lat(p, o_k));
 * length = c_last + 1. */
int64_t orc_asap(const orc_region *r, const uint32_t *order, uint32_t *cycle) {
  uint32_t n = r->n_insts;
  if (n == 0) return 0;
  uint32_t *c_of = malloc(sizeof(uint32_t) * n);
  char *placed = calloc(n, 1);
  int64_t prev = -1;
  for (uint32_t k = 0; k < n; ++k) {
    uint32_t j = order[k];
    int64_t t = prev + 1;
    for (uint32_t e = 0; e < r->n_edges; ++e)
      if (r->edge_dst[e] == j) {
        uint32_t p = r->edge_src[e];
        if (!placed[p]) { free(c_of); free(placed); return -1; } /* not topological */
        int64_t need = (int64_t)c_of[p] + r->edge_lat[e];
        if (need > t) t = need;
      }
    c_of[j] = (uint32_t)t;
    placed[j] = 1;
    cycle[k] = (uint32_t)t; /* cycle of the k-th instruction of the order */
    prev = t;
  }
  free(c_of); free(placed);
  return prev + 1;
}

/* ASAP timing of an order on the general machine model (R42, R29): in-order
 * issue; c_k = max(c_{k-1}, ready time of o_k), moved to c_{k-1} + 1 when
 * that cycle has no free slot for o_k (issue width or o_k's type); a later
 * cycle is empty.  For issue_width 1 this is orc_asap. */
int64_t orc_asap_m(const orc_region *r, const orc_machine *m, const uint32_t *order, uint32_t *cycle) {
  uint32_t n = r->n_insts;
  if (n == 0) return 0;
  uint32_t *c_of = malloc(sizeof(uint32_t) * n);
  char *placed = calloc(n, 1);
  int64_t prev = -1;
  uint32_t used = 0, used_t[4] = {0, 0, 0, 0};
  for (uint32_t k = 0; k < n; ++k) {
    uint32_t j = order[k], y = itype(r, j);
    int64_t t = prev < 0 ? 0 : prev;
    for (uint32_t e = 0; e < r->n_edges; ++e)
      if (r->edge_dst[e] == j) {
        uint32_t p = r->edge_src[e];
        if (!placed[p]) { free(c_of); free(placed); return -1; }
        int64_t need = (int64_t)c_of[p] + r->edge_lat[e];
        if (need > t) t = need;
      }
    if (t == prev && (used >= m_width(m) || used_t[y] >= m_slots(m, y))) t = prev + 1;
    if (t != prev) { used = 0; used_t[0] = used_t[1] = used_t[2] = used_t[3] = 0; }
    used++;
    used_t[y]++;
    c_of[j] = (uint32_t)t;
    placed[j] = 1;
    cycle[k] = (uint32_t)t;
    prev = t;
  }
  free(c_of); free(placed);
  return prev + 1;
}

/* ------------------------------------------------------------------------ */
/* Costs (L68-L74; R16-R18).                                                 */
/* ------------------------------------------------------------------------ */
uint32_t orc_occupancy(const orc_machine *m, uint32_t c, uint32_t prp) {
  for (uint32_t i = 0; i < m->step_count[c]; ++i)
    if (prp <= m->step_max[c][i]) return m->occ_max - i;
  return 0; /* beyond the table */
}

/* APRP(x) = the maximum PRP with the same occupancy as x (L70-L72). */
uint32_t orc_aprp(const orc_machine *m, uint32_t c, uint32_t prp) {
  for (uint32_t i = 0; i < m->step_count[c]; ++i)
    if (prp <= m->step_max[c][i]) return m->step_max[c][i];
  return prp;
}

uint32_t orc_cost_rp(const orc_machine *m, uint32_t mode, const uint32_t *prp) {
  uint32_t cost = 0;
  if (mode == 0) { /* PRP_SUM */
    for (uint32_t c = 0; c < m->n_classes; ++c) cost += prp[c];
  } else if (mode == 1) { /* APRP_SUM */
    for (uint32_t c = 0; c < m->n_classes; ++c) cost += orc_aprp(m, c, prp[c]);
  } else if (mode == 2) { /* OCC: occ_max - min_c occupancy */
    uint32_t occ = m->occ_max;
    for (uint32_t c = 0; c < m->n_classes; ++c) {
      uint32_t o = orc_occupancy(m, c, prp[c]);
      if (o < occ) occ = o;
    }
    cost = m->occ_max - occ;
  } else { /* PERP: excess over the per-class limit */
    for (uint32_t c = 0; c < m->n_classes; ++c)
      if (prp[c] > m->perp_limit[c]) cost += prp[c] - m->perp_limit[c];
  }
  return cost;
}

/* Pass-2 target per class from the pass-1 best PRP (L108, L147; R18). */
void orc_target(const orc_machine *m, uint32_t mode, const uint32_t *best, uint32_t *target) {
  for (uint32_t c = 0; c < 4; ++c) target[c] = 0xFFFFFFFFu;
  if (mode == 0) {
    for (uint32_t c = 0; c < m->n_classes; ++c) target[c] = best[c];
  } else if (mode == 1) {
    for (uint32_t c = 0; c < m->n_classes; ++c) target[c] = orc_aprp(m, c, best[c]);
  } else if (mode == 2) {
    uint32_t occ = m->occ_max;
    for (uint32_t c = 0; c < m->n_classes; ++c) {
      uint32_t o = orc_occupancy(m, c, best[c]);
      if (o < occ) occ = o;
    }
    for (uint32_t c = 0; c < m->n_classes; ++c) {
      if (occ == 0) { target[c] = 0xFFFFFFFFu; continue; }
      /* max{x : occ_c(x) >= occ}: the table entry for occupancy occ */
      uint32_t idx = m->occ_max - occ;
      uint32_t t = idx < m->step_count[c] ? m->step_max[c][idx] : m->step_max[c][m->step_count[c] - 1];
      target[c] = t > best[c] ? t : best[c];
    }
  } else {
    for (uint32_t c = 0; c < m->n_classes; ++c)
      target[c] = best[c] > m->perp_limit[c] ? best[c] : m->perp_limit[c];
  }
}

/* Lower bounds (L110, L251; R30) and ready-list UB (L180-L184; R31). */
int orc_lower_bounds(const orc_region *r, const orc_machine *mach, uint32_t mode,
                     uint32_t *lb_cost, uint32_t *lb_len, uint32_t *ub_ready) {
  model m;
  int st = model_build(&m, r, mach->n_classes);
  if (st != ORC_OK) return st;
  uint32_t n = m.n;
  uint32_t lbv[4] = {0, 0, 0, 0}, lo[4] = {0, 0, 0, 0};
  for (uint32_t c = 0; c < 4; ++c) lbv[c] = m.livein[c];
  for (uint32_t g = 0; g < r->n_regs; ++g)
    if (r->reg_flags[g] & FLAG_LIVE_OUT) lo[r->reg_class[g]]++;
  if (n > 0)
    for (uint32_t c = 0; c < 4; ++c) if (lo[c] > lbv[c]) lbv[c] = lo[c];
  for (uint32_t j = 0; j < n; ++j)
    for (uint32_t c = 0; c < m.n_classes; ++c) {
      uint32_t d = rp_defs(&m, j, c), u = 0;
      for (uint32_t k = r->use_ptr[j]; k < r->use_ptr[j + 1]; ++k)
        if (first_occurrence(r, j, k) && r->reg_class[r->use_reg[k]] == c) u++;
      if (d > lbv[c]) lbv[c] = d;
      if (u > lbv[c]) lbv[c] = u;
    }
  *lb_cost = orc_cost_rp(mach, mode, lbv);
  /* LB_len = max(1 + CPmax, ceil(n / w), max_y ceil(n_y / min(slots_y, w)))
   * (R30, R42); for the single-issue machine max(n, 1 + CPmax). */
  uint32_t w = m_width(mach);
  uint32_t l = (n + w - 1) / w;
  if (n > 0 && m.cp_max + 1 > l) l = m.cp_max + 1;
  if (w > 1)
    for (uint32_t y = 0; y < mach->n_types; ++y) {
      uint32_t ny = 0, s = m_slots(mach, y) < w ? m_slots(mach, y) : w;
      for (uint32_t j = 0; j < n; ++j) if (itype(r, j) == y) ny++;
      if ((ny + s - 1) / s > l) l = (ny + s - 1) / s;
    }
  *lb_len = l;
  /* transitive closure by DFS from each node; UB = 1 + max #independent */
  uint32_t best = 0;
  if (n > 0) {
    char *reach = calloc((size_t)n * n, 1);
    uint32_t *stack = malloc(sizeof(uint32_t) * n);
    for (uint32_t x = 0; x < n; ++x) {
      uint32_t sp = 0;
      stack[sp++] = x;
      while (sp) {
        uint32_t u = stack[--sp];
        for (uint32_t k = m.succ_ptr[u]; k < m.succ_ptr[u + 1]; ++k) {
          uint32_t v = m.succ[k];
          if (!reach[(size_t)x * n + v]) { reach[(size_t)x * n + v] = 1; stack[sp++] = v; }
        }
      }
    }
    for (uint32_t x = 0; x < n; ++x) {
      uint32_t ind = 0;
      for (uint32_t y = 0; y < n; ++y)
        if (y != x && !reach[(size_t)x * n + y] && !reach[(size_t)y * n + x]) ind++;
      if (ind > best) best = ind;
    }
    free(reach); free(stack);
    best += 1;
  }
  *ub_ready = best;
  model_free(&m);
  return ORC_OK;
}

/* ------------------------------------------------------------------------ */
/* Heuristic eta and selection (L116-L118, L122; R1-R4, R27).                 */
/* ------------------------------------------------------------------------ */
/* eta = 1 + floor(key * 65534 / max(1, keymax)), in [1, 65535] (R4). */
static uint32_t eta_of(uint64_t key, uint64_t keymax) {
  uint64_t d = keymax ? keymax : 1;
  return (uint32_t)(1 + (key * 65534u) / d);
}

static uint32_t eta1(const model *m, const rp_state *s, uint32_t j) {
  uint64_t key = (uint64_t)rp_luc(m, s, j) * (m->cp_max + 1u) + m->cp[j];
  uint64_t keymax = (uint64_t)m->max_luc * (m->cp_max + 1u) + m->cp_max;
  return eta_of(key, keymax);
}

static uint32_t eta2(const model *m, uint32_t j) { return eta_of(m->cp[j], m->cp_max); }

/* Exploit: argmax score, ties to the lowest position.  Explore (roulette):
 * r = floor(R64 * sum / 2^64); the first position whose inclusive prefix
 * sum exceeds r (R1, R27). */
uint32_t orc_select(const uint32_t *score, uint32_t count, int exploit, uint64_t r64) {
  if (exploit) {
    uint32_t best = 0;
    for (uint32_t i = 1; i < count; ++i) if (score[i] > score[best]) best = i;
    return best;
  }
  uint64_t sum = 0;
  for (uint32_t i = 0; i < count; ++i) sum += score[i];
  uint64_t r = (uint64_t)(((unsigned __int128)r64 * sum) >> 64);
  uint64_t prefix = 0;
  for (uint32_t i = 0; i < count; ++i) {
    prefix += score[i];
    if (prefix > r) return i;
  }
  return count - 1; /* unreachable: r < sum */
}

/* ------------------------------------------------------------------------ */
/* Pheromone update (L114, L120; R6-R9).                                     */
/* ------------------------------------------------------------------------ */
void orc_pheromone_update(uint16_t *tau, uint32_t n, const uint32_t *w, const orc_params *p) {
  /* next_w(i): the instruction that follows i in the winner's order; the
   * ROOT row's successor is the first instruction (R5). */
  uint32_t *next = malloc(sizeof(uint32_t) * (n + 1));
  for (uint32_t i = 0; i <= n; ++i) next[i] = UINT32_MAX;
  if (w && n > 0) {
    next[ROOT_ROW(n)] = w[0];
    for (uint32_t k = 0; k + 1 < n; ++k) next[w[k]] = w[k + 1];
  }
  for (uint32_t i = 0; i <= n; ++i)
    for (uint32_t j = 0; j < n; ++j) {
      uint64_t v = ((uint64_t)tau[(size_t)i * n + j] * p->rho_q16) >> 16; /* decay */
      if (next[i] == j) v += p->delta; /* deposit on the iteration winner's links */
      if (v < p->tau_min) v = p->tau_min;
      if (v > p->tau_max) v = p->tau_max;
      tau[(size_t)i * n + j] = (uint16_t)v;
    }
  free(next);
}

/* ------------------------------------------------------------------------ */
/* Ant construction.                                                         */
/* ------------------------------------------------------------------------ */
typedef struct {
  const model *m;
  const orc_machine *mach;
  const orc_params *p;
  uint32_t region_id;
  uint32_t target[4];
  /* scratch */
  uint32_t *pred_left, *rdy, *cand, *score, *flist;
  char *scheduled;
  rp_state rp;
  uint64_t *stats;
} ant_ctx;

typedef struct {
  uint32_t cost; /* INVALID_COST if the ant died */
  uint32_t prp[4];
  uint32_t length;
} ant_out;

/* Pass-1 ant (L108, L116-L118, L145; R19): latencies ignored, one
 * instruction per step, candidates = all ready instructions.  Written as
 * steps (begin / ready list / choose-and-commit) so that the ants of one
 * wavefront can also run in lockstep for the ready-list size limit (R45). */
static void p1_begin(ant_ctx *a) {
  const model *m = a->m;
  for (uint32_t j = 0; j < m->n; ++j) { a->pred_left[j] = m->indeg[j]; a->scheduled[j] = 0; }
  rp_init(m, &a->rp);
}

/* The ready list in ascending index order (R25) with its scores
 * tau[prev][j] * eta(j) (R1, R4); returns its size. */
static uint32_t p1_ready(ant_ctx *a, uint32_t ant, uint32_t prev, const uint16_t *tau, int greedy) {
  const model *m = a->m;
  uint32_t n = m->n, cnt = 0;
  for (uint32_t j = 0; j < n; ++j)
    if (!a->scheduled[j] && a->pred_left[j] == 0) {
      a->cand[cnt] = j;
      /* R43: with heur_mix, odd ant groups are guided by the ILP heuristic
       * (CP, eta2) instead of LUC-then-CP; the greedy schedule never is */
      uint32_t e = (!greedy && a->p->heur_mix && ((ant / a->p->group_size) & 1u)) ? eta2(m, j)
                                                                                  : eta1(m, &a->rp, j);
      a->score[cnt] = (uint32_t)tau[(size_t)prev * n + j] * e;
      cnt++;
    }
  return cnt;
}

/* Step k: select among the first `lim` ready instructions (all of them
 * unless the ready-list limit R45 is on) and commit; returns the choice. */
static uint32_t p1_commit(ant_ctx *a, uint32_t iter, uint32_t ant, uint32_t k, uint32_t cnt, uint32_t lim,
                          int greedy) {
  const model *m = a->m;
  int exploit;
  uint64_t r64 = 0;
  if (greedy) {
    exploit = 1;
  } else {
    uint32_t coin = draw_group_coin(a->p->seed, a->region_id, 1, iter, ant / a->p->group_size, k);
    exploit = (uint64_t)coin < a->p->q0_t; /* R1-R3 */
    if (!exploit) {
      uint32_t x[4];
      draw_ant(a->p->seed, a->region_id, 1, iter, ant, k, x);
      r64 = ((uint64_t)x[1] << 32) | x[0];
    }
  }
  uint32_t j = a->cand[orc_select(a->score, lim, exploit, r64)];
  if (a->stats && !greedy) {
    a->stats[ORS_SUM_R] += cnt;
    a->stats[ORS_SUM_F] += lim;
    a->stats[ORS_SUM_DEG] += m->succ_ptr[j + 1] - m->succ_ptr[j];
    a->stats[ORS_SUM_USE] += m->src->use_ptr[j + 1] - m->src->use_ptr[j];
    a->stats[ORS_SUM_DEF] += m->src->def_ptr[j + 1] - m->src->def_ptr[j];
    a->stats[ORS_PLACEMENTS]++;
  }
  rp_issue(m, &a->rp, j);
  a->scheduled[j] = 1;
  for (uint32_t q = m->succ_ptr[j]; q < m->succ_ptr[j + 1]; ++q) a->pred_left[m->succ[q]]--;
  return j;
}

static void p1_end(ant_ctx *a, ant_out *out) {
  for (uint32_t c = 0; c < 4; ++c) out->prp[c] = a->rp.prp[c];
  out->cost = orc_cost_rp(a->mach, a->p->cost_mode, a->rp.prp);
  out->length = 0;
}

static void ant_pass1(ant_ctx *a, uint32_t iter, uint32_t ant, const uint16_t *tau, int greedy,
                      uint32_t *order, ant_out *out) {
  uint32_t n = a->m->n, prev = ROOT_ROW(n);
  p1_begin(a);
  for (uint32_t k = 0; k < n; ++k) {
    uint32_t cnt = p1_ready(a, ant, prev, tau, greedy);
    prev = order[k] = p1_commit(a, iter, ant, k, cnt, cnt, greedy);
  }
  p1_end(a, out);
}

/* Scratch of one ant context (the per-ant arrays of ant_ctx). */
static int ant_scratch_alloc(ant_ctx *a, const model *m) {
  uint32_t n = m->n;
  a->pred_left = malloc(sizeof(uint32_t) * (n + 1));
  a->rdy = malloc(sizeof(uint32_t) * (n + 1));
  a->cand = malloc(sizeof(uint32_t) * (n + 1));
  a->score = malloc(sizeof(uint32_t) * (n + 1));
  a->flist = malloc(sizeof(uint32_t) * (n + 1));
  a->scheduled = malloc(n + 1);
  a->rp.rem = calloc(m->n_regs + 1, sizeof(uint32_t));
  return a->pred_left && a->rdy && a->cand && a->score && a->flist && a->scheduled && a->rp.rem;
}
static void ant_scratch_free(ant_ctx *a) {
  free(a->pred_left); free(a->rdy); free(a->cand); free(a->score); free(a->flist); free(a->scheduled);
  free(a->rp.rem);
}

/* Ready-list size limit (L214; R45): the ants of one wavefront -- the group
 * of G = group_size consecutive ant ids (R3) -- build their pass-1 schedules
 * in lockstep; at step k every ant of the group considers only the first K
 * instructions of its ready list (ascending index, R25), with K = the
 * smallest ready-list size in the group at step k (rl_limit = 1) or the
 * midpoint floor((min + max) / 2) of the smallest and largest (rl_limit = 2).
 * Ants [a0, a0 + cnt) of the group; orders[i * n ..] and outs[i] receive
 * ant a0 + i's schedule and result. */
static int pass1_group_lockstep(const ant_ctx *proto, uint32_t iter, uint32_t a0, uint32_t cnt,
                                const uint16_t *tau, uint32_t *orders, ant_out *outs) {
  const model *m = proto->m;
  uint32_t n = m->n;
  ant_ctx *g = calloc(cnt, sizeof(ant_ctx));
  uint32_t *prev = malloc(sizeof(uint32_t) * cnt), *size = malloc(sizeof(uint32_t) * cnt);
  int ok = g && prev && size;
  for (uint32_t i = 0; ok && i < cnt; ++i) {
    g[i] = *proto;
    ok = ant_scratch_alloc(&g[i], m);
    if (ok) p1_begin(&g[i]);
    prev[i] = ROOT_ROW(n);
  }
  for (uint32_t k = 0; ok && k < n; ++k) {
    uint32_t lo = UINT32_MAX, hi = 0;
    for (uint32_t i = 0; i < cnt; ++i) {
      size[i] = p1_ready(&g[i], a0 + i, prev[i], tau, 0);
      if (size[i] < lo) lo = size[i];
      if (size[i] > hi) hi = size[i];
    }
    uint32_t lim = proto->p->rl_limit == 1 ? lo : (lo + hi) / 2;
    for (uint32_t i = 0; i < cnt; ++i) /* (a midpoint above an ant's own size does not bind) */
      prev[i] = orders[(size_t)i * n + k] = p1_commit(&g[i], iter, a0 + i, k, size[i], lim < size[i] ? lim : size[i], 0);
  }
  for (uint32_t i = 0; ok && i < cnt; ++i) p1_end(&g[i], &outs[i]);
  if (g)
    for (uint32_t i = 0; i < cnt; ++i) ant_scratch_free(&g[i]);
  free(g); free(prev); free(size);
  return ok ? ORC_OK : ORC_E_ARG;
}

/* Is ant group g allowed optional stalls?  (L202-L204; R23, R44) */
static int stall_enabled_group(const orc_params *p, uint32_t g) {
  uint32_t mod = p->stall_mod, rem = p->stall_rem % mod;
  return ((g % mod) + mod - rem) % mod < p->stall_num;
}

/* Pass-2 ant (L108, L118, L147-L164, L200-L206; R19-R24), on the general
 * machine model (L64; R42).  Each loop turn either stalls (necessary, forced
 * optional, or discretionary), or places one instruction in the current
 * cycle t; the cycle is complete when issue_width instructions were placed
 * in it.  An instruction whose latency is met but whose issue slot (width or
 * type) is full this cycle counts as semi-ready with ready time t + 1.
 * The Philox step is t * issue_width + (instructions already placed in t),
 * which is t on the single-issue machine.
 * weighted (pass 4, R41): no RP target, cost = length + W * cost_rp(PRP).
 * Pruning (R24) is a GPU-only, winner-invariant shortcut; the oracle never
 * prunes. */
static void ant_pass2(ant_ctx *a, uint32_t iter, uint32_t ant, const uint16_t *tau,
                      uint32_t *order, uint32_t *cycle_of, ant_out *out) {
  const model *m = a->m;
  const orc_params *p = a->p;
  const orc_machine *mach = a->mach;
  const orc_region *src = m->src;
  uint32_t n = m->n, nc = m->n_classes, w = m_width(mach);
  for (uint32_t j = 0; j < n; ++j) { a->pred_left[j] = m->indeg[j]; a->rdy[j] = 0; a->scheduled[j] = 0; }
  rp_init(m, &a->rp);
  uint32_t prev = ROOT_ROW(n), placed = 0;
  uint64_t t = 0, k_opt = 0, last = 0;
  uint32_t used = 0, used_t[4] = {0, 0, 0, 0};
  uint32_t group = ant / p->group_size;
  int stall_enabled = stall_enabled_group(p, group); /* R23, R44 */
  int use_eta1 = p->heur_mix && (group & 1u);        /* R43 */
  uint32_t *rlist = a->cand;   /* R in ascending order */
  uint32_t *flist = a->flist;
  uint32_t *fscore = a->score;
  while (placed < n) {
    uint32_t step = (uint32_t)(t * w + used);
    uint32_t nr = 0, nf = 0, ns = 0;
    uint64_t min_s = UINT64_MAX;
    for (uint32_t j = 0; j < n; ++j) {
      if (a->scheduled[j] || a->pred_left[j]) continue;
      uint32_t y = itype(src, j);
      int slot = used < w && used_t[y] < m_slots(mach, y);
      if (a->rdy[j] <= t && slot) rlist[nr++] = j;
      else {
        uint64_t eff = a->rdy[j] <= t ? t + 1 : a->rdy[j]; /* slot-blocked: next cycle */
        ns++;
        if (eff < min_s) min_s = eff;
      }
    }
    for (uint32_t q = 0; q < nr; ++q) { /* F = RP-feasible part of R (R21) */
      uint32_t j = rlist[q];
      int ok = 1;
      for (uint32_t c = 0; c < nc; ++c)
        if ((int64_t)a->rp.live[c] + rp_delta(m, &a->rp, j, c) > (int64_t)a->target[c]) ok = 0;
      if (ok) flist[nf++] = j;
    }
    if (a->stats) { a->stats[ORS_SUM_R] += nr; a->stats[ORS_SUM_S] += ns; }
    if (nr == 0) { /* necessary stall (L153): skip ahead to the next ready time */
      t = min_s;
      used = 0; used_t[0] = used_t[1] = used_t[2] = used_t[3] = 0;
      if (a->stats) a->stats[ORS_STALL_EVENTS]++;
      continue;
    }
    if (nf == 0) {
      if (stall_enabled && ns > 0) { /* forced optional stall (L155, R22) */
        k_opt += min_s - t;
        t = min_s;
        used = 0; used_t[0] = used_t[1] = used_t[2] = used_t[3] = 0;
        if (a->stats) a->stats[ORS_STALL_EVENTS]++;
        continue;
      }
      out->cost = INVALID_COST; /* the ant is terminated (L149) */
      out->length = INVALID_COST;
      for (uint32_t c = 0; c < 4; ++c) out->prp[c] = a->rp.prp[c];
      if (a->stats) a->stats[ORS_DEAD_ANTS]++;
      return;
    }
    uint32_t x[4] = {0, 0, 0, 0};
    int have_x = 0;
    if (stall_enabled && ns > 0) { /* discretionary optional stall (L157-L164, R22) */
      int all_f_increase = 1, some_s_decrease = 0;
      for (uint32_t q = 0; q < nf; ++q) {
        int64_t mx = INT64_MIN;
        for (uint32_t c = 0; c < nc; ++c) {
          int64_t d = rp_delta(m, &a->rp, flist[q], c);
          if (d > mx) mx = d;
        }
        if (!(mx > 0)) all_f_increase = 0;
      }
      for (uint32_t j = 0; j < n; ++j) {
        if (a->scheduled[j] || a->pred_left[j]) continue;
        uint32_t y = itype(src, j);
        if (a->rdy[j] <= t && used < w && used_t[y] < m_slots(mach, y)) continue; /* in R */
        int64_t mn = INT64_MAX;
        for (uint32_t c = 0; c < nc; ++c) {
          int64_t d = rp_delta(m, &a->rp, j, c);
          if (d < mn) mn = d;
        }
        if (mn < 0) some_s_decrease = 1;
      }
      if (all_f_increase && some_s_decrease) {
        draw_ant(p->seed, a->region_id, 2, iter, ant, step, x);
        have_x = 1;
        uint32_t thr = (k_opt + 1 >= 32) ? 0u : (0xFFFFFFFFu >> (k_opt + 1));
        if (x[2] < thr) { /* probability 2^-(k_opt+1) */
          k_opt++;
          t++;
          used = 0; used_t[0] = used_t[1] = used_t[2] = used_t[3] = 0;
          if (a->stats) a->stats[ORS_STALL_EVENTS]++;
          continue;
        }
      }
    }
    for (uint32_t q = 0; q < nf; ++q)
      fscore[q] = (uint32_t)tau[(size_t)prev * n + flist[q]] *
                  (use_eta1 ? eta1(m, &a->rp, flist[q]) : eta2(m, flist[q]));
    uint32_t coin = draw_group_coin(p->seed, a->region_id, 2, iter, group, step);
    int exploit = (uint64_t)coin < p->q0_t;
    uint64_t r64 = 0;
    if (!exploit) {
      if (!have_x) draw_ant(p->seed, a->region_id, 2, iter, ant, step, x);
      r64 = ((uint64_t)x[1] << 32) | x[0];
    }
    uint32_t j = flist[orc_select(fscore, nf, exploit, r64)];
    if (a->stats) {
      a->stats[ORS_SUM_F] += nf;
      a->stats[ORS_SUM_DEG] += m->succ_ptr[j + 1] - m->succ_ptr[j];
      a->stats[ORS_SUM_USE] += m->src->use_ptr[j + 1] - m->src->use_ptr[j];
      a->stats[ORS_SUM_DEF] += m->src->def_ptr[j + 1] - m->src->def_ptr[j];
      a->stats[ORS_PLACEMENTS]++;
    }
    rp_issue(m, &a->rp, j);
    a->scheduled[j] = 1;
    cycle_of[j] = (uint32_t)t;
    last = t;
    order[placed++] = j;
    for (uint32_t q = m->succ_ptr[j]; q < m->succ_ptr[j + 1]; ++q) {
      uint32_t v = m->succ[q];
      a->pred_left[v]--;
      uint64_t need = t + m->succ_lat[q];
      if (need > a->rdy[v]) a->rdy[v] = (uint32_t)need;
    }
    prev = j;
    used++;
    used_t[itype(src, j)]++;
    if (used == w) { /* the cycle is full */
      t++;
      used = 0; used_t[0] = used_t[1] = used_t[2] = used_t[3] = 0;
    }
  }
  for (uint32_t c = 0; c < 4; ++c) out->prp[c] = a->rp.prp[c];
  out->length = n ? (uint32_t)last + 1 : 0; /* last issue cycle + 1 (R20) */
  out->cost = out->length;
  if (p->pass == 4) /* weighted single pass (L74; R41) */
    out->cost = out->length + p->ws_weight * orc_cost_rp(a->mach, p->cost_mode, a->rp.prp);
}

/* FNV-1a (64-bit) over (pass, iter, winner cost, winner ant), little endian. */
static uint64_t fnv_u32(uint64_t h, uint32_t v) {
  for (int b = 0; b < 4; ++b) {
    h ^= (v >> (8 * b)) & 0xFFu;
    h *= 0x100000001b3ull;
  }
  return h;
}

static uint32_t no_improve_limit(const orc_params *p, uint32_t n) {
  if (p->stop_no_improve != 0xFFFFFFFFu) return p->stop_no_improve;
  return n < 50 ? 1u : (n < 100 ? 2u : 3u); /* L226 */
}

/* ------------------------------------------------------------------------ */
/* The single weighted-sum pass (L74; R41): the ILP-pass construction with  */
/* no RP target, cost = length + W * cost_rp(PRP), from the heuristic order  */
/* timed ASAP.  Same iteration loop as the two passes (R5-R12).              */
/* ------------------------------------------------------------------------ */
static int weighted_pass(ant_ctx *a, const orc_region *r, const orc_machine *mach, const orc_params *p,
                         const model *m, uint16_t *tau, const uint32_t *heur_order, uint32_t lb_cost,
                         uint32_t lb_len, uint32_t *ant_order, uint32_t *ant_cycle_of, uint32_t *win_order,
                         uint32_t *win_cycle_of, uint32_t *best_order, uint32_t *best_cycle_of,
                         uint32_t *tmp_cycle, uint64_t *hash, uint64_t *stats, uint32_t *dump_cost,
                         uint32_t *dump_order, uint32_t *dump_cycle) {
  uint32_t n = m->n;
  for (uint32_t c = 0; c < 4; ++c) a->target[c] = 0xFFFFFFFFu; /* no target */
  for (uint32_t c = 0; c < 4; ++c) stats[ORS_TARGET0 + c] = a->target[c];
  int64_t init_len = orc_asap_m(r, mach, heur_order, tmp_cycle);
  uint32_t prp[4];
  orc_prp_of_order(r, mach->n_classes, heur_order, prp);
  uint32_t best = (uint32_t)init_len + p->ws_weight * orc_cost_rp(mach, p->cost_mode, prp);
  uint32_t best_len = (uint32_t)init_len;
  uint32_t lb = lb_len + p->ws_weight * lb_cost;
  for (uint32_t k = 0; k < n; ++k) {
    best_order[k] = heur_order[k];
    best_cycle_of[heur_order[k]] = tmp_cycle[k];
  }
  stats[ORS_INIT2] = best;
  for (size_t q = 0; q < (size_t)(n + 1) * n; ++q) tau[q] = (uint16_t)p->tau0;
  uint32_t nimp = 0, lim = no_improve_limit(p, n);
  int skip = p->stop_at_lb && best == lb;
  for (uint32_t it = 0; it < p->iterations && !skip; ++it) {
    uint64_t wkey = UINT64_MAX;
    uint32_t wcost = INVALID_COST, wlen = 0;
    for (uint32_t ant = 0; ant < p->ants; ++ant) {
      ant_out o;
      ant_pass2(a, it, ant, tau, ant_order, ant_cycle_of, &o);
      stats[ORS_ANT_SCHEDS]++;
      if (dump_cost) dump_cost[((size_t)1 * p->iterations + it) * p->ants + ant] = o.cost;
      if (dump_order || dump_cycle) {
        size_t base = (((size_t)1 * p->iterations + it) * p->ants + ant) * n;
        if (dump_order) memcpy(dump_order + base, ant_order, sizeof(uint32_t) * n);
        if (dump_cycle)
          for (uint32_t k = 0; k < n; ++k) dump_cycle[base + k] = ant_cycle_of[ant_order[k]];
      }
      uint64_t key = ((uint64_t)o.cost << 32) | ant; /* R10 */
      if (key < wkey) {
        wkey = key; wcost = o.cost; wlen = o.length;
        memcpy(win_order, ant_order, sizeof(uint32_t) * n);
        memcpy(win_cycle_of, ant_cycle_of, sizeof(uint32_t) * n);
      }
    }
    orc_pheromone_update(tau, n, win_order, p);
    *hash = fnv_u32(fnv_u32(fnv_u32(fnv_u32(*hash, 4), it), wcost), (uint32_t)wkey);
    if (wcost < best) { /* R11 */
      best = wcost; best_len = wlen;
      memcpy(best_order, win_order, sizeof(uint32_t) * n);
      memcpy(best_cycle_of, win_cycle_of, sizeof(uint32_t) * n);
      nimp = 0;
    } else {
      nimp++;
    }
    stats[ORS_ITERS2] = it + 1;
    if ((p->stop_at_lb && best == lb) || (lim > 0 && nimp >= lim)) break;
  }
  stats[ORS_BEST2] = best;
  stats[ORS_WS_COST] = best;
  stats[ORS_LENGTH] = best_len;
  return ORC_OK;
}

/* ------------------------------------------------------------------------ */
/* The two-pass ACO (L106-L139; R5-R13).                                     */
/* ------------------------------------------------------------------------ */
int orc_schedule(const orc_region *r, uint32_t region_id, const orc_machine *mach,
                 const orc_params *p, uint32_t *order_out, uint32_t *cycle_out,
                 uint64_t *stats, uint32_t *dump_cost, uint32_t *dump_order,
                 uint32_t *dump_cycle, uint16_t *tau_out) {
  if (p->pass < 1 || p->pass > 4 || p->cost_mode > 3 || p->group_size == 0 || p->stall_mod == 0 ||
      p->ants == 0 || p->tau_min > p->tau_max || p->tau_max > 65535u || p->ws_weight > 1024u ||
      p->heur_mix > 1u || p->rl_limit > 2u)
    return ORC_E_ARG;
  int st = machine_check(r, mach);
  if (st != ORC_OK) return st;
  model m;
  st = model_build(&m, r, mach->n_classes);
  if (st != ORC_OK) return st;
  uint32_t n = m.n;
  uint64_t local_stats[ORS_COUNT];
  if (!stats) stats = local_stats;
  memset(stats, 0, sizeof(uint64_t) * ORS_COUNT);

  ant_ctx a;
  memset(&a, 0, sizeof(a));
  a.m = &m; a.mach = mach; a.p = p; a.region_id = region_id; a.stats = stats;
  a.pred_left = malloc(sizeof(uint32_t) * (n + 1));
  a.rdy = malloc(sizeof(uint32_t) * (n + 1));
  a.cand = malloc(sizeof(uint32_t) * (n + 1));
  a.score = malloc(sizeof(uint32_t) * (n + 1));
  a.flist = malloc(sizeof(uint32_t) * (n + 1));
  a.scheduled = malloc(n + 1);
  a.rp.rem = calloc(m.n_regs + 1, sizeof(uint32_t));
  uint16_t *tau = malloc(sizeof(uint16_t) * ((size_t)(n + 1) * n + 1));
  uint32_t *ant_order = malloc(sizeof(uint32_t) * (n + 1));
  uint32_t *ant_cycle_of = malloc(sizeof(uint32_t) * (n + 1));
  uint32_t *best_order = malloc(sizeof(uint32_t) * (n + 1));
  uint32_t *win_order = malloc(sizeof(uint32_t) * (n + 1));
  uint32_t *best_cycle_of = malloc(sizeof(uint32_t) * (n + 1));
  uint32_t *win_cycle_of = malloc(sizeof(uint32_t) * (n + 1));
  uint32_t *tmp_cycle = malloc(sizeof(uint32_t) * (n + 1));
  /* R45: one wavefront's lockstep pass-1 schedules */
  uint32_t *grp_order = p->rl_limit ? malloc(sizeof(uint32_t) * ((size_t)p->group_size * n + 1)) : NULL;
  ant_out *grp_out = p->rl_limit ? malloc(sizeof(ant_out) * p->group_size) : NULL;

  uint32_t lb_cost, lb_len, ub, final_len = 0;
  orc_lower_bounds(r, mach, p->cost_mode, &lb_cost, &lb_len, &ub);
  stats[ORS_LB1] = lb_cost; stats[ORS_LBLEN] = lb_len; stats[ORS_UB_READY] = ub;
  uint64_t hash = 0xcbf29ce484222325ull;

  /* Initial pass-1 schedule: greedy list schedule on eta1 (L122; R28) --
   * the q0 = 1 ant on a uniform tau. */
  for (size_t q = 0; q < (size_t)(n + 1) * n; ++q) tau[q] = (uint16_t)p->tau0;
  ant_out best1;
  ant_pass1(&a, 0, 0, tau, 1, best_order, &best1);
  stats[ORS_INIT1] = best1.cost;
  /* the heuristic schedule H (R40): the greedy order timed ASAP */
  uint32_t *heur_order = malloc(sizeof(uint32_t) * (n + 1));
  memcpy(heur_order, best_order, sizeof(uint32_t) * n);
  ant_out heur = best1;
  stats[ORS_HEUR_LEN] = (uint64_t)orc_asap_m(r, mach, heur_order, tmp_cycle);
  stats[ORS_POLICY] = 0;
  if (p->pass == 4) { /* the single weighted-sum pass (L74; R41) */
    stats[ORS_BEST1] = best1.cost;
    st = weighted_pass(&a, r, mach, p, &m, tau, heur_order, lb_cost, lb_len, ant_order, ant_cycle_of,
                       win_order, win_cycle_of, best_order, best_cycle_of, tmp_cycle, &hash, stats,
                       dump_cost, dump_order, dump_cycle);
    final_len = (uint32_t)stats[ORS_LENGTH];
    goto report;
  }

  /* ---- pass 1 (the RP pass) ---- */
  if (p->pass & 1u) {
    uint32_t nimp = 0, lim = no_improve_limit(p, n);
    int skip = p->stop_at_lb && best1.cost == lb_cost; /* L251 */
    for (uint32_t it = 0; it < p->iterations && !skip; ++it) {
      uint64_t wkey = UINT64_MAX;
      ant_out wout;
      memset(&wout, 0, sizeof(wout));
      for (uint32_t ant = 0; ant < p->ants; ++ant) {
        ant_out o;
        if (p->rl_limit) { /* R45: the ant's wavefront was built in lockstep */
          uint32_t gs = p->group_size, a0 = ant - ant % gs;
          uint32_t gc = (a0 + gs <= p->ants ? gs : p->ants - a0);
          if (ant == a0 && pass1_group_lockstep(&a, it, a0, gc, tau, grp_order, grp_out) != ORC_OK) {
            st = ORC_E_ARG;
            goto report;
          }
          memcpy(ant_order, grp_order + (size_t)(ant - a0) * n, sizeof(uint32_t) * n);
          o = grp_out[ant - a0];
        } else {
          ant_pass1(&a, it, ant, tau, 0, ant_order, &o);
        }
        stats[ORS_ANT_SCHEDS]++;
        if (dump_cost) dump_cost[((size_t)0 * p->iterations + it) * p->ants + ant] = o.cost;
        if (dump_order)
          memcpy(dump_order + (((size_t)0 * p->iterations + it) * p->ants + ant) * n, ant_order,
                 sizeof(uint32_t) * n);
        uint64_t key = ((uint64_t)o.cost << 32) | ant; /* argmin (cost, ant), R10 */
        if (key < wkey) { wkey = key; wout = o; memcpy(win_order, ant_order, sizeof(uint32_t) * n); }
      }
      orc_pheromone_update(tau, n, win_order, p); /* decay + deposit (R8, R9) */
      hash = fnv_u32(fnv_u32(fnv_u32(fnv_u32(hash, 1), it), wout.cost), (uint32_t)wkey);
      if (wout.cost < best1.cost) { /* strict improvement (R11) */
        best1 = wout;
        memcpy(best_order, win_order, sizeof(uint32_t) * n);
        nimp = 0;
      } else {
        nimp++;
      }
      stats[ORS_ITERS1] = it + 1;
      if ((p->stop_at_lb && best1.cost == lb_cost) || (lim > 0 && nimp >= lim)) break; /* R12 */
    }
  }
  stats[ORS_BEST1] = best1.cost;

  /* ---- pass 2 (the ILP pass) ---- */
  int64_t init_len = orc_asap_m(r, mach, best_order, tmp_cycle); /* R29, R42 */
  for (uint32_t k = 0; k < n; ++k) best_cycle_of[best_order[k]] = tmp_cycle[k];
  final_len = (uint32_t)init_len;
  stats[ORS_INIT2] = (uint32_t)init_len;
  orc_target(mach, p->cost_mode, best1.prp, a.target); /* R18 */
  for (uint32_t c = 0; c < 4; ++c) stats[ORS_TARGET0 + c] = a.target[c];
  /* cycle-gap filter (L362, L393-L417; R39): pass 2 only if the input
   * schedule is at least pass2_gap cycles above LB_len */
  int gap_skip = (p->pass & 2u) && p->pass2_gap > 0 && init_len - (int64_t)lb_len < (int64_t)p->pass2_gap;
  if (gap_skip) stats[ORS_POLICY] |= 1u;
  if ((p->pass & 2u) && !gap_skip) {
    for (size_t q = 0; q < (size_t)(n + 1) * n; ++q) tau[q] = (uint16_t)p->tau0; /* R13 */
    uint32_t best_len = (uint32_t)init_len;
    uint32_t nimp = 0, lim = no_improve_limit(p, n);
    int skip = p->stop_at_lb && best_len == lb_len;
    for (uint32_t it = 0; it < p->iterations && !skip; ++it) {
      uint64_t wkey = UINT64_MAX;
      uint32_t wlen = INVALID_COST;
      for (uint32_t ant = 0; ant < p->ants; ++ant) {
        ant_out o;
        ant_pass2(&a, it, ant, tau, ant_order, ant_cycle_of, &o);
        stats[ORS_ANT_SCHEDS]++;
        if (dump_cost) dump_cost[((size_t)1 * p->iterations + it) * p->ants + ant] = o.cost;
        if (o.cost != INVALID_COST && (dump_order || dump_cycle)) {
          size_t base = (((size_t)1 * p->iterations + it) * p->ants + ant) * n;
          if (dump_order) memcpy(dump_order + base, ant_order, sizeof(uint32_t) * n);
          if (dump_cycle)
            for (uint32_t k = 0; k < n; ++k) dump_cycle[base + k] = ant_cycle_of[ant_order[k]];
        }
        if (o.cost == INVALID_COST) continue; /* only RP-feasible schedules (L118) */
        uint64_t key = ((uint64_t)o.cost << 32) | ant;
        if (key < wkey) {
          wkey = key; wlen = o.cost;
          memcpy(win_order, ant_order, sizeof(uint32_t) * n);
          memcpy(win_cycle_of, ant_cycle_of, sizeof(uint32_t) * n);
        }
      }
      int have = wkey != UINT64_MAX;
      orc_pheromone_update(tau, n, have ? win_order : NULL, p);
      hash = fnv_u32(fnv_u32(fnv_u32(fnv_u32(hash, 2), it), have ? wlen : INVALID_COST),
                     have ? (uint32_t)wkey : 0xFFFFFFFFu);
      if (have && wlen < best_len) {
        best_len = wlen;
        memcpy(best_order, win_order, sizeof(uint32_t) * n);
        memcpy(best_cycle_of, win_cycle_of, sizeof(uint32_t) * n);
        nimp = 0;
      } else {
        nimp++;
      }
      stats[ORS_ITERS2] = it + 1;
      if ((p->stop_at_lb && best_len == lb_len) || (lim > 0 && nimp >= lim)) break;
    }
    final_len = best_len;
    stats[ORS_BEST2] = best_len;
  } else {
    stats[ORS_BEST2] = (uint32_t)init_len;
  }
report:
  if (tau_out) memcpy(tau_out, tau, sizeof(uint16_t) * (size_t)(n + 1) * n);

  /* report: final order, its cycles, its PRP recomputed, cost_rp, length */
  uint32_t prp[4];
  orc_prp_of_order(r, mach->n_classes, best_order, prp);
  /* post-scheduling revert filter (L366; R40): when ACO raised the
   * occupancy by at least revert_occ but lengthened the schedule by more
   * than revert_len cycles, the heuristic schedule H is reported instead */
  if (p->revert_occ > 0) {
    uint32_t occ_f = mach->occ_max, occ_h = mach->occ_max;
    for (uint32_t c = 0; c < mach->n_classes; ++c) {
      uint32_t of = orc_occupancy(mach, c, prp[c]), oh = orc_occupancy(mach, c, heur.prp[c]);
      if (of < occ_f) occ_f = of;
      if (oh < occ_h) occ_h = oh;
    }
    if (occ_f >= occ_h + p->revert_occ && (uint64_t)final_len > stats[ORS_HEUR_LEN] + p->revert_len) {
      stats[ORS_POLICY] |= 2u;
      orc_asap_m(r, mach, heur_order, tmp_cycle);
      for (uint32_t k = 0; k < n; ++k) {
        best_order[k] = heur_order[k];
        best_cycle_of[heur_order[k]] = tmp_cycle[k];
      }
      final_len = (uint32_t)stats[ORS_HEUR_LEN];
      for (uint32_t c = 0; c < 4; ++c) prp[c] = heur.prp[c];
    }
  }
  for (uint32_t k = 0; k < n; ++k) {
    order_out[k] = best_order[k];
    cycle_out[k] = best_cycle_of[best_order[k]];
  }
  stats[ORS_COST_RP] = orc_cost_rp(mach, p->cost_mode, prp);
  stats[ORS_LENGTH] = final_len;
  for (uint32_t c = 0; c < 4; ++c) stats[ORS_PRP0 + c] = prp[c];
  stats[ORS_TRACE_HASH] = hash;

  free(a.pred_left); free(a.rdy); free(a.cand); free(a.score); free(a.flist); free(a.scheduled); free(a.rp.rem);
  free(tau); free(ant_order); free(ant_cycle_of); free(best_order); free(win_order);
  free(best_cycle_of); free(win_cycle_of); free(tmp_cycle); free(heur_order); free(grp_order); free(grp_out);
  model_free(&m);
  return st;
}

/* ------------------------------------------------------------------------ */
/* Many regions on a pool of host threads (one region per task).             */
/* ------------------------------------------------------------------------ */
typedef struct {
  const orc_region *regions;
  const uint32_t *ids;
  uint32_t count;
  const orc_machine *m;
  const orc_params *p;
  const uint64_t *off;
  uint32_t *order, *cycle;
  uint64_t *stats;
  uint32_t next;
  int status;
  pthread_mutex_t lock;
} pool_t;

static void *pool_worker(void *arg) {
  pool_t *P = arg;
  for (;;) {
    pthread_mutex_lock(&P->lock);
    uint32_t i = P->next++;
    pthread_mutex_unlock(&P->lock);
    if (i >= P->count) break;
    int st = orc_schedule(&P->regions[i], P->ids[i], P->m, P->p, P->order + P->off[i],
                          P->cycle + P->off[i], P->stats + (size_t)i * ORS_COUNT, NULL, NULL,
                          NULL, NULL);
    if (st != ORC_OK) {
      pthread_mutex_lock(&P->lock);
      if (P->status == ORC_OK) P->status = st;
      pthread_mutex_unlock(&P->lock);
    }
  }
  return NULL;
}

int orc_schedule_many(const orc_region *regions, const uint32_t *region_ids, uint32_t count,
                      const orc_machine *m, const orc_params *p, const uint64_t *out_off,
                      uint32_t *order_out, uint32_t *cycle_out, uint64_t *stats,
                      uint32_t n_threads) {
  pool_t P;
  P.regions = regions; P.ids = region_ids; P.count = count; P.m = m; P.p = p; P.off = out_off;
  P.order = order_out; P.cycle = cycle_out; P.stats = stats; P.next = 0; P.status = ORC_OK;
  pthread_mutex_init(&P.lock, NULL);
  if (n_threads < 1) n_threads = 1;
  pthread_t *th = malloc(sizeof(pthread_t) * n_threads);
  for (uint32_t t = 0; t < n_threads; ++t) pthread_create(&th[t], NULL, pool_worker, &P);
  for (uint32_t t = 0; t < n_threads; ++t) pthread_join(th[t], NULL);
  free(th);
  pthread_mutex_destroy(&P.lock);
  return P.status;
}

/* One ant on a given pheromone table (used for sampled parity at full sizes:
 * iteration-0 tables are uniform tau0, which the caller builds).  cycle_out
 * gets the cycle of the k-th placed instruction (pass 2 only). */
int orc_run_ant(const orc_region *r, uint32_t region_id, const orc_machine *mach,
                const orc_params *p, uint32_t pass, uint32_t iter, uint32_t ant,
                const uint16_t *tau, const uint32_t *target, uint32_t *order_out,
                uint32_t *cycle_out, uint32_t *prp_out, uint32_t *cost_out) {
  model m;
  int st = model_build(&m, r, mach->n_classes);
  if (st != ORC_OK) return st;
  uint32_t n = m.n;
  ant_ctx a;
  memset(&a, 0, sizeof(a));
  a.m = &m; a.mach = mach; a.p = p; a.region_id = region_id; a.stats = NULL;
  for (uint32_t c = 0; c < 4; ++c) a.target[c] = target ? target[c] : 0xFFFFFFFFu;
  a.pred_left = malloc(sizeof(uint32_t) * (n + 1));
  a.rdy = malloc(sizeof(uint32_t) * (n + 1));
  a.cand = malloc(sizeof(uint32_t) * (n + 1));
  a.score = malloc(sizeof(uint32_t) * (n + 1));
  a.flist = malloc(sizeof(uint32_t) * (n + 1));
  a.scheduled = malloc(n + 1);
  a.rp.rem = calloc(m.n_regs + 1, sizeof(uint32_t));
  uint32_t *cyc_of = calloc(n + 1, sizeof(uint32_t));
  ant_out o;
  if (pass == 1) {
    ant_pass1(&a, iter, ant, tau, 0, order_out, &o);
  } else {
    ant_pass2(&a, iter, ant, tau, order_out, cyc_of, &o);
    if (cycle_out && o.cost != INVALID_COST)
      for (uint32_t k = 0; k < n; ++k) cycle_out[k] = cyc_of[order_out[k]];
  }
  for (uint32_t c = 0; c < 4; ++c) prp_out[c] = o.prp[c];
  *cost_out = o.cost;
  free(a.pred_left); free(a.rdy); free(a.cand); free(a.score); free(a.flist); free(a.scheduled);
  free(a.rp.rem); free(cyc_of);
  model_free(&m);
  return ORC_OK;
}

/* The pass-1 greedy heuristic schedule (R28) on its own, for pins. */
int orc_greedy_pass1(const orc_region *r, const orc_machine *mach, const orc_params *p,
                     uint32_t *order_out, uint32_t *prp_out) {
  model m;
  int st = model_build(&m, r, mach->n_classes);
  if (st != ORC_OK) return st;
  uint32_t n = m.n;
  ant_ctx a;
  memset(&a, 0, sizeof(a));
  a.m = &m; a.mach = mach; a.p = p;
  a.pred_left = malloc(sizeof(uint32_t) * (n + 1));
  a.cand = malloc(sizeof(uint32_t) * (n + 1));
  a.score = malloc(sizeof(uint32_t) * (n + 1));
  a.scheduled = malloc(n + 1);
  a.rp.rem = calloc(m.n_regs + 1, sizeof(uint32_t));
  uint16_t *tau = malloc(sizeof(uint16_t) * ((size_t)(n + 1) * n + 1));
  for (size_t q = 0; q < (size_t)(n + 1) * n; ++q) tau[q] = (uint16_t)p->tau0;
  ant_out o;
  ant_pass1(&a, 0, 0, tau, 1, order_out, &o);
  for (uint32_t c = 0; c < 4; ++c) prp_out[c] = o.prp[c];
  free(a.pred_left); free(a.cand); free(a.score); free(a.scheduled); free(a.rp.rem); free(tau);
  model_free(&m);
  return ORC_OK;
}

/* eta values of the ready instructions at the start (pins for R4). */
int orc_eta_initial(const orc_region *r, const orc_machine *mach, uint32_t pass, uint32_t *eta_out) {
  model m;
  int st = model_build(&m, r, mach->n_classes);
  if (st != ORC_OK) return st;
  rp_state s;
  s.rem = calloc(m.n_regs + 1, sizeof(uint32_t));
  rp_init(&m, &s);
  for (uint32_t j = 0; j < m.n; ++j) eta_out[j] = pass == 1 ? eta1(&m, &s, j) : eta2(&m, j);
  free(s.rem);
  model_free(&m);
  return ORC_OK;
}
