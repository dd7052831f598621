/*
 * aco_oracle.h -- interface of the sequential CPU oracle.
 *
 * TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and the
 * cpu_baseline / --impl reference legs of bench.py may load liboracle.so.
 * The product path (include/aco.h, paper_conf_cgo_shobakimhlmkrg24_b200/)
 * never includes, links or calls anything in this directory, and this
 * directory never includes anything from the product path.
 *
 * What it computes: Ant Colony Optimization for register-pressure-aware
 * instruction scheduling of one basic-block DDG, in the two-pass form of
 * Shobaki et al., "Instruction Scheduling for the GPU on the GPU", CGO 2024
 * (PAPER.md L106-L164, L198-L206, L226), with every point the paper leaves
 * open fixed by the readings R1..R45 listed in DESIGN.md section 3.
 */
#ifndef ACO_ORACLE_H
#define ACO_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Status codes (same numeric meaning as documented in DESIGN.md). */
#define ORC_OK 0
#define ORC_E_ARG (-1)
#define ORC_E_DDG_CYCLE (-2)
#define ORC_E_DDG_MULTIDEF (-3)
#define ORC_E_DDG_USE_NO_EDGE (-4)
#define ORC_E_TOO_LARGE (-5)

/* One scheduling region: DDG + Def/Use sets of typed virtual
 * registers (L66).  Instruction ids are 0..n_insts-1 in program order. */
typedef struct {
  uint32_t n_insts, n_edges, n_regs;
  const uint32_t *edge_src, *edge_dst, *edge_lat;
  const uint8_t *reg_class; /* < n_classes */
  const uint8_t *reg_flags; /* bit0 LIVE_IN, bit1 LIVE_OUT */
  const uint32_t *def_ptr, *def_reg; /* CSR over instructions */
  const uint32_t *use_ptr, *use_reg; /* CSR over instructions */
  const uint8_t *inst_type; /* issue type of each instruction (R42); NULL = all type 0 */
} orc_region;

/* Occupancy model per register class (R16). */
typedef struct {
  uint32_t n_classes, occ_max;
  uint32_t step_count[4];
  uint32_t step_max[4][16]; /* max PRP giving occupancy occ_max, occ_max-1, ... */
  uint32_t perp_limit[4];
  /* general machine model (L64; R42): up to issue_width instructions per
   * cycle, at most type_slots[y] of issue type y.  issue_width <= 1 is the
   * single-issue machine of the paper's experiments (R32). */
  uint32_t issue_width, n_types;
  uint32_t type_slots[4];
} orc_machine;

typedef struct {
  uint32_t ants, iterations;
  uint64_t seed;
  uint32_t pass;      /* 1 = RP pass only, 2 = ILP pass only (pass-1 best = heuristic), 3 = both,
                         4 = single weighted-sum pass (L74; R41) */
  uint32_t cost_mode; /* 0 PRP_SUM, 1 APRP_SUM, 2 OCC, 3 PERP */
  uint64_t q0_t;      /* exploit iff group coin (u32) < q0_t; 2^32 = always */
  uint32_t group_size, stall_mod, stall_rem;
  uint32_t tau0, rho_q16, delta, tau_min, tau_max;
  uint32_t stop_no_improve; /* 0 off; 0xFFFFFFFF = paper size classes */
  uint32_t stop_at_lb;
  /* region-level compile policy (L362, L366, L393-L417; R39, R40) */
  uint32_t pass2_gap;              /* run pass 2 iff initial length - LB_len >= pass2_gap (0 = off) */
  uint32_t revert_occ, revert_len; /* revert to the heuristic schedule (revert_occ 0 = off) */
  uint32_t ws_weight;              /* pass 4: cost = length + ws_weight * cost_rp (R41) */
  uint32_t heur_mix;               /* 1: odd ant groups use the other pass's heuristic (L216-L218; R43) */
  uint32_t stall_num;              /* group g may stall iff (g - stall_rem) mod stall_mod < stall_num (R44) */
  uint32_t rl_limit;               /* pass-1 ready-list size limit per wavefront (L214; R45): 0 off, 1 min, 2 mid */
} orc_params;

/* Indices into the u64 result vector filled by orc_schedule. */
enum {
  ORS_COST_RP = 0, ORS_LENGTH, ORS_PRP0, ORS_PRP1, ORS_PRP2, ORS_PRP3,
  ORS_ITERS1, ORS_ITERS2, ORS_TRACE_HASH, ORS_BEST1, ORS_BEST2,
  ORS_LB1, ORS_LBLEN, ORS_INIT1, ORS_INIT2, ORS_TARGET0, ORS_TARGET1,
  ORS_TARGET2, ORS_TARGET3,
  /* instrumentation (summed over every ant of every iteration) */
  ORS_ANT_SCHEDS, ORS_PLACEMENTS, ORS_STALL_EVENTS, ORS_SUM_R, ORS_SUM_F,
  ORS_SUM_S, ORS_SUM_DEG, ORS_SUM_USE, ORS_SUM_DEF, ORS_SUM_MUSE_CHECKS,
  ORS_DEAD_ANTS, ORS_UB_READY,
  /* compile policy / weighted pass (R39-R41) */
  ORS_POLICY,   /* bit0: pass 2 filtered by the cycle gap; bit1: reverted to the heuristic */
  ORS_HEUR_LEN, /* length of the heuristic schedule (greedy order, ASAP) */
  ORS_WS_COST,  /* pass 4: final weighted cost */
  ORS_COUNT
};

/* Philox4x32-10 (Salmon et al., Random123), R26. */
void orc_philox4x32_10(const uint32_t ctr[4], const uint32_t key[2], uint32_t out[4]);

/* Validation (R31-R34).  Returns ORC_OK or a negative code. */
int orc_validate(const orc_region *r, uint32_t n_classes);

/* Register pressure of an instruction order (R14/R15); writes prp[c]. */
int orc_prp_of_order(const orc_region *r, uint32_t n_classes, const uint32_t *order, uint32_t *prp);

/* ASAP cycles of an order (R29); returns the length. */
int64_t orc_asap(const orc_region *r, const uint32_t *order, uint32_t *cycle);
/* Same on the general machine model (R42): in-order issue, <= issue_width per
 * cycle and <= type_slots[y] of type y per cycle. */
int64_t orc_asap_m(const orc_region *r, const orc_machine *m, const uint32_t *order, uint32_t *cycle);

/* Critical path heights (R4). */
int orc_critical_path(const orc_region *r, uint32_t *cp);

/* Cost functions (R16, R17). */
uint32_t orc_occupancy(const orc_machine *m, uint32_t c, uint32_t prp);
uint32_t orc_aprp(const orc_machine *m, uint32_t c, uint32_t prp);
uint32_t orc_cost_rp(const orc_machine *m, uint32_t mode, const uint32_t *prp);
void orc_target(const orc_machine *m, uint32_t mode, const uint32_t *best_prp, uint32_t *target);

/* Lower bounds (R30) and ready-list upper bound. */
int orc_lower_bounds(const orc_region *r, const orc_machine *m, uint32_t mode,
                     uint32_t *lb_cost, uint32_t *lb_len, uint32_t *ub_ready);

/* Selection rule (R1, R27) over scores listed in ascending index
 * order; returns the chosen position. */
uint32_t orc_select(const uint32_t *score, uint32_t count, int exploit, uint64_t r64);

/* One pheromone update (R6-R9).  tau is (n+1) x n, row n = ROOT.
 * winner_order may be NULL (no valid winner: decay only). */
void orc_pheromone_update(uint16_t *tau, uint32_t n, const uint32_t *winner_order,
                          const orc_params *p);

/* The whole two-pass ACO for one region.
 * order_out/cycle_out: n entries each.  stats: ORS_COUNT entries.
 * dump_cost:  [2][iterations][ants] (may be NULL)
 * dump_order: [2][iterations][ants][n] (may be NULL)
 * dump_cycle: [2][iterations][ants][n] (may be NULL; pass-2 cycles)
 * tau_out:    (n+1)*n, tau at the end of the last pass run (may be NULL). */
int orc_schedule(const orc_region *r, uint32_t region_id, const orc_machine *m,
                 const orc_params *p, uint32_t *order_out, uint32_t *cycle_out,
                 uint64_t *stats, uint32_t *dump_cost, uint32_t *dump_order,
                 uint32_t *dump_cycle, uint16_t *tau_out);

/* Same over many regions with a pool of host threads (bench baseline only).
 * regions[i] uses region_ids[i]; outputs are concatenated per region with
 * offsets out_off[i] (prefix sums of n_insts). Returns first error or OK. */
int orc_schedule_many(const orc_region *regions, const uint32_t *region_ids, uint32_t count,
                      const orc_machine *m, const orc_params *p, const uint64_t *out_off,
                      uint32_t *order_out, uint32_t *cycle_out, uint64_t *stats,
                      uint32_t n_threads);

/* One ant on a given pheromone table and pass-2 target (sampled parity). */
int orc_run_ant(const orc_region *r, uint32_t region_id, const orc_machine *m,
                const orc_params *p, uint32_t pass, uint32_t iter, uint32_t ant,
                const uint16_t *tau, const uint32_t *target, uint32_t *order_out,
                uint32_t *cycle_out, uint32_t *prp_out, uint32_t *cost_out);

/* The greedy pass-1 heuristic schedule (R28). */
int orc_greedy_pass1(const orc_region *r, const orc_machine *m, const orc_params *p,
                     uint32_t *order_out, uint32_t *prp_out);

/* eta of every instruction in the initial state (pass 1 or 2), R4. */
int orc_eta_initial(const orc_region *r, const orc_machine *m, uint32_t pass, uint32_t *eta_out);

#ifdef __cplusplus
}
#endif
#endif
