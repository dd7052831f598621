/*
 * aco.h -- C ABI of the B200-native ACO instruction scheduler.
 *
 * Method: Ant Colony Optimization for register-pressure-aware instruction
 * scheduling of basic-block DDGs, two-pass form (RP pass, then ILP pass), as
 * parallelised on the GPU by Shobaki et al., "Instruction Scheduling for the
 * GPU on the GPU", CGO 2024.  "L<n>" below is a line of
 * /root/reference/PAPER.md; "R<k>" is a reading in DESIGN.md section 3.
 *
 * Conventions (all entry points):
 *  - Plain C types only; no C++ or torch types cross this boundary.
 *  - Every call returns an aco_status: 0 on success, a negative code on
 *    error.  Calls never throw, never abort and never print.
 *  - The library never allocates device memory.  Device buffers (the region
 *    arena and the run workspace) are allocated by the caller (PyTorch in the
 *    Python binding) after a sizing call that passes a NULL buffer and
 *    receives the byte count in *_needed.  Buffers must be 256-byte aligned.
 *  - All device work is enqueued on the caller's CUDA stream (a cudaStream_t
 *    passed as void*; NULL = legacy default stream).  Only aco_get_results
 *    and aco_get_dump synchronise (with that stream).
 *  - A context is bound to one device and is not thread-safe.
 */
#ifndef ACO_H
#define ACO_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef int32_t aco_status;
enum {
  ACO_OK = 0,
  ACO_E_ARG = -1,             /* bad argument, duplicate edge, undefined use, ... */
  ACO_E_DDG_CYCLE = -2,       /* the DDG is not acyclic (R31) */
  ACO_E_DDG_MULTIDEF = -3,    /* a register defined twice, or a live-in defined (R34) */
  ACO_E_DDG_USE_NO_EDGE = -4, /* j uses r defined by i but the edge i->j is missing (R38) */
  ACO_E_TOO_LARGE = -5,       /* over a compiled limit (see ACO_MAX_*) */
  ACO_E_WORKSPACE = -6,       /* buffer missing or smaller than *_needed */
  ACO_E_CUDA = -7,            /* a CUDA runtime error */
  ACO_E_STATE = -8            /* call out of order (e.g. schedule before load) */
};

/* Compiled limits. */
#define ACO_MAX_INSTS 65535u   /* instruction ids are u16 on the device */
#define ACO_MAX_INDEG 255u     /* predecessor counters are u8 per ant */
#define ACO_MAX_USES 65535u    /* remaining-use counters are u16 per ant */
#define ACO_MAX_CLASSES 4u
#define ACO_MAX_LATENCY 65535u

typedef struct aco_ctx_s *aco_ctx;

/* One scheduling region = one DDG (L62): node = instruction (ids 0..n-1 in
 * program order), edge = dependency labelled with a latency in cycles (used by
 * the ILP pass only, L108), plus the Def and Use sets of typed virtual
 * registers (L66).  All pointers are HOST pointers; the data is copied during
 * aco_load_regions and may be freed when it returns. */
typedef struct {
  uint32_t region_id; /* global id, unique in the batch; part of the Philox key (R26) */
  uint32_t n_insts, n_edges, n_regs;
  const uint32_t *edge_src, *edge_dst, *edge_lat; /* [n_edges]; no duplicate (src,dst) pairs */
  const uint8_t *reg_class;                       /* [n_regs] class < n_classes (0 VGPR, 1 SGPR) */
  const uint8_t *reg_flags;                       /* [n_regs] bit0 LIVE_IN, bit1 LIVE_OUT */
  const uint32_t *def_ptr, *def_reg;              /* CSR: defs of j = def_reg[def_ptr[j]..def_ptr[j+1]) */
  const uint32_t *use_ptr, *use_reg;              /* CSR: uses of j (duplicates count once, R33) */
  const uint8_t *inst_type; /* [n_insts] issue type of each instruction for the general machine
                               model (L64; R42), < aco_machine.n_types; NULL = all type 0 */
} aco_region_desc;

/* Occupancy model per register class (L68-L72; R16, R17).  step_max[c][i] is
 * the largest PRP giving occupancy occ_max - i, ascending in i; PRP above the
 * last step has occupancy 0 and APRP(x) = x. */
typedef struct {
  uint32_t n_classes, occ_max;
  uint32_t step_count[4];
  uint32_t step_max[4][16];
  uint32_t perp_limit[4];
  /* General machine model (L64 "supports a general machine model"; R42).
   * issue_width <= 1: single issue, any instruction type per cycle (the
   * paper's experiments, R32; n_types / type_slots ignored).  Otherwise at
   * most issue_width instructions per cycle, of which at most type_slots[y]
   * of issue type y < n_types <= 4.  Affects the ILP pass (and pass 4), the
   * ASAP timing of R29 and LB_len; the RP pass ignores latencies (R19). */
  uint32_t issue_width, n_types;
  uint32_t type_slots[4];
} aco_machine;

enum { ACO_COST_PRP_SUM = 0, ACO_COST_APRP_SUM = 1, ACO_COST_OCC = 2, ACO_COST_PERP = 3 };

enum {
  ACO_FLAG_NO_PRUNE = 1u, /* disable the winner-invariant pass-2 prune (R24) */
  ACO_FLAG_DUMP = 2u,     /* record every ant (costs, orders, cycles) into the dump buffers */
  ACO_FLAG_TIMING = 4u    /* record CUDA events around every phase (see aco_get_timing) */
};

/* Run parameters (defaults in DESIGN.md section 3). */
typedef struct {
  uint32_t ants;       /* ants per region per iteration (A) */
  uint32_t iterations; /* iterations per pass (a hard cap, R12) */
  uint64_t seed;       /* Philox key (R26) */
  uint32_t pass;       /* 1 RP pass, 2 ILP pass from the heuristic, 3 both (L108),
                          4 single weighted-sum pass (L74; R41) */
  uint32_t cost_mode;  /* ACO_COST_* (R16) */
  uint64_t q0_t;       /* exploit iff group coin < q0_t; 2^32 = always (R1-R3) */
  uint32_t group_size; /* ants sharing the exploit/explore coin (L198), default 64 */
  uint32_t stall_mod, stall_rem; /* group g may take optional stalls iff g % mod == rem (L204) */
  uint32_t tau0, rho_q16, delta, tau_min, tau_max; /* pheromone, u16 units of 2^-12 (R6, R7) */
  uint32_t stop_no_improve; /* 0 = off, 0xFFFFFFFF = paper size classes 1/2/3 (L226) */
  uint32_t stop_at_lb;      /* stop a pass when its best cost equals the LB (L110, L251) */
  uint32_t flags;           /* ACO_FLAG_* */
  /* region-level compile policy (L362, L366, L393-L417; R39, R40) */
  uint32_t pass2_gap;       /* run pass 2 only if initial length - LB_len >= pass2_gap (0 off; paper 21) */
  uint32_t revert_occ;      /* report the heuristic schedule when ACO gains >= revert_occ occupancy */
  uint32_t revert_len;      /*   but lengthens the schedule by > revert_len cycles (paper 3, 63; 0 off) */
  uint32_t ws_weight;       /* pass 4: cost = length + ws_weight * cost_rp (<= 1024; R41) */
  uint32_t heur_mix;        /* 1: odd ant groups use the other pass's heuristic (L216-L218; R43) */
  uint32_t stall_num;       /* group g may stall iff (g - stall_rem) % stall_mod < stall_num (R44; paper 1) */
  uint32_t rl_limit;        /* pass-1 ready-list size limit per ant group (L214; R45): 0 off (default),
                               1 = the group's minimum ready-list size, 2 = midpoint of its min and max.
                               Not with the shared colony, nor for regions that need the
                               global-state kernels (ACO_E_ARG) */
} aco_params;

/* Per-region result (sizes fixed; the schedule itself is returned through
 * the order/cycle arrays of aco_get_results). */
typedef struct {
  uint32_t n_insts;
  uint32_t cost_rp;      /* cost of the final schedule's PRP (R16) */
  uint32_t length;       /* final schedule length = last cycle + 1 (R20) */
  uint32_t prp[4];       /* final PRP per class */
  uint32_t iters_run[2]; /* iterations run in pass 1 / pass 2 */
  uint32_t best_cost[2]; /* pass-1 best cost, pass-2 best length */
  uint32_t init_cost[2]; /* heuristic pass-1 cost, initial pass-2 length */
  uint32_t lb_cost, lb_len; /* lower bounds (R30) */
  uint32_t target[4];    /* pass-2 PRP target per class (R18) */
  uint64_t trace_hash;   /* FNV-1a over (pass, iter, winner cost, winner ant) */
  uint32_t policy;       /* bit0: pass 2 filtered by the cycle gap (R39); bit1: reverted (R40) */
  uint32_t heur_len;     /* length of the heuristic schedule (greedy order timed ASAP, R40) */
  uint32_t ws_cost;      /* pass 4: final weighted cost (R41), else 0 */
  uint32_t ants_pruned;  /* pass-2 ants cut short by the winner-invariant prune (R24), all iterations */
  uint32_t heur_prp[4];  /* PRP per class of the greedy heuristic schedule (R28), the RP pass's start */
} aco_result;

/* Create a context on CUDA device `device` for machine model *m (copied). */
aco_status aco_create(int device, const aco_machine *m, aco_ctx *out);

/* Validate and preprocess `count` regions (host C++), and copy their statics
 * into the caller's device arena with one H2D copy on `cuda_stream`.
 * Sizing: call with d_arena == NULL to get *arena_needed (validation runs).
 * All-or-nothing: on error nothing is loaded.  Region ids must be unique.
 * Replaces any previously loaded batch. */
aco_status aco_load_regions(aco_ctx ctx, const aco_region_desc *regions, uint32_t count,
                            void *d_arena, size_t arena_bytes, size_t *arena_needed,
                            void *cuda_stream);

/* Run the two-pass ACO over every loaded region (L106-L139): per pass and
 * iteration, ant construction (one ant per thread), best-ant argmin with the
 * winner replay, pheromone evaporate+deposit and the global-best epilogue.
 * Sizing: d_workspace == NULL returns *ws_needed.  The workspace must stay
 * allocated until aco_get_results/aco_get_dump return.  dump buffers
 * (ACO_FLAG_DUMP) are given with aco_set_dump before this call. */
aco_status aco_schedule_batch(aco_ctx ctx, const aco_params *p, void *d_workspace,
                              size_t ws_bytes, size_t *ws_needed, void *cuda_stream);

/* Synchronise and copy results of regions [first, first+count) (load order)
 * to host memory.  orders/cycles (may be NULL) receive the regions' final
 * instruction orders / issue cycles concatenated in load order (sum of n). */
aco_status aco_get_results(aco_ctx ctx, uint32_t first, uint32_t count, aco_result *out,
                           uint32_t *orders, uint32_t *cycles);

/* Dump buffers for ACO_FLAG_DUMP (device pointers, caller-owned), with their
 * sizes in ELEMENTS:
 *   costs : u32 [2][iterations][count][ants]            (INVALID = 0xFFFFFFFF)
 *   orders: u16 [2][iterations][sum over regions of ants * n]   (may be NULL)
 *   cycles: u32 same shape as orders, pass-2 issue cycles       (may be NULL)
 * Region r's block in a (pass, iteration) slice starts at ants * sum_{q<r} n_q.
 * aco_schedule_batch with ACO_FLAG_DUMP returns ACO_E_WORKSPACE when a given
 * buffer is smaller than the loaded batch and parameters need. */
aco_status aco_set_dump(aco_ctx ctx, uint32_t *d_costs, uint64_t costs_len, uint16_t *d_orders,
                        uint64_t orders_len, uint32_t *d_cycles, uint64_t cycles_len);

/* ---- Shared colony (config 4): the ants of the loaded regions are split
 * across ranks (one context per GPU).  Ant ids are global: this context runs
 * ants [ant_base, ant_base + p->ants) of p->ants * world ants.  Per pass and
 * iteration the caller runs
 *     aco_colony_construct(ctx, pass, iter, keys, stream)   (local ants; keys[r] = local best)
 *     allreduce(keys, MIN) over ranks, on `stream`           (int64, one per region)
 *     aco_colony_finalize(ctx, pass, iter, keys, stream)     (replay of the global winner,
 *                                                             identical pheromone update)
 * for pass in the requested passes and iter < p->iterations (stop rules are
 * evaluated identically on every rank; finished regions idle), then
 * aco_colony_end.  keys is a caller-owned device buffer of count int64:
 * key = ((cost << 32) | global ant) XOR 2^63, so a signed MIN selects the
 * lexicographically smallest (cost, ant) (R10).  The winner's order is never
 * sent: every rank replays it from its identical pheromone table.  Results
 * are bit-identical to one context running all ants (tested). */
aco_status aco_colony_begin(aco_ctx ctx, const aco_params *p, uint32_t ant_base, void *d_workspace,
                            size_t ws_bytes, size_t *ws_needed, void *cuda_stream);
aco_status aco_colony_construct(aco_ctx ctx, uint32_t pass, uint32_t iter, int64_t *d_keys, void *cuda_stream);
aco_status aco_colony_finalize(aco_ctx ctx, uint32_t pass, uint32_t iter, int64_t *d_keys, void *cuda_stream);
aco_status aco_colony_end(aco_ctx ctx, void *cuda_stream);

/* Device time of the phases of the last aco_schedule_batch run with
 * ACO_FLAG_TIMING (synchronises).  ms[0] = ant construction (all
 * k_construct launches), ms[1] = finalize (argmin + replay + pheromone +
 * epilogue), ms[2] = init + pass transition; launches[0..2] likewise.
 * Each interval is bracketed by cudaEventRecord on the launching stream. */
aco_status aco_get_timing(aco_ctx ctx, double ms[3], uint64_t launches[3]);

/* Number of kernel launches enqueued by the last aco_schedule_batch. */
aco_status aco_last_launch_count(aco_ctx ctx, uint64_t *launches);

/* Construct-kernel variants (the instantiation of the ant-construction
 * kernel each launch class uses) planned by the last aco_schedule_batch or
 * aco_colony_begin on this context, sizing calls included (the plan is made
 * without running).  codes: caller buffer of cap entries (may be NULL when
 * cap == 0); *count = number of distinct codes (ascending).  Code bits:
 * 0 4-wide candidate scan, 1 per-ant state in global memory, 2 3-4 register
 * classes, 3 u32 pass-2 cycles, 4 pheromone staged in shared memory, 5
 * word-mask bitset scan (n <= 1024), 6-7 lanes per ant (0:1 1:2 2:4 3:>=8),
 * 8 pass 2, 9 lanes >= 16, 10 lanes 32, 11 block image read through L1,
 * 12 lean pass-2 layout.  Used by the tests to prove that every variant a
 * benchmark launches is covered by an every-ant parity test. */
aco_status aco_last_variants(aco_ctx ctx, uint32_t *codes, uint32_t cap, uint32_t *count);

/* Human-readable name of a status code (static storage). */
const char *aco_status_string(aco_status st);

/* Destroy a context (does not free caller-owned device buffers). */
void aco_destroy(aco_ctx ctx);

#ifdef __cplusplus
}
#endif
#endif /* ACO_H */
