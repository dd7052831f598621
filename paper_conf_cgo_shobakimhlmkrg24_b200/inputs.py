"""Seeded synthetic inputs: scheduling regions, the machine model and parameters.

This module is the ONLY code shared by the oracle side (oracle/, tests/) and the
CUDA side (the C-ABI library).  It generates DATA -- DDGs with latency-labelled
edges and Def/Use sets of typed virtual registers -- and
holds the default configuration values; it contains none of the method's
arithmetic (no RP, no cost, no selection, no pheromone math).

Workload recipe:
  * instruction mix shaped like a GPU basic block: VALU 55 %, SALU 15 %,
    VMEM load 12 %, SMEM load 8 %, LDS load 5 %, store 5 %;
  * operands pick recent values of the needed class with geometric recency
    (p = 0.15) or, for SGPR operands, a long-lived live-in base (20 %);
  * memory ordering: every load and store depends on the last store (lat 1);
  * 4 SGPR + 8 VGPR live-in registers; unused defs are live-out with p = 0.7;
  * calibration: with recency 0.15 and 8 VGPR live-ins, 56 % of
    the n >= 50 regions of the config-3 batch have a greedy-heuristic VGPR PRP
    above 24 (round 1's 0.3 / 2 gave 35 %), so under APRP_SUM the RP pass has
    occupancy bands to search (tools/calibrate_generator.py);
  * latency profiles "mixed" (VMEM 20-80, SMEM 8-20, LDS 4-8, transcendental
    VALU 4, else 1) and "unit" (all 1);
  * region sizes for the rocPRIM-shaped batch follow Table 3.a's bucket counts
    (728 : 643 : 363 of 1,734 pass-1 regions).
"""
from __future__ import annotations

import dataclasses
from typing import List, Optional, Sequence

import numpy as np

LIVE_IN = 1
LIVE_OUT = 2
VGPR = 0
SGPR = 1


@dataclasses.dataclass
class Region:
    """One scheduling region (a basic block)."""

    n_insts: int
    edge_src: np.ndarray  # uint32 [E]
    edge_dst: np.ndarray  # uint32 [E]
    edge_lat: np.ndarray  # uint32 [E]
    reg_class: np.ndarray  # uint8 [R]
    reg_flags: np.ndarray  # uint8 [R] bit0 LIVE_IN, bit1 LIVE_OUT
    def_ptr: np.ndarray  # uint32 [n+1]
    def_reg: np.ndarray  # uint32
    use_ptr: np.ndarray  # uint32 [n+1]
    use_reg: np.ndarray  # uint32
    name: str = ""
    inst_type: Optional[np.ndarray] = None  # uint8 [n] issue type (R42); None = all type 0

    @property
    def n_edges(self) -> int:
        return int(self.edge_src.shape[0])

    @property
    def n_regs(self) -> int:
        return int(self.reg_class.shape[0])

    @staticmethod
    def from_lists(n, edges, reg_class, reg_flags, defs, uses, name="", inst_type=None):
        """edges: [(src, dst, lat)], defs/uses: per-instruction lists of reg ids."""
        e = np.asarray(edges, dtype=np.uint32).reshape(-1, 3)
        dptr = np.zeros(n + 1, np.uint32)
        uptr = np.zeros(n + 1, np.uint32)
        for j in range(n):
            dptr[j + 1] = dptr[j] + len(defs[j])
            uptr[j + 1] = uptr[j] + len(uses[j])
        dreg = np.asarray([g for d in defs for g in d], np.uint32)
        ureg = np.asarray([g for u in uses for g in u], np.uint32)
        return Region(
            n_insts=n,
            edge_src=np.ascontiguousarray(e[:, 0]),
            edge_dst=np.ascontiguousarray(e[:, 1]),
            edge_lat=np.ascontiguousarray(e[:, 2]),
            reg_class=np.asarray(reg_class, np.uint8),
            reg_flags=np.asarray(reg_flags, np.uint8),
            def_ptr=dptr,
            def_reg=dreg,
            use_ptr=uptr,
            use_reg=ureg,
            name=name,
            inst_type=None if inst_type is None else np.asarray(inst_type, np.uint8),
        )

    def defs(self, j: int) -> List[int]:
        return [int(g) for g in self.def_reg[self.def_ptr[j]:self.def_ptr[j + 1]]]

    def uses(self, j: int) -> List[int]:
        return [int(g) for g in self.use_reg[self.use_ptr[j]:self.use_ptr[j + 1]]]

    def edges(self):
        return [(int(s), int(d), int(l)) for s, d, l in zip(self.edge_src, self.edge_dst, self.edge_lat)]


# --------------------------------------------------------------------------
# Machine model: gfx906 occupancy tables (PAPER.md L70-L72 for the VGPR points;
# the rest of the VGPR table and the SGPR table are AMDGPU facts, not the paper).
# --------------------------------------------------------------------------
@dataclasses.dataclass
class Machine:
    n_classes: int = 2
    occ_max: int = 10
    steps: Sequence[Sequence[int]] = (
        (24, 28, 32, 36, 40, 48, 64, 84, 128, 256),  # VGPR: occupancy 10..1
        (80, 88, 100, 102),  # SGPR: occupancy 10..7
    )
    perp_limit: Sequence[int] = (24, 80, 0, 0)
    # general machine model (L64; R42): issue_width <= 1 = single issue, any type
    issue_width: int = 1
    n_types: int = 1
    type_slots: Sequence[int] = (1, 1, 1, 1)


GFX906 = Machine()
# Issue types of the synthetic generator (R42): VALU, SALU, memory (VMEM/SMEM/LDS/store).
TYPE_VALU, TYPE_SALU, TYPE_MEM = 0, 1, 2
# A dual-issue machine for the general-model rows: two instructions per cycle,
# at most one of each type (a VLIW-like pairing; not a GCN fact).
DUAL_ISSUE = Machine(issue_width=2, n_types=3, type_slots=(1, 1, 1, 1))

# --------------------------------------------------------------------------
# Parameters (defaults: DESIGN.md section 3).  Integers only.
# --------------------------------------------------------------------------
COST_PRP_SUM, COST_APRP_SUM, COST_OCC, COST_PERP = 0, 1, 2, 3
STOP_PAPER_CLASSES = 0xFFFFFFFF


@dataclasses.dataclass
class Params:
    ants: int = 1024
    iterations: int = 10
    seed: int = 0
    passes: int = 3  # 1 RP pass, 2 ILP pass (pass-1 best = heuristic), 3 both
    cost_mode: int = COST_APRP_SUM
    q0_t: int = 3865470566  # floor(0.9 * 2^32)
    group_size: int = 64  # the paper's wavefront (L82, L198)
    stall_mod: int = 4  # a quarter of the wavefronts may stall (L204)
    stall_rem: int = 0
    tau0: int = 4096  # 1.0 in units of 2^-12
    rho_q16: int = 52429  # decay factor 0.8 (L120) in Q0.16
    delta: int = 4096
    tau_min: int = 256
    tau_max: int = 32768
    stop_no_improve: int = 0
    stop_at_lb: int = 0
    # region-level compile policy (L362, L366; R39, R40): 0 = off
    pass2_gap: int = 0
    revert_occ: int = 0
    revert_len: int = 0
    ws_weight: int = 0  # passes == 4: cost = length + ws_weight * cost_rp (L74; R41)
    heur_mix: int = 0  # 1: odd ant groups use the other pass's heuristic (L216-L218; R43)
    stall_num: int = 1  # group g may stall iff (g - stall_rem) % stall_mod < stall_num (R44)
    rl_limit: int = 0  # pass-1 ready-list size limit per ant group (L214; R45): 0 off, 1 min, 2 mid


def paper_policy(p: "Params") -> "Params":
    """The paper's compile-time filters on top of p: stop at the LB (L251),
    size-class termination (L226), pass-2 cycle gap 21 (L362, Table 7) and
    the 3-occupancy / 63-cycle revert filter (L366)."""
    return dataclasses.replace(p, stop_at_lb=1, stop_no_improve=STOP_PAPER_CLASSES, pass2_gap=21,
                               revert_occ=3, revert_len=63)


# --------------------------------------------------------------------------
# Synthetic generator.
# --------------------------------------------------------------------------
_KINDS = ("valu", "salu", "vmem", "smem", "lds", "store")
_MIX = np.array([0.55, 0.15, 0.12, 0.08, 0.05, 0.05])


def gen_region(n: int, seed: int, profile: str = "mixed", name: str = "", recency: float = 0.15,
               v_livein: int = 8) -> Region:
    """A synthetic GPU-basic-block-like region of n instructions (2 classes)."""
    rng = np.random.default_rng(np.uint64(seed))
    reg_class: List[int] = []
    reg_flags: List[int] = []
    pools = {VGPR: [], SGPR: []}

    def new_reg(c, flags=0):
        reg_class.append(c)
        reg_flags.append(flags)
        return len(reg_class) - 1

    for _ in range(4):
        pools[SGPR].append(new_reg(SGPR, LIVE_IN))
    for _ in range(v_livein):
        pools[VGPR].append(new_reg(VGPR, LIVE_IN))
    base = pools[SGPR][0]

    def pick(c):
        if c == SGPR and rng.random() < 0.2:
            return base
        pool = pools[c]
        back = int(rng.geometric(recency)) - 1
        return pool[max(0, len(pool) - 1 - back)]

    def lat_of(kind):
        if profile == "unit":
            return 1
        if kind == "vmem":
            return int(rng.integers(20, 81))
        if kind == "smem":
            return int(rng.integers(8, 21))
        if kind == "lds":
            return int(rng.integers(4, 9))
        if kind == "valu" and rng.random() < 0.1:
            return 4
        return 1

    kinds = rng.choice(len(_KINDS), size=n, p=_MIX)
    defs: List[List[int]] = []
    uses: List[List[int]] = []
    lat = np.zeros(n, np.int64)
    def_by = {}
    last_store = -1
    edge_lat = {}

    def add_edge(s, d, l):
        key = (s, d)
        if edge_lat.get(key, -1) < l:
            edge_lat[key] = l

    for i in range(n):
        kind = _KINDS[int(kinds[i])]
        u: List[int] = []
        d: List[int] = []
        if kind == "valu":
            k = int(rng.choice([1, 2, 3], p=[0.3, 0.5, 0.2]))
            for _ in range(k):
                u.append(pick(VGPR if rng.random() < 0.8 else SGPR))
            d.append(new_reg(VGPR))
        elif kind == "salu":
            for _ in range(int(rng.integers(1, 3))):
                u.append(pick(SGPR))
            d.append(new_reg(SGPR))
        elif kind == "vmem":
            u.append(pick(VGPR))
            u.append(pick(SGPR))
            for _ in range(int(rng.choice([1, 2, 3, 4], p=[0.4, 0.2, 0.1, 0.3]))):
                d.append(new_reg(VGPR))
        elif kind == "smem":
            u.append(pick(SGPR))
            for _ in range(int(rng.integers(1, 3))):
                d.append(new_reg(SGPR))
        elif kind == "lds":
            u.append(pick(VGPR))
            d.append(new_reg(VGPR))
        else:  # store
            u.append(pick(VGPR))
            u.append(pick(VGPR))
            u.append(pick(SGPR))
        # de-duplicate uses, keep first occurrence order
        seen = set()
        u = [g for g in u if not (g in seen or seen.add(g))]
        lat[i] = lat_of(kind)
        for g in u:
            if g in def_by:
                add_edge(def_by[g], i, int(lat[def_by[g]]))
        if kind in ("vmem", "smem", "lds", "store") and last_store >= 0:
            add_edge(last_store, i, 1)
        if kind == "store":
            last_store = i
        for g in d:
            def_by[g] = i
            pools[reg_class[g]].append(g)
        defs.append(d)
        uses.append(u)

    used = set(g for ul in uses for g in ul)
    for g in range(len(reg_class)):
        if reg_flags[g] & LIVE_IN:
            continue
        if g not in used:
            if rng.random() < 0.7:
                reg_flags[g] |= LIVE_OUT
        elif rng.random() < 0.03:
            reg_flags[g] |= LIVE_OUT
    edges = sorted((s, d, l) for (s, d), l in edge_lat.items())
    itype = [TYPE_VALU if _KINDS[int(k)] == "valu" else TYPE_SALU if _KINDS[int(k)] == "salu" else TYPE_MEM
             for k in kinds]
    return Region.from_lists(n, edges, reg_class, reg_flags, defs, uses, name=name or f"synth-n{n}-s{seed}",
                             inst_type=itype)


def region_seed(base: int, region_id: int) -> int:
    """Per-region generator seed = base XOR region id (SplitMix-style mixing)."""
    z = (base ^ (region_id * 0x9E3779B97F4A7C15)) & 0xFFFFFFFFFFFFFFFF
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & 0xFFFFFFFFFFFFFFFF
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & 0xFFFFFFFFFFFFFFFF
    return z ^ (z >> 31)


def c3_sizes(count: int, base_seed: int = 3) -> np.ndarray:
    """Region sizes for the rocPRIM-shaped batch (config 3)."""
    rng = np.random.default_rng(np.uint64(base_seed))
    bucket = rng.choice(3, size=count, p=[728 / 1734, 643 / 1734, 363 / 1734])
    small = rng.integers(20, 50, size=count)
    mid = rng.integers(50, 100, size=count)
    big = np.floor(np.exp(rng.uniform(np.log(100), np.log(501), size=count))).astype(np.int64)
    big = np.clip(big, 100, 500)
    return np.where(bucket == 0, small, np.where(bucket == 1, mid, big)).astype(np.int64)


def c5_sizes(count: int, base_seed: int = 5) -> np.ndarray:
    """Region sizes for the full-suite sweep (config 5): the config-3 mix
    (85 %) plus a heavy tail log-uniform in [500, 4000] (15 %) -- Table 1
    reports regions up to 1,176 / 2,223 instructions (L240-L241); the sweep
    extends to ~4,000 (BASELINE.json)."""
    rng = np.random.default_rng(np.uint64(base_seed) + np.uint64(17))
    base = c3_sizes(count, base_seed)
    tail = np.floor(np.exp(rng.uniform(np.log(500), np.log(4001), size=count))).astype(np.int64)
    pick = rng.random(count) < 0.15
    return np.where(pick, np.clip(tail, 500, 4000), base).astype(np.int64)


def gen_batch(count: int, base_seed: int = 3, profile: str = "mixed", first_id: int = 0,
              sizes: Optional[np.ndarray] = None) -> List[Region]:
    """Regions first_id .. first_id+count-1 of the config-3 batch."""
    if sizes is None:
        sizes = c3_sizes(first_id + count, base_seed)[first_id:]
    return [gen_region(int(sizes[i]), region_seed(base_seed, first_id + i), profile,
                       name=f"c3-{first_id + i}") for i in range(count)]


def gen_regions(ids: Sequence[int], sizes: Sequence[int], base_seed: int = 3, profile: str = "mixed",
                tag: str = "c3") -> List[Region]:
    """Regions with the given global ids of a batch whose region i has size
    sizes[i] (strong scaling: any subset of the same batch, same regions)."""
    return [gen_region(int(sizes[i]), region_seed(base_seed, int(i)), profile, name=f"{tag}-{int(i)}") for i in ids]


# Config 5: n x latency profile x seed grid.
C5_SIZES = (10, 20, 50, 100, 200, 500, 1000, 2000, 4000)
C5_PROFILES = ("unit", "mixed")
C5_SEEDS = (0, 1, 2)


def c5_grid():
    """[(global id, n, profile, seed index)] of the config-5 sweep."""
    out = []
    for n in C5_SIZES:
        for prof in C5_PROFILES:
            for s in C5_SEEDS:
                out.append((len(out), n, prof, s))
    return out


def c5_region(gid: int, n: int, profile: str) -> Region:
    return gen_region(n, region_seed(5, gid), profile, name=f"c5-n{n}-{profile}-{gid}")


# --------------------------------------------------------------------------
# Hand-built fixtures (data only).  FIG1-R reconstructs PAPER.md Fig. 1 from
# its text (L143-L155, L184, L200); FIX10-A is config 1.
# --------------------------------------------------------------------------
def fig1r() -> Region:
    A, B, C, D, E, F, G = range(7)
    edges = [(A, E, 4), (B, E, 4), (C, F, 2), (D, F, 2), (E, G, 1), (F, G, 1)]
    defs = [[0], [1], [2], [3], [4], [5], [6]]
    uses = [[], [], [], [], [0, 1], [2, 3], [4, 5]]
    return Region.from_lists(7, edges, [VGPR] * 7, [0] * 7, defs, uses, name="FIG1-R")


def fix10a() -> Region:
    # registers: Sa0 Vb1 Vc2 Vd3 Sg4 Ve5 Vf6 Vh7 Vi8
    cls = [SGPR, VGPR, VGPR, VGPR, SGPR, VGPR, VGPR, VGPR, VGPR]
    defs = [[0], [1], [2], [3], [4], [5], [6], [7], [8], []]
    uses = [[], [0], [0], [0], [0], [1, 4], [2, 4], [3, 4], [5, 6], [8, 7, 0]]
    lat = [4, 6, 6, 6, 1, 2, 2, 2, 1, 1]
    def_by = {g: j for j, d in enumerate(defs) for g in d}
    edges = sorted({(def_by[g], j, lat[def_by[g]]) for j, u in enumerate(uses) for g in u})
    return Region.from_lists(10, edges, cls, [0] * 9, defs, uses, name="FIX10-A")
