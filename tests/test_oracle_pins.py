"""Pins for the CPU oracle: checks against facts the paper and mathematics fix.

Every test here pins the oracle to something OTHER than itself: the paper's
printed worked example (tests/golden/*.json, with line citations), exhaustive
enumeration (tests/brute.py, an independent interval formulation of RP),
closed forms, Random123 known-answer vectors and statistical properties.
"""
import json
import math
import os

import numpy as np
import pytest

from oracle import pyoracle as O
from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I
from tests import brute, checker

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


# ---------------------------------------------------------------- Philox (R26)
def test_philox_known_answers():
    # Random123 kat_vectors for philox4x32_10 (Salmon et al., SC'11).
    assert O.philox([0, 0, 0, 0], [0, 0]) == [0x6627E8D5, 0xE169C58D, 0xBC57AC4C, 0x9B00DBD8]
    assert O.philox([0xFFFFFFFF] * 4, [0xFFFFFFFF] * 2) == [0x408F276D, 0x41C83B0E, 0xA20BC7C6, 0x6D5451FD]
    assert O.philox([0x243F6A88, 0x85A308D3, 0x13198A2E, 0x03707344], [0xA4093822, 0x299F31D0]) == [
        0xD16CFE09, 0x94FDCCEB, 0x5001E420, 0x24126EA1]


# ------------------------------------------------------- Fig. 1 narrative (L143-L184)
LETTERS = "ABCDEFG"


def test_fig1_pass1_prp():
    g = gold("fig1_paper.json")
    f = I.fig1r()
    ant1 = [LETTERS.index(x) for x in g["order_ant1_prefix"]["value"]] + [4, 5, 6]
    ant2 = [LETTERS.index(x) for x in g["order_ant2_pass1"]["value"]]
    assert O.prp_of_order(f, ant1, 1)[0] == g["prp_ant1"]["value"]
    assert O.prp_of_order(f, ant2, 1)[0] == g["prp_ant2"]["value"]
    # independent interval formulation agrees
    assert brute.prp_interval(f, ant1, 1)[0] == g["prp_ant1"]["value"]
    assert brute.prp_interval(f, ant2, 1)[0] == g["prp_ant2"]["value"]


def test_fig1_best_pass1_prp_is_3_by_enumeration():
    g = gold("fig1_paper.json")
    f = I.fig1r()
    m = I.Machine(n_classes=1, steps=((24, 28, 32, 36, 40, 48, 64, 84, 128, 256),))
    best, _, best_len_t, count, _ = brute.optimum(f, m, 0, target=[3])
    assert best == g["prp_ant2"]["value"]  # "the best PRP at the end of the first pass is 3"
    assert best_len_t == g["len_ant2_pass2"]["value"]  # Ant 2 (10 cycles) "is optimal" (L151)
    assert count == 80


def test_fig1_ready_list_ub():
    g = gold("fig1_paper.json")
    f = I.fig1r()
    m = I.Machine(n_classes=1, steps=((24, 28, 32, 36, 40, 48, 64, 84, 128, 256),))
    _, _, ub = O.lower_bounds(f, m, 0)
    assert ub == g["ready_list_ub"]["value"]
    assert ub < g["ready_list_loose_ub"]["value"]


def test_fig1_two_ant_two_pass_run_reproduces_ant2():
    """One iteration, two ants (L143), both in a stall-enabled wavefront: the
    pass-2 winner is the paper's Ant 2 schedule A1 B2 D3 _4 _5 E6 C7 _8 F9 G10
    (L149, L153-L155, L200)."""
    g = gold("fig1_paper.json")
    f = I.fig1r()
    m = I.Machine(n_classes=1, steps=((24, 28, 32, 36, 40, 48, 64, 84, 128, 256),))
    p = I.Params(ants=2, iterations=1, seed=0, cost_mode=I.COST_PRP_SUM, stall_mod=1)
    r = O.schedule(f, 0, m, p, dump=True, dump_orders=True)
    assert r["best1"] == g["prp_ant2"]["value"]
    assert r["target0"] == g["target_prp"]["value"]
    assert r["length"] == g["len_ant2_pass2"]["value"]
    order = [LETTERS[j] for j in r["order"]]
    cyc1 = [int(c) + 1 for c in r["cycle"]]  # the paper counts cycles from 1
    assert dict(zip(order, cyc1))["D"] == g["ant2_D_cycle_1based"]["value"]
    stalls = sorted(set(range(1, r["length"] + 1)) - set(cyc1))
    assert len(stalls) == g["stalls_ant2"]["value"]
    assert g["ant2_optional_stall_cycle_1based"]["value"] in stalls
    assert g["ant2_necessary_stall_cycle_1based"]["value"] in stalls
    # PRP 2 at cycle 6: live registers right after the instruction in cycle 6
    k6 = cyc1.index(6)
    prefix = [LETTERS.index(x) for x in order]
    live = brute_live_after(f, prefix, k6)
    assert live == g["ant2_prp_at_cycle6"]["value"]
    checker.check_schedule(f, r["order"], r["cycle"], r["length"])
    assert checker.prp(f, r["order"], 1)[0] <= g["target_prp"]["value"]
    # the initial pass-2 schedule (stalls added to the pass-1 best) is longer
    assert r["init2"] > r["length"]


def brute_live_after(region, order, k):
    pos = {j: i for i, j in enumerate(order)}
    live = 0
    for g in range(region.n_regs):
        d = [j for j in range(region.n_insts) if g in region.defs(j)]
        u = [pos[j] for j in range(region.n_insts) if g in region.uses(j)]
        s = pos[d[0]]
        e = max(u) if u else s
        if s <= k < e or s == k:
            live += 1
    return live


# ------------------------------------------------------------- APRP (L70-L72)
def test_aprp_and_occupancy_points():
    g = gold("occupancy_paper.json")
    m = I.GFX906
    for key in ("aprp_24", "aprp_28"):
        lo, hi = g[key]["prp_range"]
        for x in range(lo, hi + 1):
            assert O.aprp(m, 0, x) == g[key]["value"]
    for key in ("vgpr_max_occupancy", "vgpr_occupancy_9"):
        lo, hi = g[key]["prp_range"]
        for x in range(lo, hi + 1):
            assert O.occupancy(m, 0, x) == g[key]["value"]


def test_aprp_is_max_prp_with_same_occupancy():
    """APRP(x) = max{y : occ(y) == occ(x)} (L70) checked by search."""
    m = I.GFX906
    for c in range(2):
        top = m.steps[c][-1]
        for x in range(0, top + 1):
            same = [y for y in range(0, top + 1) if O.occupancy(m, c, y) == O.occupancy(m, c, x)]
            assert O.aprp(m, c, x) == max(same)


def test_cost_modes_monotone():
    m = I.GFX906
    rng = np.random.default_rng(1)
    for _ in range(300):
        a = rng.integers(0, 120, size=2)
        b = a + rng.integers(0, 5, size=2)
        for mode in range(4):
            assert O.cost_rp(m, mode, list(a)) <= O.cost_rp(m, mode, list(b))
            assert O.cost_rp(m, mode, list(a)) == brute.cost(m, mode, list(a) + [0, 0])


def test_target_is_largest_prp_of_equal_cost():
    """Pass-2 target keeps the pass-1 best cost class (L108, L147): any PRP
    vector <= target costs no more than the best, and raising any class above
    target (PRP_SUM / APRP_SUM) would cost more."""
    m = I.GFX906
    rng = np.random.default_rng(2)
    for _ in range(200):
        best = [int(x) for x in rng.integers(0, 110, size=2)]
        for mode in (0, 1, 3):
            t = O.target(m, mode, best)
            assert O.cost_rp(m, mode, t[:2]) == O.cost_rp(m, mode, best)
            if mode in (0, 1):
                for c in range(2):
                    up = list(t[:2])
                    up[c] += 1
                    assert O.cost_rp(m, mode, up) > O.cost_rp(m, mode, best)


# ------------------------------------------------------- FIX10-A (config 1)
def test_fix10a_enumeration_facts():
    x = I.fix10a()
    m = I.GFX906
    assert x.n_edges == 15
    best, best_len, best_len_t, count, vecs = brute.optimum(x, m, 0, target=[2, 2])
    assert count == 400
    assert vecs == {(2, 2), (3, 2)}
    assert best == 4
    assert best_len == 15
    assert best_len_t == 23
    assert O.critical_path(x) == [13, 9, 9, 8, 4, 3, 3, 2, 1, 0]
    lb1, lblen, _ = O.lower_bounds(x, m, 0)
    assert lb1 <= best and lblen <= best_len
    # oracle PRP == interval PRP on every order
    for o in list(brute.topo_orders(x))[:400:7]:
        assert O.prp_of_order(x, o, 2)[:2] == brute.prp_interval(x, o, 2)[:2]
        assert O.asap(x, o)[0] == brute.asap(x, o)[0]


def test_fix10a_without_optional_stalls_no_feasible_schedule():
    """Under target (2,2) no schedule exists that stalls only when nothing is
    latency-ready -- so ants outside the stall-enabled quarter (L204) must die,
    consistent with L391 ('impossible to find an optimal schedule')."""
    x = I.fix10a()
    assert brute.no_optional_stall_schedules(x, [2, 2]) == 0
    p = I.Params(ants=128, iterations=2, seed=3, cost_mode=0)
    r = O.schedule(x, 0, I.GFX906, p, dump=True)
    if r["target0"] == 2 and r["target1"] == 2:
        costs = r["dump_cost"][1]  # pass 2
        for it in range(costs.shape[0]):
            for a in range(128):
                if (a // 64) % 4 != 0:
                    assert costs[it, a] == O.INVALID


@pytest.mark.parametrize("seed", range(10))
def test_fix10a_config1_reaches_optimum(seed):
    """Config 1: 64 ants x 20 iterations, PRP_SUM.  Hard: never below the
    enumerated optimum.  Pass 2 always meets its own target's optimum 23 when
    pass 1 reached (2,2)."""
    x = I.fix10a()
    p = I.Params(ants=64, iterations=20, seed=seed, cost_mode=0)
    r = O.schedule(x, 0, I.GFX906, p)
    checker.check_schedule(x, r["order"], r["cycle"], r["length"])
    prp = checker.prp(x, r["order"], 2)
    assert prp[:2] == r["prp"][:2]
    assert r["best1"] >= 4
    tgt = [r["target0"], r["target1"]]
    _, _, opt_t, _, _ = brute.optimum(x, I.GFX906, 0, target=tgt)
    assert r["length"] >= opt_t
    assert prp[0] <= tgt[0] and prp[1] <= tgt[1]
    if tgt == [2, 2]:
        assert r["length"] == 23


# ------------------------------------------------------- selection (R1, R27)
def test_roulette_exact_cases():
    s = [1, 2, 3]  # prefixes 1, 3, 6; r = floor(R64 * 6 / 2^64)
    def r64_for(r):
        return ((r * (1 << 64)) + 5) // 6  # smallest R64 with floor(R64*6/2^64) == r
    assert O.select(s, False, r64_for(0)) == 0
    assert O.select(s, False, r64_for(1)) == 1
    assert O.select(s, False, r64_for(2)) == 1
    assert O.select(s, False, r64_for(3)) == 2
    assert O.select(s, False, (1 << 64) - 1) == 2
    assert O.select([5, 9, 9, 1], True, 0) == 1  # argmax, ties to lowest
    assert O.select([7], False, 123) == 0


def test_roulette_frequencies_chi2():
    from scipy.stats import chisquare
    rng = np.random.default_rng(7)
    s = [1, 2, 3, 4, 10]
    N = 20000
    counts = np.zeros(len(s))
    for r in rng.integers(0, 2**63, size=N, dtype=np.uint64):
        counts[O.select(s, False, int(r) * 2 + 1)] += 1
    exp = np.array(s) / sum(s) * N
    assert chisquare(counts, exp).pvalue > 1e-3


def independent_greedy(region):
    """Textbook list scheduling [1] with priority (LUC, CP), ties to the lowest
    index -- written from the definitions, not from the oracle."""
    n = region.n_insts
    P = brute.preds_of(region)
    cp = [0] * n
    for j in reversed(range(n)):  # program order is topological
        for s, d, l in region.edges():
            if s == j:
                cp[j] = max(cp[j], l + cp[d])
    users = {}
    for j in range(n):
        for g in set(region.uses(j)):
            users.setdefault(g, set()).add(j)
    done, order = set(), []
    for _ in range(n):
        ready = [j for j in range(n) if j not in done and all(p in done for p, _ in P[j])]
        def luc(j):
            return sum(1 for g in set(region.uses(j))
                       if not (region.reg_flags[g] & 2) and users[g] - done == {j})
        j = max(ready, key=lambda j: (luc(j), cp[j], -j))
        order.append(j)
        done.add(j)
    return order


@pytest.mark.parametrize("seed", range(6))
def test_q0_one_every_ant_is_the_list_schedule(seed):
    """P1 special case: q0 = 1 on a uniform tau => every pass-1 ant of the first
    iteration equals the textbook greedy list schedule (L122)."""
    reg = I.gen_region(24, 100 + seed)
    m = I.GFX906
    p = I.Params(ants=8, iterations=1, seed=seed, q0_t=1 << 32, passes=1, cost_mode=0)
    r = O.schedule(reg, 5, m, p, dump=True, dump_orders=True)
    g = independent_greedy(reg)
    for a in range(8):
        assert list(r["dump_order"][0, 0, a]) == g
    assert list(O.greedy_pass1(reg, m, p)[0]) == g


def test_eta_normalisation_range_and_order():
    reg = I.gen_region(60, 11)
    for ps in (1, 2):
        e = O.eta_initial(reg, I.GFX906, ps)
        assert min(e) >= 1 and max(e) <= 65535
    cp = O.critical_path(reg)
    e2 = O.eta_initial(reg, I.GFX906, 2)
    for a in range(reg.n_insts):
        for b in range(reg.n_insts):
            if cp[a] < cp[b]:
                assert e2[a] <= e2[b]
    assert e2[cp.index(max(cp))] == 65535


# ------------------------------------------------------- pheromone (R6-R9)
def test_evaporation_only_trajectory_bounds():
    """Decay-only (no valid winner): tau_k lies within the floor-error band of
    tau0 * 0.8^k (L120) until it clamps at tau_min."""
    p = I.Params()
    n = 3
    tau = np.full((n + 1) * n, p.tau0, np.uint16)
    for k in range(1, 30):
        tau = O.pheromone_update(tau, n, None, p)
        exact = p.tau0 * 0.8**k
        upper = p.tau0 * (p.rho_q16 / 65536) ** k
        v = int(tau[0])
        assert np.all(tau == tau[0])
        if exact - 5 > p.tau_min:
            assert exact - 5 <= v <= upper + 1e-9
        if upper < p.tau_min:
            assert v == p.tau_min
    # reaching tau_min = tau0/16 takes ceil(log 16 / log 1.25) ~ 13 decays
    tau = np.full((n + 1) * n, p.tau0, np.uint16)
    k = 0
    while tau[0] > p.tau_min:
        tau = O.pheromone_update(tau, n, None, p)
        k += 1
    assert k in (12, 13)


def test_deposit_fixpoint_and_links():
    """A link deposited every iteration converges to the fixpoint of
    x = 0.8 x + delta, i.e. 5 * delta; only the winner's n links gain."""
    p = I.Params()
    n = 5
    w = [3, 1, 4, 0, 2]
    tau = np.full((n + 1) * n, p.tau0, np.uint16)
    for _ in range(200):
        tau = O.pheromone_update(tau, n, w, p)
    T = tau.reshape(n + 1, n)
    links = {(n, w[0])} | {(w[k], w[k + 1]) for k in range(n - 1)}
    for i in range(n + 1):
        for j in range(n):
            if (i, j) in links:
                assert abs(int(T[i, j]) - 5 * p.delta) <= 5
            else:
                assert int(T[i, j]) == p.tau_min
    one = O.pheromone_update(np.full((n + 1) * n, p.tau0, np.uint16), n, w, p).reshape(n + 1, n)
    assert int((one > one.min()).sum()) == n


def test_pheromone_clamps_at_tau_max():
    p = I.Params(delta=30000)
    n = 2
    tau = np.full((n + 1) * n, p.tau0, np.uint16)
    for _ in range(10):
        tau = O.pheromone_update(tau, n, [0, 1], p)
    assert int(tau.max()) == p.tau_max


# --------------------------------------------------- closed forms for ASAP (R29)
def test_asap_chain_and_antichain():
    n = 6
    lats = [3, 1, 7, 2, 5]
    chain = I.Region.from_lists(n, [(i, i + 1, lats[i]) for i in range(n - 1)], [], [],
                                [[] for _ in range(n)], [[] for _ in range(n)])
    L, _ = O.asap(chain, list(range(n)))
    assert L == sum(lats) + 1
    anti = I.Region.from_lists(n, [], [], [], [[] for _ in range(n)], [[] for _ in range(n)])
    assert O.asap(anti, [5, 3, 1, 0, 2, 4])[0] == n


def test_chain_is_at_lower_bound_and_skipped():
    """Heuristic cost == LB => ACO is not invoked (L251): 0 iterations run."""
    n = 8
    chain = I.Region.from_lists(n, [(i, i + 1, 1) for i in range(n - 1)], [0] * (n - 1), [0] * (n - 1),
                                [[i] for i in range(n - 1)] + [[]], [[]] + [[i - 1] for i in range(1, n)])
    p = I.Params(ants=16, iterations=5, stop_at_lb=1, cost_mode=0)
    r = O.schedule(chain, 0, I.GFX906, p)
    assert r["iters1"] == 0 and r["iters2"] == 0
    assert r["length"] == r["lblen"] == n


# ------------------------------------------ random tiny DDGs: brute force
@pytest.mark.parametrize("seed", range(12))
def test_random_tiny_regions_against_enumeration(seed):
    reg = I.gen_region(8, 1000 + seed, profile="mixed" if seed % 2 else "unit")
    m = I.GFX906
    for mode in (0, 1):
        p = I.Params(ants=32, iterations=4, seed=seed, cost_mode=mode, stall_mod=1)
        r = O.schedule(reg, seed, m, p, dump=True, dump_orders=True)
        tgt = [r["target0"], r["target1"]]
        best, best_len, best_len_t, _, _ = brute.optimum(reg, m, mode, target=tgt)
        lb1, lblen, _ = O.lower_bounds(reg, m, mode)
        assert lb1 <= best and lblen <= best_len
        assert r["best1"] >= best
        assert r["length"] >= best_len_t
        checker.check_schedule(reg, r["order"], r["cycle"], r["length"])
        prp = checker.prp(reg, r["order"])
        assert prp == r["prp"]
        assert prp[0] <= tgt[0] and prp[1] <= tgt[1]
        # every dumped ant: valid order, its reported cost recomputed independently
        for it in range(p.iterations):
            for a in range(p.ants):
                o = r["dump_order"][0, it, a]
                checker.check_order(reg, o)
                assert r["dump_cost"][0, it, a] == brute.cost(m, mode, checker.prp(reg, o))
                c2 = r["dump_cost"][1, it, a]
                if c2 != O.INVALID:
                    o2 = r["dump_order"][1, it, a]
                    y2 = r["dump_cycle"][1, it, a]
                    checker.check_schedule(reg, o2, y2, int(c2))
                    p2 = checker.prp(reg, o2)
                    assert p2[0] <= tgt[0] and p2[1] <= tgt[1]


# -------------------------------------------------------- validation (R31-R38)
def _tiny(edges, defs, uses, cls=None, flags=None, n=3):
    R = 1 + max([g for d in defs for g in d] + [g for u in uses for g in u] + [-1])
    return I.Region.from_lists(n, edges, cls or [0] * R, flags or [0] * R, defs, uses)


def test_validation_errors():
    ok = _tiny([(0, 1, 1), (1, 2, 1)], [[0], [1], []], [[], [0], [1]])
    assert O.validate(ok) == 0
    assert O.validate(_tiny([(0, 1, 1), (1, 0, 1)], [[], [], []], [[], [], []])) == -2
    assert O.validate(_tiny([(0, 0, 1)], [[], [], []], [[], [], []])) == -2
    assert O.validate(_tiny([(0, 1, 1)], [[0], [0], []], [[], [], []])) == -3
    assert O.validate(_tiny([(0, 1, 1)], [[0], [], []], [[], [], [0]])) == -4
    assert O.validate(_tiny([(0, 1, 1), (0, 1, 2)], [[], [], []], [[], [], []])) == -1
    assert O.validate(_tiny([], [[], [], []], [[], [], [0]])) == -1  # undefined, not live-in
    assert O.validate(_tiny([], [[0], [], []], [[], [], []], flags=[1])) == -3  # defines a live-in


def test_empty_and_single_instruction_regions():
    m = I.GFX906
    p = I.Params(ants=8, iterations=2)
    empty = I.Region.from_lists(0, [], [1], [1], [], [])
    r = O.schedule(empty, 0, m, p)
    assert r["length"] == 0 and r["prp"][1] == 1
    one = I.Region.from_lists(1, [], [0, 1], [0, 1], [[0]], [[1]])
    r = O.schedule(one, 0, m, p)
    assert r["length"] == 1 and list(r["order"]) == [0]
