"""Independent brute-force reference for tiny DDGs (test code, not the oracle).

Written from the problem statement with its own
formulation of register pressure -- live INTERVALS instead of the oracle's
event simulation -- so that a mistake in either shows up as a mismatch.

Interval reading of DESIGN.md R14/R15: register r of class c has
  start = position of its def (or -1 for a live-in register),
  end   = position of its last use, or +inf if LIVE_OUT (or a live-in with
          no use), or = start for a dead def;
and it is counted at point k in {-1, 0, .., n-1} iff start <= k < end or
start == k.  (A last use at k is released before k's defs: kill-before-def.)
"""
from __future__ import annotations

import math
from typing import Dict, Iterator, List, Sequence, Tuple

LIVE_IN, LIVE_OUT = 1, 2


def preds_of(region) -> Dict[int, List[Tuple[int, int]]]:
    P = {j: [] for j in range(region.n_insts)}
    for s, d, l in region.edges():
        P[d].append((s, l))
    return P


def topo_orders(region) -> Iterator[List[int]]:
    n = region.n_insts
    P = preds_of(region)
    need = [len(P[j]) for j in range(n)]
    S = {j: [] for j in range(n)}
    for s, d, _ in region.edges():
        S[s].append(d)
    order: List[int] = []
    used = [False] * n

    def rec():
        if len(order) == n:
            yield list(order)
            return
        for j in range(n):
            if not used[j] and need[j] == 0:
                used[j] = True
                order.append(j)
                for v in S[j]:
                    need[v] -= 1
                yield from rec()
                for v in S[j]:
                    need[v] += 1
                order.pop()
                used[j] = False

    yield from rec()


def prp_interval(region, order: Sequence[int], n_classes: int = 2) -> List[int]:
    n = region.n_insts
    pos = {j: k for k, j in enumerate(order)}
    inf = math.inf
    start, end = {}, {}
    for g in range(region.n_regs):
        if region.reg_flags[g] & LIVE_IN:
            start[g] = -1
    last_use: Dict[int, int] = {}
    for j in range(n):
        for g in set(region.uses(j)):
            last_use[g] = max(last_use.get(g, -1), pos[j])
        for g in region.defs(j):
            start[g] = pos[j]
    for g in range(region.n_regs):
        if g not in start:
            continue
        if region.reg_flags[g] & LIVE_OUT:
            end[g] = inf
        elif g in last_use:
            end[g] = last_use[g]
        elif region.reg_flags[g] & LIVE_IN:
            end[g] = inf
        else:
            end[g] = start[g]
    prp = [0, 0, 0, 0]
    for k in range(-1, n):
        cnt = [0, 0, 0, 0]
        for g, s in start.items():
            if (s <= k < end[g]) or s == k:
                cnt[int(region.reg_class[g])] += 1
        prp = [max(a, b) for a, b in zip(prp, cnt)]
    return prp


def asap(region, order: Sequence[int]) -> Tuple[int, List[int]]:
    """Earliest cycles for a fixed order on a single-issue machine."""
    P = preds_of(region)
    cyc: Dict[int, int] = {}
    t_prev = -1
    out = []
    for j in order:
        t = t_prev + 1
        for p, l in P[j]:
            t = max(t, cyc[p] + l)
        cyc[j] = t
        out.append(t)
        t_prev = t
    return (t_prev + 1 if order else 0), out


def aprp(steps: Sequence[int], x: int) -> int:
    for s in steps:
        if x <= s:
            return s
    return x


def cost(machine, mode: int, prp: Sequence[int]) -> int:
    nc = machine.n_classes
    if mode == 0:
        return sum(prp[:nc])
    if mode == 1:
        return sum(aprp(machine.steps[c], prp[c]) for c in range(nc))
    if mode == 2:
        occ = machine.occ_max
        for c in range(nc):
            o = 0
            for i, s in enumerate(machine.steps[c]):
                if prp[c] <= s:
                    o = machine.occ_max - i
                    break
            occ = min(occ, o)
        return machine.occ_max - occ
    return sum(max(0, prp[c] - machine.perp_limit[c]) for c in range(nc))


def optimum(region, machine, mode: int, target=None):
    """(best pass-1 cost, best unconstrained length, best length under target,
    number of orders, set of PRP vectors)."""
    best_c = math.inf
    best_len = math.inf
    best_len_t = math.inf
    count = 0
    vecs = set()
    for o in topo_orders(region):
        count += 1
        prp = prp_interval(region, o, machine.n_classes)
        vecs.add(tuple(prp[:machine.n_classes]))
        best_c = min(best_c, cost(machine, mode, prp))
        L, _ = asap(region, o)
        best_len = min(best_len, L)
        if target is not None and all(prp[c] <= target[c] for c in range(machine.n_classes)):
            best_len_t = min(best_len_t, L)
    return best_c, best_len, best_len_t, count, vecs


def no_optional_stall_schedules(region, target, n_classes=2):
    """Count complete pass-2 schedules that never stall while some instruction
    is latency-ready (only necessary stalls), and whose running peak stays
    within target -- an exhaustive DFS over the choices."""
    n = region.n_insts
    P = preds_of(region)
    found = 0
    order: List[int] = []
    cyc: Dict[int, int] = {}

    def ready_time(j):
        return max([cyc[p] + l for p, l in P[j]] + [0])

    def rec(t):
        nonlocal found
        if len(order) == n:
            prp = prp_interval(region, order, n_classes)
            if all(prp[c] <= target[c] for c in range(n_classes)):
                found += 1
            return
        avail = [j for j in range(n) if j not in cyc and all(p in cyc for p, _ in P[j])]
        R = [j for j in avail if ready_time(j) <= t]
        if not R:
            rec(min(ready_time(j) for j in avail))
            return
        for j in R:
            order.append(j)
            cyc[j] = t
            # prune on the partial peak (interval reading restricted to prefix)
            rec(t + 1)
            del cyc[j]
            order.pop()

    rec(0)
    return found


# ---------------------------------------------------------------------------
# General machine model (R42), written as a
# cycle-stepped simulation (the oracle uses a closed max() recurrence).
def asap_machine(region, order: Sequence[int], width: int, slots: Sequence[int],
                 types: Sequence[int]) -> Tuple[int, List[int]]:
    """In-order issue of `order`: at cycle t issue the next instruction if its
    operands are ready and the cycle has a free slot (width and its type),
    else move to cycle t + 1."""
    P = preds_of(region)
    cyc: Dict[int, int] = {}
    out: List[int] = []
    t, used, used_t = 0, 0, [0, 0, 0, 0]
    k = 0
    while k < len(order):
        j = order[k]
        y = int(types[j]) if types is not None else 0
        ready = max([cyc[p] + l for p, l in P[j]] + [0])
        free = used < width and (width <= 1 or used_t[y] < slots[y])
        if ready <= t and free:
            cyc[j] = t
            out.append(t)
            used += 1
            used_t[y] += 1
            k += 1
        else:
            t += 1
            used, used_t = 0, [0, 0, 0, 0]
    return (out[-1] + 1 if out else 0), out


def optimum_machine(region, machine, mode: int, target=None, weight=None):
    """Best length under target (and/or best length + weight * cost) over all
    topological orders, each timed by asap_machine."""
    w = max(1, machine.issue_width)
    best_t = math.inf
    best_w = math.inf
    for o in topo_orders(region):
        prp = prp_interval(region, o, machine.n_classes)
        L, _ = asap_machine(region, o, w, machine.type_slots, region.inst_type)
        if target is None or all(prp[c] <= target[c] for c in range(machine.n_classes)):
            best_t = min(best_t, L)
        if weight is not None:
            best_w = min(best_w, L + weight * cost(machine, mode, prp))
    return best_t, best_w


def occupancy(machine, prp: Sequence[int]) -> int:
    """min over classes of the occupancy table lookup (L68-L72)."""
    occ = machine.occ_max
    for c in range(machine.n_classes):
        o = 0
        for i, s in enumerate(machine.steps[c]):
            if prp[c] <= s:
                o = machine.occ_max - i
                break
        occ = min(occ, o)
    return occ
