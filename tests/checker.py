"""Independent validity checker for schedules (test code, not the oracle)."""
from __future__ import annotations

from typing import Sequence

from tests import brute


def check_order(region, order: Sequence[int]):
    n = region.n_insts
    assert sorted(int(x) for x in order) == list(range(n)), "not a permutation"
    pos = {int(j): k for k, j in enumerate(order)}
    for s, d, _ in region.edges():
        assert pos[s] < pos[d], f"edge {s}->{d} violated"


def check_schedule(region, order: Sequence[int], cycle: Sequence[int], length: int):
    check_order(region, order)
    cyc = {int(j): int(c) for j, c in zip(order, cycle)}
    prev = -1
    for j, c in zip(order, cycle):
        assert int(c) > prev, "cycles must strictly increase (single issue)"
        prev = int(c)
    for s, d, l in region.edges():
        assert cyc[d] >= cyc[s] + l, f"latency {s}->{d} ({l}) violated"
    if region.n_insts:
        assert length == int(cycle[-1]) + 1, "length = last issue cycle + 1"


def prp(region, order, n_classes=2):
    return brute.prp_interval(region, [int(x) for x in order], n_classes)


def check_machine_schedule(region, machine, order: Sequence[int], cycle: Sequence[int], length: int):
    """Validity on the general machine model (R42): cycles non-decreasing in
    placement order, <= issue_width per cycle, <= type_slots[y] of type y per
    cycle, every latency met, length = last issue cycle + 1."""
    check_order(region, order)
    w = max(1, machine.issue_width)
    types = region.inst_type
    per, per_t = {}, {}
    prev = -1
    for j, c in zip(order, cycle):
        c = int(c)
        assert c >= prev, "cycles must not decrease along the order"
        prev = c
        per[c] = per.get(c, 0) + 1
        y = int(types[int(j)]) if types is not None else 0
        per_t[(c, y)] = per_t.get((c, y), 0) + 1
    assert all(v <= w for v in per.values()), "issue width exceeded"
    if w > 1:
        assert all(v <= machine.type_slots[y] for (c, y), v in per_t.items()), "type slots exceeded"
    cyc = {int(j): int(c) for j, c in zip(order, cycle)}
    for s, d, l in region.edges():
        assert cyc[d] >= cyc[s] + l, f"latency {s}->{d} ({l}) violated"
    if region.n_insts:
        assert length == int(cycle[-1]) + 1, "length = last issue cycle + 1"
