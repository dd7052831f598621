"""Host logic of bench.py's oracle sampling (no GPU, no oracle call)."""
from types import SimpleNamespace

import bench


def _regs(sizes):
    return [SimpleNamespace(n_insts=n) for n in sizes]


def test_stratified_pick_largest_first_and_spans_sizes():
    sizes = [20 + (7 * i) % 481 for i in range(500)]
    regs = _regs(sizes)
    pick = bench.stratified_pick(regs, 40)
    assert len(pick) == len(set(pick)) and 30 <= len(pick) <= 40
    got = [sizes[i] for i in pick]
    assert got == sorted(got, reverse=True)
    assert got[0] == max(sizes) and got[-1] == min(sizes)


def test_stratified_pick_small_and_single():
    assert bench.stratified_pick(_regs([5]), 160) == [0]
    assert sorted(bench.stratified_pick(_regs([3, 9, 4]), 160)) == [0, 1, 2]


def test_reference_steps_partition_the_sample():
    regs = _regs([20 + (13 * i) % 481 for i in range(5000)])
    full = bench.stratified_pick(regs, 160)
    steps = 3
    per_step = bench.deal_over_steps(full, steps)
    flat = [i for p in per_step for i in p]
    assert sorted(flat) == sorted(full)
    for p in per_step:
        n = [regs[i].n_insts for i in p]
        assert n == sorted(n, reverse=True)


def test_deal_over_steps_reuses_a_small_sample():
    assert bench.deal_over_steps([7], 3) == [[7], [7], [7]]
    assert bench.deal_over_steps([1, 2, 3, 4, 5], 2) == [[1, 3, 5], [2, 4]]


def test_strong_partition_covers_the_batch_once():
    """bench.py c3 at N ranks: the LPT shares of the same batch are disjoint,
    cover every region, and regenerate the world-1 regions exactly."""
    a = bench.parse(["--workload", "c3", "--regions", "60"])
    one = bench.workload(a, 0, 1)[0][0]
    shares = [bench.workload(a, r, 3)[0][0] for r in range(3)]
    ids = sorted(i for b in shares for i in b.ids)
    assert ids == list(range(60))
    by_id = {i: r for b in shares for i, r in zip(b.ids, b.regs)}
    for i, r in zip(one.ids, one.regs):
        assert by_id[i].n_insts == r.n_insts and (by_id[i].edge_src == r.edge_src).all()


def test_c5_grid_batches():
    a = bench.parse(["--workload", "c5"])
    b = bench.workload(a, 0, 1, gen=False)[0]
    assert [x.p.iterations for x in b] == [10, 5]
    assert len(bench.I.c5_grid()) == 9 * 2 * 3
