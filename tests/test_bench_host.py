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


def test_schedule_quality_histogram():
    res = {0: {"heur_prp": [20, 3], "prp": [20, 3], "best1": 5, "init1": 5, "init2": 100, "length": 90},
           1: {"heur_prp": [30, 3], "prp": [24, 3], "best1": 4, "init1": 6, "init2": 50, "length": 50},
           2: {"heur_prp": [300, 3], "prp": [129, 3], "best1": 9, "init1": 9, "init2": 0, "length": 0}}
    q = bench.schedule_quality(res)
    assert q["regions"] == 3 and q["rp_pass_improved_cost"] == 1
    assert q["regions_by_heuristic_vgpr_band"][0] == 1 and q["regions_by_heuristic_vgpr_band"][2] == 1
    assert q["regions_by_heuristic_vgpr_band"][-1] == 1  # above the table
    assert q["regions_by_aco_vgpr_band"][0] == 2 and q["regions_by_aco_vgpr_band"][9] == 1
    assert q["heuristic_vgpr_prp_above_24"] == 2 and q["aco_vgpr_prp_above_24"] == 1
    assert q["pass2_len_gain_max_pct"] == 10.0 and q["pass2_len_gain_mean_pct"] == 5.0


def test_parity_compare_names_the_differing_fields():
    a = {f: 0 for f in bench.PARITY_FIELDS}
    a["order"] = [1, 2]
    b = dict(a)
    assert bench.parity_compare(a, b) == []
    b = dict(a, order=[2, 1], trace_hash=7)
    assert bench.parity_compare(a, b) == ["order", "trace_hash"]


def test_ncu_evidence_only_for_the_profiled_build(tmp_path, monkeypatch):
    """The committed ncu figures are reported only when their build
    fingerprint equals the fingerprint of the library sources in the tree."""
    import json
    fp = bench.build_fingerprint()
    assert len(fp) == 64 and fp == bench.build_fingerprint()
    prof = tmp_path / "profiles"
    prof.mkdir()
    monkeypatch.setattr(bench, "ROOT", str(tmp_path))
    (prof / "r02_traffic.json").write_text(json.dumps({"build_fingerprint": "0" * 64, "dram_bytes_per_launch": 1}))
    assert bench.ncu_evidence("c3")[0] is None
    (prof / "r02_traffic.json").write_text(json.dumps({"build_fingerprint": fp, "dram_bytes_per_launch": 5,
                                                       "issue_util_pct": 44.0, "source": "x"}))
    t, issue, src = bench.ncu_evidence("c3")
    assert t == 5 and issue["util_pct"] == 44.0 and src == "x"
    assert bench.ncu_evidence("c4")[0] is None
