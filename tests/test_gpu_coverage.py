"""Parity of the kernel variants and configurations round 1 left without an
oracle comparison: the 4- and 8-lane global-state
kernels, config 4 at its real shape, the shared colony on a global-state
region, the discretionary-stall and size-class-termination pins on the GPU."""
import dataclasses
import os

import pytest

from oracle import pyoracle as O
from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I
from tests import checker
from tests.test_gpu_parity import _colony_ranks, _sched, compare_results, dump_parity
from tests.test_oracle_pins_r2 import antichain, discretionary_ddg, paper_class_limit

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


@pytest.mark.parametrize("lanes", [4, 8, 16])
def test_global_state_lanes_every_ant(torch_cuda, monkeypatch, lanes):
    """Huge regions (per-ant state in global memory) with 4, 8 and 16 lanes
    per ant, both passes, every ant bit-exact (config 5 runs the 4-lane and
    config 4 the 16-lane instantiation)."""
    monkeypatch.setenv("ACO_GS_LANES", f"{lanes},{lanes}")
    monkeypatch.setenv("ACO_HUGE_SMEM", "0")  # (the global-state kernels, not the shared-memory huge path)
    regs = [I.gen_region(n, 9100 + n + lanes) for n in (1100, 1700)]
    ids = [31, 32]
    p = I.Params(ants=48, iterations=2, seed=70 + lanes, stall_mod=2)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    codes = s.variants()
    assert any(c & 2 for c in codes), codes  # the global-state kernels ran
    dump_parity(s, regs, ids, p)


@pytest.mark.parametrize("lanes", [4, 8, 16])
def test_huge_shared_state_every_ant(torch_cuda, monkeypatch, lanes):
    """Huge regions (n > 1024) with their per-ant state in shared memory
    (image and tau through L1, 4-wide strided scan, lean pass 2; configs 4
    and 5 at 8 lanes): every ant bit-exact at 4, 8 and 16 lanes per ant."""
    monkeypatch.setenv("ACO_HUGE_LANES", f"{lanes},{lanes}")
    monkeypatch.setenv("ACO_HUGE_SMEM", "1")  # (the default for n > 1024 since r03)
    regs = [I.gen_region(n, 9200 + n + lanes) for n in (1100, 1900)]
    ids = [35, 36]
    p = I.Params(ants=64, iterations=2, seed=90 + lanes, stall_mod=2)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    codes = s.variants()
    assert any((c & (1 << 11)) and not (c & (1 << 5)) for c in codes), codes  # the huge shared-state kernels ran
    dump_parity(s, regs, ids, p)


def test_config4_at_shape(torch_cuda):
    """Config 4's region (n = 2,000, seed 4, mixed latencies) at 1,024 ants x 2
    iterations in production mode (record mode, pruning on): final schedule,
    trace and iterations equal the oracle's."""
    reg = I.gen_region(2000, I.region_seed(4, 0))
    p = I.Params(ants=1024, iterations=2, seed=4)
    s = _sched()
    s.load([reg], [0]).run(p)
    g = s.results()[0]
    compare_results(g, O.schedule(reg, 0, I.GFX906, p))
    checker.check_schedule(reg, g["order"], g["cycle"], g["length"])


def test_shared_colony_on_global_state_region(torch_cuda):
    """The shared colony (4 emulated ranks x 64 ants) on a region whose state
    needs the global-state kernels: every rank replays the winner from its
    workspace scratch; results equal the oracle with 256 ants."""
    os.environ["ACO_HUGE_SMEM"] = "0"
    try:
        _colony_check()
    finally:
        del os.environ["ACO_HUGE_SMEM"]


def test_shared_colony_on_huge_shared_state_region(torch_cuda):
    """The same with the default huge-region kernels (per-ant state in shared
    memory): what config 4 runs at N > 1."""
    _colony_check()


def _colony_check():
    regs = [I.gen_region(1600, 9400)]
    ids = [3]
    p_all = I.Params(ants=256, iterations=2, seed=81)
    p_rank = dataclasses.replace(p_all, ants=64)
    ranks = _colony_ranks(regs, ids, p_rank, 4)
    ora = O.schedule(regs[0], ids[0], I.GFX906, p_all)
    for r in range(4):
        compare_results(ranks[r][0], ora, f"rank {r}")


def test_discretionary_stall_every_ant(torch_cuda):
    """The discretionary-stall DDG of tests/test_oracle_pins_r2.py (L157-L164):
    4,096 stall-enabled ants, every ant bit-exact (the stall coins and the
    decaying probability are the kernel's, the law is pinned on the oracle)."""
    reg = discretionary_ddg()
    p = I.Params(ants=4096, iterations=1, seed=123, passes=2, cost_mode=I.COST_PRP_SUM, stall_mod=1)
    s = _sched()
    s.load([reg], [9]).run(p, no_prune=True, dump=True)
    dump_parity(s, [reg], [9], p)


def test_size_class_termination_gpu(torch_cuda):
    """Paper termination classes (L226) on the GPU: regions of 49/50/99/100
    instructions that cannot improve stop after exactly 1/2/2/3 iterations."""
    sizes = (49, 50, 99, 100)
    regs = [antichain(n) for n in sizes]
    ids = [40, 41, 42, 43]
    p = I.Params(ants=64, iterations=10, seed=1, stop_no_improve=I.STOP_PAPER_CLASSES)
    s = _sched()
    s.load(regs, ids).run(p)
    for n, g in zip(sizes, s.results()):
        assert g["iters1"] == g["iters2"] == paper_class_limit(n), (n, g["iters1"], g["iters2"])


@pytest.mark.parametrize("kind", ["both", "paper", "weighted", "pass1", "pass2", "mix"])
def test_fused_run_equals_oracle_and_multilaunch(torch_cuda, monkeypatch, kind):
    """The fused single-block run (k_fused: every pass and iteration of a
    region in one block) is taken for batches with few
    ants in total; it equals the oracle and the multi-launch path bit for bit
    (final schedule, trace, iterations), for every pass mode and policy."""
    regs = [I.fix10a(), I.gen_region(60, 9700), I.gen_region(130, 9701, "unit")]
    ids = [50, 51, 52]
    base = I.Params(ants=128, iterations=6, seed=5)
    p = {"both": base, "paper": I.paper_policy(base), "weighted": dataclasses.replace(base, passes=4, ws_weight=2),
         "pass1": dataclasses.replace(base, passes=1), "pass2": dataclasses.replace(base, passes=2),
         "mix": dataclasses.replace(base, heur_mix=1, stall_num=2, cost_mode=I.COST_OCC)}[kind]
    s = _sched()
    s.load(regs, ids).run(p)
    assert s.variants() == [1 << 13], s.variants()  # k_fused
    fused = s.results()
    for k in range(len(regs)):
        compare_results(fused[k], O.schedule(regs[k], ids[k], I.GFX906, p), f"{kind} region {k}")
    monkeypatch.setenv("ACO_FUSED_ANTS", "0")
    m = _sched()
    m.load(regs, ids).run(p)
    assert (1 << 13) not in m.variants()
    for k, g in enumerate(m.results()):
        compare_results(g, O.schedule(regs[k], ids[k], I.GFX906, p), f"{kind} multi-launch region {k}")


def test_huge_kernels_for_mid_size_regions_of_few_ant_batches(torch_cuda, monkeypatch):
    """Batches with few ants in total (config 5) run regions above 400
    instructions on the huge-region kernels (strided-word scan, n <= 1024
    included): every ant bit-exact."""
    monkeypatch.setenv("ACO_HUGE_MIN_N", "400")
    regs = [I.gen_region(n, 9500 + n, "mixed" if n % 2 else "unit") for n in (450, 800, 1000)]
    ids = [41, 42, 43]
    p = I.Params(ants=64, iterations=2, seed=17, stall_mod=2)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    codes = s.variants()
    assert any((c & (1 << 11)) and not (c & (1 << 5)) for c in codes), codes  # huge (image via L1, no word mask)
    dump_parity(s, regs, ids, p)
