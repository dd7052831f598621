"""GPU parity (through the C ABI) of SURVEY 8(f) rows against the oracle:
general machine model (R42), mixed heuristics and stall fraction (R43, R44),
compile policy (R39, R40) and the weighted-sum single pass (R41).
Bit-exact: every ant in dump mode, final results in production mode."""
import dataclasses

import numpy as np
import pytest

from oracle import pyoracle as O
from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I
from tests import checker
from tests.test_gpu_parity import _sched, compare_results, dump_parity

pytestmark = pytest.mark.gpu

TRIPLE = dataclasses.replace(I.DUAL_ISSUE, issue_width=3, type_slots=(2, 1, 1, 1))


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


def ragged(tag, sizes=(1, 5, 23, 40, 64, 97, 130, 170, 260)):
    regs = [I.gen_region(n, 7000 + 31 * tag + i, "mixed" if i % 2 else "unit") for i, n in enumerate(sizes)]
    return regs, [2000 + 5 * i + tag for i in range(len(regs))]


@pytest.mark.parametrize("machine", ["dual", "triple"])
@pytest.mark.parametrize("mode", [0, 1])
def test_machine_model_every_ant(torch_cuda, machine, mode):
    m = I.DUAL_ISSUE if machine == "dual" else TRIPLE
    regs, ids = ragged(mode + (2 if machine == "triple" else 0))
    p = I.Params(ants=100, iterations=3, seed=21 + mode, cost_mode=mode, stall_mod=2)
    s = _sched(m)
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    dump_parity(s, regs, ids, p, m)
    for k, g in enumerate(s.results()):
        checker.check_machine_schedule(regs[k], m, g["order"], g["cycle"], g["length"])


def test_machine_model_prune_and_large_regions(torch_cuda):
    """Production mode (prune on) incl. a global-state region (n > 1024)."""
    regs = [I.gen_region(n, 7500 + n) for n in (60, 300, 700, 1100)]
    ids = [11, 12, 13, 14]
    p = I.Params(ants=128, iterations=3, seed=4)
    s = _sched(I.DUAL_ISSUE)
    s.load(regs, ids).run(p)
    for k, g in enumerate(s.results()):
        compare_results(g, O.schedule(regs[k], ids[k], I.DUAL_ISSUE, p), f"region {k}")


@pytest.mark.parametrize("weight", [0, 1, 3])
def test_weighted_pass_every_ant(torch_cuda, weight):
    regs, ids = ragged(10 + weight)
    p = I.Params(ants=96, iterations=3, seed=3 + weight, cost_mode=1, passes=4, ws_weight=weight)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    dump_parity(s, regs, ids, p)


def test_weighted_pass_dual_issue_and_fix10a(torch_cuda):
    x = I.fix10a()
    for W in (1, 10):
        p = I.Params(ants=64, iterations=20, seed=1, cost_mode=0, passes=4, ws_weight=W)
        s = _sched()
        s.load([x], [0]).run(p, no_prune=True, dump=True)
        dump_parity(s, [x], [0], p)
    regs, ids = ragged(20, sizes=(30, 90, 200))
    p = I.Params(ants=128, iterations=3, seed=8, passes=4, ws_weight=2)
    s = _sched(I.DUAL_ISSUE)
    s.load(regs, ids).run(p)
    for k, g in enumerate(s.results()):
        compare_results(g, O.schedule(regs[k], ids[k], I.DUAL_ISSUE, p), f"region {k}")


@pytest.mark.parametrize("passes", [1, 3])
def test_heur_mix_every_ant(torch_cuda, passes):
    regs, ids = ragged(30 + passes)
    p = I.Params(ants=100, iterations=3, seed=9, passes=passes, group_size=16, heur_mix=1)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    dump_parity(s, regs, ids, p)


@pytest.mark.parametrize("num,rem", [(0, 0), (2, 1), (3, 3)])
def test_stall_fraction_every_ant(torch_cuda, num, rem):
    regs, ids = ragged(40 + num)
    p = I.Params(ants=128, iterations=3, seed=5, group_size=16, stall_mod=4, stall_rem=rem, stall_num=num)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    dump_parity(s, regs, ids, p)


def test_compile_policy_filters(torch_cuda):
    """Cycle-gap filter and revert filter (production mode) on a batch whose
    regions straddle the thresholds; policy bits and heuristic lengths."""
    # regions of the round-1 generator calibration (recency 0.3, 2 VGPR
    # live-ins), where region 14 reverts under (revert_occ 1, revert_len 0)
    regs = [I.gen_region((60, 100, 150, 200, 250, 300)[i % 6], 1300 + i, recency=0.3, v_livein=2)
            for i in range(12, 18)]
    ids = list(range(12, 18))
    base = I.Params(ants=64, iterations=4, cost_mode=1)
    for q in (dataclasses.replace(base, pass2_gap=21), dataclasses.replace(base, pass2_gap=100000),
              dataclasses.replace(base, revert_occ=1, revert_len=0), I.paper_policy(base)):
        s = _sched()
        s.load(regs, ids).run(q)
        got = s.results()
        pol = 0
        for k, g in enumerate(got):
            ora = O.schedule(regs[k], ids[k], I.GFX906, q)
            compare_results(g, ora, f"{q} region {k}")
            pol |= g["policy"]
        if q.pass2_gap == 100000:
            assert all(g["policy"] & 1 and g["iters2"] == 0 for g in got)
        if q.revert_occ == 1:
            assert pol & 2  # region 14 reverts (see test_oracle_ext_pins)


def test_config3_sample_paper_policy(torch_cuda):
    """The paper's compile policy on a sample of the config-3 batch."""
    regs = I.gen_batch(300, base_seed=3)
    ids = list(range(300))
    p = I.paper_policy(I.Params(ants=256, iterations=10, seed=3))
    s = _sched()
    s.load(regs, ids).run(p)
    got = s.results()
    for k in range(0, 300, 13):
        compare_results(got[k], O.schedule(regs[k], ids[k], I.GFX906, p), f"region {k}")
