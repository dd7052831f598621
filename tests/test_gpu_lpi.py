"""Lane-per-instruction ants (one warp per ant, state in registers; the
latency-bound kernels of config 2) against the oracle, through the C ABI.

ACO_LPI=2 plans every eligible region (n <= 128, <= 2 classes, pass 2 on the
single-issue machine) on the lane-per-instruction variants, whatever the
batch size; every ant is compared bit for bit in dump mode (cost, order,
pass-2 cycles), the final results in production mode (record + prune).
Sizes cross the 32-instruction lane chunks (Q = 1, 2, 4) and ragged tails.
"""
import os

import numpy as np
import pytest

from oracle import pyoracle as O
from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I
from tests.test_gpu_parity import compare_results, dump_parity

pytestmark = pytest.mark.gpu

LPI_BIT = 1 << 10  # variant code: lanes = 32 (aco_internal.h variant_code)


@pytest.fixture
def lpi_forced():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    old = os.environ.get("ACO_LPI")
    os.environ["ACO_LPI"] = "2"
    yield
    if old is None:
        os.environ.pop("ACO_LPI", None)
    else:
        os.environ["ACO_LPI"] = old


def _sched(machine=I.GFX906):
    from paper_conf_cgo_shobakimhlmkrg24_b200.api import Scheduler
    return Scheduler(machine, device=0)


SIZES = [1, 2, 7, 31, 32, 33, 50, 63, 64, 65, 97, 100, 127, 128]


@pytest.mark.parametrize("mode", [0, 1, 2, 3])
def test_lpi_every_ant(lpi_forced, mode):
    regs = [I.gen_region(n, 7100 + 13 * i + mode, "mixed" if (i + mode) % 2 else "unit") for i, n in enumerate(SIZES)]
    ids = [200 + 7 * i for i in range(len(regs))]
    p = I.Params(ants=70, iterations=3, seed=40 + mode, cost_mode=mode, stall_mod=2)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    assert any(v & LPI_BIT for v in s.variants()), s.variants()
    dump_parity(s, regs, ids, p)


def test_lpi_stall_paths_every_ant(lpi_forced):
    """Every group may stall (forced, discretionary, necessary stalls) on
    long-latency regions; one pass-1 ant count that is not a warp multiple."""
    regs = [I.gen_region(n, 7300 + n, "mixed") for n in (12, 40, 90, 128)]
    ids = [1, 2, 3, 4]
    p = I.Params(ants=33, iterations=4, seed=9, stall_mod=1)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    dump_parity(s, regs, ids, p)


def test_lpi_discretionary_stall_ddg(lpi_forced):
    """The 4-instruction DDG on which the discretionary condition holds (the
    oracle pin of L157-L164), every ant."""
    from tests.test_oracle_pins_r2 import discretionary_ddg
    r = discretionary_ddg()
    p = I.Params(ants=512, iterations=2, seed=3, passes=2, cost_mode=I.COST_PRP_SUM, stall_mod=1)
    s = _sched()
    s.load([r], [9]).run(p, no_prune=True, dump=True)
    dump_parity(s, [r], [9], p)


@pytest.mark.parametrize("passes", [1, 2, 4])
def test_lpi_pass_modes_every_ant(lpi_forced, passes):
    regs = [I.gen_region(n, 7500 + n + passes) for n in (20, 45, 100)]
    ids = [5, 6, 7]
    p = I.Params(ants=64, iterations=3, seed=5 + passes, passes=passes, ws_weight=3 if passes == 4 else 0)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    dump_parity(s, regs, ids, p)


def test_lpi_config2_production(lpi_forced):
    """Config 2's region (bench --workload c2) in production mode (record,
    prune), fewer iterations: final results equal the oracle's."""
    r = I.gen_region(100, I.region_seed(2, 0))
    p = I.Params(ants=1024, iterations=12, seed=2)
    s = _sched()
    s.load([r], [0]).run(p)
    assert all(v & LPI_BIT for v in s.variants())
    compare_results(s.results()[0], O.schedule(r, 0, I.GFX906, p), "c2")


def test_lpi_auto_plan():
    """Auto mode: config 2 (one region, 1,024 ants) takes the lane-per-
    instruction variants, config 3-sized batches do not."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    if os.environ.get("ACO_LPI") not in (None, "1"):
        pytest.skip("ACO_LPI overridden")
    s = _sched()
    s.load([I.gen_region(100, I.region_seed(2, 0))], [0])
    assert all(v & LPI_BIT for v in s.plan_variants(I.Params(ants=1024, iterations=100, seed=2)))
    regs = I.gen_batch(40, base_seed=3)
    s2 = _sched()
    s2.load(regs, list(range(40)))
    assert not any(v & LPI_BIT for v in s2.plan_variants(I.Params(ants=1024, iterations=2, seed=3)))


def test_lpi_equals_group_kernels(lpi_forced):
    """Production results identical with and without the lane-per-instruction
    variants (same Philox counters, same decisions)."""
    regs = [I.gen_region(n, 7700 + n) for n in (30, 77, 120)]
    ids = [10, 11, 12]
    p = I.Params(ants=256, iterations=4, seed=21)
    a = _sched()
    a.load(regs, ids).run(p)
    ra = a.results()
    os.environ["ACO_LPI"] = "0"
    b = _sched()
    b.load(regs, ids).run(p)
    rb = b.results()
    assert not any(v & LPI_BIT for v in b.variants())
    for x, y in zip(ra, rb):
        for k in ("length", "prp", "trace_hash", "iters1", "iters2", "cost_rp"):
            assert x[k] == y[k], k
        assert np.array_equal(x["order"], y["order"]) and np.array_equal(x["cycle"], y["cycle"])


FUSED, FUSED_LPI = 1 << 13, 1 << 14


@pytest.mark.parametrize("wl,sizes,ants", [(8, (10, 25, 32), 21), (16, (40, 64), 16), (32, (100, 128), 8), (8, (7,), 2)])
def test_lpi_fused_every_ant(lpi_forced, wl, sizes, ants):
    """The fused single-block run with lane-per-instruction ants of WL lanes
    (the smallest of 8 / 16 / 32 with n <= 4 WL; an option, ACO_FUSED_LPI,
    forced here): every ant bit-exact in dump mode."""
    regs = [I.gen_region(n, 7900 + n + wl, "mixed" if i % 2 else "unit") for i, n in enumerate(sizes)]
    ids = [60 + i for i in range(len(regs))]
    # (the fused run: <= 512 ants in the batch, WL x ants <= 512 threads; 2 x 8 lanes: a partial warp)
    p = I.Params(ants=ants, iterations=4, seed=wl, stall_mod=2)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    assert s.variants() == [FUSED | FUSED_LPI * {8: 1, 16: 2, 32: 3}[wl]], s.variants()
    dump_parity(s, regs, ids, p)


@pytest.mark.parametrize("kind", ["both", "paper", "weighted", "pass1", "pass2"])
def test_lpi_fused_modes(lpi_forced, kind):
    """Config 1's shape (FIX10-A, 64 ants, 20 iterations) through the fused
    lane-per-instruction run in every pass mode and policy: final results
    equal the oracle's (production mode: record, prune)."""
    import dataclasses
    x = I.fix10a()
    base = I.Params(ants=64, iterations=20, seed=3, cost_mode=0)
    p = {"both": base, "paper": I.paper_policy(base), "weighted": dataclasses.replace(base, passes=4, ws_weight=2),
         "pass1": dataclasses.replace(base, passes=1), "pass2": dataclasses.replace(base, passes=2)}[kind]
    s = _sched()
    s.load([x], [7]).run(p)
    assert s.variants() == [FUSED | FUSED_LPI], s.variants()
    compare_results(s.results()[0], O.schedule(x, 7, I.GFX906, p), kind)
