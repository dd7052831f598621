"""Regression tests for the round-1 advisor findings: state that
outlives one call of the C ABI -- machine models shared by contexts on one
device, the plan cache, dump buffers across loads, colony calls after a
reload.  Every run is compared with the oracle."""
import dataclasses

import pytest

from oracle import pyoracle as O
from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I
from tests.test_gpu_parity import compare_results, dump_parity

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    return torch


def _sched(machine=I.GFX906):
    from paper_conf_cgo_shobakimhlmkrg24_b200.api import Scheduler
    return Scheduler(machine, device=0)


def test_contexts_with_different_machines_interleave(torch_cuda):
    """Context A (gfx906, single issue) and B (dual issue, different
    occupancy use) on one device, run A, B, A, B: each equals the oracle of
    its own machine (the machine model is bound per context, not per device)."""
    regs = [I.gen_region(n, 3100 + n) for n in (30, 90, 200)]
    ids = [1, 2, 3]
    p = I.Params(ants=128, iterations=3, seed=61)
    a, b = _sched(I.GFX906), _sched(I.DUAL_ISSUE)
    a.load(regs, ids)
    b.load(regs, ids)
    ora = {m: [O.schedule(r, i, mach, p) for r, i in zip(regs, ids)]
           for m, mach in (("a", I.GFX906), ("b", I.DUAL_ISSUE))}
    for who in ("a", "b", "a", "b"):
        s = a if who == "a" else b
        s.run(p)
        got = s.results()
        for k in range(len(regs)):
            compare_results(got[k], ora[who][k], f"{who} region {k}")


def test_colony_rerun_pass1_only(torch_cuda):
    """Two identical colony runs with passes = 1 (the second hits the plan
    cache): both equal the oracle (the pass-transition runs every time)."""
    regs = [I.gen_region(n, 3200 + n) for n in (40, 110)]
    ids = [4, 5]
    p = I.Params(ants=96, iterations=3, seed=62, passes=1)
    s = _sched()
    s.load(regs, ids)
    ora = [O.schedule(r, i, I.GFX906, p) for r, i in zip(regs, ids)]
    for _ in range(2):
        s.run_colony(p, 0, 1)
        got = s.results()
        for k in range(len(regs)):
            compare_results(got[k], ora[k], f"region {k}")


def test_dump_after_loading_a_larger_batch(torch_cuda):
    """dump=True after loading a batch of the same count but more
    instructions: the binding re-sizes the dump buffers (and the library
    checks their sizes)."""
    p = I.Params(ants=40, iterations=2, seed=63, stall_mod=2)
    s = _sched()
    small = [I.gen_region(n, 3300 + n) for n in (12, 20)]
    s.load(small, [0, 1]).run(p, no_prune=True, dump=True)
    dump_parity(s, small, [0, 1], p)
    big = [I.gen_region(n, 3400 + n) for n in (150, 260)]
    s.load(big, [0, 1]).run(p, no_prune=True, dump=True)
    dump_parity(s, big, [0, 1], p)


def test_dump_buffers_too_small_rejected(torch_cuda):
    import ctypes as C

    from paper_conf_cgo_shobakimhlmkrg24_b200 import _lib
    from paper_conf_cgo_shobakimhlmkrg24_b200.api import params_struct
    s = _sched()
    regs = [I.gen_region(50, 3500)]
    s.load(regs, [0])
    p = I.Params(ants=32, iterations=2, seed=1)
    s.set_dump(p)
    costs, od, cy = s.dump
    # claim a too-small order buffer
    st = s.lib.aco_set_dump(s.ctx, C.c_void_p(costs.data_ptr()), costs.numel(), C.c_void_p(od.data_ptr()), 10,
                            C.c_void_p(cy.data_ptr()), cy.numel())
    assert st == 0
    n = C.c_size_t(0)
    ws = torch_cuda.empty(s.workspace_bytes(p) + 256, dtype=torch_cuda.uint8, device="cuda:0")
    ps = params_struct(p, _lib.ACO_FLAG_DUMP)
    st = s.lib.aco_schedule_batch(s.ctx, C.byref(ps), C.c_void_p(ws.data_ptr()), ws.numel(), C.byref(n), None)
    assert st == _lib.ACO_E_WORKSPACE


def test_colony_calls_after_reload_need_begin(torch_cuda):
    from paper_conf_cgo_shobakimhlmkrg24_b200._lib import ACO_E_STATE, AcoError
    regs = [I.gen_region(n, 3600 + n) for n in (30, 60, 90)]
    p = I.Params(ants=64, iterations=2, seed=64)
    s = _sched()
    s.load(regs, [0, 1, 2])
    s.colony_begin(p, 0)
    s.load(regs[:1], [0])
    with pytest.raises(AcoError) as e:
        s.colony_construct(1, 0)
    assert e.value.status == ACO_E_STATE
    # a new begin on the reloaded batch works and equals the oracle
    s.run_colony(p, 0, 1)
    compare_results(s.results()[0], O.schedule(regs[0], 0, I.GFX906, p))


def test_plan_cache_colony_then_batch(torch_cuda):
    """A colony run followed by the same parameters through
    aco_schedule_batch (a different plan kind) and back."""
    regs = [I.gen_region(n, 3700 + n) for n in (35, 170)]
    ids = [8, 9]
    p = I.Params(ants=128, iterations=3, seed=65)
    s = _sched()
    s.load(regs, ids)
    ora = [O.schedule(r, i, I.GFX906, dataclasses.replace(p)) for r, i in zip(regs, ids)]
    for mode in ("colony", "batch", "colony", "batch"):
        if mode == "colony":
            s.run_colony(p, 0, 1)
        else:
            s.run(p, no_prune=True)
        got = s.results()
        for k in range(len(regs)):
            compare_results(got[k], ora[k], f"{mode} region {k}")


def test_graph_replay_equals_oracle(torch_cuda, monkeypatch):
    """Identical runs: the 1st launches directly, the 2nd captures the whole
    run as a CUDA graph, the 3rd+ replay it (also on another stream); every
    run equals the oracle, and the graph run reports the same launch count."""
    regs = [I.gen_region(n, 3800 + n) for n in (12, 40, 130, 300, 1200)]
    ids = [20, 21, 22, 23, 24]
    p = I.Params(ants=96, iterations=3, seed=66)
    ora = [O.schedule(r, i, I.GFX906, p) for r, i in zip(regs, ids)]
    s = _sched()
    s.load(regs, ids)
    counts = []
    side = torch_cuda.cuda.Stream()
    for k in range(5):
        if k == 3:
            with torch_cuda.cuda.stream(side):
                s.run(p, stream=side)
        else:
            s.run(p)
        got = s.results()
        counts.append(s.launch_count())
        for q in range(len(regs)):
            compare_results(got[q], ora[q], f"run {k} region {q}")
    assert len(set(counts)) == 1, counts
