"""Parity of the CUDA path (through the C ABI) with the CPU oracle.

Integer / index work, so the bar is BIT-EXACT: every ant's cost, order and
cycles in dump mode; the final schedule, PRP, length, iteration counts and
the per-iteration winner-trace hash in production mode.
"""
import numpy as np
import pytest

from oracle import pyoracle as O
from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I
from tests import checker

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


def compare_results(gpu, ora, ctx=""):
    assert gpu["length"] == ora["length"], ctx
    assert gpu["prp"] == ora["prp"], ctx
    assert gpu["cost_rp"] == ora["cost_rp"], ctx
    assert gpu["iters1"] == ora["iters1"] and gpu["iters2"] == ora["iters2"], ctx
    assert gpu["best1"] == ora["best1"] and gpu["best2"] == ora["best2"], ctx
    assert gpu["init1"] == ora["init1"] and gpu["init2"] == ora["init2"], ctx
    assert gpu["lb1"] == ora["lb1"] and gpu["lblen"] == ora["lblen"], ctx
    assert gpu["target"][:2] == [ora["target0"], ora["target1"]], ctx
    assert gpu["trace_hash"] == ora["trace_hash"], ctx
    assert list(gpu["order"]) == list(ora["order"]), ctx
    assert list(gpu["cycle"]) == list(ora["cycle"]), ctx
    assert gpu["policy"] == ora["policy"] and gpu["heur_len"] == ora["heur_len"], ctx
    assert gpu["ws_cost"] == ora["ws_cost"], ctx


# construct-kernel variants exercised by every-ant (dump) parity in this
# session; tests/test_zz_variant_coverage.py checks the benchmarks' variants
# against it
DUMP_VARIANTS = set()


def dump_parity(s, regions, ids, p, machine=I.GFX906):
    DUMP_VARIANTS.update(s.variants())
    c, o, y = s.dump_arrays()
    A, n_it = p.ants, p.iterations
    for k, (reg, rid) in enumerate(zip(regions, ids)):
        ora = O.schedule(reg, rid, machine, p, dump=True, dump_orders=True)
        n = reg.n_insts
        base0 = A * int(s.batch.offsets[k])
        pmask = 2 if p.passes == 4 else p.passes  # pass 4 (R41) fills the pass-2 slots
        for ps in (0, 1):
            if not (pmask & (ps + 1)):
                continue
            iters = ora["iters1"] if ps == 0 else ora["iters2"]
            for it in range(iters):
                oc = ora["dump_cost"][ps, it]
                gc = c[ps, it, k]
                assert np.array_equal(gc, oc), f"region {k} pass {ps+1} iter {it}: costs differ"
                for a in range(A):
                    if oc[a] == O.INVALID:
                        continue
                    g_ord = o[ps, it, base0 + a * n: base0 + (a + 1) * n].astype(np.uint32)
                    assert np.array_equal(g_ord, ora["dump_order"][ps, it, a]), (k, ps, it, a)
                    if ps == 1:
                        g_cyc = y[ps, it, base0 + a * n: base0 + (a + 1) * n]
                        assert np.array_equal(g_cyc, ora["dump_cycle"][ps, it, a]), (k, ps, it, a)
        compare_results(s.results(k, 1)[0], ora, f"region {k}")


def test_fig1_two_ants(torch_cuda):
    m = I.Machine(n_classes=1, steps=((24, 28, 32, 36, 40, 48, 64, 84, 128, 256),))
    f = I.fig1r()
    p = I.Params(ants=2, iterations=1, seed=0, cost_mode=0, stall_mod=1)
    s = _sched(m)
    s.load([f], [0]).run(p, no_prune=True, dump=True)
    dump_parity(s, [f], [0], p, m)
    g = s.results()[0]
    assert g["length"] == 10 and list(g["cycle"]) == [0, 1, 2, 5, 6, 8, 9]


@pytest.mark.parametrize("seed", range(10))
def test_config1_fix10a_every_ant(torch_cuda, seed):
    """Config 1: FIX10-A, 2 classes, 64 ants x 20 iterations, PRP_SUM."""
    x = I.fix10a()
    p = I.Params(ants=64, iterations=20, seed=seed, cost_mode=0)
    s = _sched()
    s.load([x], [7]).run(p, no_prune=True, dump=True)
    dump_parity(s, [x], [7], p)
    g = s.results()[0]
    checker.check_schedule(x, g["order"], g["cycle"], g["length"])


@pytest.mark.parametrize("mode", [0, 1, 2, 3])
def test_synthetic_batch_every_ant(torch_cuda, mode):
    """A ragged batch (sizes span several bitset words, mixed latencies) with
    an ant count that is not a multiple of the block or group size."""
    sizes = [1, 5, 23, 40, 64, 97, 130]
    regs = [I.gen_region(n, 500 + i + 10 * mode, "mixed" if i % 2 else "unit") for i, n in enumerate(sizes)]
    ids = [1000 + 3 * i for i in range(len(regs))]
    p = I.Params(ants=100, iterations=3, seed=11 + mode, cost_mode=mode, stall_mod=2)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    dump_parity(s, regs, ids, p)


def test_pruning_is_winner_invariant(torch_cuda):
    regs = [I.gen_region(n, 900 + n) for n in (30, 80, 150)]
    ids = [0, 1, 2]
    p = I.Params(ants=256, iterations=4, seed=5)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True)
    a = s.results()
    s.run(p, no_prune=False)
    b = s.results()
    for x, y in zip(a, b):
        for k in ("length", "prp", "trace_hash", "iters1", "iters2"):
            assert x[k] == y[k]
        assert list(x["order"]) == list(y["order"])


def test_config2_full(torch_cuda):
    """Config 2: one synthetic region n = 100, both passes, 1024 ants x 100
    iterations, production mode (pruning on), vs the oracle."""
    reg = I.gen_region(100, I.region_seed(2, 0))
    p = I.Params(ants=1024, iterations=100, seed=2)
    s = _sched()
    s.load([reg], [0]).run(p)
    g = s.results()[0]
    ora = O.schedule(reg, 0, I.GFX906, p)
    compare_results(g, ora)
    checker.check_schedule(reg, g["order"], g["cycle"], g["length"])


def test_paper_mode_stop_rules(torch_cuda):
    regs = I.gen_batch(24, base_seed=17)
    ids = list(range(24))
    p = I.Params(ants=192, iterations=8, seed=3, stop_no_improve=I.STOP_PAPER_CLASSES, stop_at_lb=1)
    s = _sched()
    s.load(regs, ids).run(p)
    g = s.results()
    _, _, stats, off = O.schedule_many(regs, ids, I.GFX906, p)
    for k in range(len(regs)):
        ora = {n: int(stats[k, i]) for n, i in O.ORS.items()}
        assert g[k]["iters1"] == ora["iters1"] and g[k]["iters2"] == ora["iters2"], k
        assert g[k]["trace_hash"] == ora["trace_hash"], k
        assert g[k]["length"] == ora["length"] and g[k]["cost_rp"] == ora["cost_rp"], k


def test_edge_regions(torch_cuda):
    empty = I.Region.from_lists(0, [], [1], [1], [], [])
    one = I.Region.from_lists(1, [], [0, 1], [0, 1], [[0]], [[1]])
    noregs = I.Region.from_lists(4, [(0, 2, 3), (1, 2, 1)], [], [], [[], [], [], []], [[], [], [], []])
    chain = I.Region.from_lists(6, [(i, i + 1, 2) for i in range(5)], [0] * 5, [0] * 5,
                                [[i] for i in range(5)] + [[]], [[]] + [[i - 1] for i in range(1, 6)])
    regs = [empty, one, noregs, chain]
    ids = [10, 11, 12, 13]
    p = I.Params(ants=40, iterations=3, seed=1, stall_mod=1)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    dump_parity(s, regs, ids, p)


def test_error_codes_through_abi(torch_cuda):
    from paper_conf_cgo_shobakimhlmkrg24_b200._lib import AcoError
    s = _sched()
    bad = I.Region.from_lists(3, [(0, 1, 1), (1, 0, 1)], [], [], [[], [], []], [[], [], []])
    with pytest.raises(AcoError) as e:
        s.load([bad], [0])
    assert e.value.status == -2
    dup = [I.gen_region(10, 1), I.gen_region(12, 2)]
    with pytest.raises(AcoError) as e:
        s.load(dup, [5, 5])
    assert e.value.status == -1


def test_config3_sampled(torch_cuda):
    """Config 3 at full size (5,000 regions, 1024 ants x 10 iterations per pass)
    in the bench's launch configuration; the oracle recomputes a sample of
    regions (the largest, the smallest and a spread) one by one."""
    regs = I.gen_batch(5000, base_seed=3)
    ids = list(range(5000))
    p = I.Params(ants=1024, iterations=10, seed=3)
    s = _sched()
    s.load(regs, ids).run(p)
    g = s.results()
    sizes = np.array([r.n_insts for r in regs])
    sample = sorted(set([int(np.argmax(sizes)), int(np.argmin(sizes))] + list(range(0, 5000, 499))))
    order, cyc, stats, off = O.schedule_many([regs[k] for k in sample], [ids[k] for k in sample], I.GFX906, p)
    for q, k in enumerate(sample):
        ora = {n: int(stats[q, i]) for n, i in O.ORS.items()}
        assert g[k]["trace_hash"] == ora["trace_hash"], k
        assert g[k]["length"] == ora["length"] and g[k]["cost_rp"] == ora["cost_rp"], k
        assert g[k]["prp"] == [ora["prp0"], ora["prp1"], ora["prp2"], ora["prp3"]], k
        a, b = int(off[q]), int(off[q + 1])  # the final schedule itself: order and issue cycles
        assert list(g[k]["order"]) == [int(x) for x in order[a:b]], k
        assert list(g[k]["cycle"]) == [int(x) for x in cyc[a:b]], k
    # every region's final schedule is valid (independent checker)
    for k in range(0, 5000, 97):
        checker.check_schedule(regs[k], g[k]["order"], g[k]["cycle"], g[k]["length"])


def _three_class(reg):
    """Move every third VGPR to a third class (exercises the 3-4 class path)."""
    cls = reg.reg_class.copy()
    v = [g for g in range(reg.n_regs) if cls[g] == 0]
    for g in v[::3]:
        cls[g] = 2
    return I.Region(reg.n_insts, reg.edge_src, reg.edge_dst, reg.edge_lat, cls, reg.reg_flags,
                    reg.def_ptr, reg.def_reg, reg.use_ptr, reg.use_reg, name=reg.name + "-3c")


M3 = I.Machine(n_classes=3, steps=((24, 28, 32, 36, 40, 48, 64, 84, 128, 256), (80, 88, 100, 102),
                                   (24, 28, 32, 36, 40, 48, 64, 84, 128, 256)),
               perp_limit=(24, 80, 24, 0))


def test_three_register_classes_every_ant(torch_cuda):
    regs = [_three_class(I.gen_region(n, 700 + n)) for n in (18, 60, 140)]
    ids = [5, 6, 7]
    for mode in (1, 3):
        p = I.Params(ants=72, iterations=2, seed=3 + mode, cost_mode=mode, stall_mod=2)
        s = _sched(M3)
        s.load(regs, ids).run(p, no_prune=True, dump=True)
        dump_parity(s, regs, ids, p, M3)


def test_large_regions_global_state_every_ant(torch_cuda):
    """Regions whose per-ant state does not fit shared memory (global-state
    kernels) and whose cycles need 32 bits, every ant vs the oracle."""
    regs = [I.gen_region(n, 9000 + n) for n in (900, 1500, 2100)]
    ids = [21, 22, 23]
    p = I.Params(ants=40, iterations=2, seed=12, stall_mod=2)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    dump_parity(s, regs, ids, p)


def test_largest_region_sampled(torch_cuda):
    """Config-5-sized region (n = 4000), production mode, vs the oracle."""
    reg = I.gen_region(4000, 4242)
    p = I.Params(ants=24, iterations=1, seed=1)
    s = _sched()
    s.load([reg], [3]).run(p)
    g = s.results()[0]
    ora = O.schedule(reg, 3, I.GFX906, p)
    compare_results(g, ora)


def _colony_ranks(regs, ids, p_rank, world):
    """Emulate `world` ranks of the shared colony on one GPU: one context per
    rank, keys combined with an elementwise MIN (what the NCCL allreduce does)."""
    import torch
    scheds = [_sched() for _ in range(world)]
    keys = []
    for r, s in enumerate(scheds):
        s.load(regs, ids)
        keys.append(s.colony_begin(p_rank, r * p_rank.ants))
    for pass_ in (1, 2):
        if not (p_rank.passes & pass_):
            continue
        for it in range(p_rank.iterations):
            for s in scheds:
                s.colony_construct(pass_, it)
            m = keys[0].clone()
            for k in keys[1:]:
                m = torch.minimum(m, k)
            for k in keys:
                k.copy_(m)
            for s in scheds:
                s.colony_finalize(pass_, it)
    for s in scheds:
        s.colony_end()
    return [s.results() for s in scheds]


def test_shared_colony_equals_single_context(torch_cuda):
    """Config 4's scheme: 4 ranks x 64 ants == one context with 256 ants ==
    the oracle with 256 ants, bit for bit (final schedule + winner trace)."""
    import dataclasses
    regs = [I.gen_region(n, 300 + n) for n in (45, 120)]
    ids = [0, 1]
    p_all = I.Params(ants=256, iterations=4, seed=8)
    p_rank = dataclasses.replace(p_all, ants=64)
    ranks = _colony_ranks(regs, ids, p_rank, 4)
    s = _sched()
    s.load(regs, ids).run(p_all, no_prune=True)
    single = s.results()
    for k, (reg, rid) in enumerate(zip(regs, ids)):
        ora = O.schedule(reg, rid, I.GFX906, p_all)
        compare_results(single[k], ora, f"single {k}")
        for r in range(4):
            compare_results(ranks[r][k], ora, f"rank {r} region {k}")


def _relat(reg, f, tag):
    """The same DDG with every edge latency mapped by f (exercises the
    pass-2 ready-time layouts: windowed 10-bit for latencies < 512, u32 beyond)."""
    lat = np.asarray([f(int(x)) for x in reg.edge_lat], np.uint32)
    return I.Region(reg.n_insts, reg.edge_src, reg.edge_dst, lat, reg.reg_class, reg.reg_flags,
                    reg.def_ptr, reg.def_reg, reg.use_ptr, reg.use_reg, name=reg.name + tag)


def test_latency_window_boundary_every_ant(torch_cuda):
    """Latencies up to exactly 511 (the compact layout's bound) and schedules
    of thousands of cycles (the ready-time window slides many times)."""
    regs = [_relat(I.gen_region(n, 800 + n), lambda x: 511 if x >= 20 else (127 if x >= 8 else x), "-l511")
            for n in (25, 70, 180)]
    ids = [31, 32, 33]
    p = I.Params(ants=72, iterations=2, seed=21, stall_mod=2)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    dump_parity(s, regs, ids, p)


def test_long_latencies_every_ant(torch_cuda):
    """Latencies of 512 and above force the u32 ready-time layout."""
    regs = [_relat(I.gen_region(n, 900 + n), lambda x: x * 8 + (600 if x >= 20 else 0), "-long") for n in (25, 70, 180)]
    ids = [41, 42, 43]
    p = I.Params(ants=72, iterations=2, seed=22, stall_mod=2)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    dump_parity(s, regs, ids, p)


def many_multiuse_region():
    """Instructions reading 9 VGPRs that each have several users: more than 7
    multi-use registers of one class per instruction (3-bit last-use counts
    do not fit -> the u32 layout)."""
    n = 24
    defs = [[g] for g in range(9)] + [[9 + k] for k in range(12)] + [[], [], []]
    uses = [[] for _ in range(9)] + [list(range(9)) for _ in range(12)] + [[9, 10, 11], [12, 13, 14], list(range(15, 21))]
    edges = set()
    for j, u in enumerate(uses):
        for g in u:
            d = next(i for i, dd in enumerate(defs) if g in dd)
            edges.add((d, j, 1 + (d % 5)))
    return I.Region.from_lists(n, sorted(edges), [0] * 21, [0] * 21, defs, uses, name="multiuse9")


def test_many_multiuse_registers_every_ant(torch_cuda):
    regs = [many_multiuse_region(), I.gen_region(40, 4242)]
    ids = [51, 52]
    p = I.Params(ants=80, iterations=3, seed=23, stall_mod=1, cost_mode=0)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    dump_parity(s, regs, ids, p)


@pytest.mark.parametrize("mode,mix", [(0, 0), (1, 0), (1, 1)])
def test_lean_layout_every_ant(torch_cuda, mode, mix):
    """Large regions (n >= 160) run pass 2 in the lean layout (u8 ready times
    relative to a 128-cycle window, kills derived from the remaining-use
    counters at evaluation): every ant bit-exact, including latencies of
    exactly 127 (the lean window's bound) and per-group mixed heuristics."""
    regs = [I.gen_region(160, 1601), _relat(I.gen_region(211, 1602), lambda x: 127 if x >= 20 else x, "-l127"),
            I.gen_region(333, 1603, "unit"), I.gen_region(420, 1604)]
    ids = [61, 62, 63, 64]
    p = I.Params(ants=96, iterations=2, seed=24 + mode, cost_mode=mode, stall_mod=2, heur_mix=mix)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    dump_parity(s, regs, ids, p)


def test_lean_equals_compact_layout(torch_cuda, monkeypatch):
    """Production mode (pruning on, no dump): the lean and the 10-bit compact
    pass-2 layouts give the same results (the layout is an implementation
    choice, not semantics)."""
    regs = [I.gen_region(n, 1700 + n) for n in (170, 260, 480)]
    ids = [71, 72, 73]
    p = I.Params(ants=256, iterations=4, seed=31)
    out = []
    for lean in ("0", "1"):
        monkeypatch.setenv("ACO_LEAN", lean)
        s = _sched()
        s.load(regs, ids).run(p)
        out.append(s.results())
    for k in range(len(regs)):
        ora = O.schedule(regs[k], ids[k], I.GFX906, p)
        for g in out:
            compare_results(g[k], ora, f"region {k}")


@pytest.mark.parametrize("mode", [1, 2])
def test_ready_list_limit_every_ant(torch_cuda, mode):
    """Pass-1 ready-list size limit (L214; R45): the ants of each group of 64
    run in lockstep and consider only the first K ready instructions, K = the
    group's minimum (mode 1) or min/max midpoint (mode 2) ready-list size;
    100 ants = a full and a partial group; regions from a single bitset word
    to the 4-wide large-region kernels."""
    regs = [I.fix10a(), I.gen_region(45, 1801), I.gen_region(130, 1802, "unit"), I.gen_region(230, 1803)]
    ids = [81, 82, 83, 84]
    p = I.Params(ants=100, iterations=3, seed=40 + mode, cost_mode=0, rl_limit=mode)
    s = _sched()
    s.load(regs, ids).run(p, no_prune=True, dump=True)
    dump_parity(s, regs, ids, p)


def test_ready_list_limit_production(torch_cuda):
    """R45 in production mode (pruning on, winner replay with the recorded
    per-group limits) at 1024 ants: results equal the oracle's."""
    regs = [I.gen_region(n, 1900 + n) for n in (60, 180, 400)]
    ids = [91, 92, 93]
    p = I.Params(ants=1024, iterations=3, seed=47, rl_limit=1)
    s = _sched()
    s.load(regs, ids).run(p)
    got = s.results()
    for k in range(len(regs)):
        compare_results(got[k], O.schedule(regs[k], ids[k], I.GFX906, p), f"region {k}")


def test_plan_cache_reruns(torch_cuda):
    """Re-running a context with the same parameters reuses its plan (host
    planning skipped); changing a parameter re-plans.  Every run equals the
    oracle for its parameters."""
    regs = [I.gen_region(n, 2000 + n) for n in (35, 120, 260)]
    ids = [101, 102, 103]
    pa = I.Params(ants=128, iterations=3, seed=51)
    pb = I.Params(ants=128, iterations=3, seed=52, cost_mode=0)
    pc = I.Params(ants=320, iterations=2, seed=53)  # a larger workspace: the binding re-sizes it
    s = _sched()
    s.load(regs, ids)
    for p in (pa, pa, pb, pa, pc, pb, pc):
        s.run(p)
        got = s.results()
        for k in range(len(regs)):
            compare_results(got[k], O.schedule(regs[k], ids[k], I.GFX906, p), f"region {k} seed {p.seed}")
