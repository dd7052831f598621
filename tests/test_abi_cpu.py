"""Host-side checks of the C-ABI library that need no GPU: it loads, exports
every symbol declared in include/aco.h, and its validation (aco_create and
the sizing call of aco_load_regions make no CUDA call) agrees with the
oracle's error codes."""
import ctypes as C
import os
import re

import pytest

from oracle import pyoracle as O
from paper_conf_cgo_shobakimhlmkrg24_b200 import _lib, build
from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    build.build()
    return _lib.load()


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "aco.h")).read()
    return sorted(set(re.findall(r"\b(aco_[a-z_]+)\s*\(", src)))


def test_exports_every_declared_symbol(lib):
    syms = declared_symbols()
    assert "aco_load_regions" in syms and "aco_schedule_batch" in syms
    for s in syms:
        assert hasattr(lib, s), s
    assert set(_lib.EXPORTS) == set(syms)


def test_status_strings(lib):
    for st in range(0, -9, -1):
        assert lib.aco_status_string(st)


def _ctx(lib):
    from paper_conf_cgo_shobakimhlmkrg24_b200.api import machine_struct
    m = machine_struct(I.GFX906)
    ctx = C.c_void_p()
    assert lib.aco_create(0, C.byref(m), C.byref(ctx)) == 0
    return ctx, m


def _size_status(lib, regions, ids=None):
    from paper_conf_cgo_shobakimhlmkrg24_b200.api import HostBatch
    ctx, m = _ctx(lib)
    b = HostBatch(regions, ids or list(range(len(regions))))
    need = C.c_size_t(0)
    st = lib.aco_load_regions(ctx, b.descs, len(regions), None, 0, C.byref(need), None)
    lib.aco_destroy(ctx)
    return st, need.value


def _tiny(edges, defs, uses, flags=None, n=3):
    R = 1 + max([g for d in defs for g in d] + [g for u in uses for g in u] + [-1])
    return I.Region.from_lists(n, edges, [0] * R, flags or [0] * R, defs, uses)


CASES = [
    _tiny([(0, 1, 1), (1, 2, 1)], [[0], [1], []], [[], [0], [1]]),
    _tiny([(0, 1, 1), (1, 0, 1)], [[], [], []], [[], [], []]),
    _tiny([(0, 0, 1)], [[], [], []], [[], [], []]),
    _tiny([(0, 1, 1)], [[0], [0], []], [[], [], []]),
    _tiny([(0, 1, 1)], [[0], [], []], [[], [], [0]]),
    _tiny([(0, 1, 1), (0, 1, 2)], [[], [], []], [[], [], []]),
    _tiny([], [[], [], []], [[], [], [0]]),
    _tiny([], [[0], [], []], [[], [], []], flags=[1]),
]


@pytest.mark.parametrize("k", range(len(CASES)))
def test_validation_matches_oracle(lib, k):
    st, _ = _size_status(lib, [CASES[k]])
    assert st == O.validate(CASES[k])


def test_sizing_call_on_synthetic_batch(lib):
    regs = I.gen_batch(40, base_seed=9)
    st, need = _size_status(lib, regs)
    assert st == 0 and need > 0
    st, _ = _size_status(lib, regs[:2], [4, 4])
    assert st == -1  # duplicate region ids


def test_too_large_region(lib):
    n = 9000
    big = I.Region.from_lists(n, [], [], [], [[] for _ in range(n)], [[] for _ in range(n)])
    st, _ = _size_status(lib, [big])
    assert st == -5


def _plan_status(lib, regions, p, colony=False):
    """Sizing calls only (NULL arena / workspace): no CUDA call is made
    (ACO_DEBUG_PLAN keeps the host metadata of a sizing-only load and prints
    the launch plan to stderr)."""
    from paper_conf_cgo_shobakimhlmkrg24_b200.api import HostBatch, params_struct
    os.environ["ACO_DEBUG_PLAN"] = "1"
    ctx, m = _ctx(lib)
    b = HostBatch(regions, list(range(len(regions))))
    need = C.c_size_t(0)
    assert lib.aco_load_regions(ctx, b.descs, len(regions), None, 0, C.byref(need), None) == 0
    ps = params_struct(p)
    ws = C.c_size_t(0)
    if colony:
        st = lib.aco_colony_begin(ctx, C.byref(ps), 0, None, 0, C.byref(ws), None)
    else:
        st = lib.aco_schedule_batch(ctx, C.byref(ps), None, 0, C.byref(ws), None)
    lib.aco_destroy(ctx)
    del os.environ["ACO_DEBUG_PLAN"]
    return st, ws.value


def test_ready_list_limit_params(lib):
    """R45: modes 0-2 plan; 3 is rejected; the shared colony rejects any
    limit (a wavefront would span ranks)."""
    regs = I.gen_batch(6, base_seed=5)
    for mode in (0, 1, 2):
        assert _plan_status(lib, regs, I.Params(ants=128, iterations=2, rl_limit=mode))[0] == 0
    assert _plan_status(lib, regs, I.Params(ants=128, iterations=2, rl_limit=3))[0] == -1
    assert _plan_status(lib, regs, I.Params(ants=128, iterations=2, rl_limit=1), colony=True)[0] == -1
    assert _plan_status(lib, regs, I.Params(ants=128, iterations=2), colony=True)[0] == 0


def test_record_mode_workspace(lib, monkeypatch):
    """Record mode (winner copied, not replayed) adds exactly the recorded
    schedules to the workspace: A x sum(n) x (2 + 4) bytes (order u16, pass-2
    cycles u32) plus A x 16 bytes per region, up to 256-byte alignment."""
    regs = I.gen_batch(12, base_seed=6)
    p = I.Params(ants=256, iterations=2)
    monkeypatch.setenv("ACO_RECORD_MB", "0")
    st0, ws0 = _plan_status(lib, regs, p)
    monkeypatch.setenv("ACO_RECORD_MB", "16384")
    st1, ws1 = _plan_status(lib, regs, p)
    assert st0 == st1 == 0
    want = p.ants * sum(r.n_insts for r in regs) * 6 + 16 * p.ants * len(regs)
    assert want <= ws1 - ws0 <= want + 3 * 256 + 3 * 16


PLAN_SNIPPET = r'''
import ctypes as C, json, os, sys
sys.path.insert(0, {root!r})
os.environ["ACO_DEBUG_PLAN"] = "1"
import bench
from paper_conf_cgo_shobakimhlmkrg24_b200 import _lib
from paper_conf_cgo_shobakimhlmkrg24_b200.api import HostBatch, machine_struct, params_struct
L = _lib.load()
a = bench.parse({argv!r})
out = []
for b in bench.workload(a, 0, 1)[0]:
    hb = HostBatch(b.regs, b.ids)
    m = machine_struct(bench.machine_of(a)); ctx = C.c_void_p()
    L.aco_create(0, C.byref(m), C.byref(ctx))
    need = C.c_size_t(0)
    assert L.aco_load_regions(ctx, hb.descs, len(b.regs), None, 0, C.byref(need), None) == 0
    ps = params_struct(b.p)
    assert L.aco_schedule_batch(ctx, C.byref(ps), None, 0, C.byref(need), None) == 0
    cnt = C.c_uint32(0); buf = (C.c_uint32 * 64)()
    L.aco_last_variants(ctx, buf, 64, C.byref(cnt))
    out.append([int(buf[i]) for i in range(cnt.value)])
print(json.dumps(out))
'''


def _plan(argv):
    """Host planning of a bench line (sizing calls, no CUDA call): the
    variants of each batch and the '[aco plan]' class lines."""
    import json
    import subprocess
    import sys
    r = subprocess.run([sys.executable, "-c", PLAN_SNIPPET.format(root=ROOT, argv=argv)], capture_output=True,
                       text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-2000:]
    classes = []
    for line in r.stderr.splitlines():
        mm = re.match(r"\[aco plan\] pass (\d) class \d+: blocks (\d+) ants/blk (\d+) lanes (\d+)", line)
        if mm:
            classes.append(tuple(int(x) for x in mm.groups()))
    return json.loads(r.stdout.strip().splitlines()[-1]), classes


def test_planner_fused_for_config1_only(lib):
    """Config 1 (64 ants, one region) runs as one fused single-block launch
    (k_fused, variant bit 13); config 2 (1,024 ants) does not."""
    v1, c1 = _plan(["--workload", "c1"])
    assert v1 == [[1 << 13]]
    v2, c2 = _plan(["--workload", "c2"])
    assert all(not (c & (1 << 13)) for c in v2[0]) and c2


def test_planner_fill_rule_spreads_few_large_regions(lib):
    """Config 2 (one region holding all the work): its ants spread over many
    small blocks in both passes (the SM fill rule), pass 1 with up to 4 lanes
    per ant; config 3 (5,000 regions) keeps its large blocks.  (Config 2
    runs on the lane-per-instruction ants by default: ACO_LPI=0 here.)"""
    os.environ["ACO_LPI"] = "0"
    try:
        _, c2 = _plan(["--workload", "c2"])
    finally:
        del os.environ["ACO_LPI"]
    for pass_ in (1, 2):
        blocks = sum(b for p, b, a, l in c2 if p == pass_)
        assert blocks >= 32, c2
    assert any(p == 1 and l == 4 for p, b, a, l in c2)
    _, c3 = _plan(["--workload", "c3", "--regions", "400"])
    assert max(a * l for p, b, a, l in c3) >= 256  # large blocks kept


def test_planner_lane_per_instruction_for_config2(lib):
    """Config 2 (one n = 100 region, 1,024 ants: the per-ant step latency
    bounds it) takes the lane-per-instruction ants in both passes: one warp
    per ant, ~148 blocks; config 3's batch never does."""
    v2, c2 = _plan(["--workload", "c2"])
    assert v2[0] and all(c & (1 << 10) for c in v2[0]), v2
    for pass_ in (1, 2):
        assert sum(b for p, b, a, l in c2 if p == pass_ and l == 32) >= 128, c2
    v3, _ = _plan(["--workload", "c3", "--regions", "400"])
    assert not any(c & (1 << 10) for c in v3[0])


def _variants_of(lib, machine, regions, p):
    """Construct variants a run would launch (sizing calls only, no CUDA)."""
    from paper_conf_cgo_shobakimhlmkrg24_b200.api import HostBatch, machine_struct, params_struct
    os.environ["ACO_DEBUG_PLAN"] = "1"
    try:
        m = machine_struct(machine)
        ctx = C.c_void_p()
        assert lib.aco_create(0, C.byref(m), C.byref(ctx)) == 0
        b = HostBatch(regions, list(range(len(regions))))
        need = C.c_size_t(0)
        assert lib.aco_load_regions(ctx, b.descs, len(regions), None, 0, C.byref(need), None) == 0
        ps = params_struct(p)
        ws = C.c_size_t(0)
        assert lib.aco_schedule_batch(ctx, C.byref(ps), None, 0, C.byref(ws), None) == 0
        cnt = C.c_uint32(0)
        assert lib.aco_last_variants(ctx, None, 0, C.byref(cnt)) == 0
        buf = (C.c_uint32 * max(1, cnt.value))()
        assert lib.aco_last_variants(ctx, buf, cnt.value, C.byref(cnt)) == 0
        lib.aco_destroy(ctx)
        return [int(buf[i]) for i in range(cnt.value)]
    finally:
        del os.environ["ACO_DEBUG_PLAN"]


def test_planner_lane_per_instruction_eligibility(lib):
    """Lane-per-instruction ants (variant bit 10) only where their
    arithmetic holds: n <= 128, <= 2 register classes, single issue in pass 2
    (pass 1 ignores the machine model, R19), no mixed heuristics (R43), a
    batch with few ants in total."""
    import dataclasses
    lpi = 1 << 10
    p = I.Params(ants=1024, iterations=3, seed=1)
    r100 = [I.gen_region(100, 11)]
    v = _variants_of(lib, I.GFX906, r100, p)
    assert v and all(c & lpi for c in v), v
    # dual issue: pass 1 keeps the lane-per-instruction ants, pass 2 does not
    v = _variants_of(lib, I.DUAL_ISSUE, r100, p)
    assert any(c & lpi and not c & 256 for c in v) and not any(c & lpi and c & 256 for c in v), v
    # three register classes, mixed heuristics, n = 129, many ants: never
    m3 = I.Machine(n_classes=3, steps=I.GFX906.steps + ((10, 20),), perp_limit=(24, 80, 10, 0))
    assert not any(c & lpi for c in _variants_of(lib, m3, r100, p))
    assert not any(c & lpi for c in _variants_of(lib, I.GFX906, r100, dataclasses.replace(p, heur_mix=1)))
    assert not any(c & lpi for c in _variants_of(lib, I.GFX906, [I.gen_region(129, 12)], p))
    assert not any(c & lpi for c in _variants_of(lib, I.GFX906, [I.gen_region(100, 13 + k) for k in range(5)], p))
    # ... unless forced (tests), which still respects eligibility
    os.environ["ACO_LPI"] = "2"
    try:
        v = _variants_of(lib, I.GFX906, [I.gen_region(100, 13 + k) for k in range(5)] + [I.gen_region(300, 20)], p)
    finally:
        del os.environ["ACO_LPI"]
    assert any(c & lpi for c in v) and any(not c & lpi for c in v), v
