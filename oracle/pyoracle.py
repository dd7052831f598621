"""ctypes binding of the sequential CPU oracle (oracle/aco_oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and the
cpu_baseline / --impl reference legs of bench.py -- never by the product
package.  Argument marshalling only; all arithmetic lives in aco_oracle.c.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from typing import Optional, Sequence

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "aco_oracle.c")
HDR = os.path.join(HERE, "aco_oracle.h")
LIB = os.path.join(HERE, "liboracle.so")

ORS_NAMES = [
    "cost_rp", "length", "prp0", "prp1", "prp2", "prp3", "iters1", "iters2", "trace_hash",
    "best1", "best2", "lb1", "lblen", "init1", "init2", "target0", "target1", "target2",
    "target3", "ant_scheds", "placements", "stall_events", "sum_R", "sum_F", "sum_S",
    "sum_deg", "sum_use", "sum_def", "sum_muse_checks", "dead_ants", "ub_ready",
    "policy", "heur_len", "ws_cost",
]
ORS = {name: i for i, name in enumerate(ORS_NAMES)}
ORS_COUNT = len(ORS_NAMES)
INVALID = 0xFFFFFFFF


def build(force: bool = False) -> str:
    """Compile liboracle.so with gcc (plain -O2, no tuning)."""
    stale = (not os.path.exists(LIB)) or any(
        os.path.getmtime(f) > os.path.getmtime(LIB) for f in (SRC, HDR))
    if force or stale:
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-fPIC", "-shared", "-pthread",
                               "-o", LIB, SRC])
    return LIB


class _Region(C.Structure):
    _fields_ = [
        ("n_insts", C.c_uint32), ("n_edges", C.c_uint32), ("n_regs", C.c_uint32),
        ("edge_src", C.c_void_p), ("edge_dst", C.c_void_p), ("edge_lat", C.c_void_p),
        ("reg_class", C.c_void_p), ("reg_flags", C.c_void_p),
        ("def_ptr", C.c_void_p), ("def_reg", C.c_void_p),
        ("use_ptr", C.c_void_p), ("use_reg", C.c_void_p), ("inst_type", C.c_void_p),
    ]


class _Machine(C.Structure):
    _fields_ = [
        ("n_classes", C.c_uint32), ("occ_max", C.c_uint32),
        ("step_count", C.c_uint32 * 4), ("step_max", (C.c_uint32 * 16) * 4),
        ("perp_limit", C.c_uint32 * 4),
        ("issue_width", C.c_uint32), ("n_types", C.c_uint32), ("type_slots", C.c_uint32 * 4),
    ]


class _Params(C.Structure):
    _fields_ = [
        ("ants", C.c_uint32), ("iterations", C.c_uint32), ("seed", C.c_uint64),
        ("pass_", C.c_uint32), ("cost_mode", C.c_uint32), ("q0_t", C.c_uint64),
        ("group_size", C.c_uint32), ("stall_mod", C.c_uint32), ("stall_rem", C.c_uint32),
        ("tau0", C.c_uint32), ("rho_q16", C.c_uint32), ("delta", C.c_uint32),
        ("tau_min", C.c_uint32), ("tau_max", C.c_uint32),
        ("stop_no_improve", C.c_uint32), ("stop_at_lb", C.c_uint32),
        ("pass2_gap", C.c_uint32), ("revert_occ", C.c_uint32), ("revert_len", C.c_uint32),
        ("ws_weight", C.c_uint32), ("heur_mix", C.c_uint32), ("stall_num", C.c_uint32),
        ("rl_limit", C.c_uint32),
    ]


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(LIB)
        vp, u32, u64 = C.c_void_p, C.c_uint32, C.c_uint64
        L.orc_philox4x32_10.argtypes = [vp, vp, vp]
        L.orc_validate.argtypes = [vp, u32]
        L.orc_prp_of_order.argtypes = [vp, u32, vp, vp]
        L.orc_asap.argtypes = [vp, vp, vp]
        L.orc_asap.restype = C.c_int64
        L.orc_asap_m.argtypes = [vp, vp, vp, vp]
        L.orc_asap_m.restype = C.c_int64
        L.orc_critical_path.argtypes = [vp, vp]
        L.orc_occupancy.argtypes = [vp, u32, u32]
        L.orc_occupancy.restype = u32
        L.orc_aprp.argtypes = [vp, u32, u32]
        L.orc_aprp.restype = u32
        L.orc_cost_rp.argtypes = [vp, u32, vp]
        L.orc_cost_rp.restype = u32
        L.orc_target.argtypes = [vp, u32, vp, vp]
        L.orc_lower_bounds.argtypes = [vp, vp, u32, vp, vp, vp]
        L.orc_select.argtypes = [vp, u32, C.c_int, u64]
        L.orc_select.restype = u32
        L.orc_pheromone_update.argtypes = [vp, u32, vp, vp]
        L.orc_schedule.argtypes = [vp, u32, vp, vp, vp, vp, vp, vp, vp, vp, vp]
        L.orc_schedule_many.argtypes = [vp, vp, u32, vp, vp, vp, vp, vp, vp, u32]
        L.orc_run_ant.argtypes = [vp, u32, vp, vp, u32, u32, u32, vp, vp, vp, vp, vp, vp]
        L.orc_greedy_pass1.argtypes = [vp, vp, vp, vp, vp]
        L.orc_eta_initial.argtypes = [vp, vp, u32, vp]
        _lib = L
    return _lib


def _ptr(a: Optional[np.ndarray]):
    return None if a is None else a.ctypes.data


class RegionRef:
    """Holds contiguous arrays alive and the ctypes struct pointing at them."""

    def __init__(self, r):
        self.arrays = [np.ascontiguousarray(x, dtype=dt) for x, dt in (
            (r.edge_src, np.uint32), (r.edge_dst, np.uint32), (r.edge_lat, np.uint32),
            (r.reg_class, np.uint8), (r.reg_flags, np.uint8), (r.def_ptr, np.uint32),
            (r.def_reg, np.uint32), (r.use_ptr, np.uint32), (r.use_reg, np.uint32))]
        # non-empty placeholders so pointers are valid
        self.arrays = [a if a.size else np.zeros(1, a.dtype) for a in self.arrays]
        a = self.arrays
        self.n = int(r.n_insts)
        it = getattr(r, "inst_type", None)
        self.types = None if it is None else np.ascontiguousarray(it, np.uint8)
        tp = None if self.types is None or not self.types.size else self.types.ctypes.data
        self.s = _Region(self.n, int(r.n_edges), int(r.n_regs), *[x.ctypes.data for x in a], tp)

    @property
    def ref(self):
        return C.byref(self.s)


def machine_struct(m) -> _Machine:
    s = _Machine()
    s.n_classes = m.n_classes
    s.occ_max = m.occ_max
    for c, steps in enumerate(m.steps):
        s.step_count[c] = len(steps)
        for i, v in enumerate(steps):
            s.step_max[c][i] = v
    for c in range(4):
        s.perp_limit[c] = m.perp_limit[c] if c < len(m.perp_limit) else 0
    s.issue_width = getattr(m, "issue_width", 1)
    s.n_types = getattr(m, "n_types", 1)
    for y, v in enumerate(getattr(m, "type_slots", (1, 1, 1, 1))):
        s.type_slots[y] = v
    return s


def params_struct(p) -> _Params:
    return _Params(p.ants, p.iterations, p.seed, p.passes, p.cost_mode, p.q0_t, p.group_size,
                   p.stall_mod, p.stall_rem, p.tau0, p.rho_q16, p.delta, p.tau_min, p.tau_max,
                   p.stop_no_improve, p.stop_at_lb, p.pass2_gap, p.revert_occ, p.revert_len,
                   p.ws_weight, p.heur_mix, p.stall_num, p.rl_limit)


def philox(ctr: Sequence[int], key: Sequence[int]):
    c = np.asarray(ctr, np.uint32)
    k = np.asarray(key, np.uint32)
    out = np.zeros(4, np.uint32)
    lib().orc_philox4x32_10(c.ctypes.data, k.ctypes.data, out.ctypes.data)
    return [int(x) for x in out]


def validate(region, n_classes=2) -> int:
    rr = RegionRef(region)
    return lib().orc_validate(rr.ref, n_classes)


def prp_of_order(region, order, n_classes=2):
    rr = RegionRef(region)
    o = np.ascontiguousarray(order, np.uint32)
    out = np.zeros(4, np.uint32)
    st = lib().orc_prp_of_order(rr.ref, n_classes, _ptr(o) if o.size else None, out.ctypes.data)
    assert st == 0, st
    return [int(x) for x in out]


def asap(region, order):
    rr = RegionRef(region)
    o = np.ascontiguousarray(order, np.uint32)
    cyc = np.zeros(max(1, len(o)), np.uint32)
    length = lib().orc_asap(rr.ref, _ptr(o) if o.size else None, cyc.ctypes.data)
    return int(length), [int(x) for x in cyc[:len(o)]]


def asap_m(region, machine, order):
    """ASAP timing on the general machine model (R42)."""
    rr = RegionRef(region)
    m = machine_struct(machine)
    o = np.ascontiguousarray(order, np.uint32)
    cyc = np.zeros(max(1, len(o)), np.uint32)
    length = lib().orc_asap_m(rr.ref, C.byref(m), _ptr(o) if o.size else None, cyc.ctypes.data)
    return int(length), [int(x) for x in cyc[:len(o)]]


def critical_path(region):
    rr = RegionRef(region)
    out = np.zeros(max(1, region.n_insts), np.uint32)
    lib().orc_critical_path(rr.ref, out.ctypes.data)
    return [int(x) for x in out[:region.n_insts]]


def occupancy(machine, c, prp):
    m = machine_struct(machine)
    return int(lib().orc_occupancy(C.byref(m), c, prp))


def aprp(machine, c, prp):
    m = machine_struct(machine)
    return int(lib().orc_aprp(C.byref(m), c, prp))


def cost_rp(machine, mode, prp):
    m = machine_struct(machine)
    a = np.zeros(4, np.uint32)
    a[:len(prp)] = prp
    return int(lib().orc_cost_rp(C.byref(m), mode, a.ctypes.data))


def target(machine, mode, best_prp):
    m = machine_struct(machine)
    a = np.zeros(4, np.uint32)
    a[:len(best_prp)] = best_prp
    out = np.zeros(4, np.uint32)
    lib().orc_target(C.byref(m), mode, a.ctypes.data, out.ctypes.data)
    return [int(x) for x in out]


def lower_bounds(region, machine, mode):
    rr = RegionRef(region)
    m = machine_struct(machine)
    a, b, c = C.c_uint32(), C.c_uint32(), C.c_uint32()
    st = lib().orc_lower_bounds(rr.ref, C.byref(m), mode, C.byref(a), C.byref(b), C.byref(c))
    assert st == 0, st
    return int(a.value), int(b.value), int(c.value)


def select(scores, exploit: bool, r64: int) -> int:
    s = np.ascontiguousarray(scores, np.uint32)
    return int(lib().orc_select(s.ctypes.data, len(s), 1 if exploit else 0, r64))


def pheromone_update(tau: np.ndarray, n: int, winner_order, params) -> np.ndarray:
    t = np.ascontiguousarray(tau, np.uint16).copy()
    p = params_struct(params)
    w = None if winner_order is None else np.ascontiguousarray(winner_order, np.uint32)
    lib().orc_pheromone_update(t.ctypes.data, n, _ptr(w), C.byref(p))
    return t


def greedy_pass1(region, machine, params):
    rr = RegionRef(region)
    m = machine_struct(machine)
    p = params_struct(params)
    order = np.zeros(max(1, region.n_insts), np.uint32)
    prp = np.zeros(4, np.uint32)
    st = lib().orc_greedy_pass1(rr.ref, C.byref(m), C.byref(p), order.ctypes.data, prp.ctypes.data)
    assert st == 0, st
    return [int(x) for x in order[:region.n_insts]], [int(x) for x in prp]


def eta_initial(region, machine, pass_):
    rr = RegionRef(region)
    m = machine_struct(machine)
    out = np.zeros(max(1, region.n_insts), np.uint32)
    st = lib().orc_eta_initial(rr.ref, C.byref(m), pass_, out.ctypes.data)
    assert st == 0, st
    return [int(x) for x in out[:region.n_insts]]


def run_ant(region, region_id, machine, params, pass_, it, ant, tau, target_prp=None):
    rr = RegionRef(region)
    m = machine_struct(machine)
    p = params_struct(params)
    n = region.n_insts
    t = np.ascontiguousarray(tau, np.uint16)
    tg = None if target_prp is None else np.asarray(list(target_prp) + [0xFFFFFFFF] * (4 - len(target_prp)), np.uint32)
    order = np.zeros(max(1, n), np.uint32)
    cyc = np.zeros(max(1, n), np.uint32)
    prp = np.zeros(4, np.uint32)
    cost = C.c_uint32()
    st = lib().orc_run_ant(rr.ref, region_id, C.byref(m), C.byref(p), pass_, it, ant, t.ctypes.data,
                           _ptr(tg), order.ctypes.data, cyc.ctypes.data, prp.ctypes.data, C.byref(cost))
    assert st == 0, st
    return dict(order=order[:n].copy(), cycle=cyc[:n].copy(), prp=[int(x) for x in prp], cost=int(cost.value))


class Result(dict):
    pass


def schedule(region, region_id, machine, params, dump=False, dump_orders=False, want_tau=False):
    """Run the whole two-pass ACO for one region; returns a dict."""
    rr = RegionRef(region)
    m = machine_struct(machine)
    p = params_struct(params)
    n = region.n_insts
    order = np.zeros(max(1, n), np.uint32)
    cyc = np.zeros(max(1, n), np.uint32)
    stats = np.zeros(ORS_COUNT, np.uint64)
    dc = do = dy = tau = None
    if dump:
        dc = np.full((2, params.iterations, params.ants), INVALID, np.uint32)
    if dump_orders:
        do = np.zeros((2, params.iterations, params.ants, max(1, n)), np.uint32)
        dy = np.zeros((2, params.iterations, params.ants, max(1, n)), np.uint32)
    if want_tau:
        tau = np.zeros(max(1, (n + 1) * n), np.uint16)
    st = lib().orc_schedule(rr.ref, region_id, C.byref(m), C.byref(p), order.ctypes.data,
                            cyc.ctypes.data, stats.ctypes.data, _ptr(dc), _ptr(do), _ptr(dy), _ptr(tau))
    if st != 0:
        raise RuntimeError(f"orc_schedule failed: {st}")
    res = Result({k: int(stats[i]) for k, i in ORS.items()})
    res["order"] = order[:n].copy()
    res["cycle"] = cyc[:n].copy()
    res["prp"] = [res["prp0"], res["prp1"], res["prp2"], res["prp3"]]
    if dump:
        res["dump_cost"] = dc
    if dump_orders:
        res["dump_order"] = do[..., :n]
        res["dump_cycle"] = dy[..., :n]
    if want_tau:
        res["tau"] = tau[:(n + 1) * n].reshape(n + 1, n) if n else tau[:0]
    return res


def schedule_many(regions, region_ids, machine, params, n_threads=None):
    """All regions on a pool of host threads; returns (orders, cycles, stats)."""
    refs = [RegionRef(r) for r in regions]
    arr = (_Region * len(refs))(*[x.s for x in refs])
    ids = np.ascontiguousarray(region_ids, np.uint32)
    sizes = np.array([r.n_insts for r in regions], np.uint64)
    off = np.zeros(len(regions) + 1, np.uint64)
    off[1:] = np.cumsum(sizes)
    order = np.zeros(max(1, int(off[-1])), np.uint32)
    cyc = np.zeros(max(1, int(off[-1])), np.uint32)
    stats = np.zeros((len(regions), ORS_COUNT), np.uint64)
    m = machine_struct(machine)
    p = params_struct(params)
    if n_threads is None:
        n_threads = os.cpu_count() or 1
    st = lib().orc_schedule_many(arr, ids.ctypes.data, len(regions), C.byref(m), C.byref(p),
                                 off.ctypes.data, order.ctypes.data, cyc.ctypes.data,
                                 stats.ctypes.data, n_threads)
    if st != 0:
        raise RuntimeError(f"orc_schedule_many failed: {st}")
    return order, cyc, stats, off
