"""Python API over the C ABI (argument marshalling only; every step of the
hot path runs in the CUDA library).  PyTorch provides device memory and streams.

    sched = Scheduler(inputs.GFX906, device=0)
    sched.load(regions)                    # aco_load_regions (host preprocessing + 1 H2D)
    sched.run(inputs.Params(ants=1024))    # aco_schedule_batch (all kernels, async)
    res = sched.results()                  # aco_get_results (sync + D2H)
"""
from __future__ import annotations

import ctypes as C
import dataclasses
from typing import List, Optional, Sequence

import numpy as np
import torch

from . import _lib
from .inputs import GFX906, Machine, Params, Region


def _stream_handle(stream: Optional[torch.cuda.Stream]) -> C.c_void_p:
    s = stream if stream is not None else torch.cuda.current_stream()
    return C.c_void_p(s.cuda_stream)


def machine_struct(m: Machine) -> _lib.Machine:
    s = _lib.Machine()
    s.n_classes = m.n_classes
    s.occ_max = m.occ_max
    for c, steps in enumerate(m.steps):
        s.step_count[c] = len(steps)
        for i, v in enumerate(steps):
            s.step_max[c][i] = v
    for c in range(4):
        s.perp_limit[c] = m.perp_limit[c] if c < len(m.perp_limit) else 0
    s.issue_width = m.issue_width
    s.n_types = m.n_types
    for y, v in enumerate(m.type_slots):
        s.type_slots[y] = v
    return s


def params_struct(p: Params, flags: int = 0) -> _lib.Params:
    return _lib.Params(p.ants, p.iterations, p.seed, p.passes, p.cost_mode, p.q0_t, p.group_size,
                       p.stall_mod, p.stall_rem, p.tau0, p.rho_q16, p.delta, p.tau_min, p.tau_max,
                       p.stop_no_improve, p.stop_at_lb, flags, p.pass2_gap, p.revert_occ, p.revert_len,
                       p.ws_weight, p.heur_mix, p.stall_num, p.rl_limit)


class HostBatch:
    """Region descriptors pointing at contiguous host arrays (kept alive here)."""

    def __init__(self, regions: Sequence[Region], region_ids: Sequence[int]):
        self.keep = []
        self.descs = (_lib.RegionDesc * len(regions))()
        for i, (r, rid) in enumerate(zip(regions, region_ids)):
            arrs = []
            for x, dt in ((r.edge_src, np.uint32), (r.edge_dst, np.uint32), (r.edge_lat, np.uint32),
                          (r.reg_class, np.uint8), (r.reg_flags, np.uint8), (r.def_ptr, np.uint32),
                          (r.def_reg, np.uint32), (r.use_ptr, np.uint32), (r.use_reg, np.uint32)):
                a = np.ascontiguousarray(x, dtype=dt)
                if a.size == 0:
                    a = np.zeros(1, dt)
                arrs.append(a)
            it = None
            if r.inst_type is not None and r.n_insts:
                it = np.ascontiguousarray(r.inst_type, dtype=np.uint8)
                arrs.append(it)
            self.keep.append(arrs)
            self.descs[i] = _lib.RegionDesc(int(rid), int(r.n_insts), int(r.n_edges), int(r.n_regs),
                                            *[a.ctypes.data for a in arrs[:9]],
                                            None if it is None else it.ctypes.data)
        self.sizes = np.array([r.n_insts for r in regions], np.int64)
        self.offsets = np.concatenate([[0], np.cumsum(self.sizes)]).astype(np.int64)


class Scheduler:
    def __init__(self, machine: Machine = GFX906, device: int = 0):
        self.lib = _lib.load()
        self.device = device
        torch.cuda.set_device(device)
        self.ctx = C.c_void_p()
        self._m = machine_struct(machine)
        _lib.check(self.lib.aco_create(device, C.byref(self._m), C.byref(self.ctx)), "aco_create")
        self.arena: Optional[torch.Tensor] = None
        self.ws: Optional[torch.Tensor] = None
        self.batch: Optional[HostBatch] = None
        self.count = 0
        self._need = {}  # workspace bytes per (params, flags) for the loaded regions
        self.params: Optional[Params] = None
        self.dump = None
        self.dump_key = None

    def __del__(self):
        try:
            if self.ctx:
                self.lib.aco_destroy(self.ctx)
                self.ctx = C.c_void_p()
        except Exception:
            pass

    # ---------------------------------------------------------------- load
    def load(self, regions: Sequence[Region], region_ids: Optional[Sequence[int]] = None,
             stream: Optional[torch.cuda.Stream] = None, batch: Optional[HostBatch] = None):
        if region_ids is None:
            region_ids = list(range(len(regions)))
        b = batch if batch is not None else HostBatch(regions, region_ids)
        need = C.c_size_t(0)
        sh = _stream_handle(stream)
        st = _lib.ACO_E_WORKSPACE
        if self.arena is not None:  # one preprocessing pass when the arena is already large enough
            st = self.lib.aco_load_regions(self.ctx, b.descs, len(regions), C.c_void_p(self.arena.data_ptr()),
                                           self.arena.numel(), C.byref(need), sh)
        if st == _lib.ACO_E_WORKSPACE:
            if need.value == 0:
                _lib.check(self.lib.aco_load_regions(self.ctx, b.descs, len(regions), None, 0, C.byref(need), sh),
                           "aco_load_regions(size)")
            self.arena = torch.empty(max(256, need.value), dtype=torch.uint8, device=f"cuda:{self.device}")
            st = self.lib.aco_load_regions(self.ctx, b.descs, len(regions), C.c_void_p(self.arena.data_ptr()),
                                           self.arena.numel(), C.byref(need), sh)
        _lib.check(st, "aco_load_regions")
        self.batch = b
        self._need = {}
        self.count = len(regions)
        self.dump = None  # dump buffers are sized for the loaded batch (sum of n)
        return self

    # ---------------------------------------------------------------- run
    def workspace_bytes(self, p: Params, flags: int = 0) -> int:
        need = C.c_size_t(0)
        ps = params_struct(p, flags)
        _lib.check(self.lib.aco_schedule_batch(self.ctx, C.byref(ps), None, 0, C.byref(need), None),
                   "aco_schedule_batch(size)")
        return need.value

    def set_dump(self, p: Params, orders: bool = True):
        """Allocate dump buffers (test/debug): costs of every ant of every
        iteration, and optionally every ant's order and pass-2 cycles."""
        dev = f"cuda:{self.device}"
        costs = torch.full((2, p.iterations, self.count, p.ants), -1, dtype=torch.int32, device=dev)
        sum_n = int(self.batch.offsets[-1])
        od = cy = None
        if orders:
            # flat [2][iterations][ants * sum_n] (+ padding so empty batches have storage)
            size = 2 * p.iterations * p.ants * sum_n + 8
            od = torch.zeros(size, dtype=torch.int16, device=dev)
            cy = torch.zeros(size, dtype=torch.int32, device=dev)
        self.dump = (costs, od, cy)
        self.dump_key = (p.ants, p.iterations)
        _lib.check(self.lib.aco_set_dump(self.ctx, C.c_void_p(costs.data_ptr()), costs.numel(),
                                         C.c_void_p(od.data_ptr()) if od is not None else None,
                                         od.numel() if od is not None else 0,
                                         C.c_void_p(cy.data_ptr()) if cy is not None else None,
                                         cy.numel() if cy is not None else 0),
                   "aco_set_dump")

    def run(self, p: Params, stream: Optional[torch.cuda.Stream] = None, no_prune: bool = False,
            dump: bool = False, timing: bool = False):
        flags = ((_lib.ACO_FLAG_NO_PRUNE if no_prune else 0) | (_lib.ACO_FLAG_DUMP if dump else 0)
                 | (_lib.ACO_FLAG_TIMING if timing else 0))
        if dump and (self.dump is None or self.dump_key != (p.ants, p.iterations)):
            self.set_dump(p)
        key = (dataclasses.astuple(p), flags)
        need = self._need.get(key)
        ps = params_struct(p, flags)
        n = C.c_size_t(0)
        if need is None and self.ws is not None:
            # new parameters or regions: try the workspace we have -- the library
            # plans once and reports the size it needs if it is too small
            st = self.lib.aco_schedule_batch(self.ctx, C.byref(ps), C.c_void_p(self.ws.data_ptr()),
                                             self.ws.numel(), C.byref(n), _stream_handle(stream))
            if st == 0:
                self._need[key] = int(n.value)
                self.params = p
                return self
            if st != _lib.ACO_E_WORKSPACE:
                _lib.check(st, "aco_schedule_batch")
            need = int(n.value)
        if need is None:  # sizing call (host planning)
            need = self.workspace_bytes(p, flags)
        self._need[key] = need
        if self.ws is None or self.ws.numel() < need:
            self.ws = torch.empty(max(256, need), dtype=torch.uint8, device=f"cuda:{self.device}")
        _lib.check(self.lib.aco_schedule_batch(self.ctx, C.byref(ps), C.c_void_p(self.ws.data_ptr()),
                                               self.ws.numel(), C.byref(n), _stream_handle(stream)),
                   "aco_schedule_batch")
        self.params = p
        return self

    # ---------------------------------------------------------------- shared colony
    def colony_begin(self, p: Params, ant_base: int, stream: Optional[torch.cuda.Stream] = None,
                     timing: bool = False):
        """Plan a shared-colony run: this context builds ants [ant_base, ant_base + p.ants)."""
        need = C.c_size_t(0)
        ps = params_struct(p, _lib.ACO_FLAG_TIMING if timing else 0)
        _lib.check(self.lib.aco_colony_begin(self.ctx, C.byref(ps), ant_base, None, 0, C.byref(need), None),
                   "aco_colony_begin(size)")
        if self.ws is None or self.ws.numel() < need.value:
            self.ws = torch.empty(max(256, need.value), dtype=torch.uint8, device=f"cuda:{self.device}")
        _lib.check(self.lib.aco_colony_begin(self.ctx, C.byref(ps), ant_base, C.c_void_p(self.ws.data_ptr()),
                                             self.ws.numel(), C.byref(need), _stream_handle(stream)),
                   "aco_colony_begin")
        self.params = p
        self.keys = torch.empty(max(1, self.count), dtype=torch.int64, device=f"cuda:{self.device}")
        return self.keys

    def colony_construct(self, pass_: int, it: int, stream: Optional[torch.cuda.Stream] = None):
        _lib.check(self.lib.aco_colony_construct(self.ctx, pass_, it, C.c_void_p(self.keys.data_ptr()),
                                                 _stream_handle(stream)), "aco_colony_construct")

    def colony_finalize(self, pass_: int, it: int, stream: Optional[torch.cuda.Stream] = None):
        _lib.check(self.lib.aco_colony_finalize(self.ctx, pass_, it, C.c_void_p(self.keys.data_ptr()),
                                                _stream_handle(stream)), "aco_colony_finalize")

    def colony_end(self, stream: Optional[torch.cuda.Stream] = None):
        _lib.check(self.lib.aco_colony_end(self.ctx, _stream_handle(stream)), "aco_colony_end")

    def run_colony(self, p: Params, rank: int, world: int, group=None, timing: bool = False):
        """Shared colony over torch.distributed (NCCL): p.ants per rank, global
        ants = p.ants * world; one int64 MIN allreduce per region per iteration."""
        from .sharding import colony_allreduce
        keys = self.colony_begin(p, rank * p.ants, timing=timing)
        pmask = 2 if p.passes == 4 else p.passes  # pass 4 runs on the pass-2 machinery (R41)
        for pass_ in (1, 2):
            if not (pmask & pass_):
                continue
            for it in range(p.iterations):
                self.colony_construct(pass_, it)
                if world > 1:
                    colony_allreduce(keys, group)
                self.colony_finalize(pass_, it)
        self.colony_end()
        return self

    def timing(self):
        """(ms[construct, finalize, init], launches[...]) of the last timed run."""
        ms = (C.c_double * 3)()
        ln = (C.c_uint64 * 3)()
        _lib.check(self.lib.aco_get_timing(self.ctx, ms, ln), "aco_get_timing")
        return [float(x) for x in ms], [int(x) for x in ln]

    def launch_count(self) -> int:
        v = C.c_uint64(0)
        _lib.check(self.lib.aco_last_launch_count(self.ctx, C.byref(v)), "aco_last_launch_count")
        return int(v.value)

    def variants(self) -> List[int]:
        """Construct-kernel variant codes of the last plan (aco_last_variants)."""
        cnt = C.c_uint32(0)
        _lib.check(self.lib.aco_last_variants(self.ctx, None, 0, C.byref(cnt)), "aco_last_variants")
        buf = (C.c_uint32 * max(1, cnt.value))()
        _lib.check(self.lib.aco_last_variants(self.ctx, buf, cnt.value, C.byref(cnt)), "aco_last_variants")
        return [int(buf[i]) for i in range(cnt.value)]

    def plan_variants(self, p: Params, flags: int = 0) -> List[int]:
        """Variants a run with these parameters would launch (a sizing call: plans, runs nothing)."""
        self.workspace_bytes(p, flags)
        return self.variants()

    # ---------------------------------------------------------------- results
    def results_raw(self, first: int = 0, count: Optional[int] = None, orders=None, cycles=None):
        """Fill caller-provided host arrays (for the e2e path); returns the Result array."""
        if count is None:
            count = self.count - first
        out = (_lib.Result * max(1, count))()
        _lib.check(self.lib.aco_get_results(self.ctx, first, count, out,
                                            None if orders is None else orders.ctypes.data,
                                            None if cycles is None else cycles.ctypes.data),
                   "aco_get_results")
        return out

    def results(self, first: int = 0, count: Optional[int] = None) -> List[dict]:
        if count is None:
            count = self.count - first
        off = self.batch.offsets
        tot = int(off[first + count] - off[first])
        orders = np.zeros(max(1, tot), np.uint32)
        cycles = np.zeros(max(1, tot), np.uint32)
        out = self.results_raw(first, count, orders, cycles)
        res = []
        for k in range(count):
            r = out[k]
            a, b = int(off[first + k] - off[first]), int(off[first + k + 1] - off[first])
            res.append(dict(
                n=r.n_insts, cost_rp=r.cost_rp, length=r.length, prp=list(r.prp),
                iters1=r.iters_run[0], iters2=r.iters_run[1], best1=r.best_cost[0], best2=r.best_cost[1],
                init1=r.init_cost[0], init2=r.init_cost[1], lb1=r.lb_cost, lblen=r.lb_len,
                target=list(r.target), trace_hash=int(r.trace_hash),
                policy=r.policy, heur_len=r.heur_len, ws_cost=r.ws_cost, ants_pruned=r.ants_pruned, heur_prp=list(r.heur_prp),
                order=orders[a:b].copy(), cycle=cycles[a:b].copy()))
        return res

    def dump_arrays(self):
        """(costs[2][I][count][A] u32, orders[2][I][A*sum_n] u16, cycles ...) as numpy."""
        torch.cuda.synchronize(self.device)
        costs, od, cy = self.dump
        c = costs.cpu().numpy().view(np.uint32)
        sl = self.params.ants * int(self.batch.offsets[-1])
        shape = (2, self.params.iterations, sl)
        o = od.cpu().numpy().view(np.uint16)[:2 * shape[1] * sl].reshape(shape) if od is not None else None
        y = cy.cpu().numpy().view(np.uint32)[:2 * shape[1] * sl].reshape(shape) if cy is not None else None
        return c, o, y

    def dump_ant(self, region: int, pass_: int, it: int, ant: int):
        c, o, y = self.dump_arrays()
        A = self.params.ants
        n = int(self.batch.sizes[region])
        base = A * int(self.batch.offsets[region]) + ant * n
        return (int(c[pass_ - 1, it, region, ant]), o[pass_ - 1, it, base:base + n].astype(np.uint32),
                y[pass_ - 1, it, base:base + n].copy())
