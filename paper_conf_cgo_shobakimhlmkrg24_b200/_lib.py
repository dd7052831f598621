"""ctypes binding of include/aco.h (libaco_b200.so).  Argument marshalling only.

The product path has no CPU fallback: if the CUDA library is missing or fails
to load, importing the binding raises.
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(HERE, "libaco_b200.so")
if os.environ.get("ACO_LIB_VARIANT"):  # A/B builds of the same sources (tools/, never the default)
    LIB_PATH = os.path.join(HERE, f"libaco_b200_{os.environ['ACO_LIB_VARIANT']}.so")

ACO_OK = 0
ACO_E_WORKSPACE = -6
ACO_E_STATE = -8
ACO_FLAG_NO_PRUNE = 1
ACO_FLAG_DUMP = 2
ACO_FLAG_TIMING = 4
INVALID = 0xFFFFFFFF

EXPORTS = [
    "aco_create", "aco_load_regions", "aco_schedule_batch", "aco_get_results", "aco_set_dump",
    "aco_last_launch_count", "aco_last_variants", "aco_get_timing", "aco_status_string", "aco_destroy",
    "aco_colony_begin", "aco_colony_construct", "aco_colony_finalize", "aco_colony_end",
]


class RegionDesc(C.Structure):
    _fields_ = [
        ("region_id", C.c_uint32), ("n_insts", C.c_uint32), ("n_edges", C.c_uint32),
        ("n_regs", C.c_uint32),
        ("edge_src", C.c_void_p), ("edge_dst", C.c_void_p), ("edge_lat", C.c_void_p),
        ("reg_class", C.c_void_p), ("reg_flags", C.c_void_p),
        ("def_ptr", C.c_void_p), ("def_reg", C.c_void_p),
        ("use_ptr", C.c_void_p), ("use_reg", C.c_void_p), ("inst_type", C.c_void_p),
    ]


class Machine(C.Structure):
    _fields_ = [
        ("n_classes", C.c_uint32), ("occ_max", C.c_uint32),
        ("step_count", C.c_uint32 * 4), ("step_max", (C.c_uint32 * 16) * 4),
        ("perp_limit", C.c_uint32 * 4),
        ("issue_width", C.c_uint32), ("n_types", C.c_uint32), ("type_slots", C.c_uint32 * 4),
    ]


class Params(C.Structure):
    _fields_ = [
        ("ants", C.c_uint32), ("iterations", C.c_uint32), ("seed", C.c_uint64),
        ("pass_", C.c_uint32), ("cost_mode", C.c_uint32), ("q0_t", C.c_uint64),
        ("group_size", C.c_uint32), ("stall_mod", C.c_uint32), ("stall_rem", C.c_uint32),
        ("tau0", C.c_uint32), ("rho_q16", C.c_uint32), ("delta", C.c_uint32),
        ("tau_min", C.c_uint32), ("tau_max", C.c_uint32),
        ("stop_no_improve", C.c_uint32), ("stop_at_lb", C.c_uint32), ("flags", C.c_uint32),
        ("pass2_gap", C.c_uint32), ("revert_occ", C.c_uint32), ("revert_len", C.c_uint32),
        ("ws_weight", C.c_uint32), ("heur_mix", C.c_uint32), ("stall_num", C.c_uint32),
        ("rl_limit", C.c_uint32),
    ]


class Result(C.Structure):
    _fields_ = [
        ("n_insts", C.c_uint32), ("cost_rp", C.c_uint32), ("length", C.c_uint32),
        ("prp", C.c_uint32 * 4), ("iters_run", C.c_uint32 * 2), ("best_cost", C.c_uint32 * 2),
        ("init_cost", C.c_uint32 * 2), ("lb_cost", C.c_uint32), ("lb_len", C.c_uint32),
        ("target", C.c_uint32 * 4), ("trace_hash", C.c_uint64),
        ("policy", C.c_uint32), ("heur_len", C.c_uint32), ("ws_cost", C.c_uint32), ("ants_pruned", C.c_uint32),
        ("heur_prp", C.c_uint32 * 4),
    ]


_lib = None


def load(path: str = LIB_PATH):
    """Load libaco_b200.so; raise (no fallback) if it is missing."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(path):
        raise RuntimeError(
            f"{path} is missing: build it with `python -m paper_conf_cgo_shobakimhlmkrg24_b200.build` "
            "(there is no CPU fallback)")
    L = C.CDLL(path)
    vp, u32, u64, sz = C.c_void_p, C.c_uint32, C.c_uint64, C.c_size_t
    L.aco_create.argtypes = [C.c_int, vp, C.POINTER(vp)]
    L.aco_load_regions.argtypes = [vp, vp, u32, vp, sz, C.POINTER(sz), vp]
    L.aco_schedule_batch.argtypes = [vp, vp, vp, sz, C.POINTER(sz), vp]
    L.aco_get_results.argtypes = [vp, u32, u32, vp, vp, vp]
    L.aco_set_dump.argtypes = [vp, vp, u64, vp, u64, vp, u64]
    L.aco_last_launch_count.argtypes = [vp, C.POINTER(C.c_uint64)]
    L.aco_last_variants.argtypes = [vp, vp, u32, C.POINTER(u32)]
    L.aco_get_timing.argtypes = [vp, vp, vp]
    L.aco_colony_begin.argtypes = [vp, vp, u32, vp, sz, C.POINTER(sz), vp]
    L.aco_colony_construct.argtypes = [vp, u32, u32, vp, vp]
    L.aco_colony_finalize.argtypes = [vp, u32, u32, vp, vp]
    L.aco_colony_end.argtypes = [vp, vp]
    L.aco_status_string.argtypes = [C.c_int32]
    L.aco_status_string.restype = C.c_char_p
    L.aco_destroy.argtypes = [vp]
    L.aco_destroy.restype = None
    for f in ("aco_create", "aco_load_regions", "aco_schedule_batch", "aco_get_results",
              "aco_set_dump", "aco_last_launch_count", "aco_last_variants", "aco_get_timing", "aco_colony_begin",
              "aco_colony_construct", "aco_colony_finalize", "aco_colony_end"):
        getattr(L, f).restype = C.c_int32
    _lib = L
    return L


class AcoError(RuntimeError):
    def __init__(self, status: int, where: str):
        msg = load().aco_status_string(status).decode()
        super().__init__(f"{where}: {msg} ({status})")
        self.status = status


def check(status: int, where: str):
    if status != ACO_OK:
        raise AcoError(status, where)
