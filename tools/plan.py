"""Print the launch plan (classes, shapes) of the C3 batch on the host: the
sizing-only path of aco_load_regions / aco_schedule_batch with ACO_DEBUG_PLAN."""
import ctypes as C
import os
import sys

os.environ["ACO_DEBUG_PLAN"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_cgo_shobakimhlmkrg24_b200 import _lib, build  # noqa: E402
from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I  # noqa: E402
from paper_conf_cgo_shobakimhlmkrg24_b200.api import HostBatch, machine_struct, params_struct  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 5000
build.build()
lib = _lib.load()
regs = I.gen_batch(n, base_seed=3)
m = machine_struct(I.GFX906)
ctx = C.c_void_p()
assert lib.aco_create(0, C.byref(m), C.byref(ctx)) == 0
b = HostBatch(regs, list(range(n)))
need = C.c_size_t(0)
assert lib.aco_load_regions(ctx, b.descs, n, None, 0, C.byref(need), None) == 0
p = params_struct(I.Params(ants=1024, iterations=10, seed=3))
ws = C.c_size_t(0)
print("status", lib.aco_schedule_batch(ctx, C.byref(p), None, 0, C.byref(ws), None), "arena", need.value, "ws", ws.value)
