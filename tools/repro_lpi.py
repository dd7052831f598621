"""Repro of tests/test_gpu_lpi.py::test_lpi_every_ant (forced lane-per-instruction ants, dump mode)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ.setdefault("ACO_LPI", "2")
import torch  # noqa: E402

from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I  # noqa: E402
from paper_conf_cgo_shobakimhlmkrg24_b200.api import Scheduler  # noqa: E402

mode = int(os.environ.get("MODE", "0"))
SIZES = [1, 2, 7, 31, 32, 33, 50, 63, 64, 65, 97, 100, 127, 128]
sel = os.environ.get("SIZES")
idx = [int(x) for x in sel.split(",")] if sel else range(len(SIZES))
regs = [I.gen_region(SIZES[i], 7100 + 13 * i + mode, "mixed" if (i + mode) % 2 else "unit") for i in idx]
ids = [200 + 7 * i for i in idx]
p = I.Params(ants=70, iterations=3, seed=40 + mode, cost_mode=mode, stall_mod=2)
s = Scheduler(I.GFX906, device=0)
s.load(regs, ids).run(p, no_prune=os.environ.get("DUMP", "1") == "1", dump=os.environ.get("DUMP", "1") == "1")
torch.cuda.synchronize()
print("ok", [r["length"] for r in s.results()])
