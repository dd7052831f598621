import sys, os, faulthandler
sys.path.insert(0, os.getcwd())
faulthandler.dump_traceback_later(50, exit=True)
import torch
from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I
from paper_conf_cgo_shobakimhlmkrg24_b200.api import Scheduler
regs = [I.fix10a(), I.gen_region(45, 1801), I.gen_region(130, 1802, "unit"), I.gen_region(230, 1803)]
for k, r in enumerate(regs):
    for ants in (64, 100):
        p = I.Params(ants=ants, iterations=1, seed=41, cost_mode=0, rl_limit=1, passes=1)
        s = Scheduler(I.GFX906, device=0)
        s.load([r], [81 + k]).run(p)
        torch.cuda.synchronize()
        print("ok region", k, "ants", ants, s.results()[0]["cost_rp"], flush=True)
