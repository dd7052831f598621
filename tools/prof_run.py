"""One aco_schedule_batch for profiling under ncu (no timing is reported).
PROF_N=<n>: PROF_REGIONS regions all of n instructions; else the C3 batch."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I  # noqa: E402
from paper_conf_cgo_shobakimhlmkrg24_b200.api import Scheduler  # noqa: E402

n = int(os.environ.get("PROF_REGIONS", "5000"))
iters = int(os.environ.get("PROF_ITERS", "10"))
size = int(os.environ.get("PROF_N", "0"))
if size:
    regs = [I.gen_region(size, I.region_seed(77, i)) for i in range(n)]
else:
    regs = I.gen_batch(n, base_seed=3)
s = Scheduler(I.GFX906, device=0)
s.load(regs, list(range(n)))
s.run(I.Params(ants=1024, iterations=iters, seed=3))
torch.cuda.synchronize()
r = s.results()
print("done", len(r), s.launch_count())
