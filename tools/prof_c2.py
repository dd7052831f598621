"""One C2 run (n = 100 region of bench --workload c2, 1,024 ants) for ncu:
PROF_ITERS iterations per pass (default 2), PROF_PASSES (default 3)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I  # noqa: E402
from paper_conf_cgo_shobakimhlmkrg24_b200.api import Scheduler  # noqa: E402

iters = int(os.environ.get("PROF_ITERS", "2"))
passes = int(os.environ.get("PROF_PASSES", "3"))
s = Scheduler(I.GFX906, device=0)
s.load([I.gen_region(100, I.region_seed(2, 0))], [0])
p = I.Params(ants=1024, iterations=iters, seed=2, passes=passes)
s.run(p)
torch.cuda.synchronize()
if os.environ.get("PROF_TIME"):
    s.run(p, timing=True)
    ms, ln = s.timing()
    print("timing", passes, iters, ms, ln)
print("done", s.results()[0]["length"], s.launch_count())
