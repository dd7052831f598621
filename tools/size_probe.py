"""Construct time split (pass 1 / pass 2) for a batch of equal huge regions:
PROBE_N (default 2000), PROBE_ANTS (8192), PROBE_REGIONS (1), PROBE_ITERS (2)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I  # noqa: E402
from paper_conf_cgo_shobakimhlmkrg24_b200.api import Scheduler  # noqa: E402

n = int(os.environ.get("PROBE_N", "2000"))
ants = int(os.environ.get("PROBE_ANTS", "8192"))
count = int(os.environ.get("PROBE_REGIONS", "1"))
iters = int(os.environ.get("PROBE_ITERS", "2"))
regs = [I.gen_region(n, I.region_seed(4, i)) for i in range(count)]
out = {}
for passes in (1, 3):
    s = Scheduler(I.GFX906, device=0)
    s.load(regs, list(range(count)))
    p = I.Params(ants=ants, iterations=iters, seed=4, passes=passes)
    s.run(p)
    torch.cuda.synchronize()
    s.run(p, timing=True)
    ms, ln = s.timing()
    out[passes] = ms
print(f"n {n} ants {ants} regions {count} iters {iters}: pass1 construct {out[1][0]:.1f} ms, "
      f"pass2 construct {out[3][0] - out[1][0]:.1f} ms, finalize(both) {out[3][1]:.1f} ms", flush=True)
