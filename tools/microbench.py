"""Per-size construct throughput: batches of equal-size regions, pass 1 alone
and both passes (pass 2 = difference), CUDA-event construct time from the
library.  Prints ns per ant-step per pass for each n (lower is better)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I  # noqa: E402
from paper_conf_cgo_shobakimhlmkrg24_b200.api import Scheduler  # noqa: E402

sizes = [int(x) for x in os.environ.get("MB_SIZES", "30,60,120,250,450").split(",")]
ants = int(os.environ.get("MB_ANTS", "1024"))
iters = int(os.environ.get("MB_ITERS", "4"))
tot = {}
for n in sizes:
    count = max(int(os.environ.get("MB_MIN_REGIONS", "160")), int(6e6 / (n * n)))
    regs = [I.gen_region(n, I.region_seed(77, i)) for i in range(count)]
    out = []
    for passes in (1, 3):
        s = Scheduler(I.GFX906, device=0)
        s.load(regs, list(range(count)))
        p = I.Params(ants=ants, iterations=iters, seed=5, passes=passes)
        s.run(p)
        torch.cuda.synchronize()
        best = None
        for _ in range(3):
            s.run(p, timing=True)
            ms, _ = s.timing()
            best = ms[0] if best is None else min(best, ms[0])
        out.append(best)
    steps = ants * iters * n * count
    p1 = out[0] * 1e6 / steps
    p2 = (out[1] - out[0]) * 1e6 / steps
    tot[n] = (p1, p2)
    print(f"n {n:4d} regions {count:5d}: pass1 {p1:7.4f} ns/ant-step  pass2 {p2:7.4f} ns/ant-step", flush=True)
