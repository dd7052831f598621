"""Where the lane-per-instruction ants stop paying: k regions of n instructions,
1,024 ants, 10 iterations x 2 passes; device ms per batch with ACO_LPI=0 (group
kernels) and ACO_LPI=2 (forced lane-per-instruction ants)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I  # noqa: E402
from paper_conf_cgo_shobakimhlmkrg24_b200.api import Scheduler  # noqa: E402


def timed(regs, p, mode):
    os.environ["ACO_LPI"] = mode
    s = Scheduler(I.GFX906, device=0)
    s.load(regs, list(range(len(regs))))
    s.run(p)
    torch.cuda.synchronize()
    ms = []
    for _ in range(3):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        s.run(p)
        b.record()
        torch.cuda.synchronize()
        ms.append(a.elapsed_time(b))
    return sorted(ms)[1]


print("| n | regions | ants total | group kernels ms | lane-per-instruction ms |")
print("|---|---|---|---|---|")
for n in (30, 60, 100, 128):
    for k in (1, 2, 4, 8, 16, 32):
        regs = [I.gen_region(n, I.region_seed(90 + n, i)) for i in range(k)]
        p = I.Params(ants=1024, iterations=10, seed=1)
        print(f"| {n} | {k} | {1024 * k} | {timed(regs, p, '0'):.2f} | {timed(regs, p, '2'):.2f} |", flush=True)
