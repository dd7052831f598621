"""Table-6 analogue: the fraction of
wavefronts (ant groups of 64) allowed to take optional stalls, 0 / 25 / 50 /
75 % (stall_num 0..3 of stall_mod 4, R44), on the config-3 regions with
n >= 100: ACO time (device, both passes) and the schedule-length improvement
relative to 0 % (mean over regions and maximum), as the paper reports them.

    python tools/table6.py > profiles/r02_table6.md
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I  # noqa: E402
from paper_conf_cgo_shobakimhlmkrg24_b200.api import Scheduler  # noqa: E402

sizes = I.c3_sizes(5000, 3)
ids = [i for i in range(5000) if sizes[i] >= 100]
regs = I.gen_regions(ids, sizes, 3)
rows = {}
for num in (0, 1, 2, 3):
    p = I.Params(ants=1024, iterations=10, seed=3, stall_num=num)
    s = Scheduler(I.GFX906, device=0)
    s.load(regs, ids)
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
    s.run(p, timing=True)
    cms = s.timing()[0][0]
    res = s.results()
    rows[num] = (float(np.median(ms)), cms, np.array([r["length"] for r in res], float),
                 np.array([r["init2"] for r in res], float), np.array([r["cost_rp"] for r in res]))
t0, _, l0, i0, _ = rows[0]
print(f"Config-3 regions with n >= 100: {len(regs)} (of 5,000), A = 1024, I = 10 per pass, APRP_SUM, stop rules off.\n")
print("| % groups inserting optional stalls | 0 % | 25 % | 50 % | 75 % |")
print("|---|---|---|---|---|")
print("| ACO time per batch (ms) | " + " | ".join(f"{rows[k][0]:.1f}" for k in range(4)) + " |")
print("| % increase in ACO time | - | " + " | ".join(f"{100 * (rows[k][0] / t0 - 1):.2f} %" for k in (1, 2, 3)) + " |")
print("| mean % improvement in schedule length | - | " + " | ".join(
    f"{100 * np.mean((l0 - rows[k][2]) / l0):.2f} %" for k in (1, 2, 3)) + " |")
print("| max % improvement in schedule length | - | " + " | ".join(
    f"{100 * np.max((l0 - rows[k][2]) / l0):.2f} %" for k in (1, 2, 3)) + " |")
print("| regions whose pass-2 result is its input schedule (no improvement) | " + " | ".join(
    f"{int(np.sum(rows[k][2] == rows[k][3]))}" for k in range(4)) + " |")
print("\nPaper (Radeon VII, rocPRIM regions n >= 100, Table 6): +8.65 / +12.30 / +20.28 % ACO time, "
      "0.27 / 0.30 / 0.95 % mean and 15.75 / 15.75 / 23.58 % max length improvement.")
