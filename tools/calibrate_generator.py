"""Generator calibration: the fraction of config-3 regions with
n >= 50 whose greedy pass-1 heuristic schedule has VGPR PRP above 24 (the
first APRP band), for a grid of the generator's knobs (geometric operand
recency, VGPR live-ins).  Uses the oracle's greedy heuristic (R28).

    PYTHONPATH=. python tools/calibrate_generator.py [regions]
"""
import itertools
import sys

import numpy as np

from oracle import pyoracle as O
from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I

count = int(sys.argv[1]) if len(sys.argv) > 1 else 800
p = I.Params()
sizes = I.c3_sizes(count, 3)
for rec, vl in itertools.product([0.3, 0.2, 0.15, 0.1], [2, 8]):
    v, ns = [], []
    for i in range(count):
        n = int(sizes[i])
        if n < 50:
            continue
        r = I.gen_region(n, I.region_seed(3, i), recency=rec, v_livein=vl)
        v.append(O.greedy_pass1(r, I.GFX906, p)[1][0])
        ns.append(n)
    v, ns = np.array(v), np.array(ns)
    by = [(lo, round(float((v[(ns >= lo) & (ns < hi)] > 24).mean()), 2)) for lo, hi in ((50, 100), (100, 200), (200, 501))]
    print(f"recency {rec} v_livein {vl}: frac VGPR PRP > 24 = {(v > 24).mean():.2f}, median {np.median(v)}, by size {by}")
