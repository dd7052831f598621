"""Config 5 as SURVEY 8(d) defines it: for every n in {10 .. 4000}, the six
regions {unit, mixed} x seeds {0, 1, 2} (A = 1024, I = 10, 5 for n >= 2000),
GPU throughput, construct roofline fraction and GPU / oracle ratio per n.

    python tools/c5_sweep.py [--steps 3] > profiles/r02_c5_sweep.md

GPU: aco_schedule_batch over the six regions, CUDA events (device time per
batch, median of --steps; construct time from a run with per-phase events).
Oracle: the sequential CPU oracle on one region per n with a bounded sample
(32 ants x 2 iterations per pass), single host thread: ant-schedules/s and
the SURVEY 8(d) algorithmic bytes per ant-step from its instrumentation.
"""
import argparse
import dataclasses
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
from oracle import pyoracle as O  # noqa: E402
from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I  # noqa: E402
from paper_conf_cgo_shobakimhlmkrg24_b200.api import Scheduler  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--steps", type=int, default=3)
ap.add_argument("--sizes", default=",".join(str(n) for n in I.C5_SIZES))
args = ap.parse_args()
sizes = [int(x) for x in args.sizes.split(",")]
grid = I.c5_grid()
mhz = 1965.0
peak = 148 * 128 * mhz * 1e6 / 1e9
print("| n | regions | I | GPU ms / batch | ant-schedules/s | ant-steps/s | construct ms | B / ant-step (oracle) "
      "| smem roofline frac | oracle ant-schedules/s (1 thread) | GPU / oracle (1 thread) | GPU / oracle (16 threads, ideal) | parity |")
print("|---|---|---|---|---|---|---|---|---|---|---|---|---|")
for n in sizes:
    sel = [g for g in grid if g[1] == n]
    regs = [I.c5_region(g[0], g[1], g[2]) for g in sel]
    ids = [g[0] for g in sel]
    p = I.Params(ants=1024, iterations=5 if n >= 2000 else 10, seed=5)
    s = Scheduler(I.GFX906, device=0)
    s.load(regs, ids)
    for _ in range(3):
        s.run(p)
    torch.cuda.synchronize()
    ms = []
    for _ in range(args.steps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        s.run(p)
        b.record()
        torch.cuda.synchronize()
        ms.append(a.elapsed_time(b))
    step = float(np.median(ms))
    s.run(p, timing=True)
    cms = s.timing()[0][0]
    res = s.results()
    scheds = sum(p.ants * (r["iters1"] + r["iters2"]) for r in res)
    ant_steps = sum(p.ants * r["n"] * (r["iters1"] + r["iters2"]) for r in res)
    # oracle: one region (mixed, seed 0), bounded sample, one thread; parity of the sample
    ps = dataclasses.replace(p, ants=32, iterations=2)
    k = [i for i, g in enumerate(sel) if g[2] == "mixed"][0]
    t0 = time.perf_counter()
    ores, stats, dt, osched = bench.run_oracle([regs[k]], [ids[k]], ps, I.GFX906, threads=1)
    bpas = bench.bytes_per_ant_step(stats)
    orate = osched / dt
    s2 = Scheduler(I.GFX906, device=0)
    s2.load([regs[k]], [ids[k]]).run(ps)
    par = "ok" if not bench.parity_compare(bench.gpu_digest(s2.results()[0]), ores[0]) else "MISMATCH"
    rate = scheds / (step / 1000.0)
    frac = bpas * ant_steps / (cms / 1000.0) / 1e9 / peak
    print(f"| {n} | {len(regs)} | {p.iterations} | {step:.2f} | {rate:.3e} | {ant_steps / (step / 1000.0):.3e} | {cms:.2f} | "
          f"{bpas:.0f} | {frac:.4f} | {orate:.0f} | {rate / orate:.0f} | {rate / (16 * orate):.0f} | {par} |", flush=True)
