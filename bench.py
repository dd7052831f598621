#!/usr/bin/env python
"""Benchmark: region-batch ACO throughput (ant-schedules/s) on 1..N B200s.

One STEP = one full two-pass ACO run (aco_schedule_batch: every pass and
iteration of every region: construction, argmin + winner copy, pheromone
update, epilogue) over one batch of synthetic regions.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload c3|c2|c1|c4|c5]
                  [--scaling strong|weak] [--parity sample|all|off]
                  [--machine gfx906|dual] [--passes 3|4 --ws-weight W] [--policy off|paper]
                  [--heur-mix 0|1] [--stall-num k] [--rl-limit 0|1|2]
  python bench.py --impl reference ...     # the CPU oracle on a bounded sample

Workloads (BASELINE.json configs): c1 FIX10-A; c2 one n = 100 region; c3
(default, the metric's config) the 5,000 rocPRIM-shaped regions, LPT-
partitioned across the N ranks (strong scaling; --scaling weak gives every
rank its own 5,000); c4 one n = 2,000 region with 8,192 ants x 20 iterations
per pass, ONE shared colony across the N ranks (one int64 MIN allreduce per
iteration over NCCL); c5 the SURVEY 8(d) sweep n in {10..4000} x {unit,
mixed} x 3 seeds (I = 10, 5 for n >= 2,000), LPT-partitioned.

Multi-GPU: launched by torchrun, one process per GPU.  Regions shard with no
data-path collective (global region ids key the Philox streams, so a region's
result does not depend on the rank running it); NCCL carries only the
barrier, the max-over-ranks time and the result gather for the parity check.
"""
from __future__ import annotations

import argparse
import dataclasses
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_cgo_shobakimhlmkrg24_b200 import inputs as I  # noqa: E402
from paper_conf_cgo_shobakimhlmkrg24_b200 import sharding  # noqa: E402

METRIC = "ant-schedules/s"
C3_REGIONS = 5000
# result fields compared bit for bit by the parity check (oracle vs GPU)
PARITY_FIELDS = ("order", "cycle", "prp", "length", "cost_rp", "iters1", "iters2", "best1", "best2",
                 "init1", "init2", "lb1", "lblen", "trace_hash")


def parse(argv=None):
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="c3", choices=["c3", "c2", "c1", "c4", "c5"])
    ap.add_argument("--scaling", default="strong", choices=["strong", "weak"],
                    help="c3/c5 at N > 1: partition the same batch (strong) or one batch per rank (weak)")
    ap.add_argument("--machine", default="gfx906", choices=["gfx906", "dual"])
    ap.add_argument("--passes", type=int, default=3, choices=[1, 2, 3, 4])
    ap.add_argument("--ws-weight", type=int, default=4)
    ap.add_argument("--policy", default="off", choices=["off", "paper"])
    ap.add_argument("--heur-mix", type=int, default=0)
    ap.add_argument("--stall-num", type=int, default=1)
    ap.add_argument("--rl-limit", type=int, default=0, help="pass-1 ready-list size limit (R45): 1 min, 2 mid")
    ap.add_argument("--regions", type=int, default=C3_REGIONS, help="regions of the c3 batch")
    ap.add_argument("--ants", type=int, default=None)
    ap.add_argument("--iterations", type=int, default=None)
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-sample", type=int, default=160, help="regions in the oracle sample")
    ap.add_argument("--parity", default="sample", choices=["sample", "all", "off"],
                    help="compare GPU results with the oracle on the cpu_baseline sample, on every region, or not")
    ap.add_argument("--parity-log", default=None, help="write the per-region parity log here (--parity all)")
    return ap.parse_args(argv)


# ---------------------------------------------------------------- workloads
@dataclasses.dataclass
class Batch:
    regs: list
    ids: list
    p: I.Params


def base_params(args, p):
    p = dataclasses.replace(p, passes=args.passes, ws_weight=args.ws_weight if args.passes == 4 else 0,
                            heur_mix=args.heur_mix, stall_num=args.stall_num, rl_limit=args.rl_limit)
    if args.policy == "paper":
        p = I.paper_policy(p)
    return p


def workload(args, rank: int, world: int, gen: bool = True):
    """(batches for this rank, config dict, scaling) -- every batch is one
    aco_schedule_batch call per step (c5: one per iteration count).
    gen=False: parameters only (no regions generated)."""
    strong = args.scaling == "strong"
    if args.workload == "c3":
        R = args.regions
        p = base_params(args, I.Params(ants=args.ants or 1024, iterations=args.iterations or 10, seed=3))
        if strong or world == 1:
            sizes = I.c3_sizes(R, 3)
            ids = sharding.lpt_partition(sizes, world, p.ants, p.iterations)[rank]
            regs = I.gen_regions(ids, sizes, 3) if gen else []
            cfg = {"workload": "c3-rocprim-shaped-batch", "regions": R, "regions_this_rank_0": None}
        else:
            regs = I.gen_batch(R, base_seed=3, first_id=rank * R) if gen else []
            ids = list(range(rank * R, (rank + 1) * R))
            cfg = {"workload": "c3-rocprim-shaped-batch", "regions_per_gpu": R}
        cfg.update({"sizes": "20-500 (Table 3.a buckets)", "latency": "mixed"})
        batches = [Batch(regs, list(ids), p)]
        scaling = "strong" if strong else "weak"
    elif args.workload == "c5":
        grid = I.c5_grid()
        p10 = base_params(args, I.Params(ants=args.ants or 1024, iterations=args.iterations or 10, seed=5))
        p5 = dataclasses.replace(p10, iterations=args.iterations or 5)
        batches = []
        for big, p in ((False, p10), (True, p5)):
            sel = [g for g in grid if (g[1] >= 2000) == big]
            sizes = {g[0]: g[1] for g in sel}
            gids = [g[0] for g in sel]
            if world > 1:
                part = sharding.lpt_partition([sizes[i] for i in gids], world, p.ants, p.iterations)[rank]
                gids = [gids[k] for k in part]
            regs = [I.c5_region(g[0], g[1], g[2]) for g in sel if g[0] in set(gids)] if gen else []
            batches.append(Batch(regs, [g[0] for g in sel if g[0] in set(gids)], p))
        cfg = {"workload": "c5-suite-sweep", "regions": len(grid), "sizes": list(I.C5_SIZES),
               "latency": list(I.C5_PROFILES), "seeds": len(I.C5_SEEDS),
               "iterations_per_pass": "10 (n < 2000), 5 (n >= 2000)"}
        scaling = "strong"
    elif args.workload == "c4":
        total = args.ants or 8192
        p = base_params(args, I.Params(ants=total // world, iterations=args.iterations or 20, seed=4))
        batches = [Batch([I.gen_region(2000, I.region_seed(4, 0))], [0], p)]
        cfg = {"workload": "c4-shared-colony-n2000", "regions": 1, "ants_total": total,
               "ants_per_gpu": total // world, "latency": "mixed"}
        scaling = "strong"
    elif args.workload == "c2":
        p = base_params(args, I.Params(ants=args.ants or 1024, iterations=args.iterations or 100, seed=2))
        batches = [Batch([I.gen_region(100, I.region_seed(2, 0))], [rank], p)]
        cfg = {"workload": "c2-single-region-n100", "regions_per_gpu": 1, "latency": "mixed",
               "multi_gpu": "replicas only (one region does not shard)"}
        scaling = "weak"
    else:
        p = base_params(args, I.Params(ants=args.ants or 64, iterations=args.iterations or 20, seed=0, cost_mode=0))
        batches = [Batch([I.fix10a()], [rank], p)]
        cfg = {"workload": "c1-fix10a", "regions_per_gpu": 1,
               "multi_gpu": "replicas only (one region does not shard)"}
        scaling = "weak"
    p = batches[0].p
    passes = {1: "RP", 2: "ILP", 3: "RP+ILP", 4: f"weighted single pass (W={p.ws_weight})"}[p.passes]
    cfg.pop("regions_this_rank_0", None)
    cfg.update({"ants": p.ants if args.workload != "c4" else cfg["ants_total"],
                "iterations_per_pass": cfg.get("iterations_per_pass", p.iterations), "passes": passes,
                "cost": ["PRP_SUM", "APRP_SUM", "OCC", "PERP"][p.cost_mode],
                "stop_rules": "paper policy (LB, size classes, gap 21, revert 3/63)" if args.policy == "paper"
                else "off (fixed work)",
                "machine": "gfx906 single issue" if args.machine == "gfx906" else "dual issue (VALU/SALU/MEM)"})
    if args.heur_mix:
        cfg["heur_mix"] = 1
    if args.stall_num != 1:
        cfg["stall_groups"] = f"{args.stall_num}/{p.stall_mod}"
    if args.rl_limit:
        cfg["ready_list_limit"] = {1: "group min", 2: "group min/max midpoint"}[args.rl_limit]
    return batches, cfg, scaling


def machine_of(args):
    return I.DUAL_ISSUE if args.machine == "dual" else I.GFX906


# ---------------------------------------------------------------- helpers
class ClockSampler:
    """nvidia-smi clocks + throttle reasons during the timed region."""

    def __init__(self, index: int):
        self.index = index
        self.samples = []
        self._stop = threading.Event()
        self._t = None

    def _run(self):
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}",
                                  "--format=csv,noheader,nounits", "-lms", "200"],
                                 stdout=subprocess.PIPE, text=True)
        except Exception:
            return
        while not self._stop.is_set():
            line = p.stdout.readline()
            if not line:
                break
            self.samples.append([x.strip() for x in line.split(",")])
        p.terminate()

    def start(self):
        self._t = threading.Thread(target=self._run, daemon=True)
        self._t.start()
        time.sleep(0.3)

    def stop(self):
        time.sleep(0.25)
        self._stop.set()
        if self._t:
            self._t.join(timeout=3)
        sm = [float(s[0]) for s in self.samples if s and s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if len(s) > 1 and s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4)
                          if len(s) > 3 + i and s[3 + i].lower() == "active"})
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples)}


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f)
    except Exception:
        return {}


def host_cpu():
    """CPU model and thread count of the host (lscpu)."""
    model = None
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            if line.lower().startswith("model name"):
                model = line.split(":", 1)[1].strip()
    except Exception:
        pass
    return {"model": model, "threads": os.cpu_count()}


def build_fingerprint():
    """sha256 of the library's sources + nvcc flags (matches a profile to its build)."""
    from paper_conf_cgo_shobakimhlmkrg24_b200 import build as B
    return B.source_fingerprint()


def ncu_evidence(workload: str):
    """DRAM traffic and issue-slot figures of the construct launches from the
    committed ncu --set full capture (profiles/r03_traffic.json, else the
    round-2 one) -- used only when that capture profiled this very build
    (same source fingerprint)."""
    tj = None
    for name in ("r03_traffic.json", "r02_traffic.json"):
        try:
            with open(os.path.join(ROOT, "profiles", name)) as f:
                tj = json.load(f)
            break
        except Exception:
            continue
    if tj is None:
        return None, None, "no committed capture"
    if workload != "c3":
        return None, None, "capture is of the c3 batch"
    sha = build_fingerprint()
    if tj.get("build_fingerprint") != sha:
        return None, None, f"committed capture is of another build ({str(tj.get('build_fingerprint'))[:12]} vs {sha[:12]})"
    issue = {"util_pct": tj.get("issue_util_pct"), "warps_active_pct": tj.get("warps_active_pct"),
             "source": tj.get("issue_source")}
    return tj.get("dram_bytes_per_launch"), issue, tj.get("source")


def bytes_per_ant_step(stats: np.ndarray) -> float:
    """SURVEY 8(d) algorithmic bytes per ant-step from oracle instrumentation:
    8.5|F| + 2|R| + 12 deg + 6 |Use| + 2 |Def| + 16 per placed instruction."""
    from oracle.pyoracle import ORS
    s = stats.sum(axis=0).astype(np.float64)
    pl = s[ORS["placements"]]
    b = (8.5 * s[ORS["sum_F"]] + 2.0 * s[ORS["sum_R"]] + 12.0 * s[ORS["sum_deg"]] + 6.0 * s[ORS["sum_use"]]
         + 2.0 * s[ORS["sum_def"]] + 16.0 * pl)
    return float(b / max(pl, 1.0))


def cpu_sample_params(args, p):
    """Bounded oracle sample: fewer ants / iterations where the full workload
    would take minutes on the host (c4: one n = 2,000 region; c5: regions up
    to 4,000 instructions); the per-ant-schedule cost is what is measured."""
    if args.workload == "c4":
        return dataclasses.replace(p, ants=64, iterations=2), "64 ants x 2 iterations per pass of the n = 2,000 region"
    if args.workload == "c5":
        return dataclasses.replace(p, ants=32, iterations=2), "32 ants x 2 iterations per pass"
    return p, "full A x I x passes"


def stratified_pick(regs, sample: int):
    """Indices of a size-stratified sample, largest region first (the oracle's
    thread pool takes regions in the order given: largest first keeps one big
    region from running alone at the end; per-region results do not depend on it)."""
    k = min(sample, len(regs))
    order = np.argsort([r.n_insts for r in regs], kind="stable")
    pick = set(int(order[int(i)]) for i in np.linspace(0, len(regs) - 1, k))
    return sorted(pick, key=lambda i: (-regs[i].n_insts, i))


def deal_over_steps(full, steps: int):
    """Round-robin a sample over the steps (a sample smaller than the step
    count is reused whole by the steps it does not reach)."""
    return [full[s::steps] or full for s in range(steps)]


def run_oracle(regs, ids, p, machine, threads=None):
    """The oracle as it stands over regions on the host's threads: (per-region
    result dicts, stats, seconds, ant-schedules)."""
    from oracle import pyoracle as O
    threads = threads or os.cpu_count() or 1
    t0 = time.perf_counter()
    order, cyc, stats, off = O.schedule_many(regs, ids, machine, p, n_threads=threads)
    dt = time.perf_counter() - t0
    res = []
    for k in range(len(regs)):
        d = {n: int(stats[k, i]) for n, i in O.ORS.items()}
        d["prp"] = [d["prp0"], d["prp1"], d["prp2"], d["prp3"]]
        a, b = int(off[k]), int(off[k + 1])
        d["order"] = [int(x) for x in order[a:b]]
        d["cycle"] = [int(x) for x in cyc[a:b]]
        res.append(d)
    return res, stats, dt, float(stats[:, O.ORS["ant_scheds"]].sum())


def cpu_baseline(regs, ids, p, sample: int, machine=I.GFX906, note="full A x I x passes", pick=None):
    """The oracle as it stands on a bounded, stratified sample of the same
    workload: (baseline dict, stats, picked indices, oracle results, seconds,
    ant-schedules)."""
    if pick is None:
        pick = stratified_pick(regs, sample)
    sub = [regs[i] for i in pick]
    sid = [ids[i] for i in pick]
    threads = os.cpu_count() or 1
    res, stats, dt, scheds = run_oracle(sub, sid, p, machine, threads)
    base = {"value": scheds / dt, "unit": METRIC, "cores": min(threads, len(sub)), "kind": "oracle",
            "host": host_cpu(),
            "sample": f"{len(sub)} of {len(regs)} regions (stratified by size, largest first), {note}, "
                      f"{scheds:.0f} ant-schedules in {dt:.1f} s on {min(threads, len(sub))} host threads"}
    return base, stats, pick, res, dt, scheds


def gpu_digest(r: dict) -> dict:
    """The fields of a GPU result compared with the oracle (plain Python types)."""
    return {"order": [int(x) for x in r["order"]], "cycle": [int(x) for x in r["cycle"]],
            "prp": [int(x) for x in r["prp"]], "length": r["length"], "cost_rp": r["cost_rp"],
            "iters1": r["iters1"], "iters2": r["iters2"], "best1": r["best1"], "best2": r["best2"],
            "init1": r["init1"], "init2": r["init2"], "lb1": r["lb1"], "lblen": r["lblen"],
            "trace_hash": r["trace_hash"]}


# APRP bands of the gfx906 VGPR table (R17): upper bound of each band
VGPR_BANDS = (24, 28, 32, 36, 40, 48, 64, 84, 128, 256)


def schedule_quality(res: dict) -> dict:
    """Histogram of the heuristic (greedy, R28) and final ACO VGPR PRP over the
    regions' occupancy bands, plus how many regions the RP pass improved
    (final cost below the heuristic cost) and the mean / max pass-2 length
    gain over its input schedule -- the RP pass visibly doing work."""
    def band(x):
        for i, b in enumerate(VGPR_BANDS):
            if x <= b:
                return i
        return len(VGPR_BANDS)
    h = [0] * (len(VGPR_BANDS) + 1)
    a = [0] * (len(VGPR_BANDS) + 1)
    for r in res.values():
        h[band(r["heur_prp"][0])] += 1
        a[band(r["prp"][0])] += 1
    imp = sum(1 for r in res.values() if r["best1"] < r["init1"])
    gains = [(r["init2"] - r["length"]) / r["init2"] for r in res.values() if r["init2"]]
    return {"vgpr_band_upper": list(VGPR_BANDS) + ["more"], "regions_by_heuristic_vgpr_band": h,
            "regions_by_aco_vgpr_band": a, "regions": len(res), "rp_pass_improved_cost": imp,
            "heuristic_vgpr_prp_above_24": sum(h[1:]), "aco_vgpr_prp_above_24": sum(a[1:]),
            "pass2_len_gain_mean_pct": round(100 * float(np.mean(gains)), 2) if gains else None,
            "pass2_len_gain_max_pct": round(100 * float(np.max(gains)), 2) if gains else None}


def parity_compare(gpu: dict, ora: dict):
    """Names of the fields where the GPU result differs from the oracle's."""
    return [f for f in PARITY_FIELDS if gpu[f] != ora[f]]


# ---------------------------------------------------------------- main arm
def main(argv=None):
    args = parse(argv)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))

    if args.impl == "reference":
        return reference_arm(args, world, rank)

    import torch
    import torch.distributed as dist
    from paper_conf_cgo_shobakimhlmkrg24_b200.api import HostBatch, Scheduler

    # (test knobs: ACO_BENCH_ONE_GPU=1 puts every rank on cuda:0 and
    # ACO_BENCH_BACKEND=gloo lets such ranks talk -- a dry run of the N > 1
    # path on a one-GPU box; the product runs are one rank per GPU over NCCL)
    if os.environ.get("ACO_BENCH_ONE_GPU") == "1":
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        backend = os.environ.get("ACO_BENCH_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    batches, cfg, scaling = workload(args, rank, world)
    machine = machine_of(args)
    colony = args.workload == "c4" and world > 1  # one region, ants split across ranks
    hosts = [HostBatch(b.regs, b.ids) for b in batches]
    scheds = [Scheduler(machine, device=local) for _ in batches]
    stream = torch.cuda.current_stream()
    for s, b, h in zip(scheds, batches, hosts):
        s.load(b.regs, b.ids, batch=h)
    flush = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=f"cuda:{local}")

    def barrier():
        if world > 1:
            dist.barrier()

    def run(timing=False):
        for s, b in zip(scheds, batches):
            if not b.regs and not colony:
                continue
            if colony:
                s.run_colony(b.p, rank, world, timing=timing)
            else:
                s.run(b.p, timing=timing)

    for _ in range(max(3, args.warmup)):
        run()
    torch.cuda.synchronize()

    # ---- timed region: K steps, no per-phase events inside (ACO_FLAG_TIMING off)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.steps)]
    launches = 0
    clk = ClockSampler(local)
    clk.start()
    barrier()
    torch.cuda.synchronize()
    for k in range(args.steps):
        flush.zero_()  # L2 flush between timed steps (outside the events)
        ev[k][0].record(stream)
        run()
        ev[k][1].record(stream)
        launches += sum(s.launch_count() for s, b in zip(scheds, batches) if b.regs or colony)
    torch.cuda.synchronize()
    barrier()
    clocks = clk.stop()
    step_ms = sum(a.elapsed_time(b) for a, b in ev)
    t = torch.tensor([step_ms], dtype=torch.float64, device=f"cuda:{local}")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    max_ms = float(t.item())
    res = {}  # global id -> GPU result (this rank)
    for s, b in zip(scheds, batches):
        if b.regs:
            for rid, r in zip(b.ids, s.results()):
                res[rid] = r
    scheds_rank = sum(b.p.ants * (r["iters1"] + r["iters2"]) for s, b in zip(scheds, batches)
                      for r in (res[i] for i in b.ids)) * args.steps
    if colony:  # every rank holds the same region: count its own ants once
        scheds_rank = batches[0].p.ants * sum(res[i]["iters1"] + res[i]["iters2"] for i in batches[0].ids) * args.steps
    pruned = sum(r["ants_pruned"] for r in res.values())
    p2_ants = sum(b.p.ants * res[i]["iters2"] for b in batches for i in b.ids)
    tot = torch.tensor([float(scheds_rank), float(pruned), float(p2_ants)], dtype=torch.float64,
                       device=f"cuda:{local}")
    if world > 1:
        dist.all_reduce(tot, op=dist.ReduceOp.SUM)
    total_scheds = float(tot[0].item())
    value = total_scheds / (max_ms / 1000.0)
    prune_frac = float(tot[1].item()) / max(1.0, float(tot[2].item()))

    # ---- phase split and construct time (roofline): the same K steps again
    # with per-phase CUDA events on the launching streams (ACO_FLAG_TIMING)
    phase_ms = np.zeros(3)
    phase_launches = np.zeros(3)
    for k in range(args.steps):
        flush.zero_()
        run(timing=True)
        for s, b in zip(scheds, batches):
            if b.regs or colony:
                ms, ln = s.timing()
                phase_ms += ms
                phase_launches += ln
    torch.cuda.synchronize()

    # ---- end to end through the public API: host inputs -> H2D -> run -> D2H results
    e2e_ms = []
    sum_n = sum(int(h.offsets[-1]) for h in hosts)
    outs = [(np.zeros(max(1, int(h.offsets[-1])), np.uint32), np.zeros(max(1, int(h.offsets[-1])), np.uint32))
            for h in hosts]
    e2e_phase = []  # (load, run, results) host wall-clock ms per step (diagnostic split of e2e)
    for _ in range(max(1, args.e2e_steps)):
        barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for s, b, h in zip(scheds, batches, hosts):
            s.load(b.regs, b.ids, batch=h)
        t1 = time.perf_counter()
        run()
        t2 = time.perf_counter()
        for s, b, (o, c) in zip(scheds, batches, outs):
            if b.regs:
                s.results_raw(0, len(b.regs), o, c)
        e2e_ms.append((time.perf_counter() - t0) * 1000.0)
        e2e_phase.append(((t1 - t0) * 1000.0, (t2 - t1) * 1000.0, (time.perf_counter() - t2) * 1000.0))
    h2d = sum(int(s.arena.numel()) for s in scheds if s.arena is not None)
    n_regs = sum(len(b.regs) for b in batches)
    d2h = int(n_regs * 72 + 4 * 2 * sum_n)  # aco_result + orders + cycles
    e = torch.tensor([float(np.median(e2e_ms))], dtype=torch.float64, device=f"cuda:{local}")
    if world > 1:
        dist.all_reduce(e, op=dist.ReduceOp.MAX)
    e2e_value = total_scheds / args.steps / (float(e.item()) / 1000.0)

    # ---- gather every rank's results (global id -> digest) to rank 0 for the parity check
    local_digest = {rid: gpu_digest(r) for rid, r in res.items()}
    if world > 1 and not colony:
        all_digest = sharding.gather_results(local_digest, world, rank)
    else:
        all_digest = local_digest

    out = None
    if rank == 0:
        peaks = measured_peaks()
        cpu, bpas, parity = None, None, None
        step_ratio = 1.0
        n_cmp, n_ok, bad, log = 0, 0, [], []

        def check(rid, n, gdig, ora):
            nonlocal n_cmp, n_ok
            diff = parity_compare(gdig, ora)
            n_cmp += 1
            n_ok += not diff
            if diff:
                bad.append({"region": rid, "fields": diff})
            log.append(f"{rid} n={n} {'ok' if not diff else 'MISMATCH ' + ','.join(diff)} "
                       f"len={ora['length']} cost={ora['cost_rp']} hash={ora['trace_hash']:016x}")

        parity_note = None
        if world == 1 and not args.no_cpu_baseline:
            # the oracle on a stratified sample (per batch; c5 has two), on all host threads
            share = max(4, args.cpu_sample if args.workload != "c5" else 24)
            parts, stats_all, secs, scheds_cpu = [], [], 0.0, 0.0
            nominal_steps = 0.0  # A x n x iterations of the sample (what A x n per pass-iteration counts)
            for s, b in zip(scheds, batches):
                ps, note = cpu_sample_params(args, b.p)
                k = share if len(batches) == 1 else max(2, share // len(batches))
                base, stats, pick, ores, dt, sc = cpu_baseline(b.regs, b.ids, ps, k, machine, note)
                parts.append(base)
                stats_all.append(stats)
                nominal_steps += sum(ps.ants * b.regs[i].n_insts * (ores[q]["iters1"] + ores[q]["iters2"])
                                     for q, i in enumerate(pick))
                secs += dt
                scheds_cpu += sc
                if args.parity == "off":
                    continue
                if ps == b.p:  # the timed run's own results
                    gd = {b.ids[i]: all_digest[b.ids[i]] for i in pick}
                else:  # reduced sample parameters: one more GPU run with them, same regions
                    s.run(ps)
                    rr = s.results()
                    gd = {b.ids[i]: gpu_digest(rr[i]) for i in pick}
                    parity_note = f"GPU re-run with the cpu_baseline sample parameters ({note})"
                for q, i in enumerate(pick):
                    check(b.ids[i], b.regs[i].n_insts, gd[b.ids[i]], ores[q])
            cpu = dict(parts[0])
            cpu["value"] = round(scheds_cpu / max(secs, 1e-9), 1)
            if len(parts) > 1:
                cpu["sample"] = " + ".join(x["sample"] for x in parts)
            bpas = bytes_per_ant_step(np.concatenate(stats_all))
            from oracle.pyoracle import ORS
            placed = float(np.concatenate(stats_all)[:, ORS["placements"]].sum())
            step_ratio = placed / max(1.0, nominal_steps)  # < 1: pass-2 ants that die early
        if args.parity != "off" and (n_cmp == 0 or args.parity == "all") and args.workload not in ("c4", "c5"):
            # the oracle with the run's own parameters on a small stratified
            # sample (N > 1: every rank's results gathered to rank 0), or on
            # every region of the batch (--parity all)
            all_regs = [(r, i, b.p) for b in batches for r, i in zip(b.regs, b.ids)]
            if world > 1 and args.workload == "c3":  # rank 0 holds its share: regenerate the batch
                all_regs = [(r, i, b.p) for b in workload(args, 0, 1)[0] for r, i in zip(b.regs, b.ids)
                            if i in all_digest]
            regs_ = [x[0] for x in all_regs]
            pick = list(range(len(regs_))) if args.parity == "all" else stratified_pick(regs_, 24)
            if args.parity == "all":
                n_cmp, n_ok, bad, log = 0, 0, [], []
            t0 = time.perf_counter()
            pp = all_regs[0][2]
            ores, _, _, _ = run_oracle([all_regs[i][0] for i in pick], [all_regs[i][1] for i in pick], pp, machine)
            for q, i in enumerate(pick):
                check(all_regs[i][1], all_regs[i][0].n_insts, all_digest[all_regs[i][1]], ores[q])
            parity_note = (f"every region ({time.perf_counter() - t0:.0f} s of oracle)" if args.parity == "all"
                           else f"{len(pick)} regions stratified by size, all ranks' results gathered to rank 0")
        elif args.parity != "off" and n_cmp == 0:
            parity_note = "not in this run (c4/c5 at N > 1: every-ant parity of these variants is in tests/)"
        if n_cmp or parity_note:
            parity = {"regions": n_cmp, "bit_exact": n_ok, "mismatches": bad[:8], "fields": list(PARITY_FIELDS),
                      "sample": parity_note or "the cpu_baseline sample (stratified by size)"}
        if args.parity_log and log:
            with open(args.parity_log, "w") as f:
                f.write(f"# parity {args.workload} N={world}: {n_ok}/{n_cmp} regions bit-exact vs the oracle "
                        f"({', '.join(PARITY_FIELDS)})\n")
                f.write("\n".join(log) + "\n")
        # roofline of the dominant kernel (ant construction):
        # algorithmic shared-memory bytes (SURVEY 8(d) per ant-step figure from
        # the oracle's instrumentation of the sample) x ant-steps per launch,
        # over the construct launches' CUDA-event time; peak = the SM shared
        # memory crossbar, 148 SMs x 128 B/clk x the SM clock seen under load.
        construct_ms = phase_ms[0] / max(1, args.steps)
        # ant-steps the method performs: A x n per region and pass-iteration,
        # scaled by the oracle sample's placements / (A x n x iterations)
        # (an ant that dies in pass 2 stops early; the GPU's prune is not
        # counted as work the method must do, nor subtracted)
        ant_steps_nominal = sum(b.p.ants * sum(r.n_insts * (res[i]["iters1"] + res[i]["iters2"])
                                               for r, i in zip(b.regs, b.ids)) for b in batches)
        ant_steps = int(round(ant_steps_nominal * step_ratio))
        sm_mhz = clocks.get("sm_mhz") or peaks.get("sm_max_mhz", 1965.0)
        smem_peak = 148 * 128 * sm_mhz * 1e6 / 1e9  # GB/s
        roof = None
        if bpas is not None and construct_ms > 0:
            n_launch = phase_launches[0] / max(1, args.steps)
            achieved = bpas * ant_steps / (construct_ms / 1000.0) / 1e9
            traffic, issue, tsrc = ncu_evidence(args.workload)
            roof = {"bound": "smem", "achieved": round(achieved, 1), "peak": round(smem_peak, 1),
                    "unit": "GB/s", "frac": round(achieved / smem_peak, 4), "traffic": traffic,
                    "traffic_source": tsrc, "issue_slots_ncu": issue,
                    "algorithmic_bytes_per_launch": round(bpas * ant_steps / max(1.0, n_launch)),
                    "kernel": "k_construct (all classes)", "bytes_per_ant_step": round(bpas, 2),
                    "ant_steps_per_step": ant_steps, "ant_steps_nominal": ant_steps_nominal,
                    "ant_steps_source": f"A x n x iterations scaled by the oracle sample's placements ratio "
                                        f"{step_ratio:.4f}", "launches_per_step": n_launch,
                    "construct_ms_per_step": round(construct_ms, 3),
                    "ant_steps_per_s": round(ant_steps / (construct_ms / 1000.0), 1),
                    "peak_source": f"guide: 148 SM x 128 B/clk x {sm_mhz:.0f} MHz (smem crossbar, no measured peak)"}
        par = (f"shared colony x{world} (NCCL int64 MIN allreduce per iteration)" if args.workload == "c4"
               else (f"regions LPT-partitioned x{world}" if scaling == "strong" else f"regions x{world}")
               if args.workload in ("c3", "c5") else f"replicas x{world}")
        out = {
            "metric": METRIC, "value": round(value, 1), "unit": METRIC, "n_gpus": world,
            "steps": args.steps, "warmup": max(3, args.warmup),
            "ms_per_step": round(max_ms / args.steps, 3), "higher_is_better": True,
            "scaling": scaling, "vs_baseline": None, "dtype": "u32/u16 fixed-point (integer only)",
            "data": "synthetic",
            "config": dict(cfg, l2="flushed between timed steps (256 MB write)", parallelism=par),
            "aco_ms_per_batch": round(max_ms / args.steps, 3),
            "phase_ms_per_step": {"construct": round(phase_ms[0] / args.steps, 3),
                                  "finalize": round(phase_ms[1] / args.steps, 3),
                                  "init": round(phase_ms[2] / args.steps, 3),
                                  "note": "from K further steps with per-phase events (value is timed without them)"},
            "pruned_pass2_ant_frac": round(prune_frac, 4),
            "gpu_launches": int(launches),
            "e2e": {"value": round(e2e_value, 1), "unit": METRIC, "h2d_bytes_per_step": h2d,
                    "d2h_bytes_per_step": d2h, "ms_per_step": round(float(e.item()), 3),
                    "host_split_ms": dict(zip(("load", "run", "results"),
                                              [round(float(x), 3) for x in np.median(np.array(e2e_phase), axis=0)])),
                    "host_split_note": "rank 0 wall clock around the public calls (load: host preprocessing + "
                                       "H2D; run: planning + launch enqueue (asynchronous); results: waits for "
                                       "the device, then D2H)"},
            "clocks": clocks, "roofline": roof, "cpu_baseline": cpu, "parity": parity,
            "schedule_quality": schedule_quality(res) if args.workload != "c4" or not colony else None,
        }
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return out


# ---------------------------------------------------------------- reference arm
def reference_arm(args, world, rank):
    """--impl reference: the oracle (as it stands) on the host cores.  Every
    step runs the SAME stratified sample of this arm's workload (the value
    does not depend on --steps); the sample is shrunk only when K steps of it
    would exceed the time budget, never below 4 regions per host thread."""
    if rank != 0:
        return None
    batches, cfg, scaling = workload(args, 0, 1)
    threads = os.cpu_count() or 1
    budget_s = float(os.environ.get("ACO_REF_BUDGET_S", "240"))
    b = max(batches, key=lambda x: sum(r.n_insts for r in x.regs))
    ps, note = cpu_sample_params(args, b.p)
    full = stratified_pick(b.regs, args.cpu_sample)
    # size the per-step sample: time one step of the full sample, shrink if K of them would not fit
    times, scheds = [], 0.0
    res0, _, dt0, s0 = run_oracle([b.regs[i] for i in full], [b.ids[i] for i in full], ps, machine_of(args), threads)
    pick = full
    if dt0 * args.steps > budget_s:
        keep = max(4 * threads, int(len(full) * budget_s / (dt0 * args.steps)))
        pick = stratified_pick([b.regs[i] for i in full], min(len(full), keep))
        pick = [full[i] for i in pick]
    for _ in range(args.steps):
        _, _, dt, s = run_oracle([b.regs[i] for i in pick], [b.ids[i] for i in pick], ps, machine_of(args), threads)
        times.append(dt)
        scheds += s
    tot_s = sum(times)
    value = scheds / tot_s
    out = {"metric": METRIC, "value": round(value, 1), "unit": METRIC, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": round(1000 * tot_s / args.steps, 3), "higher_is_better": True,
           "scaling": scaling, "vs_baseline": None, "dtype": "u32/u16 fixed-point (integer only)",
           "data": "synthetic", "config": cfg, "impl": "reference",
           "cpu_baseline": {"value": round(value, 1), "unit": METRIC, "cores": min(threads, len(pick)),
                            "kind": "oracle", "host": host_cpu(),
                            "regions_per_step": len(pick), "threads": threads,
                            "sample": f"every step: the same {len(pick)} regions (stratified by size, largest first) "
                                      f"of the {cfg['workload']} workload, {note}; {scheds / args.steps:.0f} "
                                      f"ant-schedules per step on {threads} host threads"},
           "e2e": {"value": round(value, 1), "unit": METRIC, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)
    return out


if __name__ == "__main__":
    main()
