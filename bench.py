#!/usr/bin/env python
"""Benchmark: region-batch ACO throughput (ant-schedules/s) on 1..N B200s.

One STEP = one full two-pass ACO run (aco_schedule_batch: every pass and
iteration of every region: construction, argmin + winner replay, pheromone
update, epilogue) over one batch of synthetic regions.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--workload c3|c2|c1|c4|c5]
                  [--machine gfx906|dual] [--passes 3|4 --ws-weight W] [--policy off|paper]
                  [--heur-mix 0|1] [--stall-num k] [--rl-limit 0|1|2]
  python bench.py --impl reference ...     # the CPU oracle on a bounded sample

Workloads (BASELINE.json configs): c1 FIX10-A; c2 one n = 100 region; c3
(default, the metric's config) 5,000 rocPRIM-shaped regions per GPU (weak
scaling); c4 one n = 2,000 region with 8,192 ants per iteration as ONE shared
colony across the N ranks (strong scaling: 8,192 / N ants per rank, one int64
MIN allreduce per iteration over NCCL); c5 the full-suite sweep, 1,000
regions per GPU up to 4,000 instructions (weak scaling).

Multi-GPU: launched by torchrun, one process per GPU.  Regions shard with no
data-path collective (each rank schedules its own batch with globally unique
region ids); NCCL is used only for the barrier and the max-over-ranks time.
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

METRIC = "ant-schedules/s"
C3_REGIONS = 5000


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="c3", choices=["c3", "c2", "c1", "c4", "c5"])
    ap.add_argument("--machine", default="gfx906", choices=["gfx906", "dual"])
    ap.add_argument("--passes", type=int, default=3, choices=[1, 2, 3, 4])
    ap.add_argument("--ws-weight", type=int, default=4)
    ap.add_argument("--policy", default="off", choices=["off", "paper"])
    ap.add_argument("--heur-mix", type=int, default=0)
    ap.add_argument("--stall-num", type=int, default=1)
    ap.add_argument("--rl-limit", type=int, default=0, help="pass-1 ready-list size limit (R45): 1 min, 2 mid")
    ap.add_argument("--regions", type=int, default=C3_REGIONS, help="regions per rank (c3)")
    ap.add_argument("--ants", type=int, default=None)
    ap.add_argument("--iterations", type=int, default=None)
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-sample", type=int, default=160, help="regions in the oracle sample")
    return ap.parse_args()


def workload(args, rank: int):
    """(regions, region_ids, params, config dict) for this rank."""
    if args.workload == "c3":
        n = args.regions
        first = rank * n
        regs = I.gen_batch(n, base_seed=3, first_id=first)
        ids = list(range(first, first + n))
        p = I.Params(ants=args.ants or 1024, iterations=args.iterations or 10, seed=3)
        cfg = {"workload": "c3-rocprim-shaped-batch", "regions_per_gpu": n,
               "sizes": "20-500 (Table 3.a buckets)", "latency": "mixed"}
    elif args.workload == "c2":
        regs = [I.gen_region(100, I.region_seed(2, rank))]
        ids = [rank]
        p = I.Params(ants=args.ants or 1024, iterations=args.iterations or 100, seed=2)
        cfg = {"workload": "c2-single-region-n100", "regions_per_gpu": 1, "latency": "mixed"}
    elif args.workload == "c4":
        regs = [I.gen_region(2000, I.region_seed(4, 0))]
        ids = [0]  # ONE region shared by all ranks (shared colony)
        world = int(os.environ.get("WORLD_SIZE", "1"))
        total = args.ants or 8192
        p = I.Params(ants=total // world, iterations=args.iterations or 10, seed=4)
        cfg = {"workload": "c4-shared-colony-n2000", "regions": 1, "ants_total": total,
               "ants_per_gpu": total // world, "latency": "mixed"}
    elif args.workload == "c5":
        n = args.regions if args.regions != C3_REGIONS else 1000
        first = rank * n
        sizes = I.c5_sizes(first + n, base_seed=5)[first:]
        regs = I.gen_batch(n, base_seed=5, first_id=first, sizes=sizes)
        ids = list(range(first, first + n))
        p = I.Params(ants=args.ants or 1024, iterations=args.iterations or 5, seed=5)
        cfg = {"workload": "c5-suite-sweep", "regions_per_gpu": n, "sizes": "20-4000 (c3 mix + 15% tail 500-4000)",
               "max_n": int(max(r.n_insts for r in regs)), "latency": "mixed"}
    else:
        regs = [I.fix10a()]
        ids = [rank]
        p = I.Params(ants=args.ants or 64, iterations=args.iterations or 20, seed=0, cost_mode=0)
        cfg = {"workload": "c1-fix10a", "regions_per_gpu": 1}
    p = dataclasses.replace(p, passes=args.passes, ws_weight=args.ws_weight if args.passes == 4 else 0,
                            heur_mix=args.heur_mix, stall_num=args.stall_num,
                            rl_limit=args.rl_limit)
    if args.policy == "paper":
        p = I.paper_policy(p)
    passes = {1: "RP", 2: "ILP", 3: "RP+ILP", 4: f"weighted single pass (W={p.ws_weight})"}[p.passes]
    cfg.update({"ants": p.ants, "iterations_per_pass": p.iterations, "passes": passes,
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
    return regs, ids, p, cfg


def machine_of(args):
    return I.DUAL_ISSUE if args.machine == "dual" else I.GFX906


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
    """Round-robin the sample over the steps (a sample smaller than the step
    count is reused whole by the steps it does not reach)."""
    return [full[s::steps] or full for s in range(steps)]


def cpu_baseline(regs, ids, p, sample: int, machine=I.GFX906, note="full A x I x passes", pick=None):
    """The oracle as it stands on a bounded, stratified sample of the same workload."""
    from oracle import pyoracle as O
    if pick is None:
        pick = stratified_pick(regs, sample)
    sub = [regs[i] for i in pick]
    sid = [ids[i] for i in pick]
    threads = os.cpu_count() or 1
    t0 = time.perf_counter()
    _, _, stats, _ = O.schedule_many(sub, sid, machine, p, n_threads=threads)
    dt = time.perf_counter() - t0
    scheds = float(stats[:, O.ORS["ant_scheds"]].sum())
    return {"value": scheds / dt, "unit": METRIC, "cores": min(threads, len(sub)), "kind": "oracle",
            "sample": f"{len(sub)} of {len(regs)} regions (stratified by size), {note}, "
                      f"{scheds:.0f} ant-schedules in {dt:.1f} s"}, stats


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))

    if args.impl == "reference":
        return reference_arm(args, world, rank)

    import torch
    import torch.distributed as dist
    from paper_conf_cgo_shobakimhlmkrg24_b200.api import HostBatch, Scheduler

    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    regs, ids, p, cfg = workload(args, rank)
    machine = machine_of(args)
    colony = args.workload == "c4" and world > 1  # one region, ants split across ranks
    batch = HostBatch(regs, ids)
    sched = Scheduler(machine, device=local)
    stream = torch.cuda.current_stream()
    sched.load(regs, ids, batch=batch)
    flush = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device=f"cuda:{local}")

    def barrier():
        if world > 1:
            dist.barrier()

    def run(timing=False):
        if colony:
            sched.run_colony(p, rank, world, timing=timing)
        else:
            sched.run(p, timing=timing)

    for _ in range(max(3, args.warmup)):
        run()
    torch.cuda.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(args.steps)]
    phase_ms = np.zeros(3)
    phase_launches = np.zeros(3)
    launches = 0
    clk = ClockSampler(local)
    clk.start()
    barrier()
    torch.cuda.synchronize()
    for k in range(args.steps):
        flush.zero_()  # L2 flush between timed steps (outside the events)
        ev[k][0].record(stream)
        run(timing=True)
        ev[k][1].record(stream)
        ms, ln = sched.timing()  # syncs; events inside the library, same stream
        phase_ms += ms
        phase_launches += ln
        launches += sched.launch_count()
    torch.cuda.synchronize()
    barrier()
    clocks = clk.stop()
    step_ms = sum(a.elapsed_time(b) for a, b in ev)
    t = torch.tensor([step_ms], dtype=torch.float64, device=f"cuda:{local}")
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    max_ms = float(t.item())
    res = sched.results()
    iters = sum(r["iters1"] + r["iters2"] for r in res)
    scheds_rank = p.ants * iters * args.steps
    tot = torch.tensor([float(scheds_rank)], dtype=torch.float64, device=f"cuda:{local}")
    if world > 1:
        dist.all_reduce(tot, op=dist.ReduceOp.SUM)
    value = float(tot.item()) / (max_ms / 1000.0)

    # ---- end to end through the public API: host inputs -> H2D -> run -> D2H results
    e2e_ms = []
    h2d = d2h = 0
    sum_n = int(batch.offsets[-1])
    orders = np.zeros(max(1, sum_n), np.uint32)
    cycles = np.zeros(max(1, sum_n), np.uint32)
    for _ in range(max(1, args.e2e_steps)):
        barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        sched.load(regs, ids, batch=batch)
        run()
        sched.results_raw(0, len(regs), orders, cycles)
        e2e_ms.append((time.perf_counter() - t0) * 1000.0)
    h2d = int(sched.arena.numel()) if sched.arena is not None else 0
    d2h = int(len(regs) * 64 + 4 * 2 * sum_n)
    e = torch.tensor([float(np.median(e2e_ms))], dtype=torch.float64, device=f"cuda:{local}")
    if world > 1:
        dist.all_reduce(e, op=dist.ReduceOp.MAX)
    e2e_value = float(tot.item()) / args.steps / (float(e.item()) / 1000.0)

    out = None
    if rank == 0:
        peaks = measured_peaks()
        cpu = None
        bpas = None
        if world == 1 and not args.no_cpu_baseline:
            ps, note = cpu_sample_params(args, p)
            cpu, stats = cpu_baseline(regs, ids, ps, args.cpu_sample if args.workload != "c5" else 24,
                                      machine, note)
            bpas = bytes_per_ant_step(stats)
        # roofline of the dominant kernel (ant construction):
        # algorithmic shared-memory bytes (SURVEY 8(d) per ant-step figure from
        # the oracle's instrumentation of the sample) x ant-steps per launch,
        # over the construct launches' CUDA-event time; peak = the SM shared
        # memory crossbar, 148 SMs x 128 B/clk x the SM clock seen under load.
        construct_ms = phase_ms[0] / max(1, args.steps)
        ant_steps = p.ants * sum(r["n"] * (r["iters1"] + r["iters2"]) for r in res)
        sm_mhz = clocks.get("sm_mhz") or peaks.get("sm_max_mhz", 1965.0)
        smem_peak = 148 * 128 * sm_mhz * 1e6 / 1e9  # GB/s
        roof = None
        if bpas is not None and construct_ms > 0:
            n_launch = phase_launches[0] / max(1, args.steps)
            achieved = bpas * ant_steps / (construct_ms / 1000.0) / 1e9
            traffic, tsrc, issue = None, None, None
            try:  # DRAM bytes per construct launch from the committed ncu --set full capture
                with open(os.path.join(ROOT, "profiles", "r01_traffic.json")) as f:
                    tj = json.load(f)
                if args.workload == "c3":
                    traffic, tsrc = tj["dram_bytes_per_launch"], tj["source"]
                    # the bound that actually binds: SM issue slots, from ncu
                    issue = {"util_pct": tj.get("issue_util_pct"), "warps_active_pct": tj.get("warps_active_pct"),
                             "source": tj.get("issue_source")}
            except Exception:
                pass
            roof = {"bound": "smem", "achieved": round(achieved, 1), "peak": round(smem_peak, 1),
                    "unit": "GB/s", "frac": round(achieved / smem_peak, 4), "traffic": traffic,
                    "traffic_source": tsrc, "issue_slots_ncu": issue,
                    "algorithmic_bytes_per_launch": round(bpas * ant_steps / max(1.0, n_launch)),
                    "kernel": "k_construct (all classes)", "bytes_per_ant_step": round(bpas, 2),
                    "ant_steps_per_step": ant_steps, "launches_per_step": n_launch,
                    "construct_ms_per_step": round(construct_ms, 3),
                    "ant_steps_per_s": round(ant_steps / (construct_ms / 1000.0), 1),
                    "peak_source": f"guide: 148 SM x 128 B/clk x {sm_mhz:.0f} MHz (smem crossbar, no measured peak)"}
        out = {
            "metric": METRIC, "value": round(value, 1), "unit": METRIC, "n_gpus": world,
            "steps": args.steps, "warmup": max(3, args.warmup),
            "ms_per_step": round(max_ms / args.steps, 3), "higher_is_better": True,
            "scaling": "strong" if args.workload == "c4" else "weak",
            "vs_baseline": None, "dtype": "u32/u16 fixed-point (integer only)", "data": "synthetic",
            "config": dict(cfg, l2="flushed between timed steps (256 MB write)",
                           parallelism=f"shared colony x{world} (NCCL int64 MIN allreduce per iteration)"
                           if args.workload == "c4" else f"regions x{world}"),
            "aco_ms_per_batch": round(max_ms / args.steps, 3),
            "phase_ms_per_step": {"construct": round(phase_ms[0] / args.steps, 3),
                                  "finalize": round(phase_ms[1] / args.steps, 3),
                                  "init": round(phase_ms[2] / args.steps, 3)},
            "gpu_launches": int(launches),
            "e2e": {"value": round(e2e_value, 1), "unit": METRIC, "h2d_bytes_per_step": h2d,
                    "d2h_bytes_per_step": d2h, "ms_per_step": round(float(e.item()), 3)},
            "clocks": clocks, "roofline": roof, "cpu_baseline": cpu,
        }
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return out


def reference_arm(args, world, rank):
    """--impl reference: the oracle (as it stands) on the host cores, on a
    bounded sample of this arm's workload per step."""
    if rank != 0:
        return None
    regs, ids, p, cfg = workload(args, 0)
    cpu_times = []
    scheds = 0.0
    ps, note = cpu_sample_params(args, p)
    for _ in range(args.warmup):
        pass  # the oracle has no warm-up state
    # the --cpu-sample stratified sample, dealt round-robin over the steps
    # (each step a smaller stratified sample, largest region first)
    full = stratified_pick(regs, max(args.cpu_sample, 4 * args.steps))
    per_step = deal_over_steps(full, args.steps)
    for s in range(args.steps):
        cpu, stats = cpu_baseline(regs, ids, ps, 0, machine_of(args), note, pick=per_step[s])
        from oracle.pyoracle import ORS
        s = float(stats[:, ORS["ant_scheds"]].sum())
        scheds += s
        cpu_times.append(s / cpu["value"])
    tot_s = sum(cpu_times)
    value = scheds / tot_s
    out = {"metric": METRIC, "value": round(value, 1), "unit": METRIC, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": round(1000 * tot_s / args.steps, 3), "higher_is_better": True,
           "scaling": "strong" if args.workload == "c4" else "weak", "vs_baseline": None, "dtype": "u32/u16 fixed-point (integer only)",
           "data": "synthetic", "config": cfg, "impl": "reference",
           "cpu_baseline": {"value": round(value, 1), "unit": METRIC, "cores": os.cpu_count(), "kind": "oracle",
                            "sample": f"per step about {max(1, len(full) // args.steps)} regions (a stratified sample of "
                                      f"{len(full)} dealt over the steps, largest first) of the {cfg['workload']} workload, {note}"},
           "e2e": {"value": round(value, 1), "unit": METRIC, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)
    return out


if __name__ == "__main__":
    main()
