"""Write the round's ncu summary (markdown) from a verification run's outputs:
launch list by kernel, per-launch --set full metrics of the first iteration,
the top pass-2 class's stall reasons and code-region breakdown, and the
config-4 global-state kernel.

    python tools/make_ncu_summary.py gpurun_out/final > profiles/r02_final_ncu_summary.md
"""
import csv
import io
import os
import subprocess
import sys

D = sys.argv[1]
T = os.path.dirname(os.path.abspath(__file__))


def run(*args):
    return subprocess.run([sys.executable, *args], capture_output=True, text=True).stdout


def stalls(raw):
    rows = list(csv.reader(open(raw)))
    out = []
    for r in rows[2:]:
        d = dict(zip(rows[0], r))
        items = []
        for k, v in sorted(d.items()):
            if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("_per_issue_active.ratio"):
                try:
                    if float(v) >= 0.1:
                        items.append((k[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")], float(v)))
                except ValueError:
                    pass
        keys = ["gpu__time_duration.sum", "sm__warps_active.avg.pct_of_peak_sustained_active",
                "sm__inst_issued.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
                "smsp__thread_inst_executed_per_inst_executed.ratio", "l1tex__t_sector_hit_rate.pct"]
        out.append((d.get("Kernel Name", "")[:80], {k: d.get(k) for k in keys}, items))
    return out


TAG = os.environ.get("TAG", "r03")
print(f"# {TAG} final ncu evidence: C3 batch (5,000 regions, 1,024 ants x 10 iterations x 2 passes) on one B200\n")
print(f"Build: the final kernels (`profiles/{TAG}_traffic.json` carries its source fingerprint; bench.py")
print(f"reports the issue-slot / DRAM figures below only for that build).  Commands: `tools/gpu_{TAG}_final4.sh`.")
print("ncu serialises launches and runs them cold: compare shares, not absolutes.\n")
print("## Launch list by kernel (every launch of the bench command under ncu)\n")
print("```")
print(run(os.path.join(T, "launch_summary.py"), os.path.join(D, "launches.csv"), "0").strip())
print("```\n")
print("## Full-set metrics per launch (first iteration, both passes)\n")
print(open(os.path.join(D, "ncu_table.md")).read())
print(f"\nRoll-up (time-weighted over the construct launches; `{TAG}_traffic.json`):\n")
print("```")
print(open(os.path.join(D, f"{TAG}_traffic.json")).read().strip())
print("```\n")
for title, raw, src, ranges in (
        ("Top pass-2 class `k_construct<2,1,1,0,0,0,2,1,1>` (lean layout, image through L1)", "prof_top_raw.csv",
         "prof_top_source.csv", None),
        ("Config 4's global-state kernel (n = 2,000, 8,192 ants, 16 lanes per ant)", "prof_gs_raw.csv", None, None),
        ("Config 4's huge-region kernels (n = 2,000, 8,192 ants: per-ant state in shared memory, 8 lanes per ant)",
         "prof_c4_raw.csv", None, None),
        ("Config 2: lane-per-instruction ants (k_construct<P, 32, ...>) and the one-launch finalize",
         "prof_c2_raw.csv", None, None)):
    p = os.path.join(D, raw)
    if not os.path.exists(p):
        continue
    print(f"## {title}\n")
    for name, m, items in stalls(p):
        print(f"`{name}`: " + ", ".join(f"{k.split('.')[0].replace('__', ' ')} {v}" for k, v in m.items()))
        print("stall reasons per issued instruction: " + ", ".join(f"{k} {v:.2f}" for k, v in items) + "\n")
    if src and os.path.exists(os.path.join(D, src)):
        print("```")
        print(run(os.path.join(T, "src_lines.py"), os.path.join(D, src), "25").strip())
        print("```\n")
