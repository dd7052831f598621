"""Markdown table of a bench matrix directory (bench_<line>.json files)."""
import json
import os
import sys

D = sys.argv[1]
names = {'c3': 'C3 (headline)', 'c1': 'C1 FIX10-A, 64 × 20 × 2', 'c2': 'C2 n = 100, 1024 × 100 × 2',
         'c4': 'C4 n = 2,000, 8,192 ants × 20 × 2', 'c5': 'C5 SURVEY grid (54 regions, n ≤ 4,000)',
         'c3_dual': 'C3 dual-issue machine', 'c3_weighted': 'C3 weighted single pass (W = 4)',
         'c3_paper_policy': 'C3 paper compile policy', 'c3_heur_mix': 'C3 mixed heuristics',
         'c3_stall50': 'C3 50 % stalling groups', 'c3_rl_min': 'C3 ready-list limit, min (R45)',
         'c3_rl_mid': 'C3 ready-list limit, mid (R45)'}


def f(x):
    return f"{x / 1e6:.2f} M" if x >= 1e6 else f"{x / 1e3:.0f} K" if x >= 1e3 else f"{x:.0f}"


print("| line | ms / step | ant-schedules/s | e2e (ms / step) | oracle (host, 16 threads) | roofline frac | parity (bit-exact / compared) |")
print("|---|---|---|---|---|---|---|")
for k, label in names.items():
    p = os.path.join(D, f"bench_{k}.json")
    if not os.path.exists(p):
        continue
    try:
        d = json.load(open(p))
    except ValueError:
        continue
    r = d.get('roofline') or {}
    cb = d.get('cpu_baseline') or {}
    par = d.get('parity') or {}
    print(f"| {label} | {d['ms_per_step']:.3f} | {f(d['value'])} | {f(d['e2e']['value'])} ({d['e2e']['ms_per_step']:.1f}) | "
          f"{f(cb.get('value', 0))} | {r.get('frac')} | {par.get('bit_exact')} / {par.get('regions')} |")
p = os.path.join(D, "bench_c3_reference.json")
if os.path.exists(p):
    d = json.load(open(p))
    print(f"\nReference arm (`--impl reference`): {f(d['value'])} ant-schedules/s "
          f"({d['cpu_baseline']['regions_per_step']} regions per step on {d['cpu_baseline']['threads']} threads).")
