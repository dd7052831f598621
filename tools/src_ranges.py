"""Instruction and stall shares of an ncu source page aggregated over named
line ranges of aco_kernels.cu (ranges given as name:lo-hi,...)."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
ranges = [(x.split(":")[0], *map(int, x.split(":")[1].split("-"))) for x in sys.argv[2].split(",")]
hi = [i for i, r in enumerate(rows) if r and r[0] == "Line No"] + [len(rows)]
best = None
for a, b in zip(hi, hi[1:]):
    h = rows[a]
    ie, ss = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
    lines = []
    for r in rows[a + 1:b]:
        try:
            lines.append((int(r[0]), int(r[ie] or 0), int(r[ss] or 0)))
        except (ValueError, IndexError):
            continue
    if best is None or len(lines) > len(best):
        best = lines
ti = sum(x[1] for x in best) or 1
ts = sum(x[2] for x in best) or 1
for name, lo, hi_ in ranges:
    i = sum(x[1] for x in best if lo <= x[0] <= hi_)
    s = sum(x[2] for x in best if lo <= x[0] <= hi_)
    print(f"{name:24s} {100 * i / ti:5.1f}% inst {100 * s / ts:5.1f}% stall")
i = sum(x[1] for x in best if not any(lo <= x[0] <= h for _, lo, h in ranges))
s = sum(x[2] for x in best if not any(lo <= x[0] <= h for _, lo, h in ranges))
print(f"{'(other)':24s} {100 * i / ti:5.1f}% inst {100 * s / ts:5.1f}% stall")
