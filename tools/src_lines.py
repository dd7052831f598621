"""Per-CUDA-line instruction and stall shares of an ncu source page
(--page source --csv --print-source cuda,sass), largest section = kernel file."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
hi = [i for i, r in enumerate(rows) if r and r[0] == "Line No"] + [len(rows)]
best = None
for a, b in zip(hi, hi[1:]):
    h = rows[a]
    ie, ss = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
    lines = []
    for r in rows[a + 1:b]:
        try:
            lines.append((int(r[ie] or 0), int(r[ss] or 0), r[0], r[1]))
        except (ValueError, IndexError):
            continue
    if best is None or len(lines) > len(best):
        best = lines
tot = sum(x[0] for x in best) or 1
ts = sum(x[1] for x in best) or 1
print(f"warp-inst {tot:.3e}  stall samples {ts}")
for x, s, ln, src in sorted(best, key=lambda t: -t[1])[:top]:
    print(f"{100 * x / tot:5.1f}% inst {100 * s / ts:5.1f}% stall L{ln:>5} {src.strip()[:96]}")
