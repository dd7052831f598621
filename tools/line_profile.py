"""Aggregate an ncu source page (cuda,sass) by CUDA source line."""
import csv
import subprocess
import sys
from collections import defaultdict


def main(rep, src_path, top=40, key="inst"):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr = rows[2]
    data = rows[3:]
    iE = hdr.index('Instructions Executed')
    iT = hdr.index('Thread Instructions Executed')
    iW = hdr.index('Warp Stall Sampling (All Samples)')
    src = open(src_path).read().split('\n')
    agg = defaultdict(lambda: [0.0, 0.0, 0.0])
    cur = None
    for r in data:
        if r[0].strip().isdigit():
            cur = int(r[0])
        try:
            e, t, w = float(r[iE] or 0), float(r[iT] or 0), float(r[iW] or 0)
        except (ValueError, IndexError):
            continue
        if cur:
            agg[cur][0] += e
            agg[cur][1] += t
            agg[cur][2] += w
    tot = sum(v[0] for v in agg.values())
    totw = sum(v[2] for v in agg.values())
    print(f"{rows[1][1][:100]}\n warp-inst {tot:.3g}  thread/warp-inst {sum(v[1] for v in agg.values()) / tot:.1f}")
    idx = 0 if key == "inst" else 2
    for ln, (e, t, w) in sorted(agg.items(), key=lambda x: -x[1][idx])[:top]:
        print(f"L{ln:4d} {100 * e / tot:5.1f}% inst {100 * w / totw:5.1f}% stall  act {t / max(e, 1):4.1f} | {src[ln - 1].strip()[:88]}")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], int(sys.argv[3]) if len(sys.argv) > 3 else 40,
         sys.argv[4] if len(sys.argv) > 4 else "inst")
