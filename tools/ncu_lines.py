"""Aggregate an ncu source page (--print-source cuda,sass --csv) by CUDA
source line: warp-stall samples per line with the dominant stall reasons."""
import csv
import sys


def main(path, top=40):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if r and r[0] == "Line No")
    h = rows[hi]
    si = h.index("Warp Stall Sampling (All Samples)")
    reasons = [i for i, x in enumerate(h) if x.startswith("stall_") and "Not Issued" not in x]
    tot_by_reason = {h[i]: 0 for i in reasons}
    lines = []
    for r in rows[hi + 1:]:
        if not r or not r[0] or len(r) <= si:
            continue
        try:
            s = int(r[si])
        except ValueError:
            continue
        rs = {h[i]: int(r[i]) for i in reasons if r[i].isdigit()}
        for k, v in rs.items():
            tot_by_reason[k] += v
        lines.append((s, r[0], r[1], rs))
    tot = sum(x[0] for x in lines) or 1
    print(f"samples {tot}")
    print("by reason:", ", ".join(f"{k[6:]} {100 * v / tot:.1f}%" for k, v in
                                  sorted(tot_by_reason.items(), key=lambda x: -x[1]) if v))
    for s, ln, src, rs in sorted(lines, reverse=True)[:top]:
        top3 = sorted(rs.items(), key=lambda x: -x[1])[:3]
        print(f"{100 * s / tot:5.1f}% L{ln:>5} {src.strip()[:80]:80s} " +
              " ".join(f"{k[6:]}:{100 * v / max(1, s):.0f}%" for k, v in top3 if v))


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 40)
