"""Summarise an ncu --csv launch list (gpu__time_duration and friends) by kernel."""
import csv
import sys
from collections import defaultdict


def load(path):
    rows = list(csv.reader(open(path)))
    hdr, by = None, defaultdict(dict)
    for r in rows:
        if 'Kernel Name' in r:
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            e = by[d['ID']]
            e[d['Metric Name']] = d['Metric Value']
            e['name'], e['grid'], e['block'] = d['Kernel Name'], d['Grid Size'], d['Block Size']
    return by


def main(path, top=30):
    by = load(path)
    tot = sum(float(v['gpu__time_duration.sum']) for v in by.values())
    agg = defaultdict(lambda: [0, 0.0])
    for v in by.values():
        k = v['name'].split('(')[0]
        agg[k][0] += 1
        agg[k][1] += float(v['gpu__time_duration.sum'])
    print(f"total {tot / 1e6:.3f} ms over {len(by)} launches")
    for k, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"  {100 * t / tot:5.1f}%  {t / 1e6:9.3f} ms  {c:4d}x  {k}")
    print("top launches:")
    for k, v in sorted(by.items(), key=lambda x: -float(x[1]['gpu__time_duration.sum']))[:top]:
        t = float(v['gpu__time_duration.sum'])
        extra = ""
        if 'sm__warps_active.avg.pct_of_peak_sustained_active' in v:
            extra = (f" warps {float(v['sm__warps_active.avg.pct_of_peak_sustained_active']):5.1f}%"
                     f" issue {float(v['sm__inst_issued.avg.pct_of_peak_sustained_active']):5.1f}%"
                     f" inst {float(v['smsp__inst_executed.sum']) / 1e9:.2f}G")
        print(f"  {t / 1e6:8.3f} ms {v['name'][:44]:44s} grid {v['grid']:>14} blk {v['block']:>12}{extra}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 30)
