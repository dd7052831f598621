"""Markdown table of per-launch ncu --set full metrics (raw csv page) and the
DRAM traffic / issue-slot roll-up of the construct launches (r01_traffic.json)."""
import csv
import json
import sys

COLS = [('kernel', 'Kernel Name'), ('grid', 'Grid Size'), ('block', 'Block Size'), ('ms', 'gpu__time_duration.sum'),
        ('warps%', 'sm__warps_active.avg.pct_of_peak_sustained_active'),
        ('issue%', 'sm__inst_issued.avg.pct_of_peak_sustained_active'),
        ('lanes/inst', 'smsp__thread_inst_executed_per_inst_executed.ratio'),
        ('blk/SM (smem)', 'launch__occupancy_limit_shared_mem'), ('blk/SM (regs)', 'launch__occupancy_limit_registers'),
        ('smem wavefronts %', 'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed'),
        ('L1 hit %', 'l1tex__t_sector_hit_rate.pct'), ('L2 hit %', 'lts__t_sector_hit_rate.pct'),
        ('dram rd MB', 'dram__bytes_read.sum'), ('dram wr MB', 'dram__bytes_write.sum')]
SCALE = {'byte': 1, 'Kbyte': 1e3, 'Mbyte': 1e6, 'Gbyte': 1e9, 'nsecond': 1e-6, 'usecond': 1e-3, 'msecond': 1.0}


def main(path, traffic_out=None, source="", so_sha256=None):
    rows = list(csv.reader(open(path)))
    h, u = rows[0], rows[1]

    def num(r, k):
        return float(r[h.index(k)].replace(',', '')) * SCALE.get(u[h.index(k)], 1.0)

    print('| ' + ' | '.join(c[0] for c in COLS) + ' |')
    print('|' + '---|' * len(COLS))
    tw = acc = accw = dram = 0.0
    nc = 0
    for r in rows[2:]:
        name = r[h.index('Kernel Name')]
        vals = []
        for c, k in COLS:
            if c == 'kernel':
                vals.append('`' + name.split('(')[0].replace('void aco::', '').replace('aco::', '') + '`')
            elif c == 'ms' or c.startswith('dram'):
                x = num(r, k)
                vals.append(f"{x / 1e6:.2f}" if c.startswith('dram') else f"{x:.2f}")
            else:
                v = r[h.index(k)]
                try:
                    vals.append(f"{float(v):.1f}")
                except ValueError:
                    vals.append(v)
        print('| ' + ' | '.join(vals) + ' |')
        if 'k_construct' in name:
            t = num(r, 'gpu__time_duration.sum')
            tw += t
            acc += t * num(r, 'sm__inst_issued.avg.pct_of_peak_sustained_active')
            accw += t * num(r, 'sm__warps_active.avg.pct_of_peak_sustained_active')
            dram += num(r, 'dram__bytes_read.sum') + num(r, 'dram__bytes_write.sum')
            nc += 1
    if traffic_out and nc:
        json.dump({"kernel": "k_construct (all classes)", "dram_bytes_per_launch": int(dram / nc), "launches": nc,
                   "source": source, "issue_util_pct": round(acc / tw, 1), "warps_active_pct": round(accw / tw, 1),
                   "issue_source": "time-weighted sm__inst_issued.avg.pct_of_peak_sustained_active (and "
                                   "sm__warps_active) over the same construct launches",
                   "build_fingerprint": so_sha256},
                  open(traffic_out, 'w'), indent=1)


if __name__ == "__main__":
    # ncu_table.py prof_raw.csv [traffic.json source-text [build fingerprint of the profiled library]]
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else None, sys.argv[3] if len(sys.argv) > 3 else "",
         sys.argv[4] if len(sys.argv) > 4 else None)
