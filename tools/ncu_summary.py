"""Summarise an ncu report: key metrics, stall mix and instruction mix per kernel (text)."""
import collections
import csv
import io
import subprocess
import sys

KEYS = ['gpu__time_duration.sum', 'smsp__inst_executed.sum', 'smsp__issue_active.avg.pct_of_peak_sustained_active',
        'sm__warps_active.avg.pct_of_peak_sustained_active', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed', 'l1tex__throughput.avg.pct_of_peak_sustained_active',
        'sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active', 'launch__registers_per_thread',
        'launch__occupancy_limit_shared_mem', 'launch__occupancy_limit_registers', 'sm__cycles_elapsed.avg']


def raw(rep):
    out = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


def main(rep, with_ops=True):
    hdr, units, rows = raw(rep)
    for row in rows:
        name = row[hdr.index('Kernel Name')]
        print(name[:80])
        for k in KEYS:
            if k in hdr:
                print(f"    {k:60s} {row[hdr.index(k)]} {units[hdr.index(k)]}")
        st = []
        for i, h in enumerate(hdr):
            if 'pcsamp_warps_issue_stalled' in h and 'not_issued' not in h:
                try:
                    st.append((float(row[i]), h.replace('smsp__pcsamp_warps_issue_stalled_', '')))
                except ValueError:
                    pass
        tot = sum(v for v, _ in st) or 1
        print('    stalls: ' + ', '.join(f'{h} {100 * v / tot:.0f}%' for v, h in sorted(st, reverse=True)[:8]))


if __name__ == '__main__':
    main(sys.argv[1])
