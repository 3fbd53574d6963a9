#!/usr/bin/env python
"""Summarise ncu outputs for profiles/: a launch list (--csv --metrics gpu__time_duration.sum)
or a --set full report (.ncu-rep, read with `ncu -i ... --page raw --csv`)."""
import collections
import csv
import io
import subprocess
import sys

KEYS = ['launch__grid_size', 'launch__registers_per_thread', 'gpu__time_duration.sum', 'dram__bytes_read.sum',
        'dram__bytes_write.sum', 'lts__t_bytes.sum', 'sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active',
        'sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_elapsed',
        'sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active',
        'sm__warps_active.avg.pct_of_peak_sustained_active', 'smsp__issue_active.avg.pct_of_peak_sustained_active',
        'l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum']
STALLS = 'smsp__average_warps_issue_stalled_'


def launch_list(path):
    lines = [l for l in open(path) if not l.startswith('==')]
    rows = list(csv.DictReader(io.StringIO(''.join(lines))))
    agg = collections.OrderedDict()
    for r in rows:
        k = r['Kernel Name'].split('(')[0]
        agg.setdefault(k, []).append(float(r['Metric Value']) / 1e3)  # us
    tot = sum(sum(v) for v in agg.values())
    out = ['kernel | launches | total_ms | mean_us | share']
    for k, v in agg.items():
        out.append('%s | %d | %.3f | %.2f | %.1f%%' % (k, len(v), sum(v) / 1e3, sum(v) / len(v), 100 * sum(v) / tot))
    out.append('total device time %.3f ms over %d launches (cold-cache, serialised under ncu)' % (
        tot / 1e3, sum(len(v) for v in agg.values())))
    return '\n'.join(out)


def report(path):
    txt = subprocess.run(['ncu', '-i', path, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(txt)))
    h, u = r[0], r[1]
    out = []
    for v in r[2:]:
        out.append('kernel: ' + v[h.index('Kernel Name')])
        for k in KEYS:
            if k in h:
                out.append('  %s = %s %s' % (k, v[h.index(k)], u[h.index(k)]))
        for i, k in enumerate(h):
            if k.startswith(STALLS) and k.endswith('_per_issue_active.ratio'):
                try:
                    if float(v[i]) >= 0.05:
                        out.append('  %s = %s' % (k, v[i]))
                except ValueError:
                    pass
    return '\n'.join(out)


if __name__ == '__main__':
    p = sys.argv[1]
    print(report(p) if p.endswith('.ncu-rep') else launch_list(p))
