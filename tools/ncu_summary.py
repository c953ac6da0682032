"""Summarise an ncu --set full report: SOL, issue, pipes, stalls, instruction regions."""
import csv, io, subprocess, sys
from collections import defaultdict

rep = sys.argv[1]
def page(*a):
    return subprocess.run(['ncu', '-i', rep] + list(a), capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(page('--page', 'raw', '--csv', '--print-units', 'base'))))
d = dict(zip(r[0], r[2] if len(r) > 2 else r[1]))
keys = ['gpu__time_duration.sum', 'sm__throughput.avg.pct_of_peak_sustained_elapsed',
        'smsp__issue_active.avg.pct_of_peak_sustained_active', 'sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active',
        'sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_elapsed', 'sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active',
        'sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active', 'sm__warps_active.avg.pct_of_peak_sustained_active',
        'smsp__thread_inst_executed_per_inst_executed.ratio', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'launch__registers_per_thread', 'smsp__inst_executed.sum']
for k in keys:
    if k in d: print(f'{k:70s} {d[k]}')
ks = [k for k in r[0] if k.startswith('smsp__pcsamp_warps_issue_stalled') and not k.endswith('not_issued')]
vals = []
for k in ks:
    try: vals.append((float(d[k].replace(',', '')), k))
    except ValueError: pass
tot = sum(v for v, _ in vals) or 1
print('stalls:', ', '.join(f"{k.replace('smsp__pcsamp_warps_issue_stalled_', '')} {v/tot*100:.1f}%" for v, k in sorted(vals, reverse=True)[:8]))
src = list(csv.reader(io.StringIO(page('--page', 'source', '--csv', '--print-source', 'sass'))))
h = src[1]; rows = [dict(zip(h, x)) for x in src[2:] if len(x) == len(h)]
tot_i = sum(float(x['Instructions Executed'] or 0) for x in rows) or 1
reg = defaultdict(lambda: [0, 0.0])
for x in rows:
    ie = float(x['Instructions Executed'] or 0)
    if ie: reg[round(ie / 1e6, 1)][0] += 1; reg[round(ie / 1e6, 1)][1] += ie
print(f'total warp instructions {tot_i:.3e}')
for k, (n, ie) in sorted(reg.items(), key=lambda t: -t[1][1])[:6]:
    print(f'  executed {k:7.1f}M times x {n:3d} instructions = {ie/tot_i*100:5.1f}%')
