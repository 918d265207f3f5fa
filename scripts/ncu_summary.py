"""Print the key ncu metrics of every kernel in a .ncu-rep (run here, no GPU)."""
import csv
import subprocess
import sys

KEYS = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'sm__warps_active.avg.pct_of_peak_sustained_active', 'launch__registers_per_thread',
        'sm__inst_executed.sum', 'smsp__issue_active.avg.pct_of_peak_sustained_active',
        'launch__occupancy_limit_registers', 'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum',
        'smsp__thread_inst_executed_per_inst_executed.ratio', 'gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed']
out = subprocess.run(['ncu', '-i', sys.argv[1], '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
h, u = rows[0], rows[1]
for r in rows[2:]:
    d = dict(zip(h, r))
    print(d['Kernel Name'][:80])
    for k in KEYS:
        if k in d:
            print(f'   {k:60s} {d[k]} {u[h.index(k)]}')
    st = [(k.replace('smsp__pcsamp_warps_issue_stalled_', ''), float(d[k].replace(',', '') or 0)) for k in h
          if k.startswith('smsp__pcsamp_warps_issue_stalled_') and not k.endswith('not_issued')]
    tot = sum(v for _, v in st) or 1
    print('   stalls:', ', '.join(f'{k} {100 * v / tot:.1f}%' for k, v in sorted(st, key=lambda x: -x[1])[:10]))
    pipes = [(k.split('pipe_')[1].split('.')[0], d[k]) for k in h
             if k.startswith('sm__inst_executed_pipe_') and k.endswith('.avg.pct_of_peak_sustained_active')]
    print('   pipes %:', ', '.join(f'{p} {v}' for p, v in pipes if v and float(v.replace(',', '')) > 1))
