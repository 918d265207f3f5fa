"""Summarise an ncu launch list (gpu__time_duration per kernel name)."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = [i for i, r in enumerate(rows) if 'Kernel Name' in r][0]
h = rows[hdr]
ki, vi = h.index('Kernel Name'), h.index('Metric Value')
d = collections.OrderedDict()
for r in rows[hdr + 1:]:
    if len(r) > vi:
        d.setdefault(r[ki][:90], []).append(float(r[vi].replace(',', '')))
skip = ('at::', 'synth::', 'at_cuda_detail', 'compute_cuda_kernel', '<unnamed>')
for k, v in d.items():
    if not any(s in k for s in skip):
        print(f"{sum(v) / len(v) / 1e3:9.1f} us x{len(v):3d}  {k}")
