"""Per-opcode and top per-instruction stall breakdown from an ncu source-page
CSV (ncu -i rep --page source --csv --print-source sass)."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdrs = [i for i, r in enumerate(rows) if r and r[0] == 'Address']
h = rows[hdrs[0]]
end = hdrs[1] - 1 if len(hdrs) > 1 else len(rows)
data = [r for r in rows[hdrs[0] + 1:end] if len(r) == len(h)]
reasons = [c for c in h if c.startswith('stall_') and 'Not Issued' not in c]
src = h.index('Source')
tot = sum(float(r[h.index('Warp Stall Sampling (All Samples)')] or 0) for r in data)
by = collections.defaultdict(collections.Counter)
for r in data:
    t = r[src].split()
    if not t:
        continue
    op = (t[1] if t[0].startswith('@') else t[0]).split('.')[0]
    for c in reasons:
        by[op][c] += float(r[h.index(c)] or 0)
print('total samples', tot)
for op, cnt in sorted(by.items(), key=lambda kv: -sum(kv[1].values()))[:12]:
    s = sum(cnt.values())
    top = ', '.join(f'{k[6:]} {100 * v / tot:.1f}' for k, v in cnt.most_common(4) if v)
    print(f'{op:8s} {100 * s / tot:5.1f}%  [{top}]')
# top instructions by long_sb
ls = h.index('stall_long_sb')
print('top long_sb instructions:')
for r in sorted(data, key=lambda r: -float(r[ls] or 0))[:6]:
    print('   ', r[ls], r[src][:80])
