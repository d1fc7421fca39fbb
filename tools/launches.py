"""Summarise an ncu --metrics gpu__time_duration.sum CSV launch list."""
import csv, sys, re, collections
rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if 'Kernel Name' in r][0]
h = rows[hi]; ki = h.index('Kernel Name'); vi = h.index('Metric Value'); ui = h.index('Metric Unit')
only = sys.argv[2] if len(sys.argv) > 2 else None
seq = []
for r in rows[hi + 1:]:
    name = r[ki]
    m = re.search(r'(\w+_kernel)(<[^>]*>)?', name)
    short = (m.group(1) + (m.group(2) or '')) if m else name.split('(')[0][:50]
    if 'spbla' not in name and only:
        continue
    v = float(r[vi].replace(',', '')); unit = r[ui]
    if unit == 'usecond': v *= 1e3
    if unit == 'msecond': v *= 1e6
    seq.append((short, v))
for s, v in seq:
    print(f"{s:45s} {v/1e3:12.1f} us")
