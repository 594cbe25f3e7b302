"""Summarise an ncu --metrics gpu__time_duration.sum CSV launch list."""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
h = next(i for i, r in enumerate(rows) if 'Kernel Name' in r)
H = rows[h]; ki, vi = H.index('Kernel Name'), H.index('Metric Value')
gi = H.index('Grid Size') if 'Grid Size' in H else None
agg = collections.OrderedDict()
for r in rows[h + 1:]:
    k = r[ki].split('(CUtensor')[0][:60] + (' ' + r[gi] if gi is not None else '')
    a = agg.setdefault(k, [0, 0.0])
    a[0] += 1; a[1] += float(r[vi].replace(',', ''))
tot = sum(v[1] for v in agg.values())
for k, (n, t) in agg.items():
    print(f"{n:4d} {t/n/1000:9.2f} us/launch {100*t/tot:5.1f}%  {k}")
