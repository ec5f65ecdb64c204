"""Summarise an ncu --csv launch list (gpu__time_duration + dram bytes) per kernel for the last
timed tree (launches after the last k_grad).  Usage: launch_summary.py launches.csv [all]"""
import collections
import csv
import sys

lines = open(sys.argv[1]).read().splitlines()
start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
rows = list(csv.reader(lines[start:]))
h = rows[0]
iK, iM, iV, iID = h.index('Kernel Name'), h.index('Metric Name'), h.index('Metric Value'), h.index('ID')
d = collections.defaultdict(dict)
for r in rows[1:]:
    if len(r) < len(h):
        continue
    d[int(r[iID])][r[iM]] = float(r[iV].replace(',', ''))
    d[int(r[iID])]['name'] = r[iK]
ids = sorted(d)
grads = [i for i in ids if 'k_grad' in d[i]['name']]
start = 0 if (len(sys.argv) > 2 or not grads) else grads[-1]
agg = collections.OrderedDict()
for i in ids:
    if i < start:
        continue
    n = d[i]['name'].split('(')[0].replace('void ', '').split('::')[-1]
    a = agg.setdefault(n, [0, 0.0, 0.0])
    a[0] += 1
    a[1] += d[i].get('gpu__time_duration.sum', 0) / 1e6
    a[2] += d[i].get('dram__bytes_read.sum', 0) + d[i].get('dram__bytes_write.sum', 0)
tot = sum(a[1] for a in agg.values())
for n, a in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{n:34s} n={a[0]:4d} {a[1]:9.3f} ms {100 * a[1] / tot:5.1f}%  {a[2] / 1e9:8.2f} GB  "
          f"{a[2] / 1e9 / (a[1] / 1e3 + 1e-12):7.0f} GB/s")
print(f"total {tot:.3f} ms over {sum(a[0] for a in agg.values())} launches")
