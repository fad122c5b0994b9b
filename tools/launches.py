"""Summarise an ncu --metrics gpu__time_duration.sum launch list (csv)."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hi = [i for i, r in enumerate(rows) if 'Kernel Name' in r][0]
h = rows[hi]
ki, mi = h.index('Kernel Name'), h.index('Metric Value')
agg = collections.defaultdict(lambda: [0, 0.0])
tot = 0
seq = []
for r in rows[hi + 1:]:
    if len(r) <= mi:
        continue
    v = float(r[mi].replace(',', '')) / 1e3
    name = r[ki].split('(')[0].replace('void ', '')
    agg[name][0] += 1
    agg[name][1] += v
    tot += v
    seq.append((name, v))
print(f'total {tot:.1f} us over {len(seq)} launches')
for k, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1])[:int(sys.argv[2]) if len(sys.argv) > 2 else 25]:
    print(f'{k:48s} {c:5d} {t:10.1f} us {100 * t / tot:5.1f}%  avg {t / c:8.1f}')
