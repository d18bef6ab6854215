"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV) per kernel."""
import csv
import re
import sys
from collections import OrderedDict

rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if 'Kernel Name' in r)
h = rows[hi]
ki, vi, ui = h.index('Kernel Name'), h.index('Metric Value'), h.index('Metric Unit')
agg = OrderedDict()
for r in rows[hi + 1:]:
    name = re.sub(r'\(spg::Prob.*|\(int, const.*|\(const .*|\(long long.*', '', r[ki]).replace('void ', '')[:60]
    v = float(r[vi].replace(',', ''))
    scale = {'ns': 1e-3, 'us': 1, 'usecond': 1, 'msecond': 1e3, 'nsecond': 1e-3}.get(r[ui], 1)
    agg.setdefault(name, []).append(v * scale)
tot = sum(sum(v) for v in agg.values())
for k, v in agg.items():
    print(f"{k:62s} n={len(v):3d} avg={sum(v)/len(v):9.1f} us  share={sum(v)/tot*100:5.1f}%")
