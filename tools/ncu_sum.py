"""Per-kernel summary of an ncu --csv --metrics launch list (time, DRAM bytes, warp instructions)."""
import csv
import re
import sys
from collections import OrderedDict

rows = list(csv.reader(open(sys.argv[1])))
hi = next(i for i, r in enumerate(rows) if 'Kernel Name' in r)
h = rows[hi]
ki, mi, vi, ii = h.index('Kernel Name'), h.index('Metric Name'), h.index('Metric Value'), h.index('ID')
d = OrderedDict()
for r in rows[hi + 1:]:
    name = re.sub(r'\(spg::.*|\(int, const.*|\(const .*|\(long long.*|\(unsigned.*', '', r[ki]).replace('void ', '')[:58]
    d.setdefault((r[ii], name), {})[r[mi]] = float(r[vi].replace(',', ''))
agg = OrderedDict()
for (_, n), m in d.items():
    a = agg.setdefault(n, [0, 0.0, 0.0, 0.0, 0.0])
    a[0] += 1
    a[1] += m.get('gpu__time_duration.sum', 0)
    a[2] += m.get('dram__bytes_read.sum', 0)
    a[3] += m.get('dram__bytes_write.sum', 0)
    a[4] += m.get('smsp__inst_executed.sum', 0)
tot = sum(a[1] for a in agg.values())
for n, a in agg.items():
    c = a[0]
    print(f"{n:58s} n={c:2d} t={a[1]/c/1e3:8.1f}us share={a[1]/tot*100:5.1f}% rd={a[2]/c/1e6:7.1f}MB "
          f"wr={a[3]/c/1e6:7.1f}MB inst={a[4]/c/1e6:7.1f}M")
