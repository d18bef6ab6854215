"""Per-launch DRAM traffic of the numeric phase (k_numeric) from an ncu launch list
(tools/round_capture.sh metrics) -> <out dir>/traffic_<config>.json (copied to profiles/, where
bench.py reads it).   python tools/traffic.py launches.csv webbase1m [out_dir]"""
import csv
import json
import re
import sys
from collections import defaultdict

src, config = sys.argv[1], sys.argv[2]
rows = list(csv.reader(open(src)))
hi = next(i for i, r in enumerate(rows) if 'Kernel Name' in r)
h = rows[hi]
ki, mi, vi, ii = h.index('Kernel Name'), h.index('Metric Name'), h.index('Metric Value'), h.index('ID')
per = defaultdict(lambda: defaultdict(float))
for r in rows[hi + 1:]:
    per[(int(r[ii]), re.sub(r'\(.*', '', r[ki]))][r[mi]] = float(r[vi].replace(',', ''))
num = [(k, m) for k, m in sorted(per.items()) if re.search(r'k_numeric|k_pack_b', k[1])]
main = [m for k, m in num if re.search(r'k_numeric<', k[1])]
n = len(main)
tot = sum(m['dram__bytes_read.sum'] + m['dram__bytes_write.sum'] for _, m in num)
out = {"numeric_dram_bytes_per_launch": tot / n, "launches": n, "source": src,
       "kernels": sorted({k[1] for k, _ in num}),
       "how": "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum --clock-control none, python bench.py --profile"}
odir = sys.argv[3] if len(sys.argv) > 3 else "profiles"
json.dump(out, open(f"{odir}/traffic_{config}.json", "w"), indent=1)
print(json.dumps(out))
