"""Per-CUDA-source-line summary of an ncu report: warp-stall samples and instructions executed.
ncu -i rep --page source --csv --print-source cuda,sass > x.csv; python tools/ncu_src.py x.csv [top]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1], errors="replace")))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
cur, hdr, out = None, None, []
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        cur = r[1].split("/")[-1]
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or r[0] == "Function Name" or not r[0].isdigit():
        continue
    try:
        s = int(r[hdr.index("Warp Stall Sampling (All Samples)")] or 0)
        n = int(r[hdr.index("Instructions Executed")] or 0)
    except ValueError:
        continue
    out.append((s, n, f"{cur}:{r[0]}", r[1].strip()[:90]))
ts = sum(x[0] for x in out) or 1
tn = sum(x[1] for x in out) or 1
print(f"samples {ts}  warp-instructions {tn}")
for s, n, loc, src in sorted(out, reverse=True)[:top]:
    print(f"{100*s/ts:5.1f}% stall  {100*n/tn:5.1f}% inst  {loc:18s} {src}")
