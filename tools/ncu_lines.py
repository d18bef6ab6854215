"""Per-source-line instruction / stall summary from `ncu --page source --csv --print-source cuda,sass`."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 20
cur_file = cur_fn = hdr = None
agg = {}
for r in rows:
    if not r:
        continue
    if r[0] == 'File Path':
        cur_file = r[1].split('/')[-1]
        continue
    if r[0] == 'Function Name':
        cur_fn = r[1][:60]
        continue
    if r[0] == 'Line No':
        hdr = r
        ie = hdr.index('Instructions Executed')
        ti = hdr.index('Thread Instructions Executed')
        ws = hdr.index('Warp Stall Sampling (All Samples)')
        continue
    if hdr and r[0].isdigit() and r[2] == '-':
        key = (cur_fn, cur_file, int(r[0]), r[1][:80])
        a = agg.setdefault(key, [0, 0, 0])
        a[0] += float(r[ie] or 0)
        a[1] += float(r[ti] or 0)
        a[2] += float(r[ws] or 0)
for fn in sorted(set(k[0] for k in agg)):
    items = [(k, v) for k, v in agg.items() if k[0] == fn]
    tot = sum(v[0] for k, v in items)
    tots = sum(v[2] for k, v in items) or 1
    print("==", fn, "total warp inst %.1fM" % (tot / 1e6))
    for k, v in sorted(items, key=lambda kv: -kv[1][0])[:top]:
        print(f"  {k[1][:10]}:{k[2]:4d} inst {v[0]/tot*100:5.1f}% lanes {v[1]/max(v[0],1):5.1f} "
              f"stall {v[2]/tots*100:5.1f}%  {k[3]}")
