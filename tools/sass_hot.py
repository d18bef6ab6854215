"""Hot spots of an `ncu --page source --csv --print-source sass` export: instructions executed and
stall samples per contiguous SASS block (split at branch targets / labels), largest first."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
ia, isrc, ist, iex = h.index("Address"), h.index("Source"), h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
ins = [(r[ia], r[isrc].strip(), int(r[ist] or 0), int(r[iex] or 0)) for r in rows[2:] if len(r) > iex and r[iex].isdigit()]
tot_ex = sum(x[3] for x in ins)
tot_st = sum(x[2] for x in ins)
print(f"total instructions executed {tot_ex/1e6:.1f}M, stall samples {tot_st}")
# group consecutive instructions with the same execution count (basic blocks)
blocks = []
for k, x in enumerate(ins):
    if blocks and blocks[-1]["ex"] == x[3]:
        blocks[-1]["n"].append(k)
    else:
        blocks.append({"ex": x[3], "n": [k]})
for b in blocks:
    b["tot"] = b["ex"] * len(b["n"])
    b["st"] = sum(ins[k][2] for k in b["n"])
top = sorted(blocks, key=lambda b: -b["tot"])[: int(sys.argv[2]) if len(sys.argv) > 2 else 12]
for b in top:
    k0 = b["n"][0]
    print(f"--- block @{k0} len {len(b['n'])} exec/inst {b['ex']/1e6:.2f}M total {b['tot']/1e6:.1f}M ({100*b['tot']/tot_ex:.1f}%) stalls {b['st']} ({100*b['st']/max(tot_st,1):.1f}%)")
    for k in b["n"][:60]:
        print(f"   {k:5d} {ins[k][1][:90]:90s} st={ins[k][2]}")
