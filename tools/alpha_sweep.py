#!/usr/bin/env python
"""alpha sweep (Fig. 10): C = A.B for two distinct Chung-Lu
power-law matrices with the same exponent alpha, n = 100K / 500K / 1M rows, alpha 3.0 .. 6.5.
Times symbolic + numeric with the heavy/light split (default thresholds) and two single-kernel
baselines — every row through a block-per-row bitmap (FORCE_CLASS = HEAVY: the GPU analogue of
[13]'s dense per-row accumulator, the one-path extreme of P:L233 the paper compares against) and
every row that fits through the tile kernel (LIGHT_MAX = 4096, the strongest light-only setting)
— checks that all give the same C (the default is oracle-checked in tests/), and reports the
split's speedup over the better baseline.  Fig. 10's claim: the gain falls as alpha
grows (fewer heavy rows); the summary line fits speedup vs alpha per size.

  python tools/alpha_sweep.py [--steps 5] [--out profiles/r01_alpha_sweep.jsonl]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_ramamoorthybsk15_b200 as spg  # noqa: E402
import workloads as W  # noqa: E402
from sweep import time_plan  # noqa: E402


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--steps", type=int, default=5)
    p.add_argument("--out", default=None)
    p.add_argument("--sizes", default="100000,500000,1000000")
    p.add_argument("--alphas", default="3.0,3.5,4.0,4.5,5.0,5.5,6.0,6.5")
    a = p.parse_args()
    rows = []
    for n in [int(x) for x in a.sizes.split(",")]:
        for al in [float(x) for x in a.alphas.split(",")]:
            # average degree 8, caps 2000, correlated hubs (sigma 6), two seeds: A != B
            A = W.chung_lu(n, n, al, 8 * n, 2000.0, 2000.0, 6.0, 1.1, 101)
            B = W.chung_lu(n, n, al, 8 * n, 2000.0, 2000.0, 6.0, 1.1, 202)
            dA = spg.DeviceCSR.from_host(A, "cuda")
            dB = spg.DeviceCSR.from_host(B, "cuda")
            ts, tn, st, dig = time_plan(dA, dB, a.steps)
            ts1, tn1, st1, dig1 = time_plan(dA, dB, a.steps, force_class=5)
            ts2, tn2, st2, dig2 = time_plan(dA, dB, a.steps, light_max_flops=4096, tile_flops=1024)
            F = st["flops"]
            same = all(d[0] == dig[0] and d[2] == dig[2] and abs(d[1] - dig[1]) <= 1e-9 * abs(dig[1]) for d in (dig1, dig2))
            best_single = min(ts1 + tn1, ts2 + tn2)
            line = {"n": n, "alpha": al, "nnzA": A.nnz, "nnzB": B.nnz, "flops": F, "nnzC": dig[0],
                    "split_ms": ts + tn, "block_per_row_ms": ts1 + tn1, "max_tiles_ms": ts2 + tn2,
                    "split_gflops": 2 * F / ((ts + tn) * 1e-3) / 1e9,
                    "speedup_vs_block_per_row": (ts1 + tn1) / (ts + tn),
                    "speedup_vs_best_single": best_single / (ts + tn),
                    "same_result": same, "class_rows": st["class_rows"], "class_flops": st["class_flops"]}
            rows.append(line)
            print(json.dumps(line), flush=True)
            if a.out:
                with open(a.out, "a") as fh:
                    fh.write(json.dumps(line) + "\n")
            del dA, dB
            torch.cuda.empty_cache()
    for n in sorted({r["n"] for r in rows}):  # trend of the split's gain with alpha (Fig. 10)
        rs = [r for r in rows if r["n"] == n]
        x = np.array([r["alpha"] for r in rs])
        for key in ("speedup_vs_block_per_row", "speedup_vs_best_single"):
            y = np.array([r[key] for r in rs])
            slope = float(np.polyfit(x, y, 1)[0]) if len(rs) > 1 else 0.0
            line = {"summary": key, "n": n, "slope_per_alpha": slope, "falls_with_alpha": slope < 0}
            print(json.dumps(line), flush=True)
            if a.out:
                with open(a.out, "a") as fh:
                    fh.write(json.dumps(line) + "\n")


if __name__ == "__main__":
    main()
