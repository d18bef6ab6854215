#!/usr/bin/env python
"""alpha sweep (Fig. 10): C = A.B for two distinct Chung-Lu
power-law matrices with the same exponent alpha, n = 100K / 500K / 1M rows, alpha 3.0 .. 6.5.
Times symbolic + numeric with the heavy/light split (default thresholds) and with a single path
(every non-empty row through one kernel: FORCE_CLASS = HUGE, the uncached bitmap kernel — the
T_light = infinity extreme of P:L233 that the paper compares against [13]), checks that both
give the same C, and reports the split's speedup.

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
    for n in [int(x) for x in a.sizes.split(",")]:
        for al in [float(x) for x in a.alphas.split(",")]:
            # average degree 8, caps 2000, correlated hubs (sigma 6), two seeds: A != B
            A = W.chung_lu(n, n, al, 8 * n, 2000.0, 2000.0, 6.0, 1.1, 101)
            B = W.chung_lu(n, n, al, 8 * n, 2000.0, 2000.0, 6.0, 1.1, 202)
            dA = spg.DeviceCSR.from_host(A, "cuda")
            dB = spg.DeviceCSR.from_host(B, "cuda")
            ts, tn, st, dig = time_plan(dA, dB, a.steps)
            ts1, tn1, st1, dig1 = time_plan(dA, dB, a.steps, force_class=6)
            F = st["flops"]
            line = {"n": n, "alpha": al, "nnzA": A.nnz, "nnzB": B.nnz, "flops": F, "nnzC": dig[0],
                    "split_ms": ts + tn, "single_path_ms": ts1 + tn1,
                    "split_gflops": 2 * F / ((ts + tn) * 1e-3) / 1e9,
                    "speedup": (ts1 + tn1) / (ts + tn),
                    "same_result": dig[0] == dig1[0] and dig[2] == dig1[2] and abs(dig[1] - dig1[1]) <= 1e-9 * abs(dig[1]),
                    "class_rows": st["class_rows"]}
            print(json.dumps(line), flush=True)
            if a.out:
                with open(a.out, "a") as fh:
                    fh.write(json.dumps(line) + "\n")
            del dA, dB
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
