#!/usr/bin/env python
"""Threshold sweep (Fig. 8): time symbolic + numeric of
C = A.A on a config for a grid of class thresholds, and check that C does not change.

  python tools/sweep.py [--config webbase1m] [--steps 10] [--out profiles/sweep.jsonl]
"""
import argparse
import itertools
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ipps_ramamoorthybsk15_b200 as spg  # noqa: E402
import workloads as W  # noqa: E402


def time_plan(dA, dB, steps, **opts):
    h = spg.spg_create(0, None, dA.vals.dtype)
    if "tile_flops" in opts and "light_max_flops" in opts:
        spg.spg_set_option(h, "light_max_flops", 0)  # light + tile <= TILE_PMAX after every call
    for k, v in opts.items():
        spg.spg_set_option(h, k, v)
    rp = torch.empty(dA.nrows + 1, dtype=torch.int64, device="cuda")
    nnz, _, _ = spg.spg_spgemm_symbolic(h, dA, dB, rp)
    col = torch.empty(max(nnz, 1), dtype=torch.int32, device="cuda")
    val = torch.empty(max(nnz, 1), dtype=dA.vals.dtype, device="cuda")
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    ts, tn = [], []
    for s in range(steps + 2):
        flush.zero_()
        e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        e[0].record()
        spg.spg_spgemm_symbolic(h, dA, dB, rp)
        e[1].record()
        spg.spg_spgemm_numeric(h, dA, dB, rp, col, val)
        e[2].record()
        torch.cuda.synchronize()
        if s >= 2:
            ts.append(e[0].elapsed_time(e[1]))
            tn.append(e[1].elapsed_time(e[2]))
    st = spg.spg_get_stats(h)
    digest = (int(rp[-1].item()), float(val[:nnz].double().sum().item()), int(col[:nnz].long().sum().item()))
    spg.spg_spgemm_free(h)
    return float(np.median(ts)), float(np.median(tn)), st, digest


LIGHT = [int(x) for x in os.environ.get("SWEEP_LIGHT", "0,256,512,1024,2048").split(",")]
TILE = [int(x) for x in os.environ.get("SWEEP_TILE", "1024,2048").split(",")]
HEAVY = [int(x) for x in os.environ.get("SWEEP_HEAVY", "4096,8192").split(",")]
PMAX = int(os.environ.get("SWEEP_PMAX", "6144"))


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--config", default="webbase1m")
    p.add_argument("--steps", type=int, default=10)
    p.add_argument("--out", default=None)
    p.add_argument("--concurrent", type=int, default=1)
    a = p.parse_args()
    A, B = W.make(a.config)
    dA = spg.DeviceCSR.from_host(A, "cuda")
    dB = dA if B is A else spg.DeviceCSR.from_host(B, "cuda")
    # (light_max, tile_flops, heavy_max): light rows (f <= light_max) go to the tile kernel,
    # light_max + tile_flops <= SWEEP_PMAX (rows above TILE_PMAX - tile_flops are solo tiles);
    # heavy rows up to heavy_max to the cached bitmap
    grid = [(lm, tf, hm) for lm in LIGHT for tf in TILE for hm in HEAVY if lm + tf <= PMAX]
    ref = None
    for lm, tf, hm in grid:
        ts, tn, st, dig = time_plan(dA, dB, a.steps, tile_flops=tf, light_max_flops=lm, heavy_max_flops=hm,
                                    concurrent=a.concurrent)
        ref = ref or dig
        F = st["flops"]
        line = {"config": a.config, "light_max": lm, "tile_flops": tf, "heavy_max": hm, "symbolic_ms": ts,
                "numeric_ms": tn, "gflops": 2 * F / ((ts + tn) * 1e-3) / 1e9, "class_rows": st["class_rows"],
                "same_result": dig[0] == ref[0] and dig[2] == ref[2] and abs(dig[1] - ref[1]) <= 1e-9 * abs(ref[1])}
        print(json.dumps(line), flush=True)
        if a.out:
            with open(a.out, "a") as fh:
                fh.write(json.dumps(line) + "\n")


if __name__ == "__main__":
    main()
