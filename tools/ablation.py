#!/usr/bin/env python
"""Ablations (Fig. 9): the same C = A.A with parts of the
design switched off or replaced, every variant checked to give the default's C (the default
itself is checked against the oracle in tests/test_gpu_parity.py).

  default              heavy/light split: tiles for light rows, bitmap blocks for heavy rows
  no_single            FORCE_CLASS = LIGHT: rows with one non-empty B row sorted like any other
  max_tiles            LIGHT_MAX_FLOPS = 4096, TILE_FLOPS = 1024: every row that fits a tile is
                       sorted in tiles (the strongest light-kernel-only configuration)
  block_per_row        FORCE_CLASS = HEAVY: every row through a block with a dense bitmap — the
                       GPU analogue of [13]'s warp-per-row dense PartialOutput,
                       i.e. one path for all rows
  unsorted_workqueue   FORCE_CLASS = HUGE, HEAVY_ORDER = 0: one kernel, rows dequeued in natural
                       order (the paper's Unsorted-Workqueue, L251)
  sorted_workqueue     FORCE_CLASS = HUGE, HEAVY_ORDER = 2: one kernel, rows dequeued largest
                       first (the paper's Sorted-Workqueue: rows by size, no class kernels, L253)
  serial               CONCURRENT = 0: class kernels one after another on one stream
  autotune             AUTOTUNE = 1: thresholds timed on the first call (f1)
  csrmm_*              sparse x dense A x D (n = 64): split (default 256 stored entries) vs
                       every row a warp (light_nnz = inf) vs every row a block (light_nnz = 0)

  python tools/ablation.py [--config webbase1m] [--steps 10] [--out profiles/r02_ablation.jsonl]
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

VARIANTS = {
    "default": {},
    "no_single": {"force_class": 3},
    "max_tiles": {"light_max_flops": 4096, "tile_flops": 1024},
    "block_per_row": {"force_class": 5},
    "unsorted_workqueue": {"force_class": 6, "heavy_order": 0},
    "sorted_workqueue": {"force_class": 6, "heavy_order": 2},
    "serial": {"concurrent": 0},
    "autotune": {"autotune": 1},
}


def emit(line, out):
    print(json.dumps(line), flush=True)
    if out:
        with open(out, "a") as fh:
            fh.write(json.dumps(line) + "\n")


def time_csrmm(dA, D, steps, light):
    h = spg.spg_create(0, None, dA.vals.dtype)
    spg.spg_set_option(h, "csrmm_light_nnz", light)
    C = torch.empty(dA.nrows, D.shape[1], dtype=D.dtype, device="cuda")
    ts = []
    for s in range(steps + 2):
        e = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
        e[0].record()
        spg.spg_csrmm(h, dA, D, C)
        e[1].record()
        torch.cuda.synchronize()
        if s >= 2:
            ts.append(e[0].elapsed_time(e[1]))
    spg.spg_spgemm_free(h)
    return float(np.median(ts)), float(C.double().sum().item())


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--config", default="webbase1m")
    p.add_argument("--steps", type=int, default=10)
    p.add_argument("--skip", default="", help="comma-separated variants to skip (slow ones on big configs)")
    p.add_argument("--out", default=None)
    a = p.parse_args()
    skip = set(a.skip.split(",")) if a.skip else set()
    A, B = W.make(a.config)
    dA = spg.DeviceCSR.from_host(A, "cuda")
    dB = dA if B is A else spg.DeviceCSR.from_host(B, "cuda")
    ref = None
    for name, opts in VARIANTS.items():
        if name in skip:
            continue
        ts, tn, st, dig = time_plan(dA, dB, a.steps, **opts)
        ref = ref or dig
        F = st["flops"]
        emit({"config": a.config, "variant": name, "options": opts, "symbolic_ms": ts, "numeric_ms": tn,
              "gflops": 2 * F / ((ts + tn) * 1e-3) / 1e9, "class_rows": st["class_rows"],
              "light_max": st["light_max"], "tile_flops": st["tile_flops"],
              "same_result": dig[0] == ref[0] and dig[2] == ref[2] and abs(dig[1] - ref[1]) <= 1e-9 * abs(ref[1])},
             a.out)
    # sparse x dense: the heavy/light split of rows by stored entries
    n = 64
    D = torch.rand(A.ncols, n, dtype=dA.vals.dtype, device="cuda") + 1.0
    nnz_flops = 2.0 * A.nnz * n
    base = None
    for name, light in [("csrmm_split", 256), ("csrmm_warp_per_row", 1 << 30), ("csrmm_block_per_row", 0)]:
        t, dig = time_csrmm(dA, D, a.steps, light)
        base = base or dig
        emit({"config": a.config, "variant": name, "n": n, "light_nnz": light, "ms": t,
              "gflops": nnz_flops / (t * 1e-3) / 1e9, "same_result": abs(dig - base) <= 1e-9 * abs(base)}, a.out)


if __name__ == "__main__":
    main()
