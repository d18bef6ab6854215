#!/usr/bin/env python
"""Ablations (Fig. 9): the same C = A.A with parts of the
design switched off, each checked to give the same C.

  default          heavy/light split, SINGLE shortcut, concurrent streams
  no_single        FORCE_CLASS = LIGHT: SINGLE rows sorted like any light row
  no_tiles         LIGHT_MAX_FLOPS = 0: every row on the heavy (bitmap) path
  heavy_path_only  FORCE_CLASS = HEAVY: every row through the cached bitmap when it fits
  single_path      FORCE_CLASS = HUGE: every row through the uncached bitmap (one kernel, rows
                   in queue order: the GPU analogue of the paper's Unsorted-Workqueue)
  warp_rows        WARP_MAX_FLOPS = 256: light rows <= 256 flops one warp per row
  serial           CONCURRENT = 0: class kernels one after another on one stream

  python tools/ablation.py [--config webbase1m] [--steps 10] [--out profiles/r01_ablation.jsonl]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))

import paper_conf_ipps_ramamoorthybsk15_b200 as spg  # noqa: E402
import workloads as W  # noqa: E402
from sweep import time_plan  # noqa: E402

VARIANTS = {
    "default": {},
    "no_single": {"force_class": 3},
    "no_tiles": {"light_max_flops": 0},
    "heavy_path_only": {"force_class": 5},
    "single_path": {"force_class": 6},
    "warp_rows": {"warp_max_flops": 256},
    "serial": {"concurrent": 0},
}


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--config", default="webbase1m")
    p.add_argument("--steps", type=int, default=10)
    p.add_argument("--out", default=None)
    a = p.parse_args()
    A, B = W.make(a.config)
    dA = spg.DeviceCSR.from_host(A, "cuda")
    dB = dA if B is A else spg.DeviceCSR.from_host(B, "cuda")
    ref = None
    for name, opts in VARIANTS.items():
        ts, tn, st, dig = time_plan(dA, dB, a.steps, **opts)
        ref = ref or dig
        F = st["flops"]
        line = {"config": a.config, "variant": name, "options": opts, "symbolic_ms": ts, "numeric_ms": tn,
                "gflops": 2 * F / ((ts + tn) * 1e-3) / 1e9, "class_rows": st["class_rows"],
                "same_result": dig[0] == ref[0] and dig[2] == ref[2] and abs(dig[1] - ref[1]) <= 1e-9 * abs(ref[1])}
        print(json.dumps(line), flush=True)
        if a.out:
            with open(a.out, "a") as fh:
                fh.write(json.dumps(line) + "\n")


if __name__ == "__main__":
    main()
