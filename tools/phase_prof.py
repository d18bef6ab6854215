"""Per-phase clock64 totals of the light tile kernel (library built with SPG_NVCC_FLAGS=-DSPG_PHASE_PROF)."""
import ctypes
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import paper_conf_ipps_ramamoorthybsk15_b200 as spg  # noqa: E402
import workloads as W  # noqa: E402

lib = ctypes.CDLL(os.path.join(ROOT, "paper_conf_ipps_ramamoorthybsk15_b200", "libspg.so"))
A, B = W.make(sys.argv[1] if len(sys.argv) > 1 else "webbase1m")
dA = spg.DeviceCSR.from_host(A, "cuda")
plan = spg.SpGEMM(0, torch.float64)
for _ in range(3):
    plan(dA, dA)
torch.cuda.synchronize()
buf = (ctypes.c_ulonglong * 16)()
lib.spg_debug_phase_clk(buf, 1)
for _ in range(5):
    plan(dA, dA)
torch.cuda.synchronize()
lib.spg_debug_phase_clk(buf, 0)
names = ["collect", "rows", "expand", "bad check", "bucket scan", "scatter", "heads", "ranks", "between batches"]
tot = sum(buf[i] for i in range(9))
for i, n in enumerate(names):
    print(f"{n:16s} {buf[i] / tot * 100:5.1f}%")
