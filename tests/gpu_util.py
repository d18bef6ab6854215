"""Helpers for GPU parity tests: run the CUDA path through the C ABI and compare with the
oracle element by element (DESIGN.md §5 comparison rule)."""
from __future__ import annotations

import numpy as np
import torch

import oracle
import paper_conf_ipps_ramamoorthybsk15_b200 as spg

RTOL = {np.dtype(np.float64): 1e-12, np.dtype(np.float32): 1e-5}   # BASELINE.json north_star


def to_dev(M):
    return spg.DeviceCSR.from_host(M, "cuda")


def run_gpu(A, B, **opts):
    """Symbolic + numeric through the C ABI; returns host (row_ptr int64, col int32, val, stats)."""
    dA = to_dev(A)
    dB = dA if B is A else to_dev(B)
    then = opts.pop("_then", {})
    plan = spg.SpGEMM(0, dA.vals.dtype, **opts)
    for k, v in then.items():
        plan.set_option(k, v)
    try:
        C = plan(dA, dB)
        torch.cuda.synchronize()
        st = plan.stats()
        return (C.row_ptr.cpu().numpy(), C.col_idx.cpu().numpy(), C.vals.cpu().numpy(), st)
    finally:
        plan.close()


def compare(A, B, got, ref=None, exact_values=False, nthreads=8):
    rp, col, val = got[:3]
    if ref is None:
        ref = oracle.spgemm(A, B, nthreads=nthreads)
    orp, ocol, oval, oabs = ref
    np.testing.assert_array_equal(rp, orp, err_msg="C_row_ptr differs")
    np.testing.assert_array_equal(col, ocol, err_msg="C_col_idx differs")
    v = val.astype(np.float64)
    if exact_values:
        np.testing.assert_array_equal(v, oval, err_msg="values differ (exact expected)")
        return
    rtol = RTOL[np.dtype(A.vals.dtype)]
    err = np.abs(v - oval)
    bound = rtol * oabs
    bad = err > bound
    if bad.any():
        k = int(np.argmax(bad))
        raise AssertionError(f"{int(bad.sum())} values out of tolerance; first at {k}: gpu={v[k]!r} "
                             f"oracle={oval[k]!r} abs={oabs[k]!r} rtol={rtol}")
