"""Oracle — TEST INFRASTRUCTURE ONLY (see oracle.cpp header).

Plain CPU reference for C = A x B (Row-Row / Gustavson formulation, PAPER.md L62;
like-tuple addition and sorted output).  Only `tests/`,
`__graft_entry__.smoke()` and `bench.py`'s cpu_baseline / `--impl reference` legs may
import this package.  It shares no code with `paper_conf_ipps_ramamoorthybsk15_b200`.

Every function here is pinned by `tests/test_oracle.py` (no function is "parity unpinned").
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.cpp")
_lib = None

_P = ctypes.c_void_p
_I32 = ctypes.c_int32


def build() -> str:
    """Compile oracle.cpp -> liboracle.so in-tree (plain g++, no CUDA)."""
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-pthread", _SRC, "-o", tmp])
        os.replace(tmp, _SO)
    return _SO


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        lib.orc_row_flops.argtypes = [_I32, _P, _P, _P, _P]
        lib.orc_bins.argtypes = [_I32, _P, _P, _P]
        lib.orc_split_points.argtypes = [_I32, _P, _I32, _P]
        common = [_I32, _I32, _I32, _P, _P, _P, _I32, _P, _P, _P, ctypes.c_int]
        lib.orc_spgemm_count.argtypes = common + [_P, ctypes.c_int]
        lib.orc_spgemm_fill.argtypes = common + [_P, _P, _P, _P, ctypes.c_int]
        lib.orc_csrmm.argtypes = [_I32, _P, _P, _P, ctypes.c_int, _P, ctypes.c_int64, _P, _P]
        _lib = lib
    return _lib


def _c(a, dt):
    return np.ascontiguousarray(a, dtype=dt)


def row_flops(A, B) -> np.ndarray:
    """f_i (int64) = number of intermediate products of row i."""
    lib = _load()
    rpA, colA, rpB = _c(A.row_ptr, np.int32), _c(A.col_idx, np.int32), _c(B.row_ptr, np.int32)
    f = np.empty(A.nrows, np.int64)
    lib.orc_row_flops(A.nrows, rpA.ctypes.data, colA.ctypes.data, rpB.ctypes.data, f.ctypes.data)
    return f


def bins(f: np.ndarray):
    """(bin int32[M], hist int64[65]); bin = -1 for f = 0 else ceil(log2 f); hist[b+1] = #rows in bin b."""
    lib = _load()
    f = _c(f, np.int64)
    b = np.empty(f.shape[0], np.int32)
    h = np.zeros(65, np.int64)
    lib.orc_bins(f.shape[0], f.ctypes.data, b.ctypes.data, h.ctypes.data)
    return b, h


def split_points(f: np.ndarray, P: int) -> np.ndarray:
    """Flop-balanced row split points s[0..P]."""
    lib = _load()
    f = _c(f, np.int64)
    s = np.empty(P + 1, np.int32)
    lib.orc_split_points(f.shape[0], f.ctypes.data, P, s.ctypes.data)
    return s


def _args(A, B, r0, r1):
    assert A.ncols == B.nrows, "dimension mismatch"
    is64 = 1 if np.dtype(A.vals.dtype) == np.float64 else 0
    vdt = np.float64 if is64 else np.float32
    arrs = [_c(A.row_ptr, np.int32), _c(A.col_idx, np.int32), _c(A.vals, vdt),
            _c(B.row_ptr, np.int32), _c(B.col_idx, np.int32), _c(B.vals, vdt)]
    args = [r0, r1, A.nrows, arrs[0].ctypes.data, arrs[1].ctypes.data, arrs[2].ctypes.data,
            B.nrows, arrs[3].ctypes.data, arrs[4].ctypes.data, arrs[5].ctypes.data, is64]
    return args, arrs


def spgemm_count(A, B, r0: int = 0, r1: int | None = None, nthreads: int = 1) -> np.ndarray:
    """c_i = nnz of row i of C for rows [r0, r1) (int64)."""
    r1 = A.nrows if r1 is None else r1
    args, keep = _args(A, B, r0, r1)
    c = np.empty(r1 - r0, np.int64)
    _load().orc_spgemm_count(*args, c.ctypes.data, nthreads)
    return c


def spgemm(A, B, r0: int = 0, r1: int | None = None, nthreads: int = 1, with_abs: bool = True):
    """C rows [r0, r1) as (row_ptr int64[r1-r0+1] starting at 0, col int32, val float64, abs float64|None)."""
    r1 = A.nrows if r1 is None else r1
    c = spgemm_count(A, B, r0, r1, nthreads)
    rp = np.zeros(r1 - r0 + 1, np.int64)
    np.cumsum(c, out=rp[1:])
    nnz = int(rp[-1])
    col = np.empty(nnz, np.int32)
    val = np.empty(nnz, np.float64)
    ab = np.empty(nnz, np.float64) if with_abs else None
    args, keep = _args(A, B, r0, r1)
    _load().orc_spgemm_fill(*args, rp.ctypes.data, col.ctypes.data, val.ctypes.data,
                            ab.ctypes.data if with_abs else None, nthreads)
    return rp, col, val, ab


def csrmm(A, D: np.ndarray):
    """Sparse x dense C = A x D (PAPER.md L289's CSTMM): (C float64 [M, n], abs float64 [M, n])."""
    D = np.ascontiguousarray(D, dtype=np.float64)
    assert D.ndim == 2 and D.shape[0] == A.ncols, "dimension mismatch"
    is64 = 1 if np.dtype(A.vals.dtype) == np.float64 else 0
    vdt = np.float64 if is64 else np.float32
    rp, ci, v = _c(A.row_ptr, np.int32), _c(A.col_idx, np.int32), _c(A.vals, vdt)
    n = D.shape[1]
    C = np.empty((A.nrows, n), np.float64)
    ab = np.empty((A.nrows, n), np.float64)
    _load().orc_csrmm(A.nrows, rp.ctypes.data, ci.ctypes.data, v.ctypes.data, is64, D.ctypes.data, n,
                      C.ctypes.data, ab.ctypes.data)
    return C, ab
