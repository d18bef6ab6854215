"""Seeded synthetic workloads (input recipe only — no SpGEMM arithmetic lives here).

Shared by `oracle` tests, GPU parity tests and `bench.py`; see DESIGN.md §3 for the
recipe and why each config has the shape it has.  The generators are C++
(`gen.cpp`, built in-tree into `libspg_workloads.so`) so that the 134M-entry R-MAT
config is produced in seconds; every draw is a pure function of (seed, stream,
index), so the matrices are identical on every machine and thread count.

Configs mirror BASELINE.json `configs` (0-based):
  [0] cl10k       Chung-Lu 10k x 10k, alpha 2.1, ~50k nnz, fp64
  [1] webbase1m   webbase-1M shape (Table I): 1,000,005 rows, 3.1M nnz, alpha 2.1, fp64
  [2] webgoogle   web-Google shape: 916,428 rows, 5.1M nnz, alpha 3.75, fp64
      citpatents  cit-Patents shape: 3,774,768 rows, 16.5M nnz, alpha 3.90, fp64
  [3] ab2m        C = A.B, two 2M-row power-law matrices with different exponents, fp32
  [4] rmat23      R-MAT scale 23, edge factor 16, GTgraph defaults, fp64
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "libspg_workloads.so")
_SRC = os.path.join(_HERE, "gen.cpp")
_lib = None


def build() -> str:
    """Compile gen.cpp -> libspg_workloads.so (in-tree) if missing or stale."""
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["g++", "-O3", "-std=c++17", "-shared", "-fPIC", "-pthread", _SRC, "-o", tmp])
        os.replace(tmp, _SO)
    return _SO


def _load():
    global _lib
    if _lib is None:
        lib = ctypes.CDLL(build())
        lib.wl_chung_lu.restype = ctypes.c_void_p
        lib.wl_chung_lu.argtypes = [ctypes.c_int32, ctypes.c_int32, ctypes.c_double, ctypes.c_double,
                                    ctypes.c_int64, ctypes.c_double, ctypes.c_double, ctypes.c_double,
                                    ctypes.c_double, ctypes.c_uint64]
        lib.wl_rmat.restype = ctypes.c_void_p
        lib.wl_rmat.argtypes = [ctypes.c_int32, ctypes.c_int32, ctypes.c_double, ctypes.c_double,
                                ctypes.c_double, ctypes.c_uint64]
        lib.wl_sizes.argtypes = [ctypes.c_void_p, ctypes.POINTER(ctypes.c_int32),
                                 ctypes.POINTER(ctypes.c_int32), ctypes.POINTER(ctypes.c_int64)]
        lib.wl_copy.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int]
        lib.wl_free.argtypes = [ctypes.c_void_p]
        _lib = lib
    return _lib


@dataclass
class CSR:
    """0-based CSR with int32 indices (host numpy arrays)."""
    nrows: int
    ncols: int
    row_ptr: np.ndarray  # int32[nrows+1]
    col_idx: np.ndarray  # int32[nnz]
    vals: np.ndarray     # float64 or float32 [nnz]

    @property
    def nnz(self) -> int:
        return int(self.col_idx.shape[0])

    @property
    def dtype(self):
        return self.vals.dtype


def _extract(h, dtype) -> CSR:
    lib = _load()
    nr, nc, nnz = ctypes.c_int32(), ctypes.c_int32(), ctypes.c_int64()
    lib.wl_sizes(h, ctypes.byref(nr), ctypes.byref(nc), ctypes.byref(nnz))
    rp = np.empty(nr.value + 1, np.int32)
    ci = np.empty(nnz.value, np.int32)
    dt = np.dtype(dtype)
    va = np.empty(nnz.value, dt)
    lib.wl_copy(h, rp.ctypes.data, ci.ctypes.data, va.ctypes.data, 1 if dt == np.float64 else 0)
    lib.wl_free(h)
    return CSR(nr.value, nc.value, rp, ci, va)


def chung_lu(n_rows: int, n_cols: int, alpha: float, nnz: int, row_cap: float, col_cap: float,
             sigma: float, m_factor: float, seed: int, dtype=np.float64, alpha_c: float | None = None) -> CSR:
    """Chung-Lu power-law matrix. sigma < 0 = independent column ranks."""
    h = _load().wl_chung_lu(n_rows, n_cols, alpha, alpha if alpha_c is None else alpha_c, nnz,
                            row_cap, col_cap, sigma, m_factor, seed)
    return _extract(h, dtype)


def rmat(scale: int, edge_factor: int = 16, a: float = 0.45, b: float = 0.15, c: float = 0.15,
         seed: int = 7, dtype=np.float64) -> CSR:
    """R-MAT with GTgraph default quadrant probabilities (a,b,c,d)=(.45,.15,.15,.25) ([3])."""
    return _extract(_load().wl_rmat(scale, edge_factor, a, b, c, seed), dtype)


def random_csr(nrows: int, ncols: int, density: float, seed: int, dtype=np.float64,
               values: str = "uniform12", canonical: bool = True, empty_row_frac: float = 0.0) -> CSR:
    """Small uniformly-random CSR for tests (numpy RNG, seeded).

    values: "uniform12" -> U[1,2);  "int" -> small signed integers in [-8, 8] (exact sums);
            "int_pos" -> integers in [1, 8].
    canonical=False keeps duplicate (row, col) draws and shuffles columns inside rows.
    """
    rng = np.random.default_rng(seed)
    nnz = int(round(nrows * ncols * density))
    rows = rng.integers(0, max(nrows, 1), nnz) if nrows > 0 else np.zeros(0, np.int64)
    cols = rng.integers(0, max(ncols, 1), nnz) if ncols > 0 else np.zeros(0, np.int64)
    if empty_row_frac > 0 and nrows > 0:
        dead = rng.random(nrows) < empty_row_frac
        keep = ~dead[rows]
        rows, cols = rows[keep], cols[keep]
    if canonical:
        key = np.unique(rows.astype(np.int64) * max(ncols, 1) + cols)
        rows, cols = key // max(ncols, 1), key % max(ncols, 1)
    else:
        order = np.argsort(rows, kind="stable")
        rows, cols = rows[order], cols[order]
    counts = np.bincount(rows, minlength=nrows) if nrows > 0 else np.zeros(0, np.int64)
    rp = np.zeros(nrows + 1, np.int32)
    rp[1:] = np.cumsum(counts)
    n = rows.shape[0]
    if values == "uniform12":
        v = 1.0 + rng.random(n)
    elif values == "int":
        v = rng.integers(-8, 9, n).astype(np.float64)
    elif values == "int_pos":
        v = rng.integers(1, 9, n).astype(np.float64)
    else:
        raise ValueError(values)
    return CSR(nrows, ncols, rp, cols.astype(np.int32), v.astype(dtype))


# --- BASELINE.json configs ----------------------------------------------------------------
# Parameters and their provenance are tabulated in DESIGN.md §3.
CONFIGS = {
    "cl10k": dict(kind="chung_lu", n=10_000, alpha=2.1, nnz=50_000, row_cap=2000, col_cap=2000,
                  sigma=6.0, m_factor=1.13, seed=1, dtype="float64"),
    "webbase1m": dict(kind="chung_lu", n=1_000_005, alpha=2.1, nnz=3_105_536, row_cap=4700, col_cap=30000,
                      sigma=5.15, m_factor=1.055, seed=2, dtype="float64"),
    "webgoogle": dict(kind="chung_lu", n=916_428, alpha=3.75, nnz=5_105_039, row_cap=500, col_cap=7000,
                      sigma=6.0, m_factor=1.01, seed=2, dtype="float64"),
    "citpatents": dict(kind="chung_lu", n=3_774_768, alpha=3.90, nnz=16_518_948, row_cap=800, col_cap=3200,
                       sigma=6.0, m_factor=1.01, seed=2, dtype="float64"),
    "ab2m": dict(kind="ab", n=2_000_000, dtype="float32",
                 A=dict(alpha=2.1, nnz=8_000_000, row_cap=5000, col_cap=30000, sigma=-1.0, m_factor=1.0, seed=11),
                 B=dict(alpha=3.0, nnz=16_000_000, row_cap=2000, col_cap=2000, sigma=-1.0, m_factor=1.0, seed=12)),
    "rmat23": dict(kind="rmat", scale=23, edge_factor=16, a=0.45, b=0.15, c=0.15, seed=7, dtype="float64"),
}
CONFIG_ORDER = ["cl10k", "webbase1m", "webgoogle", "citpatents", "ab2m", "rmat23"]


def make(name: str):
    """Return (A, B) for a named config; for C = A.A configs, B is A (same object)."""
    cfg = CONFIGS[name]
    dt = np.dtype(cfg["dtype"])
    if cfg["kind"] == "chung_lu":
        A = chung_lu(cfg["n"], cfg["n"], cfg["alpha"], cfg["nnz"], cfg["row_cap"], cfg["col_cap"],
                     cfg["sigma"], cfg["m_factor"], cfg["seed"], dt)
        return A, A
    if cfg["kind"] == "rmat":
        A = rmat(cfg["scale"], cfg["edge_factor"], cfg["a"], cfg["b"], cfg["c"], cfg["seed"], dt)
        return A, A
    if cfg["kind"] == "ab":
        n = cfg["n"]
        mats = []
        for key in ("A", "B"):
            p = cfg[key]
            mats.append(chung_lu(n, n, p["alpha"], p["nnz"], p["row_cap"], p["col_cap"], p["sigma"],
                                 p["m_factor"], p["seed"], dt))
        return mats[0], mats[1]
    raise ValueError(name)
