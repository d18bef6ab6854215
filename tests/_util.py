"""Test helpers: golden-file parsing and dense conversions (no SpGEMM arithmetic here)."""
from __future__ import annotations

import os

import numpy as np

from workloads import CSR

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def read_golden(name: str) -> dict:
    """Parse a golden text file: '#' comments, section headers (bare words), rows of numbers."""
    out, cur = {}, None
    with open(os.path.join(GOLDEN, name)) as fh:
        for line in fh:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            toks = line.split()
            try:
                row = [float(t) for t in toks]
            except ValueError:
                cur = line
                out[cur] = []
                continue
            out[cur].append(row)
    return {k: np.array(v) for k, v in out.items()}


def dense_to_csr(D: np.ndarray, dtype=np.float64) -> CSR:
    """Stored entries = nonzeros of D (row-major order, ascending columns)."""
    D = np.asarray(D)
    rows, cols = np.nonzero(D)
    rp = np.zeros(D.shape[0] + 1, np.int32)
    np.add.at(rp, rows + 1, 1)
    rp = np.cumsum(rp).astype(np.int32)
    return CSR(D.shape[0], D.shape[1], rp, cols.astype(np.int32), D[rows, cols].astype(dtype))


def csr_to_dense(M: CSR) -> np.ndarray:
    """Dense value matrix; duplicate stored entries are summed."""
    D = np.zeros((M.nrows, M.ncols), np.float64)
    rows = np.repeat(np.arange(M.nrows), np.diff(M.row_ptr))
    np.add.at(D, (rows, M.col_idx), M.vals.astype(np.float64))
    return D


def csr_pattern(M: CSR) -> np.ndarray:
    """Boolean matrix of stored positions (explicit zeros count as stored)."""
    P = np.zeros((M.nrows, M.ncols), bool)
    rows = np.repeat(np.arange(M.nrows), np.diff(M.row_ptr))
    P[rows, M.col_idx] = True
    return P


def identity(n: int, dtype=np.float64) -> CSR:
    return CSR(n, n, np.arange(n + 1, dtype=np.int32), np.arange(n, dtype=np.int32), np.ones(n, dtype))


def permutation_matrix(perm: np.ndarray, dtype=np.float64) -> CSR:
    """P with P[i, perm[i]] = 1, so (P.A)[i,:] = A[perm[i], :]."""
    n = perm.shape[0]
    return CSR(n, n, np.arange(n + 1, dtype=np.int32), perm.astype(np.int32), np.ones(n, dtype))


def rows_of(rp: np.ndarray) -> np.ndarray:
    return np.repeat(np.arange(rp.shape[0] - 1), np.diff(rp))
