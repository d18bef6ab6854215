"""Pins for the oracle (CPU only).  Each test checks the oracle against something other
than itself: the paper's printed worked example, closed forms, brute force, invariants,
or an independent library routine on inputs where it is exact.  A plausible mistake in
the oracle (a dropped term, a wrong index, a transposed operand, a lost duplicate)
fails at least one of them."""
from __future__ import annotations

import numpy as np
import pytest
import scipy.sparse as sp

import oracle
import workloads as W
from tests._util import (csr_pattern, csr_to_dense, dense_to_csr, identity, permutation_matrix,
                         read_golden, rows_of)

# --- PAPER.md Fig. 2 (L66-L82) -----------------------------------------------------------
def test_fig2_worked_example():
    g = read_golden("fig2.txt")
    A, B = dense_to_csr(g["A"]), dense_to_csr(g["B"])
    rp, col, val, ab = oracle.spgemm(A, B)
    Cd = np.zeros((4, 3))
    Cd[rows_of(rp), col] = val
    np.testing.assert_array_equal(Cd, g["C"])                      # printed rows L69-L72
    np.testing.assert_array_equal(np.diff(rp), g["c"].ravel())       # c = [2 2 3 3]
    assert rp[-1] == 10
    # structure: exactly the printed nonzeros (no entry of C(1,:)/C(2,:) is stored at a 0)
    np.testing.assert_array_equal(Cd != 0, g["C"] != 0)
    f = oracle.row_flops(A, B)
    np.testing.assert_array_equal(f, g["f"].ravel())                 # f = [2 2 4 4]
    assert f.sum() == 12
    np.testing.assert_array_equal(ab, val)                           # positive data: abs == sum


# --- dense triple loop + Boolean pattern product --------------------------------------------
def _dense_check(A, B):
    rp, col, val, ab = oracle.spgemm(A, B)
    Da, Db = csr_to_dense(A), csr_to_dense(B)
    # textbook triple loop on tiny inputs (integer data => exact in any order)
    M, K, N = Da.shape[0], Da.shape[1], Db.shape[1]
    Cd = np.zeros((M, N))
    for i in range(M):
        for j in range(N):
            s = 0.0
            for k in range(K):
                s += Da[i, k] * Db[k, j]
            Cd[i, j] = s
    pat = (csr_pattern(A).astype(np.int64) @ csr_pattern(B).astype(np.int64)) > 0
    got_pat = np.zeros((M, N), bool)
    got_pat[rows_of(rp), col] = True
    np.testing.assert_array_equal(got_pat, pat)                       # structure
    got = np.zeros((M, N))
    got[rows_of(rp), col] = val
    np.testing.assert_array_equal(got, Cd)                            # values (exact)
    for i in range(M):                                                # sorted, unique columns
        seg = col[rp[i]:rp[i + 1]]
        assert np.all(np.diff(seg) > 0)
    # |sum| <= abs, and abs is exactly the triple loop over |a||b| on the pattern
    absd = np.abs(Da) @ np.abs(Db)
    np.testing.assert_array_equal(ab, absd[rows_of(rp), col]) if _canonical(A) and _canonical(B) else None
    assert np.all(np.abs(val) <= ab)
    return rp, col, val


def _canonical(M):
    for i in range(M.nrows):
        seg = M.col_idx[M.row_ptr[i]:M.row_ptr[i + 1]]
        if np.any(np.diff(seg) <= 0):
            return False
    return True


@pytest.mark.parametrize("seed", range(6))
@pytest.mark.parametrize("shape", [(7, 5, 9), (12, 12, 12), (1, 9, 3), (9, 1, 4), (16, 20, 6)])
def test_dense_tiny_signed_int(seed, shape):
    M, K, N = shape
    A = W.random_csr(M, K, 0.35, seed, values="int", empty_row_frac=0.2)
    B = W.random_csr(K, N, 0.35, seed + 100, values="int", empty_row_frac=0.2)
    _dense_check(A, B)


@pytest.mark.parametrize("seed", range(4))
def test_dense_tiny_noncanonical(seed):
    """Duplicate and unsorted stored entries: duplicates are summed (Gustavson), explicit
    zeros are structure (readings R2, R9)."""
    A = W.random_csr(10, 8, 0.5, seed, values="int", canonical=False)
    B = W.random_csr(8, 11, 0.5, seed + 7, values="int", canonical=False)
    rng = np.random.default_rng(seed)
    for M in (A, B):   # shuffle inside rows
        for i in range(M.nrows):
            s, e = M.row_ptr[i], M.row_ptr[i + 1]
            p = rng.permutation(e - s) + s
            M.col_idx[s:e], M.vals[s:e] = M.col_idx[p], M.vals[p]
    _dense_check(A, B)


def test_explicit_zeros_and_cancellation_are_kept():
    # A(0,0)=1, A(0,1)=-1 ; B(0,0)=2, B(1,0)=2, B(1,1)=0 (explicit zero)
    A = W.CSR(1, 2, np.array([0, 2], np.int32), np.array([0, 1], np.int32), np.array([1.0, -1.0]))
    B = W.CSR(2, 2, np.array([0, 1, 3], np.int32), np.array([0, 0, 1], np.int32), np.array([2.0, 2.0, 0.0]))
    rp, col, val, ab = oracle.spgemm(A, B)
    np.testing.assert_array_equal(col, [0, 1])         # both stored, although both are 0.0
    np.testing.assert_array_equal(val, [0.0, 0.0])
    np.testing.assert_array_equal(ab, [4.0, 0.0])


def test_empty_shapes():
    for (M, K, N) in [(0, 0, 0), (0, 5, 3), (4, 0, 3), (4, 5, 0), (3, 3, 3)]:
        A = W.random_csr(M, K, 0.0, 1)
        B = W.random_csr(K, N, 0.0, 2)
        rp, col, val, ab = oracle.spgemm(A, B)
        assert rp.shape == (M + 1,) and rp[-1] == 0 and col.size == 0
        np.testing.assert_array_equal(oracle.row_flops(A, B), np.zeros(M))


# --- identity / permutation -------------------------------------------------------------------
@pytest.mark.parametrize("seed", range(3))
def test_identity_and_permutation(seed):
    A = W.random_csr(30, 30, 0.1, seed)
    I = identity(30)
    for (X, Y, ref) in [(A, I, A), (I, A, A)]:
        rp, col, val, _ = oracle.spgemm(X, Y)
        np.testing.assert_array_equal(rp, ref.row_ptr)
        np.testing.assert_array_equal(col, ref.col_idx)
        np.testing.assert_array_equal(val, ref.vals)
    perm = np.random.default_rng(seed).permutation(30)
    P = permutation_matrix(perm)
    rp, col, val, _ = oracle.spgemm(P, A)
    for i in range(30):
        s, e = A.row_ptr[perm[i]], A.row_ptr[perm[i] + 1]
        np.testing.assert_array_equal(col[rp[i]:rp[i + 1]], A.col_idx[s:e])
        np.testing.assert_array_equal(val[rp[i]:rp[i + 1]], A.vals[s:e])
    # A.P moves column j of A to column perm[j]
    rp, col, val, _ = oracle.spgemm(A, P)
    got = np.zeros((30, 30))
    got[rows_of(rp), col] = val
    ref = np.zeros((30, 30))
    ref[:, perm] = csr_to_dense(A)
    np.testing.assert_array_equal(got, ref)
    np.testing.assert_array_equal(np.diff(rp), np.diff(A.row_ptr))


# --- invariants on a power-law workload --------------------------------------------------------
def test_invariants_cl10k():
    A, B = W.make("cl10k")
    f = oracle.row_flops(A, B)
    rp, col, val, ab = oracle.spgemm(A, B, nthreads=4)
    c = np.diff(rp)
    assert np.all(c <= f)                                   # c_i <= f_i
    assert rp[-1] <= f.sum()                                # nnz(C) <= F
    lenB = np.diff(B.row_ptr)
    lb = np.zeros(A.nrows, np.int64)
    np.maximum.at(lb, rows_of(A.row_ptr), lenB[A.col_idx])
    assert np.all(c >= lb)                                  # c_i >= max len_B (canonical B)
    # C.1 = A.(B.1): row sums, computed independently with scipy SpMV
    Sa = sp.csr_matrix((A.vals, A.col_idx, A.row_ptr), shape=(A.nrows, A.ncols))
    Sb = sp.csr_matrix((B.vals, B.col_idx, B.row_ptr), shape=(B.nrows, B.ncols))
    rs = np.add.reduceat(val, rp[:-1][c > 0]) if rp[-1] else np.zeros(0)
    ref = Sa @ (Sb @ np.ones(B.ncols))
    got = np.zeros(A.nrows)
    got[c > 0] = rs
    np.testing.assert_allclose(got, ref, rtol=1e-12)
    np.testing.assert_array_equal(ab, val)                  # positive data


def test_row_sum_exact_integer():
    A = W.random_csr(200, 150, 0.05, 3, values="int")
    B = W.random_csr(150, 170, 0.05, 4, values="int")
    rp, col, val, _ = oracle.spgemm(A, B)
    got = np.zeros(200)
    np.add.at(got, rows_of(rp), val)
    ref = csr_to_dense(A) @ (csr_to_dense(B) @ np.ones(170))
    np.testing.assert_array_equal(got, ref)


# --- scipy on strictly positive data (scipy drops numerical zeros, so positive only) ----------
@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_scipy_positive(dtype):
    A = W.random_csr(400, 300, 0.02, 5, dtype=dtype)
    B = W.random_csr(300, 350, 0.02, 6, dtype=dtype)
    rp, col, val, ab = oracle.spgemm(A, B)
    Sa = sp.csr_matrix((A.vals.astype(np.float64), A.col_idx, A.row_ptr), shape=(400, 300))
    Sb = sp.csr_matrix((B.vals.astype(np.float64), B.col_idx, B.row_ptr), shape=(300, 350))
    C = (Sa @ Sb).tocsr()
    C.sort_indices()
    np.testing.assert_array_equal(rp, C.indptr)
    np.testing.assert_array_equal(col, C.indices)
    np.testing.assert_allclose(val, C.data, rtol=1e-13)


def test_scipy_positive_cl10k_threads():
    A, B = W.make("cl10k")
    rp1, col1, val1, _ = oracle.spgemm(A, B, nthreads=1)
    rp4, col4, val4, _ = oracle.spgemm(A, B, nthreads=4)
    np.testing.assert_array_equal(rp1, rp4)
    np.testing.assert_array_equal(col1, col4)
    np.testing.assert_array_equal(val1, val4)
    Sa = sp.csr_matrix((A.vals, A.col_idx, A.row_ptr), shape=(A.nrows, A.ncols))
    C = (Sa @ Sa).tocsr()
    C.sort_indices()
    np.testing.assert_array_equal(rp1, C.indptr)
    np.testing.assert_array_equal(col1, C.indices)
    np.testing.assert_allclose(val1, C.data, rtol=1e-12)


def test_row_range():
    A, B = W.make("cl10k")
    rp, col, val, _ = oracle.spgemm(A, B)
    r0, r1 = 1234, 5678
    rq, cq, vq, _ = oracle.spgemm(A, B, r0, r1)
    np.testing.assert_array_equal(rq, rp[r0:r1 + 1] - rp[r0])
    np.testing.assert_array_equal(cq, col[rp[r0]:rp[r1]])
    np.testing.assert_array_equal(vq, val[rp[r0]:rp[r1]])


# --- row flops, bins, split points -----------------------------------------------------------
def test_row_flops_bruteforce():
    A = W.random_csr(40, 30, 0.1, 9, canonical=False)
    B = W.random_csr(30, 25, 0.2, 10, canonical=False)
    f = oracle.row_flops(A, B)
    for i in range(A.nrows):
        n = 0
        for p in range(A.row_ptr[i], A.row_ptr[i + 1]):
            k = A.col_idx[p]
            for q in range(B.row_ptr[k], B.row_ptr[k + 1]):
                n += 1
        assert f[i] == n
    # one-entry rows: c_i = len_B(k_i) exactly (canonical B)
    A1 = W.CSR(30, 30, np.arange(31, dtype=np.int32), np.arange(30, dtype=np.int32)[::-1].copy(), np.ones(30))
    Bc = W.random_csr(30, 25, 0.2, 11)
    c = oracle.spgemm_count(A1, Bc)
    np.testing.assert_array_equal(c, np.diff(Bc.row_ptr)[::-1])


def test_bins_closed_form():
    f = np.array([0, 1, 2, 3, 4, 5, 31, 32, 33, 1024, 1025, 2**31 - 1, 2**31, 2**31 + 1, 2**40], np.int64)
    b, h = oracle.bins(f)
    exp = [-1 if x == 0 else (int(x) - 1).bit_length() for x in f]
    np.testing.assert_array_equal(b, exp)
    assert h.sum() == f.size and h[0] == 1
    for bb in range(64):
        assert h[bb + 1] == sum(1 for e in exp if e == bb)


@pytest.mark.parametrize("seed", range(5))
@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_split_points_bruteforce(seed, P):
    rng = np.random.default_rng(seed)
    M = int(rng.integers(0, 40))
    f = rng.integers(0, 6, M).astype(np.int64) * (rng.random(M) < 0.7)
    s = oracle.split_points(f, P)
    Pf = np.concatenate([[0], np.cumsum(f)])
    F = int(Pf[-1])
    assert s[0] == 0 and s[P] == M
    for r in range(1, P):
        cand = [i for i in range(M + 1) if Pf[i] * P >= r * F]
        assert s[r] == min(cand)
    assert np.all(np.diff(s) >= 0)
    # balance: every block's flops is at most F/P + max f
    if M:
        for r in range(P):
            blk = Pf[s[r + 1]] - Pf[s[r]]
            assert blk * P <= F + P * int(f.max())


def test_split_points_large_values():
    f = np.array([2**40, 1, 2**40, 3], np.int64)
    s = oracle.split_points(f, 2)
    assert list(s) == [0, 3, 4]   # Pf = [0, 2^40, 2^40+1, 2^41+1, 2^41+4]


# --- sparse x dense (csrmm) ------------------------------------------------------
@pytest.mark.parametrize("seed", range(4))
@pytest.mark.parametrize("shape", [(7, 5, 3), (12, 12, 33), (1, 9, 1), (9, 1, 4), (20, 16, 70)])
def test_csrmm_dense_triple_loop(seed, shape):
    """Against a textbook triple loop over the dense form of A (signed small integers: exact)."""
    M, K, n = shape
    A = W.random_csr(M, K, 0.35, seed, values="int", empty_row_frac=0.2)
    D = np.random.default_rng(seed).integers(-8, 9, size=(K, n)).astype(np.float64)
    Ad = csr_to_dense(A)
    ref = np.zeros((M, n))
    for i in range(M):
        for j in range(n):
            for k in range(K):
                ref[i, j] += Ad[i, k] * D[k, j]
    C, ab = oracle.csrmm(A, D)
    np.testing.assert_array_equal(C, ref)
    np.testing.assert_array_equal(ab, np.abs(Ad) @ np.abs(D))


def test_csrmm_identity_and_duplicates():
    """I x D = D; duplicate stored entries of A add (Gustavson semantics)."""
    D = np.random.default_rng(3).standard_normal((6, 5))
    C, _ = oracle.csrmm(identity(6), D)
    np.testing.assert_array_equal(C, D)
    A = W.CSR(1, 6, np.array([0, 3], np.int32), np.array([2, 2, 4], np.int32), np.array([1.0, 2.0, -1.0]))
    C, ab = oracle.csrmm(A, D)
    np.testing.assert_allclose(C[0], 3.0 * D[2] - D[4], rtol=1e-15)
    np.testing.assert_allclose(ab[0], 3.0 * np.abs(D[2]) + np.abs(D[4]), rtol=1e-15)


def test_csrmm_matches_spgemm_with_dense_b():
    """A x D equals the SpGEMM oracle's A x B with B the CSR form of D (all entries stored)."""
    A = W.random_csr(15, 10, 0.3, 4)
    D = np.random.default_rng(4).uniform(1, 2, size=(10, 7))
    B = dense_to_csr(D)
    rp, col, val, _ = oracle.spgemm(A, B)
    C, _ = oracle.csrmm(A, D)
    Cs = np.zeros_like(C)
    for i in range(15):
        Cs[i, col[rp[i]:rp[i + 1]]] = val[rp[i]:rp[i + 1]]
    np.testing.assert_allclose(C, Cs, rtol=1e-14)
