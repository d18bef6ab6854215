"""Input generators: determinism, canonical CSR, and the shape targets DESIGN.md §3 states."""
import numpy as np
import pytest

import workloads as W


def _check_canonical(A):
    assert A.row_ptr[0] == 0 and A.row_ptr[-1] == A.nnz
    assert np.all(np.diff(A.row_ptr) >= 0)
    assert A.col_idx.min(initial=0) >= 0 and A.col_idx.max(initial=-1) < A.ncols
    starts = A.row_ptr[:-1]
    d = np.diff(A.col_idx.astype(np.int64))
    first = np.zeros(A.nnz, bool)
    first[starts[starts < A.nnz]] = True
    assert np.all(d[~first[1:]] > 0)          # strictly ascending inside each row


def test_deterministic_and_canonical():
    A1, _ = W.make("cl10k")
    A2, _ = W.make("cl10k")
    np.testing.assert_array_equal(A1.row_ptr, A2.row_ptr)
    np.testing.assert_array_equal(A1.col_idx, A2.col_idx)
    np.testing.assert_array_equal(A1.vals, A2.vals)
    _check_canonical(A1)
    assert 1.0 <= A1.vals.min() and A1.vals.max() < 2.0


def test_cl10k_shape():
    A, _ = W.make("cl10k")
    lens = np.diff(A.row_ptr)
    assert A.nrows == 10_000 and 45_000 < A.nnz < 55_000
    assert lens.max() > 500                    # heavy rows exist (scale-free)
    assert (lens >= 60).sum() < 200            # "very few rows with >= 60 nonzeros"


def test_rmat_small_and_fp32():
    A = W.rmat(10, 8, seed=3, dtype=np.float32)
    _check_canonical(A)
    assert A.nrows == 1024 and A.vals.dtype == np.float32
    assert 0.9 * 8 * 1024 < A.nnz <= 8 * 1024
    assert 1.0 <= A.vals.min() and A.vals.max() < 2.0


def test_random_csr_noncanonical_keeps_duplicates():
    A = W.random_csr(5, 3, 2.0, 1, canonical=False)
    assert A.nnz == 30                        # 5*3*2 draws, duplicates kept


@pytest.mark.slow
def test_webbase_shape():
    A, _ = W.make("webbase1m")
    assert A.nrows == 1_000_005
    assert abs(A.nnz - 3_105_536) / 3_105_536 < 0.01
    lens = np.diff(A.row_ptr)
    assert (lens >= 60).sum() < 0.01 * A.nrows        # Fig. 1: very few rows >= 60 nnz
