"""GPU parity: the CUDA path (through the C ABI) against the oracle, element by element.

Structure (row_ptr, col_idx) must be identical; values within |gpu - sum| <= rtol * sum|a*b|
(rtol 1e-12 fp64, 1e-5 fp32 — BASELINE.json north_star) or bit-exact where the inputs make
every partial sum exact (small integers, the Fig. 2 example)."""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
import workloads as W
from tests._util import dense_to_csr, identity, permutation_matrix, read_golden
from tests.gpu_util import compare, run_gpu, to_dev

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # collected on CPU boxes only with -m gpu
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ipps_ramamoorthybsk15_b200 as spg  # noqa: E402

FORCE = [-1, 2, 3, 4, 5, 6]   # natural, TINY.. HUGE (TINY = SINGLE shortcut off)


def test_native_library_is_loaded():
    import paper_conf_ipps_ramamoorthybsk15_b200.binding as b
    lib = b.load()
    assert lib._name.endswith("libspg.so")
    assert "sm_100a" in spg.spg_version()


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_fig2_bit_exact(dtype):
    g = read_golden("fig2.txt")
    A, B = dense_to_csr(g["A"], dtype), dense_to_csr(g["B"], dtype)
    for force in FORCE:
        got = run_gpu(A, B, force_class=force)
        compare(A, B, got, exact_values=True)
        np.testing.assert_array_equal(np.diff(got[0]), [2, 2, 3, 3])


@pytest.mark.parametrize("seed", range(4))
@pytest.mark.parametrize("shape", [(37, 29, 41), (200, 150, 300), (1, 50, 7), (64, 1, 64)])
@pytest.mark.parametrize("force", FORCE)
def test_random_int_exact(seed, shape, force):
    M, K, N = shape
    A = W.random_csr(M, K, 0.15, seed, values="int", empty_row_frac=0.1)
    B = W.random_csr(K, N, 0.15, seed + 50, values="int", empty_row_frac=0.1)
    compare(A, B, run_gpu(A, B, force_class=force), exact_values=True)


@pytest.mark.parametrize("force", FORCE)
def test_power_law_rows_span_all_classes(force):
    """Chung-Lu rows from 1 to ~10k products: every class, several merge rounds, ragged tails."""
    A, B = W.make("cl10k")
    got = run_gpu(A, B, force_class=force)
    compare(A, B, got)
    st = got[3]
    if force == -1:
        for c in (1, 2, 3, 4, 5, 6):
            assert st["class_rows"][c] > 0, (spg.CLASS_NAMES[c], st["class_rows"])
    f = oracle.row_flops(A, B)
    assert st["flops"] == f.sum() and st["f_max"] == f.max()
    _, hist = oracle.bins(f)
    np.testing.assert_array_equal(st["bin_hist"], hist)


@pytest.mark.parametrize("heavy_max,tile,light_max", [(64, 64, 40), (256, 128, 64), (8192, 2048, 1024),
                                                      (8192, 2048, 2048), (0, 1, 0), (4096, 16, 4000),
                                                      (33, 4000, 32), (8192, 3072, 4096), (8192, 1024, 4096),
                                                      (8192, 4096, 4096)])
def test_thresholds_do_not_change_result(heavy_max, tile, light_max):
    """the threshold moves work between kernels, never changes C (tile 1: a tile
    per light row; light_max 0: every row on the heavy path; heavy_max 0: every heavy row HUGE)."""
    A, B = W.make("cl10k")
    ref = oracle.spgemm(A, B, nthreads=8)
    # light rows above 4096 - tile are solo tiles; light_max <= 4096 (TILE_PMAX)
    got = run_gpu(A, B, light_max_flops=0, tile_flops=tile, heavy_max_flops=heavy_max, _then={"light_max_flops": light_max})
    compare(A, B, got, ref=ref)


def test_autotune_picks_a_candidate_and_keeps_the_result():
    """SPG_OPT_AUTOTUNE (f1): the first symbolic call on a structure times the candidate
    thresholds; whichever wins, C is the oracle's (thresholds never change C)."""
    A, B = W.make("cl10k")
    got = run_gpu(A, B, autotune=1)
    compare(A, B, got)
    st = got[3]
    assert (st["light_max"], st["tile_flops"]) in [(1024, 3072), (2048, 2048), (3072, 1024), (4096, 2048), (512, 3584)]


@pytest.mark.parametrize("alpha", [3.0, 6.5])
def test_alpha_sweep_pair_variants(alpha):
    """The f3 alpha-sweep workload (two distinct Chung-Lu matrices with the same exponent, n =
    100K) through compare() with the default split and every baseline the
    sweep times: block per row ([13]-style one path), max tiles, and the Unsorted- / Sorted-
    Workqueue analogues (FORCE_CLASS = HUGE, HEAVY_ORDER 0 / 2)."""
    n = 100000
    A = W.chung_lu(n, n, alpha, 8 * n, 2000.0, 2000.0, 6.0, 1.1, 101)
    B = W.chung_lu(n, n, alpha, 8 * n, 2000.0, 2000.0, 6.0, 1.1, 202)
    ref = oracle.spgemm(A, B, nthreads=8)
    for opts in ({}, {"force_class": 5}, {"light_max_flops": 4096, "tile_flops": 1024},
                 {"force_class": 6, "heavy_order": 0}, {"force_class": 6, "heavy_order": 2}):
        compare(A, B, run_gpu(A, B, **opts), ref=ref)


@pytest.mark.parametrize("light", [0, 1024, 2048])
def test_heavy_rows_as_big_tiles(light):
    """SPG_OPT_HEAVY_SORT = 1: the register-cached heavy bins sorted in big tiles (8192
    products, 1024 threads) instead of the column bitmap — same C as the oracle."""
    A, B = W.make("cl10k")
    ref = oracle.spgemm(A, B, nthreads=8)
    compare(A, B, run_gpu(A, B, heavy_sort=1, light_max_flops=light), ref=ref)
    A2 = W.chung_lu(30000, 30000, 2.1, 150000, 4000, 4000, 5.0, 1.1, 17)
    compare(A2, A2, run_gpu(A2, A2, heavy_sort=1, light_max_flops=light))


@pytest.mark.parametrize("opts", [{}, {"heavy_max_flops": 4096}, {"heavy_max_flops": 6000, "heavy_order": 0},
                                  {"concurrent": 0}, {"huge_slots": 3}])
def test_heavy_dual_queue(opts):
    """SPG_OPT_HEAVY_DUAL = 1: HUGE-kernel blocks take rows from the front of [HUGE ; HEAVY2]
    and register-cached HEAVY2 blocks from the back — every row is processed
    exactly once whichever side claims it, so C equals the oracle's at any split."""
    A = W.chung_lu(30000, 30000, 2.1, 150000, 4000, 4000, 5.0, 1.1, 17)
    ref = oracle.spgemm(A, A, nthreads=8)
    compare(A, A, run_gpu(A, A, heavy_dual=1, heavy_sort=0, **opts), ref=ref)


@pytest.mark.parametrize("name", ["webbase1m", "ab2m"])
def test_heavy_dual_queue_full_config(name):
    """The dual-ended queue on the BASELINE shapes with many HUGE and HEAVY2 rows: C equals the
    oracle's on every row."""
    A, B = W.make(name)
    got = run_gpu(A, B, heavy_dual=1)
    compare(A, B, got, nthreads=max(1, __import__("os").cpu_count() or 1))


def test_heavy_dual_queue_reused_handle():
    """The claim generation advances per symbolic pass: a handle re-run on the same and on a new
    structure (plan grows, rerun inside symbolic) keeps processing every row once."""
    A1, _ = W.make("cl10k")
    A2 = W.chung_lu(30000, 30000, 2.1, 150000, 4000, 4000, 5.0, 1.1, 17)
    plan = spg.SpGEMM(0, torch.float64, heavy_dual=1, heavy_sort=0)
    for A in (A1, A2, A1, A2):
        dA = spg.DeviceCSR.from_host(A, "cuda:0")
        C = plan(dA, dA)
        torch.cuda.synchronize()
        compare(A, A, (C.row_ptr.cpu().numpy(), C.col_idx.cpu().numpy(), C.vals.cpu().numpy()))
    plan.close()


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_packed_b_numeric(dtype):
    """SPG_OPT_PACK_B = 1: numeric gathers B through the packed {column, value} copy (automatic
    only for B > 64 MB, i.e. rmat23) — same C as the oracle, repeats included."""
    A = W.chung_lu(20000, 20000, 2.1, 80000, 3000, 3000, 6.0, 1.1, 5, dtype)
    compare(A, A, run_gpu(A, A, pack_b=1))


def test_fp32_power_law():
    A = W.chung_lu(20000, 20000, 2.1, 80000, 3000, 3000, 6.0, 1.1, 5, np.float32)
    B = W.chung_lu(20000, 20000, 3.0, 160000, 1000, 1000, -1.0, 1.0, 6, np.float32)
    for force in (-1, 6):
        compare(A, B, run_gpu(A, B, force_class=force))


def test_rectangular_and_empty():
    cases = [(0, 5, 3, 0.0), (4, 0, 3, 0.0), (4, 5, 0, 0.0), (6, 6, 6, 0.0), (1, 1, 1, 1.0), (300, 2, 500, 0.4)]
    for (M, K, N, d) in cases:
        A = W.random_csr(M, K, d, 1, values="int")
        B = W.random_csr(K, N, d, 2, values="int")
        for force in (-1, 3, 6):
            compare(A, B, run_gpu(A, B, force_class=force), exact_values=True)


def test_noncanonical_A():
    """A with duplicate and unsorted entries (B canonical): duplicates are summed."""
    A = W.random_csr(300, 200, 0.05, 3, values="int", canonical=False)
    rng = np.random.default_rng(0)
    for i in range(A.nrows):
        s, e = A.row_ptr[i], A.row_ptr[i + 1]
        p = rng.permutation(e - s) + s
        A.col_idx[s:e], A.vals[s:e] = A.col_idx[p], A.vals[p]
    B = W.random_csr(200, 250, 0.05, 4, values="int")
    for force in FORCE:
        compare(A, B, run_gpu(A, B, force_class=force), exact_values=True)


def test_identity_permutation():
    A, _ = W.make("cl10k")
    I = identity(A.nrows)
    for (X, Y) in [(A, I), (I, A)]:
        rp, col, val, _ = run_gpu(X, Y)
        np.testing.assert_array_equal(rp, A.row_ptr)
        np.testing.assert_array_equal(col, A.col_idx)
        np.testing.assert_array_equal(val, A.vals)
    perm = np.random.default_rng(1).permutation(A.nrows)
    rp, col, val, _ = run_gpu(permutation_matrix(perm), A)
    lens = np.diff(A.row_ptr)[perm]
    np.testing.assert_array_equal(np.diff(rp), lens)


def test_long_rows_huge_tier_dense():
    """Rows of up to ~60k products over a 40k-column space: HUGE tier with dense extraction."""
    rng = np.random.default_rng(7)
    K, N = 400, 40000
    B = W.random_csr(K, N, 0.004, 8)                        # ~160 per row
    A = W.random_csr(64, K, 0.9, 9)                         # ~360 B rows per A row
    compare(A, B, run_gpu(A, B))
    compare(A, B, run_gpu(A, B, force_class=6, huge_slots=3))


def test_numeric_rerun_new_values():
    A, B = W.make("cl10k")
    dA = to_dev(A)
    plan = spg.SpGEMM(0, torch.float64)
    C = plan.symbolic(dA, dA)
    plan.numeric(dA, dA, C)
    # same structure pointers, new values: the plan is reusable
    dA2 = spg.DeviceCSR(dA.nrows, dA.ncols, dA.row_ptr, dA.col_idx, dA.vals * 2.0)
    plan.numeric(dA2, dA2, C)
    torch.cuda.synchronize()
    A2 = W.CSR(A.nrows, A.ncols, A.row_ptr, A.col_idx, A.vals * 2.0)
    compare(A2, A2, (C.row_ptr.cpu().numpy(), C.col_idx.cpu().numpy(), C.vals.cpu().numpy()))
    plan.close()


def test_host_path_matches_device_path():
    A, B = W.make("cl10k")
    h = spg.spg_create(0, None, torch.float64)
    try:
        rp = np.empty(A.nrows + 1, np.int64)
        nnz = spg.spg_spgemm_host_symbolic(h, A, A, rp)
        col = np.empty(nnz, np.int32)
        val = np.empty(nnz, np.float64)
        spg.spg_spgemm_host_numeric(h, col, val)
    finally:
        spg.spg_spgemm_free(h)
    compare(A, B, (rp, col, val))


def test_split_points_exact():
    A, B = W.make("cl10k")
    f = oracle.row_flops(A, B)
    h = spg.spg_create(0, None, torch.float64)
    try:
        dA = to_dev(A)
        for P in (1, 2, 3, 4, 8, 13):
            s = spg.spg_split_points(h, dA, dA, P)
            np.testing.assert_array_equal(s, oracle.split_points(f, P))
    finally:
        spg.spg_spgemm_free(h)


def test_split_points_flop_prefix_beyond_2_32():
    """The flop prefix (one-pass look-back scan over ~60 tiles) passes 2^32: 120000 rows of one
    entry each, most pointing at a 65535-long B row (4.4e9 products), some at a 1000-long row,
    every seventh empty.  Only the analysis and the scan run (no symbolic)."""
    M = 120000
    i = np.arange(M)
    has = (i % 7) != 0
    col = np.where(i % 3 == 0, 1, 0).astype(np.int32)[has]
    rp = np.concatenate([[0], np.cumsum(has)]).astype(np.int32)
    A = W.CSR(M, 2, rp, col, np.ones(col.shape[0]))
    bcol = np.concatenate([np.arange(65535), np.arange(1000)]).astype(np.int32)
    B = W.CSR(2, 65535, np.array([0, 65535, 66535], np.int32), bcol, np.ones(bcol.shape[0]))
    f = oracle.row_flops(A, B)
    assert int(f.sum()) > 2**32
    h = spg.spg_create(0, None, torch.float64)
    try:
        dA, dB = to_dev(A), to_dev(B)
        for P in (1, 2, 3, 8, 13):
            np.testing.assert_array_equal(spg.spg_split_points(h, dA, dB, P), oracle.split_points(f, P))
    finally:
        spg.spg_spgemm_free(h)


def test_error_paths():
    A = W.random_csr(10, 8, 0.3, 1)
    B = W.random_csr(9, 8, 0.3, 2)
    dA, dB = to_dev(A), to_dev(B)
    plan = spg.SpGEMM(0, torch.float64)
    with pytest.raises(spg.SpgError, match="DIMENSION_MISMATCH"):
        plan.symbolic(dA, dB)
    B2 = W.random_csr(8, 8, 0.3, 2)
    dB2 = to_dev(B2)
    C = spg.DeviceCSR64(10, 8, torch.zeros(11, dtype=torch.int64, device="cuda"),
                        torch.empty(0, dtype=torch.int32, device="cuda"),
                        torch.empty(0, dtype=torch.float64, device="cuda"))
    with pytest.raises(spg.SpgError, match="BAD_STATE"):
        plan.numeric(dA, dB2, C)
    with pytest.raises(spg.SpgError, match="INVALID_ARGUMENT"):
        plan.set_option("force_class", 1)
    with pytest.raises(spg.SpgError, match="INVALID_ARGUMENT"):
        plan.set_option("light_max_flops", 5000)  # > TILE_PMAX (4096)
    # value arrays of another dtype are rejected before they reach the C side (it would read
    # fp32 data as fp64)
    dA32 = spg.DeviceCSR(dA.nrows, dA.ncols, dA.row_ptr, dA.col_idx, dA.vals.float())
    with pytest.raises(TypeError):
        plan.symbolic(dA32, dB2)
    # validation: unsorted B rows and out-of-range columns are reported, not executed
    plan.set_option("validate", 1)
    Bu = W.random_csr(8, 8, 0.5, 3)
    r = int(np.argmax(np.diff(Bu.row_ptr) >= 2))
    s0 = Bu.row_ptr[r]
    Bu.col_idx[s0], Bu.col_idx[s0 + 1] = Bu.col_idx[s0 + 1], Bu.col_idx[s0]
    with pytest.raises(spg.SpgError, match="strictly ascending"):
        plan.symbolic(dA, to_dev(Bu))
    bad = W.random_csr(8, 8, 0.3, 4)
    bad.col_idx[0] = 99
    with pytest.raises(spg.SpgError, match="out of range"):
        plan.symbolic(dA, to_dev(bad))
    # nnz beyond SPG_MAX_NNZ (2^31 - 4097) is refused on the host, before any device access
    import ctypes
    from paper_conf_ipps_ramamoorthybsk15_b200 import binding as Bd
    big = Bd.spg_csr(10, 8, 2**31 - 4096, dA.row_ptr.data_ptr(), dA.col_idx.data_ptr(), dA.vals.data_ptr())
    nnz, rb, re = ctypes.c_int64(), ctypes.c_int32(), ctypes.c_int32()
    rp = torch.zeros(11, dtype=torch.int64, device="cuda")
    st = Bd.load().spg_spgemm_symbolic(plan.h, ctypes.byref(big), ctypes.byref(dB2.c()), ctypes.c_void_p(rp.data_ptr()),
                                       ctypes.byref(nnz), ctypes.byref(rb), ctypes.byref(re))
    assert Bd.STATUS_NAMES[st] == "SPG_ERR_INDEX_OVERFLOW"
    plan.close()


def test_repeat_record_field_limits():
    """A repeat record holds its A entry relative to the row in 23 bits: a repeated product
    2^23 or more entries into its A row is reported (NOT_SUPPORTED), one just below is exact."""
    for K, want_error in ((2**23 + 3, True), (2**23 - 2, False)):
        # one A row over all K columns; B rows 0, K-2 and K-1 hold column 0, the rest are empty:
        # three products of column 0 (one output, two repeats), at least one late in the row
        rpB = np.zeros(K + 1, dtype=np.int32)
        rpB[1:] = 1
        rpB[K - 1:] = 2
        rpB[K] = 3
        B = W.CSR(K, 4, rpB, np.zeros(3, dtype=np.int32), np.array([1.0, 2.0, 3.0]))
        A = W.CSR(1, K, np.array([0, K], dtype=np.int32), np.arange(K, dtype=np.int32), np.ones(K))
        if want_error:
            plan = spg.SpGEMM(0, torch.float64)
            with pytest.raises(spg.SpgError, match="NOT_SUPPORTED"):
                plan.symbolic(to_dev(A), to_dev(B))
            plan.close()
        else:
            rp, col, val, _ = run_gpu(A, B)
            assert list(rp) == [0, 1] and list(col) == [0] and float(val[0]) == 6.0


def test_concurrent_and_serial_agree():
    A, B = W.make("cl10k")
    ref = oracle.spgemm(A, B, nthreads=8)
    compare(A, B, run_gpu(A, B, concurrent=0), ref=ref)
    compare(A, B, run_gpu(A, B, concurrent=1, timing=1), ref=ref)


# ---- BASELINE.json configs at full size --------------------------------------------------
@pytest.mark.parametrize("name", ["webbase1m", "webgoogle", "citpatents", "ab2m"])
def test_config_full_parity(name):
    A, B = W.make(name)
    got = run_gpu(A, B)
    compare(A, B, got, nthreads=max(1, __import__("os").cpu_count() or 1))
    st = got[3]
    assert st["flops"] == int(oracle.row_flops(A, B).sum())


@pytest.mark.slow
def test_rmat23_full_parity_streamed():
    """R-MAT scale 23 (BASELINE.json configs[4]: 8.4M rows, F = 5.29e9, nnz(C) ~ 5.28e9; the
    GTgraph generator of PAPER.md L277): EVERY row compared element by element with the
    multi-threaded oracle, streamed in row chunks of ~96M outputs (C copied back chunk by chunk):
    C_row_ptr exact, C_col_idx exact, values within 1e-12 * sum|a*b|.  Also the row-sum invariant
    C.1 = A.(A.1) on the device.  This config alone reaches N > 2^22 (the N-dependent default
    thresholds) and multi-column-tile bitmap rows."""
    import os
    import time
    t_start = time.time()
    A, _ = W.make("rmat23")
    dA = to_dev(A)
    plan = spg.SpGEMM(0, torch.float64)
    C = plan(dA, dA)
    torch.cuda.synchronize()
    st = plan.stats()
    f = oracle.row_flops(A, A)
    assert st["flops"] == int(f.sum())
    rp = C.row_ptr.cpu().numpy()
    T = os.cpu_count() or 1
    # chunks of rows with ~96M outputs
    target = 96 << 20
    cuts = [0]
    while cuts[-1] < A.nrows:
        r = int(np.searchsorted(rp, rp[cuts[-1]] + target, side="right")) - 1
        cuts.append(max(cuts[-1] + 1, min(A.nrows, r)))
    checked = 0
    for r0, r1 in zip(cuts[:-1], cuts[1:]):
        orp, ocol, oval, oabs = oracle.spgemm(A, A, r0, r1, nthreads=T)
        s, e = int(rp[r0]), int(rp[r1])
        np.testing.assert_array_equal(rp[r0:r1 + 1] - s, orp, err_msg=f"C_row_ptr differs in rows [{r0}, {r1})")
        np.testing.assert_array_equal(C.col_idx[s:e].cpu().numpy(), ocol, err_msg=f"C_col_idx differs in rows [{r0}, {r1})")
        v = C.vals[s:e].cpu().numpy()
        bad = np.abs(v - oval) > 1e-12 * oabs
        assert not bad.any(), f"{int(bad.sum())} values out of tolerance in rows [{r0}, {r1})"
        checked += e - s
    assert checked == int(rp[-1])
    # row sums on the device in chunks of rows
    x = torch.ones(A.ncols, dtype=torch.float64, device="cuda")
    Ad = torch.sparse_csr_tensor(dA.row_ptr.long(), dA.col_idx.long(), dA.vals, (A.nrows, A.ncols))
    ref = Ad @ (Ad @ x)
    got = torch.empty(A.nrows, dtype=torch.float64, device="cuda")
    step = 1 << 18
    for r0 in range(0, A.nrows, step):
        r1 = min(A.nrows, r0 + step)
        s, e = int(rp[r0]), int(rp[r1])
        off = C.row_ptr[r0:r1 + 1] - s
        got[r0:r1] = torch.segment_reduce(C.vals[s:e], "sum", offsets=off, axis=0)
    torch.testing.assert_close(got, ref, rtol=1e-12, atol=0)
    plan.close()
    print(f"rmat23: {checked} outputs of {A.nrows} rows checked against the oracle on {T} threads "
          f"in {time.time() - t_start:.0f} s")


# ---- non-canonical B (SPG_OPT_INPUT_CANONICAL = 0) -----------------------------------------
@pytest.mark.parametrize("force", [-1, 3, 6])
def test_noncanonical_B_library_sorts(force):
    A = W.random_csr(120, 90, 0.08, 11, values="int", canonical=False)
    B = W.random_csr(90, 140, 0.08, 12, values="int", canonical=False)
    rng = np.random.default_rng(3)
    for M in (A, B):
        for i in range(M.nrows):
            s, e = M.row_ptr[i], M.row_ptr[i + 1]
            p = rng.permutation(e - s) + s
            M.col_idx[s:e], M.vals[s:e] = M.col_idx[p], M.vals[p]
    got = run_gpu(A, B, input_canonical=0, force_class=force)
    compare(A, B, got, exact_values=True)


def test_noncanonical_B_numeric_rerun():
    A, _ = W.make("cl10k")
    Bn = W.random_csr(A.ncols, 3000, 0.002, 4, canonical=False)
    dA, dB = to_dev(A), to_dev(Bn)
    plan = spg.SpGEMM(0, torch.float64, input_canonical=0)
    C = plan.symbolic(dA, dB)
    plan.numeric(dA, dB, C)
    dB2 = spg.DeviceCSR(dB.nrows, dB.ncols, dB.row_ptr, dB.col_idx, dB.vals * 3.0)
    plan.numeric(dA, dB2, C)
    torch.cuda.synchronize()
    B2 = W.CSR(Bn.nrows, Bn.ncols, Bn.row_ptr, Bn.col_idx, Bn.vals * 3.0)
    compare(A, B2, (C.row_ptr.cpu().numpy(), C.col_idx.cpu().numpy(), C.vals.cpu().numpy()))
    plan.close()


# ---- multi-GPU pipeline: virtual ranks (partitioned rows on one GPU) and a real 1-rank comm --
@pytest.mark.parametrize("P", [2, 3, 4, 8])
def test_virtual_ranks_concatenate_to_full(P):
    A, B = W.make("cl10k")
    ref = oracle.spgemm(A, B, nthreads=8)
    f = oracle.row_flops(A, B)
    s_ref = oracle.split_points(f, P)
    dA = to_dev(A)
    rps, cols, vals = [], [], []
    for r in range(P):
        h = spg.spg_create_dist(0, None, torch.float64, None, r, P)
        try:
            rp = torch.empty(A.nrows + 1, dtype=torch.int64, device="cuda")
            nnz, rb, re = spg.spg_spgemm_symbolic(h, dA, dA, rp)
            assert (rb, re) == (int(s_ref[r]), int(s_ref[r + 1]))
            col = torch.empty(max(nnz, 1), dtype=torch.int32, device="cuda")
            val = torch.empty(max(nnz, 1), dtype=torch.float64, device="cuda")
            spg.spg_spgemm_numeric(h, dA, dA, rp, col, val)
            torch.cuda.synchronize()
            st = spg.spg_get_stats(h)
            assert st["flops_total"] == f.sum() and st["flops"] == f[rb:re].sum()
            rps.append(rp[: re - rb + 1].cpu().numpy())
            cols.append(col[:nnz].cpu().numpy())
            vals.append(val[:nnz].cpu().numpy())
        finally:
            spg.spg_spgemm_free(h)
    off = 0
    full_rp = [np.zeros(1, np.int64)]
    for rp in rps:
        full_rp.append(rp[1:] + off)
        off += int(rp[-1])
    got = (np.concatenate(full_rp), np.concatenate(cols), np.concatenate(vals))
    compare(A, B, got, ref=ref)


def test_nccl_single_rank_broadcast_allgatherv():
    A, B = W.make("cl10k")
    uid = spg.spg_get_unique_id()
    h = spg.spg_create_dist(0, None, torch.float64, uid, 0, 1)
    try:
        dA = to_dev(A)
        spg.spg_broadcast_csr(h, dA, 0)
        rp = torch.empty(A.nrows + 1, dtype=torch.int64, device="cuda")
        nnz, rb, re = spg.spg_spgemm_symbolic(h, dA, dA, rp)
        col = torch.empty(nnz, dtype=torch.int32, device="cuda")
        val = torch.empty(nnz, dtype=torch.float64, device="cuda")
        spg.spg_spgemm_numeric(h, dA, dA, rp, col, val)
        assert spg.spg_allgather_nnz(h, nnz) == nnz
        full = spg.DeviceCSR64(A.nrows, A.ncols, torch.empty(A.nrows + 1, dtype=torch.int64, device="cuda"),
                               torch.empty(nnz, dtype=torch.int32, device="cuda"),
                               torch.empty(nnz, dtype=torch.float64, device="cuda"))
        spg.spg_allgatherv_c(h, spg.DeviceCSR64(A.nrows, A.ncols, rp, col, val), full)
        torch.cuda.synchronize()
        compare(A, B, (full.row_ptr.cpu().numpy(), full.col_idx.cpu().numpy(), full.vals.cpu().numpy()))
    finally:
        spg.spg_spgemm_free(h)


def test_nccl_single_rank_async_broadcast_and_scatter():
    """One real NCCL rank: B replicated with the asynchronous broadcast (values overlap symbolic),
    A != B row blocks scattered from the root (ncclSend/Recv to itself), C = A_local x B."""
    A = W.chung_lu(6000, 5000, 2.1, 30000, 1500, 1500, 6.0, 1.1, 21)
    B = W.chung_lu(5000, 7000, 3.0, 40000, 800, 800, -1.0, 1.0, 22)
    ref = oracle.spgemm(A, B, nthreads=8)
    uid = spg.spg_get_unique_id()
    h = spg.spg_create_dist(0, None, torch.float64, uid, 0, 1)
    try:
        dA, dB = to_dev(A), to_dev(B)
        spg.spg_broadcast_csr_async(h, dB, 0)
        rb, re, nz = spg.spg_scatter_plan(h, dA, dB, 0)
        assert (rb, re, nz) == (0, A.nrows, A.nnz)
        loc = spg.DeviceCSR(re - rb, A.ncols, torch.empty(re - rb + 1, dtype=torch.int32, device="cuda"),
                            torch.empty(nz, dtype=torch.int32, device="cuda"),
                            torch.empty(nz, dtype=torch.float64, device="cuda"))
        spg.spg_scatter_rows(h, dA, 0, loc)
        torch.cuda.synchronize()
        np.testing.assert_array_equal(loc.row_ptr.cpu().numpy(), A.row_ptr)
        np.testing.assert_array_equal(loc.col_idx.cpu().numpy(), A.col_idx)
        # symbolic on the dist handle (one rank: all rows), numeric after the async values
        rp = torch.empty(A.nrows + 1, dtype=torch.int64, device="cuda")
        nnz, _, _ = spg.spg_spgemm_symbolic(h, loc, dB, rp)
        col = torch.empty(nnz, dtype=torch.int32, device="cuda")
        val = torch.empty(nnz, dtype=torch.float64, device="cuda")
        spg.spg_spgemm_numeric(h, loc, dB, rp, col, val)
        torch.cuda.synchronize()
        compare(A, B, (rp.cpu().numpy(), col.cpu().numpy(), val.cpu().numpy()), ref=ref)
    finally:
        spg.spg_spgemm_free(h)


def _two_process_worker(rank, world, port, out_q):
    """One process per rank on the SAME GPU: virtual-rank handles (the library's partitioned
    pipeline) with the process group on gloo; C blocks gathered by dist.allgatherv_c."""
    import os
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, root)
    import torch.distributed as tdist
    import oracle as O
    import workloads as WW
    import paper_conf_ipps_ramamoorthybsk15_b200 as S
    from paper_conf_ipps_ramamoorthybsk15_b200 import dist as D
    tdist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        A, B = WW.make("cl10k")
        dA = S.DeviceCSR.from_host(A, "cuda")
        h = S.spg_create_dist(0, None, torch.float64, None, rank, world)
        rp = torch.empty(A.nrows + 1, dtype=torch.int64, device="cuda")
        nnz, rb, re = S.spg_spgemm_symbolic(h, dA, dA, rp)
        col = torch.empty(max(nnz, 1), dtype=torch.int32, device="cuda")
        val = torch.empty(max(nnz, 1), dtype=torch.float64, device="cuda")
        S.spg_spgemm_numeric(h, dA, dA, rp, col, val)
        torch.cuda.synchronize()
        splits = S.spg_split_points(h, dA, dA, world)
        frp, fcol, fval = D.allgatherv_c(rp[: re - rb + 1].cpu().numpy(), col[:nnz].cpu().numpy(),
                                         val[:nnz].cpu().numpy(), splits)
        S.spg_spgemm_free(h)
        t = D.max_over_ranks(float(rank + 1))
        if rank == 0:
            ref = O.spgemm(A, B, nthreads=4)
            err = np.abs(fval - ref[2]) <= 1e-12 * ref[3] if frp[-1] == ref[0][-1] else False
            out_q.put((np.array_equal(frp, ref[0]), np.array_equal(fcol, ref[1]), bool(np.all(err)), t,
                       [int(x) for x in splits]))
    finally:
        tdist.destroy_process_group()


def test_two_processes_virtual_ranks_gloo():
    import socket
    import torch.multiprocessing as mp
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        port = so.getsockname()[1]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_two_process_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=600)
        assert p.exitcode == 0
    rp_ok, col_ok, val_ok, t, splits = q.get(timeout=10)
    assert rp_ok and col_ok and val_ok and t == 2.0
    A, B = W.make("cl10k")
    np.testing.assert_array_equal(splits, oracle.split_points(oracle.row_flops(A, B), 2))


# ---- light/medium kernels hand rows to the general kernel: many runs, clustered columns -----
def test_fallback_many_short_runs():
    """f ~ 100-1500 made of one-product runs: more runs than the ESC2 run table holds."""
    rng = np.random.default_rng(21)
    K, N = 5000, 200000
    B = W.random_csr(K, N, 1.0 / N, 22, values="int")          # ~1 entry per B row
    A = W.random_csr(400, K, 0.0, 23, values="int")
    rows, cols = [], []
    for i in range(A.nrows):
        n = int(rng.integers(40, 1500))
        rows += [i] * n
        cols += list(rng.choice(K, n, replace=False))
    D = np.zeros((A.nrows, K), np.float64)
    D[rows, cols] = rng.integers(1, 5, len(rows))
    A = dense_to_csr(D)
    compare(A, B, run_gpu(A, B), exact_values=True)


def test_fallback_clustered_columns():
    """All products of a row land in a narrow column range of a wide matrix: skewed buckets."""
    rng = np.random.default_rng(31)
    K, N = 300, 1 << 20
    rp = np.arange(0, K * 40 + 1, 40, dtype=np.int32)
    col = np.concatenate([np.sort(rng.choice(256, 40, replace=False)) for _ in range(K)]).astype(np.int32)
    B = W.CSR(K, N, rp, col, rng.integers(1, 5, K * 40).astype(np.float64))
    A = W.random_csr(200, K, 0.05, 32, values="int")
    compare(A, B, run_gpu(A, B), exact_values=True)


def test_columns_up_to_2_31():
    """B with 2^31 - 1 columns (the int32 limit), its first and last column used: light rows whose
    column range spans everything (bucket widths up to 2^31), heavy rows as big tiles (B wider
    than 2^20 columns) and HUGE rows making 2048 bitmap column-tile passes."""
    rng = np.random.default_rng(41)
    N = 2**31 - 1
    K = 3000
    rows = []
    for k in range(K):
        c = rng.choice(N - 2, 30, replace=False) + 1
        if k % 97 == 0:
            c[0] = 0
        if k % 89 == 0:
            c[1] = N - 1
        rows.append(np.unique(c))
    rp = np.concatenate([[0], np.cumsum([len(r) for r in rows])]).astype(np.int32)
    B = W.CSR(K, N, rp, np.concatenate(rows).astype(np.int32),
              rng.integers(-4, 5, int(rp[-1])).astype(np.float64))
    lens = np.concatenate([rng.integers(0, 6, 480), np.full(14, 200), np.full(6, 400)])
    rng.shuffle(lens)
    arp = np.concatenate([[0], np.cumsum(lens)]).astype(np.int32)
    acol = np.concatenate([np.sort(rng.choice(K, n, replace=False)) for n in lens]).astype(np.int32)
    A = W.CSR(len(lens), K, arp, acol, rng.integers(-4, 5, int(arp[-1])).astype(np.float64))
    got = run_gpu(A, B)
    st = got[3]
    assert st["heavy_rows"] >= 20 and st["class_rows"][6] >= 6  # HUGE rows were exercised
    compare(A, B, got, exact_values=True)


# ---- sparse x dense (csrmm) ---------------------------------------------------
def _csrmm_gpu(A, D, **opts):
    dA = to_dev(A)
    Dd = torch.from_numpy(np.ascontiguousarray(D)).to("cuda")
    return spg.csrmm(dA, Dd, **opts).cpu().numpy()


@pytest.mark.parametrize("n", [1, 7, 32, 100, 129])
@pytest.mark.parametrize("light", [0, 16, 256, 1 << 30])
def test_csrmm_int_exact(n, light):
    """Small signed integers: every partial sum exact, so C must equal the oracle bit for bit,
    whichever rows are light (a warp per row) or heavy (a block per row)."""
    A = W.random_csr(300, 200, 0.2, 3, values="int", empty_row_frac=0.1)
    D = np.random.default_rng(n).integers(-8, 9, size=(200, n)).astype(np.float64)
    C = _csrmm_gpu(A, D, csrmm_light_nnz=light)
    ref, _ = oracle.csrmm(A, D)
    np.testing.assert_array_equal(C, ref)


@pytest.mark.parametrize("dtype", [np.float64, np.float32])
def test_csrmm_power_law(dtype):
    """Chung-Lu rows of 1 .. ~2000 stored entries (light and heavy rows), positive values."""
    A = W.chung_lu(20000, 15000, 2.1, 90000, 2000, 2000, 6.0, 1.1, 9, dtype)
    D = np.random.default_rng(1).uniform(1, 2, size=(15000, 48)).astype(dtype)
    C = _csrmm_gpu(A, D)
    ref, ab = oracle.csrmm(A, D.astype(np.float64))
    rtol = 1e-12 if dtype == np.float64 else 1e-5
    assert np.all(np.abs(C.astype(np.float64) - ref) <= rtol * ab)


def test_csrmm_strided_and_empty():
    A = W.random_csr(50, 40, 0.1, 5, values="int", empty_row_frac=0.5)
    Dfull = np.random.default_rng(2).integers(-4, 5, size=(40, 20)).astype(np.float64)
    dA = to_dev(A)
    Dd = torch.from_numpy(Dfull).to("cuda")[:, 3:14]          # ldd = 20, n = 11
    C = torch.full((50, 16), -7.0, dtype=torch.float64, device="cuda")[:, :11]
    h = spg.spg_create(0, None, torch.float64)
    try:
        spg.spg_csrmm(h, dA, Dd, C)
        torch.cuda.synchronize()
    finally:
        spg.spg_spgemm_free(h)
    ref, _ = oracle.csrmm(A, Dfull[:, 3:14])
    np.testing.assert_array_equal(C.cpu().numpy(), ref)
