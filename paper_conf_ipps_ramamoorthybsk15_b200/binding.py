"""Thin ctypes binding over libspg.so (include/spg.h).  Argument marshalling only: every step
of the SpGEMM runs in the library's CUDA kernels.  PyTorch supplies device memory, streams
and process groups.  There is no CPU fallback: if the extension cannot be loaded, or no CUDA
device is present, calls raise."""
from __future__ import annotations

import ctypes
import os
from ctypes import POINTER, byref, c_char_p, c_float, c_int, c_int32, c_int64, c_void_p
from dataclasses import dataclass

import torch

_HERE = os.path.dirname(os.path.abspath(__file__))
SO_PATH = os.path.join(_HERE, "libspg.so")

# status codes (spg_status)
SPG_OK = 0
STATUS_NAMES = {0: "SPG_OK", 1: "SPG_ERR_INVALID_ARGUMENT", 2: "SPG_ERR_DIMENSION_MISMATCH",
                3: "SPG_ERR_INDEX_OVERFLOW", 4: "SPG_ERR_OUT_OF_MEMORY", 5: "SPG_ERR_CUDA", 6: "SPG_ERR_NCCL",
                7: "SPG_ERR_BAD_STATE", 8: "SPG_ERR_NOT_SUPPORTED"}
# dtypes
SPG_FP32, SPG_FP64 = 0, 1
# row classes
CLASS_NAMES = ["empty", "single", "tiny", "light", "medium", "heavy", "huge"]
NUM_CLASSES = 7
# options
OPTIONS = {"light_max_flops": 0, "tile_flops": 1, "heavy_max_flops": 2, "force_class": 3, "validate": 4,
           "input_canonical": 5, "timing": 6, "huge_slots": 7, "concurrent": 8, "autotune": 9,
           "csrmm_light_nnz": 10, "heavy_order": 11, "pack_b": 12,
           "heavy_sort": 13, "heavy_dual": 14}

EXPORTED = ["spg_create", "spg_set_option", "spg_get_option", "spg_spgemm_free", "spg_last_error", "spg_get_stats",
            "spg_version", "spg_spgemm_symbolic", "spg_spgemm_numeric", "spg_spgemm_host_symbolic",
            "spg_spgemm_host_numeric", "spg_get_unique_id", "spg_create_dist", "spg_broadcast_csr",
            "spg_allgather_nnz", "spg_allgatherv_c", "spg_split_points", "spg_broadcast_csr_async",
            "spg_scatter_plan", "spg_scatter_rows", "spg_csrmm"]


class spg_csr(ctypes.Structure):
    _fields_ = [("nrows", c_int32), ("ncols", c_int32), ("nnz", c_int64), ("row_ptr", c_void_p),
                ("col_idx", c_void_p), ("vals", c_void_p)]


class spg_stats(ctypes.Structure):
    _fields_ = [("flops", c_int64), ("flops_total", c_int64), ("f_max", c_int64), ("nnz_c", c_int64),
                ("row_begin", c_int32), ("row_end", c_int32),
                ("class_rows", c_int64 * NUM_CLASSES), ("class_flops", c_int64 * NUM_CLASSES),
                ("bin_hist", c_int64 * 65), ("tiles", c_int64), ("heavy_rows", c_int64),
                ("dup_products", c_int64), ("plan_bytes", c_int64), ("ms_analysis", c_float), ("ms_symbolic", c_float),
                ("ms_numeric", c_float), ("ms_light", c_float), ("ms_heavy", c_float),
                ("light_max", c_int32), ("tile_flops", c_int32),
                ("launches_symbolic", c_int32), ("launches_numeric", c_int32)]

    def to_dict(self) -> dict:
        d = {k: getattr(self, k) for k, _ in self._fields_}
        for k in ("class_rows", "class_flops", "bin_hist"):
            d[k] = list(d[k])
        return d


class SpgError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS_NAMES.get(status, status)}: {msg}")
        self.status = status


_lib = None


def load(build_if_missing: bool = True):
    """Load libspg.so (building it in-tree with nvcc if it is missing or stale)."""
    global _lib
    if _lib is not None:
        return _lib
    if build_if_missing:
        from . import build as _b
        try:
            _b.build()
        except (FileNotFoundError, OSError):
            if not os.path.exists(SO_PATH):
                raise
    if not os.path.exists(SO_PATH):
        raise ImportError(f"{SO_PATH} is missing: run `python -m paper_conf_ipps_ramamoorthybsk15_b200.build`")
    lib = ctypes.CDLL(SO_PATH)
    H = c_void_p
    P = c_void_p
    sig = {
        "spg_create": [POINTER(H), c_int, P, c_int],
        "spg_set_option": [H, c_int, c_int64],
        "spg_get_option": [H, c_int, POINTER(c_int64)],
        "spg_spgemm_free": [H],
        "spg_last_error": [H],
        "spg_get_stats": [H, POINTER(spg_stats)],
        "spg_version": [],
        "spg_spgemm_symbolic": [H, POINTER(spg_csr), POINTER(spg_csr), P, POINTER(c_int64), POINTER(c_int32),
                                POINTER(c_int32)],
        "spg_spgemm_numeric": [H, POINTER(spg_csr), POINTER(spg_csr), P, P, P],
        "spg_spgemm_host_symbolic": [H, POINTER(spg_csr), POINTER(spg_csr), P, POINTER(c_int64)],
        "spg_spgemm_host_numeric": [H, P, P],
        "spg_get_unique_id": [P],
        "spg_create_dist": [POINTER(H), c_int, P, c_int, P, c_int, c_int],
        "spg_broadcast_csr": [H, POINTER(spg_csr), c_int],
        "spg_allgather_nnz": [H, c_int64, POINTER(c_int64)],
        "spg_allgatherv_c": [H, P, P, P, P, P, P],
        "spg_split_points": [H, POINTER(spg_csr), POINTER(spg_csr), c_int32, P],
        "spg_broadcast_csr_async": [H, POINTER(spg_csr), c_int],
        "spg_scatter_plan": [H, POINTER(spg_csr), POINTER(spg_csr), c_int, POINTER(c_int32), POINTER(c_int32),
                             POINTER(c_int64)],
        "spg_scatter_rows": [H, POINTER(spg_csr), c_int, POINTER(spg_csr)],
        "spg_csrmm": [H, POINTER(spg_csr), P, c_int64, c_int32, P, c_int64],
    }
    for name, args in sig.items():
        fn = getattr(lib, name)
        fn.argtypes = args
        fn.restype = c_int
    lib.spg_last_error.restype = c_char_p
    lib.spg_version.restype = c_char_p
    _lib = lib
    return lib


def _check(h, status: int):
    if status != SPG_OK:
        msg = load().spg_last_error(h)
        raise SpgError(status, msg.decode() if msg else "")


# ---- device CSR --------------------------------------------------------------------------
@dataclass
class DeviceCSR:
    """CSR on a CUDA device: int32 row_ptr/col_idx, fp32/fp64 values (torch tensors)."""
    nrows: int
    ncols: int
    row_ptr: torch.Tensor
    col_idx: torch.Tensor
    vals: torch.Tensor

    @property
    def nnz(self) -> int:
        return int(self.col_idx.numel())

    @property
    def dtype(self):
        return self.vals.dtype

    def c(self) -> spg_csr:
        return spg_csr(self.nrows, self.ncols, self.nnz, self.row_ptr.data_ptr(),
                       self.col_idx.data_ptr() if self.nnz else None,
                       self.vals.data_ptr() if self.nnz else None)

    @staticmethod
    def from_host(m, device="cuda") -> "DeviceCSR":
        """From any object with nrows/ncols/row_ptr/col_idx/vals numpy arrays."""
        t = lambda a: torch.from_numpy(a).to(device)  # noqa: E731
        return DeviceCSR(int(m.nrows), int(m.ncols), t(m.row_ptr), t(m.col_idx), t(m.vals))


@dataclass
class DeviceCSR64:
    """Result of an SpGEMM: int64 row offsets, int32 columns."""
    nrows: int
    ncols: int
    row_ptr: torch.Tensor
    col_idx: torch.Tensor
    vals: torch.Tensor
    row_begin: int = 0

    @property
    def nnz(self) -> int:
        return int(self.col_idx.numel())


def _dt(dtype) -> int:
    if dtype in (torch.float64, "float64", "fp64"):
        return SPG_FP64
    if dtype in (torch.float32, "float32", "fp32"):
        return SPG_FP32
    raise ValueError(f"unsupported dtype {dtype}")


def _stream_ptr(stream):
    if stream is None:
        stream = torch.cuda.current_stream()
    return c_void_p(stream.cuda_stream)


# ---- the C ABI, one Python function per entry point ------------------------------------------
def spg_version() -> str:
    return load().spg_version().decode()


def spg_create(device: int = 0, stream=None, dtype=torch.float64) -> int:
    if not torch.cuda.is_available():
        raise RuntimeError("spg: no CUDA device (the library has no CPU path)")
    h = c_void_p()
    with torch.cuda.device(device):
        st = _stream_ptr(stream)
    _check(None, load().spg_create(byref(h), device, st, _dt(dtype)))
    return h.value


def spg_set_option(h, name, value: int):
    opt = OPTIONS[name] if isinstance(name, str) else int(name)
    _check(h, load().spg_set_option(h, opt, int(value)))


def spg_get_option(h, name) -> int:
    opt = OPTIONS[name] if isinstance(name, str) else int(name)
    v = c_int64()
    _check(h, load().spg_get_option(h, opt, byref(v)))
    return v.value


def spg_spgemm_free(h):
    _check(None, load().spg_spgemm_free(h))


def spg_last_error(h) -> str:
    return load().spg_last_error(h).decode()


def spg_get_stats(h) -> dict:
    s = spg_stats()
    _check(h, load().spg_get_stats(h, byref(s)))
    return s.to_dict()


def spg_spgemm_symbolic(h, A: DeviceCSR, B: DeviceCSR, C_row_ptr: torch.Tensor):
    """Returns (nnzC, row_begin, row_end); C_row_ptr (int64, device) is filled."""
    assert C_row_ptr.dtype == torch.int64 and C_row_ptr.is_cuda
    nnz, rb, re = c_int64(), c_int32(), c_int32()
    a, b = A.c(), B.c()
    _check(h, load().spg_spgemm_symbolic(h, byref(a), byref(b), c_void_p(C_row_ptr.data_ptr()), byref(nnz),
                                         byref(rb), byref(re)))
    return nnz.value, rb.value, re.value


def spg_spgemm_numeric(h, A: DeviceCSR, B: DeviceCSR, C_row_ptr: torch.Tensor, C_col_idx: torch.Tensor,
                       C_vals: torch.Tensor):
    a, b = A.c(), B.c()
    _check(h, load().spg_spgemm_numeric(h, byref(a), byref(b), c_void_p(C_row_ptr.data_ptr()),
                                        c_void_p(C_col_idx.data_ptr() if C_col_idx.numel() else None),
                                        c_void_p(C_vals.data_ptr() if C_vals.numel() else None)))


def _host_csr(m) -> spg_csr:
    return spg_csr(int(m.nrows), int(m.ncols), int(m.col_idx.shape[0]), m.row_ptr.ctypes.data,
                   m.col_idx.ctypes.data if m.col_idx.shape[0] else None,
                   m.vals.ctypes.data if m.vals.shape[0] else None)


def spg_spgemm_host_symbolic(h, A, B, C_row_ptr) -> int:
    """A, B, C_row_ptr: host (numpy) arrays — ideally in pinned memory.  Returns nnzC."""
    nnz = c_int64()
    a, b = _host_csr(A), _host_csr(B)
    _check(h, load().spg_spgemm_host_symbolic(h, byref(a), byref(b), c_void_p(C_row_ptr.ctypes.data), byref(nnz)))
    return nnz.value


def spg_spgemm_host_numeric(h, C_col_idx, C_vals):
    _check(h, load().spg_spgemm_host_numeric(h, c_void_p(C_col_idx.ctypes.data if C_col_idx.size else None),
                                             c_void_p(C_vals.ctypes.data if C_vals.size else None)))


def spg_get_unique_id() -> bytes:
    buf = ctypes.create_string_buffer(128)
    _check(None, load().spg_get_unique_id(buf))
    return buf.raw


def spg_create_dist(device: int, stream, dtype, uid, rank: int, nranks: int) -> int:
    """uid = None creates a virtual rank (partitioned rows, no communicator)."""
    h = c_void_p()
    with torch.cuda.device(device):
        st = _stream_ptr(stream)
    buf = ctypes.create_string_buffer(uid, 128) if uid is not None else None
    _check(None, load().spg_create_dist(byref(h), device, st, _dt(dtype), buf, rank, nranks))
    return h.value


def spg_broadcast_csr(h, m: DeviceCSR, root: int):
    c = m.c()
    _check(h, load().spg_broadcast_csr(h, byref(c), root))


def spg_csrmm(h, A: DeviceCSR, D: torch.Tensor, C: torch.Tensor):
    """C (M x n) = A x D (K x n); D and C row-major device tensors (strided rows allowed)."""
    assert D.dim() == 2 and C.dim() == 2 and D.stride(1) == 1 and C.stride(1) == 1
    assert D.shape[0] == A.ncols and C.shape == (A.nrows, D.shape[1])
    a = A.c()
    _check(h, load().spg_csrmm(h, byref(a), c_void_p(D.data_ptr() if D.numel() else None), D.stride(0),
                               int(D.shape[1]), c_void_p(C.data_ptr() if C.numel() else None), C.stride(0)))


def csrmm(A: DeviceCSR, D: torch.Tensor, **options) -> torch.Tensor:
    """C = A x D (sparse x dense) on A's device (one-shot handle)."""
    dt = A.vals.dtype
    if D.dtype != dt:
        raise TypeError(f"D must be {dt}")
    h = spg_create(A.row_ptr.device.index or 0, None, dt)
    try:
        for k, v in options.items():
            spg_set_option(h, k, v)
        C = torch.empty(A.nrows, D.shape[1], dtype=dt, device=A.row_ptr.device)
        spg_csrmm(h, A, D.contiguous(), C)
        torch.cuda.current_stream().synchronize()
        return C
    finally:
        spg_spgemm_free(h)


def spg_broadcast_csr_async(h, m: DeviceCSR, root: int):
    c = m.c()
    _check(h, load().spg_broadcast_csr_async(h, byref(c), root))


def spg_scatter_plan(h, A, B: DeviceCSR, root: int):
    """A: DeviceCSR on the root; elsewhere any object with nrows/ncols (its tensors are not read).
    Returns (row_begin, row_end, nnz_local)."""
    a = A.c() if isinstance(A, DeviceCSR) else spg_csr(int(A.nrows), int(A.ncols), 0, None, None, None)
    b = B.c()
    rb, re, nz = c_int32(), c_int32(), c_int64()
    _check(h, load().spg_scatter_plan(h, byref(a), byref(b), root, byref(rb), byref(re), byref(nz)))
    return rb.value, re.value, nz.value


def spg_scatter_rows(h, A, root: int, A_local: DeviceCSR):
    a = A.c() if isinstance(A, DeviceCSR) else spg_csr(int(A.nrows), int(A.ncols), 0, None, None, None)
    loc = A_local.c()
    _check(h, load().spg_scatter_rows(h, byref(a), root, byref(loc)))


def spg_allgather_nnz(h, nnz_local: int) -> int:
    t = c_int64()
    _check(h, load().spg_allgather_nnz(h, nnz_local, byref(t)))
    return t.value


def spg_allgatherv_c(h, C_local: DeviceCSR64, C_full: DeviceCSR64):
    p = lambda t: c_void_p(t.data_ptr() if t.numel() else None)  # noqa: E731
    _check(h, load().spg_allgatherv_c(h, p(C_local.row_ptr), p(C_local.col_idx), p(C_local.vals),
                                      p(C_full.row_ptr), p(C_full.col_idx), p(C_full.vals)))


def spg_split_points(h, A: DeviceCSR, B: DeviceCSR, P: int):
    import numpy as np
    s = np.empty(P + 1, np.int32)
    a, b = A.c(), B.c()
    _check(h, load().spg_split_points(h, byref(a), byref(b), P, c_void_p(s.ctypes.data)))
    return s


# ---- convenience ---------------------------------------------------------------------------
class SpGEMM:
    """Owns an spg handle.  `plan = SpGEMM(); C = plan(A, B)` runs symbolic + numeric."""

    def __init__(self, device: int = 0, dtype=torch.float64, stream=None, **options):
        self.device = device
        self.dtype = dtype
        self.h = spg_create(device, stream, dtype)
        for k, v in options.items():
            spg_set_option(self.h, k, v)

    def set_option(self, name, value):
        spg_set_option(self.h, name, value)

    def _check(self, *mats):
        """The C side reads every value array as the handle's dtype: reject anything else."""
        for m in mats:
            for t in (m.row_ptr, m.col_idx):
                if t.dtype != torch.int32 or not t.is_contiguous():
                    raise TypeError("row_ptr / col_idx must be contiguous int32 tensors")
            if m.vals.numel() and (m.vals.dtype != self.dtype or not m.vals.is_contiguous()):
                raise TypeError(f"values must be contiguous {self.dtype}, got {m.vals.dtype}")

    def symbolic(self, A: DeviceCSR, B: DeviceCSR) -> DeviceCSR64:
        self._check(A, B)
        rp = torch.empty(A.nrows + 1, dtype=torch.int64, device=A.row_ptr.device)
        nnz, rb, re = spg_spgemm_symbolic(self.h, A, B, rp)
        n = re - rb
        col = torch.empty(nnz, dtype=torch.int32, device=rp.device)
        val = torch.empty(nnz, dtype=self.dtype, device=rp.device)
        return DeviceCSR64(n, B.ncols, rp[: n + 1], col, val, rb)

    def numeric(self, A: DeviceCSR, B: DeviceCSR, C: DeviceCSR64) -> DeviceCSR64:
        self._check(A, B)
        if C.vals.numel() and (C.vals.dtype != self.dtype or not C.vals.is_contiguous()):
            raise TypeError(f"C values must be contiguous {self.dtype}")
        spg_spgemm_numeric(self.h, A, B, C.row_ptr, C.col_idx, C.vals)
        return C

    def __call__(self, A: DeviceCSR, B: DeviceCSR) -> DeviceCSR64:
        return self.numeric(A, B, self.symbolic(A, B))

    def stats(self) -> dict:
        return spg_get_stats(self.h)

    def close(self):
        if self.h:
            spg_spgemm_free(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


def spgemm(A: DeviceCSR, B: DeviceCSR, **options) -> DeviceCSR64:
    """C = A x B on A's device (one-shot; creates and frees a handle)."""
    plan = SpGEMM(A.row_ptr.device.index or 0, A.vals.dtype, **options)
    try:
        C = plan(A, B)
        torch.cuda.current_stream().synchronize()
        return C
    finally:
        plan.close()
