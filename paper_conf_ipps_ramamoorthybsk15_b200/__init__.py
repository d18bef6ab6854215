"""Heavy/light-row Gustavson SpGEMM for B200 (sm_100a).

C = A x B for CSR matrices, the hot path of Ramamoorthy et al., "A Novel Heterogeneous
Algorithm for Multiplying Scale-Free Sparse Matrices" (IPDPS-W 2015), rebuilt as
class-specialised CUDA kernels behind a C ABI (include/spg.h, libspg.so).  This package
is the thin Python binding; see DESIGN.md.
"""
from .binding import (CLASS_NAMES, OPTIONS, DeviceCSR, DeviceCSR64, SpGEMM, SpgError, load, spg_allgather_nnz,
                      spg_allgatherv_c, csrmm, spg_broadcast_csr, spg_broadcast_csr_async, spg_create, spg_csrmm, spg_create_dist, spg_get_option,
                      spg_get_stats, spg_get_unique_id, spg_last_error, spg_set_option, spg_spgemm_free,
                      spg_spgemm_host_numeric, spg_spgemm_host_symbolic, spg_spgemm_numeric, spg_spgemm_symbolic,
                      spg_scatter_plan, spg_scatter_rows, spg_split_points, spg_version, spgemm)

__all__ = ["CLASS_NAMES", "OPTIONS", "DeviceCSR", "DeviceCSR64", "SpGEMM", "SpgError", "load", "spgemm",
           "spg_allgather_nnz", "spg_allgatherv_c", "spg_broadcast_csr", "spg_broadcast_csr_async",
           "spg_scatter_plan", "spg_scatter_rows", "spg_csrmm", "csrmm", "spg_create", "spg_create_dist",
           "spg_get_option", "spg_get_stats", "spg_get_unique_id", "spg_last_error", "spg_set_option",
           "spg_spgemm_free", "spg_spgemm_host_numeric", "spg_spgemm_host_symbolic", "spg_spgemm_numeric",
           "spg_spgemm_symbolic", "spg_split_points", "spg_version"]
