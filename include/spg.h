/* spg.h — C ABI of the heavy/light-row Gustavson SpGEMM for B200 (sm_100a).
 *
 * Computes C = A x B for sparse A (M x K) and B (K x N) in CSR form, following the
 * Row-Row formulation of PAPER.md L62 (§II-A.a): C(i,:) = sum_k A(i,j_k) * B(j_k,:).
 * Rows of A are classified by their intermediate-product (flop) count into light and
 * heavy classes and each class runs on the kernel suited to it — the paper's
 * "right work to the right processor" (Phase I thresholds L112,
 * L128-132) recast as light-row (warp) and heavy-row (thread-block / dense
 * accumulator) kernels on one GPU instead of a CPU+GPU split.  Like-tuples are added and
 * the output holds distinct, column-sorted entries (Phase IV).
 *
 * Conventions
 *   - 0-based CSR.  row_ptr and col_idx are int32; input nnz must be < 2^31.
 *   - C row offsets are int64 (nnz(C) can exceed 2^31).  Column indices of
 *     C are int32, strictly ascending within each row.
 *   - Values are fp64 or fp32 (the handle's dtype), identical for A, B and C.  Products
 *     are accumulated in the value type (reading R5).
 *   - Every structurally produced entry is stored, even when its value is 0.0
 *     (explicit zeros in the inputs are structure; reading R2).
 *   - Matrix pointers passed to spg_spgemm_* are DEVICE pointers on the handle's device.
 *     The spg_spgemm_host_* entry points take HOST pointers and do the copies themselves.
 *   - A: any column order, duplicates allowed (they are summed).  B: each row's columns
 *     must be strictly ascending ("canonical") unless SPG_OPT_INPUT_CANONICAL is set to 0,
 *     in which case the library sorts and de-duplicates a copy of B first.
 *
 * Ownership and threading
 *   - The caller owns A, B and C.  The handle owns all workspace (row flops, classes, the item
 *     list, the plan — 4 bytes per intermediate product (8 for rows with an A row or a referenced
 *     B row longer than 65535 entries) plus 1 byte per product of the largest rows — and the NCCL
 *     communicator) and caches the symbolic analysis that spg_spgemm_numeric consumes.
 *     spg_spgemm_free releases everything.
 *   - A handle is bound to one device and one CUDA stream and is not thread-safe;
 *     several handles may coexist.
 *   - All work is stream-ordered on the handle's stream.  spg_spgemm_symbolic blocks the
 *     host exactly once (to read nnz(C)); spg_spgemm_numeric returns asynchronously.
 *
 * Errors
 *   - Every function returns a status and never throws, exits or aborts across the ABI.
 *   - CUDA / NCCL failures map to SPG_ERR_CUDA / SPG_ERR_NCCL; spg_last_error(h) gives
 *     the detail.  Asynchronous kernel faults surface at the next synchronising call.
 *   - nnz of an input is at most SPG_MAX_NNZ = 2^31 - 4097 (kernels form entry indices a block
 *     stride past a row range in 32-bit arithmetic); larger inputs give SPG_ERR_INDEX_OVERFLOW.
 *   - Always checked: null pointers, A.ncols == B.nrows, nnz consistency with row_ptr
 *     (host-side when the value is known), dtype, call order (SPG_ERR_BAD_STATE), and
 *     per-row flop counts < 2^31 (SPG_ERR_INDEX_OVERFLOW, reported by symbolic), and repeated
 *     products within the first 2^23 stored entries of their A row (SPG_ERR_NOT_SUPPORTED,
 *     reported by symbolic: a repeat's record holds its A entry relative to the row in 23 bits).
 *   - Index ranges and ordering of device inputs are checked only under SPG_OPT_VALIDATE.
 *   - Values are not bitwise reproducible run to run when a row has repeated columns: the
 *     repeated products are added with atomics in a nondeterministic order (R6).
 *     Structure (C_row_ptr, C_col_idx) is deterministic.
 */
#ifndef SPG_H
#define SPG_H

#include <stdint.h>

#define SPG_MAX_NNZ (((int64_t)1 << 31) - 4097) /* largest nnz of an input matrix */

#ifdef __cplusplus
extern "C" {
#endif

typedef struct spg_ctx* spg_handle;

typedef enum {
  SPG_OK = 0,
  SPG_ERR_INVALID_ARGUMENT = 1,   /* null pointer, bad option, malformed CSR (validate)   */
  SPG_ERR_DIMENSION_MISMATCH = 2, /* A.ncols != B.nrows                                    */
  SPG_ERR_INDEX_OVERFLOW = 3,     /* input nnz > SPG_MAX_NNZ, or a row's flop count >= 2^31 */
  SPG_ERR_OUT_OF_MEMORY = 4,      /* workspace allocation failed                           */
  SPG_ERR_CUDA = 5,               /* CUDA runtime error (see spg_last_error)               */
  SPG_ERR_NCCL = 6,               /* NCCL error (see spg_last_error)                       */
  SPG_ERR_BAD_STATE = 7,          /* numeric before symbolic, or with different inputs     */
  SPG_ERR_NOT_SUPPORTED = 8       /* e.g. N too large for the dense heavy-row tier         */
} spg_status;

typedef enum { SPG_FP32 = 0, SPG_FP64 = 1 } spg_dtype;

/* A CSR matrix.  For spg_spgemm_symbolic / _numeric all pointers are device pointers;
 * for spg_spgemm_host_* they are host pointers.  vals may be NULL for symbolic. */
typedef struct {
  int32_t nrows;
  int32_t ncols;
  int64_t nnz;            /* must equal row_ptr[nrows] and be < 2^31 */
  const int32_t* row_ptr; /* [nrows + 1] */
  const int32_t* col_idx; /* [nnz]       */
  const void* vals;       /* [nnz] fp32 or fp64, per the handle dtype */
} spg_csr;

/* Row classes (PAPER.md L104 logical reordering A = [A_H; A_L]).
 * f_i = number of intermediate products of row i.  The heavy/light threshold t of the paper
 * (Phase I) is SPG_OPT_LIGHT_MAX_FLOPS: rows with f_i <= t are "light"
 * (TINY / LIGHT / MEDIUM: tiles of consecutive rows, sorted by one thread block each), the rest
 * "heavy" (one thread block and a shared-memory column bitmap per row).  SINGLE rows (one
 * non-empty B row) are copied; they ride in tiles when f_i <= t. */
typedef enum {
  SPG_CLASS_EMPTY = 0,  /* f_i = 0: no work, c_i = 0                                         */
  SPG_CLASS_SINGLE = 1, /* exactly one non-empty B row referenced: scaled copy, c_i = f_i    */
  SPG_CLASS_TINY = 2,   /* light, f_i <= 32                                                  */
  SPG_CLASS_LIGHT = 3,  /* light, 32 < f_i <= 256                                            */
  SPG_CLASS_MEDIUM = 4, /* light, 256 < f_i <= LIGHT_MAX_FLOPS                               */
  SPG_CLASS_HEAVY = 5,  /* heavy, f_i <= HEAVY_MAX_FLOPS: products cached in registers       */
  SPG_CLASS_HUGE = 6,   /* heavy, larger: products re-gathered per pass                      */
  SPG_NUM_CLASSES = 7
} spg_row_class;

typedef enum {
  SPG_OPT_LIGHT_MAX_FLOPS = 0,  /* heavy/light threshold t: 0..4096; light rows
                                   above 4096 - TILE_FLOPS are tiles of their own;
                                   default 2048 with tile 2048 (tools/sweep_quick.sh, profiles/);
                                   when B has > 2^22 columns and neither option was set: 4096
                                   with tile 1024.  0 sends every non-SINGLE row to the heavy
                                   path                                                         */
  SPG_OPT_TILE_FLOPS = 1,       /* nominal products per light tile, default 2048               */
  SPG_OPT_HEAVY_MAX_FLOPS = 2,  /* 0..8192, default 8192; heavy rows above are HUGE            */
  SPG_OPT_FORCE_CLASS = 3,      /* -1 (default) or a class id c >= TINY: the SINGLE shortcut is
                                   off, and c >= HEAVY sends every non-empty row to the heavy
                                   path (HUGE: uncached) — the threshold extremes of PAPER.md L233 */
  SPG_OPT_VALIDATE = 4,         /* 1: check CSR indices/order on the device (extra sync)      */
  SPG_OPT_INPUT_CANONICAL = 5,  /* 1 (default): caller promises B rows strictly ascending;
                                   0: the library canonicalises a copy of B                   */
  SPG_OPT_TIMING = 6,           /* 1: record per-phase CUDA-event times into the stats        */
  SPG_OPT_HUGE_SLOTS = 7,       /* max concurrent heavy-row blocks per bin (0 = full occupancy) */
  SPG_OPT_CONCURRENT = 8,       /* 1 (default): light and heavy kernels on concurrent streams  */
  SPG_OPT_AUTOTUNE = 9,         /* 1: the first symbolic call on a new A/B structure times five
                                   (LIGHT_MAX_FLOPS, TILE_FLOPS) candidates and keeps the fastest
                                   (spg_stats.light_max / tile_flops report the choice); 0
                                   (default): the fixed defaults above                         */
  SPG_OPT_CSRMM_LIGHT_NNZ = 10, /* spg_csrmm: rows with more stored entries are heavy (a block
                                   per row), the rest light (a warp per row); default 256      */
  SPG_OPT_HEAVY_ORDER = 11,     /* order in which heavy-row blocks take rows from their queues:
                                   0 natural (row order), 1 (default) largest rows first in the
                                   HUGE / HEAVY2 bins, 2 largest first in every bin (rows ordered
                                   by f_i in 8 classes per octave) — with
                                   FORCE_CLASS = HUGE the GPU analogues of the paper's Unsorted-
                                   and Sorted-Workqueue                    */
  SPG_OPT_PACK_B = 12,          /* numeric gathers B through a packed {column, value} copy (one
                                   sector per output instead of two; the copy is made by every
                                   numeric call, 16 B per B entry for fp64): -1 (default) when
                                   B's columns + values exceed 64 MB (B not L2-resident), 0 never,
                                   1 always                                                     */
  SPG_OPT_HEAVY_SORT = 13,      /* HEAVY rows (f <= 8192) are sorted like tiles in "big tiles" of
                                   8192 products (1024 threads) instead of the column bitmap:
                                   -1 (default) when B has more than 2^20 columns (the bitmap
                                   would need several column-tile passes per row), 0 never,
                                   1 always                                                     */
  SPG_OPT_HEAVY_DUAL = 14       /* 1: the HUGE and HEAVY2 bins share one dual-ended work queue
                                   (cpuOffset / gpuOffset): over the list
                                   [HUGE rows ; HEAVY2 rows], each largest first, the HUGE-kernel
                                   blocks take rows from the front and the register-cached HEAVY2
                                   blocks from the back, so the split between the two kernels is
                                   set at run time.  0 (default): each bin its own queue.  No
                                   effect when HEAVY_SORT puts HEAVY2 rows in big tiles         */
} spg_option;

typedef struct {
  int64_t flops;                          /* F = sum f_i over this rank's rows           */
  int64_t flops_total;                    /* F over all rows (equal to flops at P = 1)  */
  int64_t f_max;                          /* max f_i over this rank's rows               */
  int64_t nnz_c;                          /* nnz(C) of this rank's rows                  */
  int32_t row_begin, row_end;             /* this rank's rows [row_begin, row_end)       */
  int64_t class_rows[SPG_NUM_CLASSES];    /* rows per class (this rank)                  */
  int64_t class_flops[SPG_NUM_CLASSES];   /* products per class (this rank)              */
  int64_t bin_hist[65];                   /* rows with f = 0 (index 0) and with
                                             ceil(log2 f) = b (index b + 1), all rows    */
  int64_t tiles;                          /* tiles of the last symbolic call              */
  int64_t heavy_rows;                     /* rows on the heavy (bitmap) path             */
  int64_t dup_products;                   /* products adding to an output another product
                                             created (f - c summed over rows)            */
  int64_t plan_bytes;                     /* bytes of the plan numeric reads             */
  float ms_analysis;                      /* SPG_OPT_TIMING: row analysis + classify     */
  float ms_symbolic;                      /*   symbolic kernels + row_ptr scan            */
  float ms_numeric;                       /*   numeric (last numeric call)                */
  float ms_light;                         /*   symbolic light-tile kernel                 */
  float ms_heavy;                         /*   symbolic heavy-row kernels                 */
  int32_t light_max;                      /* thresholds the last symbolic call used      */
  int32_t tile_flops;
  int32_t launches_symbolic;              /* kernels launched by the last symbolic call  */
  int32_t launches_numeric;               /* kernels launched by the last numeric call   */
} spg_stats;

/* ---- handle ------------------------------------------------------------------------ */
/* stream: a cudaStream_t (NULL = legacy default stream) on `device`. */
spg_status spg_create(spg_handle* h, int device, void* cuda_stream, spg_dtype dtype);
spg_status spg_set_option(spg_handle h, spg_option opt, int64_t value);
spg_status spg_get_option(spg_handle h, spg_option opt, int64_t* value);
spg_status spg_spgemm_free(spg_handle h);
const char* spg_last_error(spg_handle h);   /* never NULL; valid until the next call on h */
spg_status spg_get_stats(spg_handle h, spg_stats* out);
const char* spg_version(void);

/* ---- SpGEMM (device pointers) ------------------------------------------------------ */
/* Phase I (row analysis, classification) + symbolic.  Writes the exact row offsets of
 * C for this rank's rows [row_begin, row_end): C_row_ptr[0] = 0,
 * C_row_ptr[i - row_begin + 1] - C_row_ptr[i - row_begin] = nnz of row i of C.
 * C_row_ptr: device int64[(row_end - row_begin) + 1], capacity for A.nrows + 1 suffices.
 * nnzC / row_begin / row_end: host outputs (row_begin/row_end may be NULL).
 * Blocks the host once (nnzC readback). */
spg_status spg_spgemm_symbolic(spg_handle h, const spg_csr* A, const spg_csr* B, int64_t* C_row_ptr,
                               int64_t* nnzC, int32_t* row_begin, int32_t* row_end);

/* Numeric phase (Phase IV "add like-tuples, compact"): symbolic sorted every
 * row's products and left a plan — for each output of C, in C order, the A entry and B entry of
 * one of its products, then the repeated products; numeric streams C in output order,
 * C(i,r) = a·b, then adds the repeats — C comes out sorted and compacted.  Requires a preceding
 * symbolic call on this handle with the same A/B structure (checked by pointers, shapes and nnz
 * only: a different structure at recycled addresses is not detected — the caller's contract) and
 * the same C_row_ptr contents.  C_col_idx: device int32[nnzC];
 * C_vals: device fp32/fp64[nnzC].  Values of A and B may differ from the symbolic call
 * (re-run numeric on new values with the same structure).  Asynchronous. */
spg_status spg_spgemm_numeric(spg_handle h, const spg_csr* A, const spg_csr* B, const int64_t* C_row_ptr,
                              int32_t* C_col_idx, void* C_vals);

/* ---- sparse x dense (the CSTMM extension) ------------------------------ */
/* C = A x D with A CSR (device, the handle's dtype), D dense K x n row-major (leading dimension
 * ldd >= n), C dense M x n row-major (ldc >= n), both device pointers.  C(i,:) = sum_k
 * A(i,k) D(k,:) (Row-Row); rows with <= SPG_OPT_CSRMM_LIGHT_NNZ stored entries run
 * one warp per row, longer rows one thread block per row.  Every C(i,j) is written (0 for empty
 * rows).  Asynchronous on the handle's stream; the summation order of a heavy row's entries is
 * fixed (deterministic). */
spg_status spg_csrmm(spg_handle h, const spg_csr* A, const void* D, int64_t ldd, int32_t n, void* C, int64_t ldc);

/* ---- SpGEMM (host pointers; the end-to-end path) ------------------------------------ */
/* Copies A and B (host) into handle-owned device buffers, runs symbolic, copies C's row
 * offsets back.  C_row_ptr: host int64[A.nrows + 1].  Synchronous. */
spg_status spg_spgemm_host_symbolic(spg_handle h, const spg_csr* A, const spg_csr* B, int64_t* C_row_ptr,
                                    int64_t* nnzC);
/* Runs numeric on the buffers of the last host_symbolic call and copies C's columns and
 * values to the host arrays (int32[nnzC], value type[nnzC]).  Synchronous. */
spg_status spg_spgemm_host_numeric(spg_handle h, int32_t* C_col_idx, void* C_vals);

/* ---- multi-GPU ---------------------------------------------------- */
/* Rows of A are split into contiguous blocks balanced on the flop prefix:
 *   s_0 = 0, s_P = M, s_r = min{ i : Pf[i] * P >= r * F },  Pf the exclusive prefix of f.
 * Rank r computes rows [s_r, s_{r+1}) of C.  B (and A) must be resident on every rank —
 * spg_broadcast_csr replicates a matrix from `root` over NCCL. */
spg_status spg_get_unique_id(void* id128);   /* ncclGetUniqueId (128 bytes), call on one rank */
/* A handle for rank `rank` of `nranks`: symbolic/numeric compute only this rank's rows.
 * id128 = NULL creates a VIRTUAL rank (no communicator; collectives return BAD_STATE) — the
 * partitioned pipeline can then be run block by block on one GPU. */
spg_status spg_create_dist(spg_handle* h, int device, void* cuda_stream, spg_dtype dtype, const void* id128,
                           int rank, int nranks);
/* In-place broadcast of a device CSR (row_ptr, col_idx, vals) whose buffers are already
 * allocated with the right sizes on every rank. */
spg_status spg_broadcast_csr(spg_handle h, spg_csr* m, int root);
/* As spg_broadcast_csr, but only the structure (row_ptr, col_idx) is broadcast on the handle's
 * stream; the values go over an internal communication stream, so a following
 * spg_spgemm_symbolic (structure only) overlaps them.  The next spg_spgemm_numeric on this
 * handle waits for the values (valB broadcast overlapped with symbolic). */
spg_status spg_broadcast_csr_async(spg_handle h, spg_csr* m, int root);
/* A != B (the paper ships A's row blocks to its devices): A lives on `root` only.
 * Every rank passes A's dimensions (pointers may be NULL off the root) and the replicated B.
 * The root computes the flop-balanced split points (same formula as above) and broadcasts them;
 * every rank learns its rows [row_begin, row_end) and their entry count.  Synchronous. */
spg_status spg_scatter_plan(spg_handle h, const spg_csr* A, const spg_csr* B, int root, int32_t* row_begin,
                            int32_t* row_end, int64_t* nnz_local);
/* After spg_scatter_plan: the root sends every rank its row block (ncclSend / ncclRecv group).
 * A_local: device buffers allocated by the caller for (row_end - row_begin) rows and nnz_local
 * entries; its row offsets come out starting at 0.  The rank then multiplies A_local x B with a
 * single-GPU handle; the row blocks of C concatenate in rank order.  Stream-ordered. */
spg_status spg_scatter_rows(spg_handle h, const spg_csr* A, int root, spg_csr* A_local);

/* Gathers every rank's C row block into full C on every rank (allgatherv through grouped
 * ncclBroadcast).  C_row_ptr_full: device int64[M+1]; C_col_full/C_val_full sized for
 * the total nnz (= sum of all ranks' nnzC; query with spg_allgather_nnz). */
spg_status spg_allgather_nnz(spg_handle h, int64_t nnz_local, int64_t* nnz_total);
spg_status spg_allgatherv_c(spg_handle h, const int64_t* C_row_ptr_local, const int32_t* C_col_local,
                            const void* C_val_local, int64_t* C_row_ptr_full, int32_t* C_col_full, void* C_val_full);

/* Flop-balanced split points for P parts of the rows of A (device A/B, host out int32[P+1]),
 * computed on the device with the same kernels the distributed path uses. */
spg_status spg_split_points(spg_handle h, const spg_csr* A, const spg_csr* B, int32_t P, int32_t* s_out);

#ifdef __cplusplus
}
#endif
#endif /* SPG_H */
