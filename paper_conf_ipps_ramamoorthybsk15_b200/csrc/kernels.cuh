// kernels.cuh — declarations shared by the kernel translation units and the C-ABI layer.
//
// Pipeline:
//   analysis   k_row_flops: f_i, run flags, log2 histogram
//   classify   k_classify: row path (light tile kernel / heavy bitmap kernel / identity copy),
//              heavy row lists and their plan (EQ) offsets; scan of light flops -> PL; k_tiles:
//              tile cut points in light-product space, plan offsets of light rows
//   symbolic   k_light_rank (tiles of light rows) and k_bitmap_rank (heavy rows) sort every row's
//              products by column and emit the gather plan: for the first product of each
//              distinct column of row i, EQ[Ro_i + rank] = {A entry, B entry}; every other
//              product goes to the dup list.  c_i = #distinct.
//   plan       k_plan: per-row EQ-to-C offset (or the SINGLE row's run), chunk -> first row
//   numeric    k_numeric: C in chunks of NUM_CH outputs, one coalesced pass — C(i, r) =
//              valA[e]·valB[q] from EQ (Phase IV of PAPER.md L154-156: the sort moved to the
//              symbolic phase, so numeric re-runs are a stream); k_numeric_dup adds the dup list.
#pragma once
#include "common.cuh"

namespace spg {

struct ClassParams {
  int light_max;   // f <= light_max -> light (tile) kernel
  int heavy_max;   // f <= heavy_max -> register-cached bitmap kernel, else HUGE (uncached)
  int tile_cap;    // nominal products per tile; rows above TILE_PMAX - tile_cap are solo tiles
  int force;       // -1 or a class id >= CLS_TINY
  int single_ok;   // B rows canonical -> SINGLE (identity) shortcut allowed
  int warp_max;    // light rows with f <= warp_max -> warp-per-row kernel (0: none)
};

struct HeavyLists {
  int* rows[NUM_LISTS];
};

// Small per-call device scratch (zeroed at the start of every symbolic call).
struct Small {
  int counts[8];            // per bitmap bin: rows
  int qhead[8];             // per bitmap bin: dynamic row-queue heads (counts + 8)
  int fb[16];               // fallback rows from the light kernel: [0] rows, [8] queue head
  int ntiles;
  int err;
  int r_ok;                 // EQ capacity sufficient (written by k_tiles)
  int amax;                 // longest row of A
  int nch_need;             // numeric chunks (+1) the plan needed
  int tqhead;               // light tiles: dynamic queue head
  unsigned long long dupn;  // non-first products (dup list entries)
  long long heavy_total;    // products of heavy rows (EQ offsets of heavy rows, relative)
  long long fr;             // products of rows with a gather plan (light + heavy)
  unsigned long long hist[65];
  unsigned long long cstats[2 * NUM_CLS + 2];
};

// Problem view passed to the symbolic kernels.  Row indices in lists / cls / Ro / crow are
// local (i - row_begin).
//
// Gather plan (the symbolic phase's output, consumed by numeric): row i's distinct columns, in
// ascending order, are described by EQ[Ro_i + r] = {A entry e, B entry q} of the first product
// (in the kernel's visiting order) that produced the column of rank r; every other product of
// the column is a dup entry {li, r, e, q}.  Numeric is then C(i, r) = valA[e]·valB[q] (+ dups):
// a coalesced stream in output order (Phase IV's "sort, mark, add like-tuples, compact" of
// PAPER.md L154-156 with the sort moved to symbolic, so numeric re-runs on new values are cheap).
struct SymProb {
  const int* __restrict__ rpA;
  const int* __restrict__ colA;
  const int* __restrict__ rpB;
  const int* __restrict__ colB;
  const int* frow;          // f_i (global row index)
  const uint8_t* cls;       // path per local row
  const long long* Ro;      // EQ offset per local row (-1: no plan: empty / SINGLE)
  int2* EQ;                 // gather plan, indexed Ro_i + rank
  int4* dup;                // dup list
  unsigned long long* dupn; // its length (may exceed dupcap: then the host grows it and reruns)
  long long dupcap;
  uint8_t* fl8;             // uncached bitmap rows: first-claim flag per product (Ro_i + offset)
  long long* crow;          // C row offsets (local); symbolic writes counts at [li + 1]
  const int* r_ok;
  const long long* heavy_total;  // heavy rows' plan size (final after k_classify)
  long long r_cap;               // plan capacity (entries)
  int row_begin, row_end;
  int lgN;                  // ceil(log2 N), N = columns of B
};

// Append a non-first product to the dup list (all 32 lanes must call).  The caller reserved the
// slots [base, base + n) of its row / tile / batch with one global atomic (the count is known before
// the ranks are written: products - distinct columns); *s_cnt (shared) hands them out per warp.
__device__ __forceinline__ void dup_push(const SymProb& P, bool d, int li, int rank, int e, int q,
                                         unsigned long long base, int* s_cnt) {
  const unsigned m = __ballot_sync(FULL, d);
  if (!m) return;
  const int lane = threadIdx.x & 31, leader = __ffs(m) - 1;
  int o = 0;
  if (lane == leader) o = atomicAdd(s_cnt, __popc(m));
  const unsigned long long b = base + (unsigned long long)(__shfl_sync(FULL, o, leader) + __popc(m & lanemask_lt()));
  if (d && (long long)b < P.dupcap) P.dup[b] = make_int4(li, rank, e, q);
}

// Numeric phase: chunks of NUM_CH consecutive outputs of C (one block each).
constexpr int NUM_CH = 2048;
constexpr int NUM_NT = 256;

template <typename V>
struct NumProb {
  const V* __restrict__ valA;
  const int* __restrict__ colB;
  const V* __restrict__ valB;
  const int2* __restrict__ EQ;
  const int4* __restrict__ dup;
  const long long* __restrict__ crow;   // C row offsets (local)
  const long long* __restrict__ nd;     // per local row: EQ index (or B index, SINGLE) minus C offset
  const int* __restrict__ ne;           // per local row: -1, or the A entry of a SINGLE row
  const int* __restrict__ chunk_row;    // row holding the first output of each chunk
  long long nnz;                        // outputs (this rank)
  long long ndup;
  void* packB;                          // optional packed {column, value} copy of B (one gather)
  long long nB;
  int nch;
  int mloc;
  int* ccol;
  V* cval;
};

// analysis.cu
cudaError_t launch_row_flops(cudaStream_t st, int M, const int* rpA, const int* colA, int K, const int* rpB, int* f,
                             uint8_t* nz, unsigned long long* hist, int* err, int* amax);
cudaError_t launch_classify(cudaStream_t st, int sms, const int* f, const uint8_t* nz, int rb, int re,
                            const ClassParams& prm, uint8_t* cls, int* fl, long long* Ro, const HeavyLists& lists,
                            Small* small, long long* crow, long long* PL);
cudaError_t launch_tiles(cudaStream_t st, int sms, const int* f, int rb, int re, int tile_cap, const uint8_t* cls,
                         const long long* PL, long long* Ro, uint8_t* tflag, int* tiles, Small* small,
                         long long r_cap);
cudaError_t launch_sort_list(cudaStream_t st, const HeavyLists& lists, int bin, const int* f, int rb,
                             const Small* small);
size_t scan_tmp_elems(long long n);
int scan_launches(long long n);
template <typename Tin>
cudaError_t launch_incl_scan(cudaStream_t st, const Tin* in, long long* out, long long n, long long* tmp);
cudaError_t launch_split_points(cudaStream_t st, const long long* Pf, int M, int P, int* s);
cudaError_t launch_validate(cudaStream_t st, int sms, int M, const int* rp, const int* ci, int ncols, long long nnz,
                            int check_sorted, int* err);
cudaError_t launch_rebase(cudaStream_t st, long long* rp_full, int M, int P, const int* splits, const long long* off);
cudaError_t launch_iota(cudaStream_t st, int* p, long long n);
template <typename V>
cudaError_t launch_fill(cudaStream_t st, V* p, long long n, V v);
cudaError_t launch_narrow(cudaStream_t st, const long long* in, int* out, long long n);

// k_light.cu — symbolic ranks of the light rows, one tile per block iteration.
cudaError_t light_configure();
int light_occupancy();
cudaError_t launch_light_rank(cudaStream_t st, int grid, const SymProb& P, const int* tiles, const int* ntiles, int* tqhead,
                              const uint8_t* tflag, const long long* PL, int* fb_list, int* fb_count);

// k_warp.cu — symbolic plan of the smallest light rows, one warp per row.
int warp_occupancy();
cudaError_t launch_warp_rank(cudaStream_t st, int grid, const SymProb& P, const int* list, const int* count);

// k_heavy.cu — symbolic ranks of heavy rows (column bitmap), per bin or over an explicit list.
cudaError_t heavy_configure();
int heavy_occupancy(int bin);
cudaError_t launch_heavy_rank(int bin, cudaStream_t st, int grid, const SymProb& P, const int* list,
                              const int* count, long long N, int fallback);

// k_numeric.cu — numeric plan (end of symbolic) and numeric phase.
cudaError_t launch_plan(cudaStream_t st, int sms, const long long* crow, int mloc, const int* rpA, const int* colA,
                        const int* rpB, const uint8_t* cls, const long long* Ro, int rb, long long* nd, int* ne,
                        int* chunk_row, int chcap, Small* small);
template <typename V>
cudaError_t numeric_configure();
template <typename V>
int numeric_occupancy();
template <typename V>
cudaError_t launch_numeric(cudaStream_t st, int grid, const NumProb<V>& P);

}  // namespace spg
