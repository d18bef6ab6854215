// kernels.cuh — declarations shared by the kernel translation units and the C-ABI layer.
//
// Pipeline:
//   analysis   k_row_flops: f_i, run flags, log2 histogram, per-A-entry row and in-row product
//              offset (rowA, Pe)
//   classify   k_classify: row path (light tile kernel / heavy bitmap kernel / identity copy),
//              heavy row lists and their R offsets; scan of light flops -> PL; k_tiles: tile
//              cut points in light-product space, R offsets of light rows
//   symbolic   k_light_rank (tiles of light rows) and k_bitmap_rank (heavy rows) compute, for
//              every product of row i, its rank among the distinct columns of C(i,:) plus a
//              first-occurrence flag: R[Ro_i + j] = rank | RFLAG·first.  c_i = #distinct.
//   plan       k_cut_count / k_cut_write: row-aligned output windows of C (end of symbolic)
//   numeric    k_num_windows / k_num_large: every product of a window's rows is scattered by
//              its rank into shared memory and the window is written out coalesced (the
//              Phase IV merge of PAPER.md L154-156, with the sort moved to the symbolic phase
//              so numeric re-runs are a stream over R).
#pragma once
#include "common.cuh"

namespace spg {

struct ClassParams {
  int light_max;   // f <= light_max -> light (tile) kernel
  int heavy_max;   // f <= heavy_max -> register-cached bitmap kernel, else HUGE (uncached)
  int tile_cap;    // nominal products per tile (light_max + tile_cap <= TILE_PMAX)
  int force;       // -1 or a class id >= CLS_TINY
  int single_ok;   // B rows canonical -> SINGLE (identity) shortcut allowed
};

struct HeavyLists {
  int* rows[NUM_BINS];
};

// Small per-call device scratch (zeroed at the start of every symbolic call).
struct Small {
  int counts[8];            // per bitmap bin: rows
  int qhead[8];             // per bitmap bin: dynamic row-queue heads (counts + 8)
  int fb[16];               // fallback rows from the light kernel: [0] rows, [8] queue head
  int ntiles;
  int err;
  int r_ok;                 // R capacity sufficient (written by k_tiles)
  int amax;                 // longest row of A
  int nwunits;              // numeric units: windows
  int nlunits;              //   large rows
  int ea0;                  // first A entry of this rank's rows
  int lqhead;               // large-row numeric kernel: queue head
  long long heavy_total;    // products of heavy rows (R offsets of heavy rows, relative)
  long long fr;             // products needing R (light + heavy)
  unsigned long long hist[65];
  unsigned long long cstats[2 * NUM_CLS + 2];
};

// Problem view passed to the symbolic kernels.  Row indices in lists / cls / Ro / crow are
// local (i - row_begin).
struct SymProb {
  const int* __restrict__ rpA;
  const int* __restrict__ colA;
  const int* __restrict__ rpB;
  const int* __restrict__ colB;
  const int* frow;          // f_i (global row index)
  const uint8_t* cls;       // path per local row
  const long long* Ro;      // R offset per local row (-1: identity / empty)
  unsigned* R;              // rank array
  long long* crow;          // C row offsets (local); symbolic writes counts at [li + 1]
  const int* r_ok;
  int row_begin, row_end;
  int lgN;                  // ceil(log2 N), N = columns of B
};

// Output window of the numeric phase: starts at C position pos (local), first row `row`.
struct Cut {
  long long pos;
  int row;
  int pad;
};

// Numeric work unit: outputs [lo, lo + c) of C (local positions) from local A entries [ea, eb).
struct __align__(16) Unit {
  long long lo;
  int ea, eb, c, pad;
};

// Problem view of the numeric kernel.
template <typename V>
struct NumProb {
  const V* __restrict__ valA;
  const int* __restrict__ colB;
  const V* __restrict__ valB;
  const unsigned* __restrict__ R;
  const int4* __restrict__ rec0;     // per local A entry: {B start, length, R index lo, hi}
  const int4* __restrict__ rec1;     //   {C offset of its row lo, hi, first rank, last rank}
  const Unit* __restrict__ wunits;
  const Unit* __restrict__ lunits;
  const Small* small;                // unit counts, ea0
  int* lqhead;                       // large-row kernel: dynamic queue head
  int* gq_pos;                       //   per-block overflow queues of non-first products
  V* gq_val;                         //   (NUM_GDUP entries per block)
  int* ccol;
  V* cval;
};

// analysis.cu
cudaError_t launch_row_flops(cudaStream_t st, int M, const int* rpA, const int* colA, int K, const int* rpB, int* f,
                             uint8_t* nz, int* rowA, int* Pe, unsigned long long* hist, int* err, int* amax);
cudaError_t launch_classify(cudaStream_t st, int sms, const int* f, const uint8_t* nz, int rb, int re,
                            const ClassParams& prm, uint8_t* cls, int* fl, long long* Ro, const HeavyLists& lists,
                            Small* small, long long* crow);
cudaError_t launch_tiles(cudaStream_t st, int sms, const int* f, int rb, int re, int tile_cap, const uint8_t* cls,
                         const long long* PL, long long* Ro, uint8_t* tflag, int* tiles, Small* small,
                         long long r_cap);
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
cudaError_t launch_light_rank(cudaStream_t st, int grid, const SymProb& P, const int* tiles, const int* ntiles,
                              const uint8_t* tflag, const long long* PL, int* fb_list, int* fb_count);

// k_heavy.cu — symbolic ranks of heavy rows (column bitmap), per bin or over an explicit list.
cudaError_t heavy_configure();
int heavy_occupancy(int bin);
cudaError_t launch_heavy_rank(int bin, cudaStream_t st, int grid, const SymProb& P, const int* list,
                              const int* count, long long N);

// k_numeric.cu — numeric plan (end of symbolic) and numeric phase.
cudaError_t launch_plan(cudaStream_t st, int sms, const long long* crow, int mloc, const int* rpA, const int* colA,
                        const int* rpB, const int* rowA, const int* Pe, const long long* Ro, const unsigned* R, int rb,
                        int re, long long nnzA_upper, int* cnt, long long* coff, long long* scan_tmp, Cut* cuts,
                        Unit* wunits, Unit* lunits, int lcap, int4* rec0, int4* rec1, Small* small);
int plan_launches(long long mloc);
template <typename V>
cudaError_t numeric_configure();
template <typename V>
int numeric_occupancy(int which);  // 0: windows, 1..3: large-row kernel configuration 0..2
template <typename V>
cudaError_t launch_num_windows(cudaStream_t st, int grid, const NumProb<V>& P);
template <typename V>
cudaError_t launch_num_large(cudaStream_t st, int grid, int cfg, const NumProb<V>& P);

}  // namespace spg
