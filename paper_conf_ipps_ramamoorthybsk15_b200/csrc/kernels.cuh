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
//   numeric    k_numeric: windows of NUM_W consecutive outputs of C; every product of the
//              window's rows is scattered by its rank into shared memory and the window is
//              written out coalesced (the Phase IV merge of PAPER.md L154-156, with the sort
//              moved to the symbolic phase so numeric re-runs are a stream over R).
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

// Problem view of the numeric kernel.
template <typename V>
struct NumProb {
  const int* __restrict__ rpA;
  const int* __restrict__ colA;
  const V* __restrict__ valA;
  const int* __restrict__ rpB;
  const int* __restrict__ colB;
  const V* __restrict__ valB;
  const int* __restrict__ rowA;   // global row of each A entry
  const int* __restrict__ Pe;     // in-row product offset of each A entry
  const long long* __restrict__ Ro;
  const unsigned* __restrict__ R;
  const long long* __restrict__ crow;
  const int* __restrict__ wrow;   // first local row of each window
  int* ccol;
  V* cval;
  long long nnzC;
  int nwin;
  int row_begin, mloc;
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

// k_numeric.cu — numeric phase.
template <typename V>
cudaError_t numeric_configure();
cudaError_t launch_window_rows(cudaStream_t st, const long long* crow, int mloc, int* wrow, int nwin);
template <typename V>
cudaError_t launch_numeric(cudaStream_t st, const NumProb<V>& P);

}  // namespace spg
