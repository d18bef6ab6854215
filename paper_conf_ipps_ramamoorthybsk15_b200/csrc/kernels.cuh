// kernels.cuh — declarations shared by the kernel translation units and the C-ABI layer.
#pragma once
#include "common.cuh"

namespace spg {

struct ClassParams {
  int light_max;   // f <= light_max -> LIGHT (warp merge), 32 < light_max <= LIGHT_CAP
  int medium_max;  // f <= medium_max -> MEDIUM (256-thread block)
  int heavy_max;   // f <= heavy_max -> HEAVY (512-thread block), else HUGE
  int force;       // -1 or a class id >= CLS_TINY
  int single_ok;   // B rows canonical -> SINGLE shortcut allowed
};

struct BinLists {
  int* rows[NUM_BINS];
};

// Problem view passed to the class kernels.  crow is the int64 C row-offset array of this
// rank's rows (index i - row_begin); symbolic writes counts at [i - row_begin + 1].
template <typename V>
struct Prob {
  const int* __restrict__ rpA;
  const int* __restrict__ colA;
  const V* __restrict__ valA;
  const int* __restrict__ rpB;
  const int* __restrict__ colB;
  const V* __restrict__ valB;
  const int* sp;    // per row: index of one A entry whose B row is non-empty (row analysis)
  const int* frow;  // per row: f_i (row analysis)
  int row_begin;
  int lgN;          // ceil(log2(N)), N = columns of B (>= 0)
  long long* crow;
  int* ccol;
  V* cval;
  int* fb_list;     // numeric: rows the light/medium kernels hand to the general kernel
  int* fb_count;    // [0] = rows, [16] = queue head of the general kernel
};

// analysis.cu
cudaError_t launch_row_flops(cudaStream_t st, int M, const int* rpA, const int* colA, int K, const int* rpB, int* f,
                             uint8_t* nz, int* sp, unsigned long long* hist, int* err, int* amax);
cudaError_t launch_classify(cudaStream_t st, int sms, const int* f, const uint8_t* nz, int rb, int re,
                            const ClassParams& prm, const BinLists& lists, int* counts, unsigned long long* cstats,
                            long long* crow);
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

// Class kernels: one launcher per bin and phase.  `count` is the device-side bin size; `grid`
// is chosen by the caller (persistent grid-stride loops inside).  N = columns of B.
template <typename V>
struct BinLaunch {
  static cudaError_t launch(int bin, cudaStream_t st, int grid, bool numeric, const Prob<V>& P, const int* list,
                            const int* count, long long N);
  static int rows_per_block(int bin);
  static int max_blocks_per_sm(int bin, bool numeric);
  static cudaError_t configure();  // opt-in dynamic shared memory sizes (once per device)
  // general (HUGE-tier) kernel over an explicit row list, e.g. the fallback list
  static cudaError_t launch_general(cudaStream_t st, int grid, const Prob<V>& P, const int* list, const int* count,
                                    long long N);
};

}  // namespace spg
