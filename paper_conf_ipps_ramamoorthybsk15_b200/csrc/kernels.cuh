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

struct ClassLists {
  int* rows[NUM_CLS];
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
  int row_begin;
  long long* crow;
  int* ccol;
  V* cval;
};

// Dense-accumulator workspace of the HUGE tier (one slot per resident block).
template <typename V>
struct HugeWs {
  unsigned* bm;     // [slots][nbw] touched-column bitmap words (kept zero between rows)
  V* acc;           // [slots][N]   dense PartialOutput (kept zero between rows; numeric only)
  long long nbw;    // bitmap words per slot = ceil(N / 32)
  int nl1;          // level-1 summary words = ceil(nbw / 32) (in shared memory)
  long long N;
};

// analysis.cu
cudaError_t launch_row_flops(cudaStream_t st, int M, const int* rpA, const int* colA, int K, const int* rpB, int* f,
                             uint8_t* nz, unsigned long long* hist, int* err);
cudaError_t launch_classify(cudaStream_t st, int sms, const int* f, const uint8_t* nz, int rb, int re,
                            const int* range_d, const ClassParams& prm, const ClassLists& lists, int* counts,
                            unsigned long long* cstats, long long* crow);
size_t scan_tmp_elems(long long n);
int scan_launches(long long n);
template <typename Tin>
cudaError_t launch_incl_scan(cudaStream_t st, const Tin* in, long long* out, long long n, long long* tmp);
cudaError_t launch_split_points(cudaStream_t st, const long long* Pf, int M, int P, int* s);
cudaError_t launch_validate(cudaStream_t st, int sms, int M, const int* rp, const int* ci, int ncols, long long nnz,
                            int check_sorted, int* err);
cudaError_t launch_rebase(cudaStream_t st, long long* rp_full, int M, int P, const int* splits, const long long* off);

// kernels.cu — one launcher per (class, phase).  `count` is the device-side class size;
// `grid` is chosen by the caller (persistent grid-stride loops inside).
template <typename V>
struct ClassLaunch {
  static cudaError_t tiny(cudaStream_t, int grid, bool numeric, const Prob<V>&, const int* list, const int* count);
  static cudaError_t light(cudaStream_t, int grid, bool numeric, const Prob<V>&, const int* list, const int* count);
  static cudaError_t medium(cudaStream_t, int grid, bool numeric, const Prob<V>&, const int* list, const int* count);
  static cudaError_t heavy(cudaStream_t, int grid, bool numeric, const Prob<V>&, const int* list, const int* count);
  static cudaError_t single(cudaStream_t, int grid, const Prob<V>&, const int* list, const int* count);
  static cudaError_t huge(cudaStream_t, int grid, bool numeric, const Prob<V>&, const int* list, const int* count,
                          const HugeWs<V>&);
  static cudaError_t configure();  // opt-in dynamic shared memory sizes (once per device)
  static int max_blocks_per_sm(int cls, bool numeric);
  static size_t huge_smem(int nl1);
};

}  // namespace spg
