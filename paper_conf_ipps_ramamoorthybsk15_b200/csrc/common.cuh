// common.cuh — shared device helpers for the SpGEMM kernels (sm_100a).
#pragma once
#include <cstdint>
#include <climits>
#include <cuda_runtime.h>

namespace spg {

constexpr unsigned FULL = 0xffffffffu;
constexpr int KEY_INF = INT_MAX;  // sentinel column (> any valid column: N <= INT_MAX)

// Row classes — must match spg_row_class in include/spg.h.
enum : int { CLS_EMPTY = 0, CLS_SINGLE, CLS_TINY, CLS_LIGHT, CLS_MEDIUM, CLS_HEAVY, CLS_HUGE, NUM_CLS };

// Internal work lists ("bins"): a class may be split by kernel geometry (TINY by sub-warp width).
enum : int {
  BIN_SINGLE = 0, BIN_T4, BIN_T8, BIN_T16, BIN_T32,   // TINY: one W-lane group per row
  BIN_L64, BIN_L128, BIN_L256,                        // LIGHT: one warp per row, CAP = 64/128/256
  BIN_M512, BIN_M1024, BIN_M2048,                     // MEDIUM: one block per row, CAP = 512/1024/2048
  BIN_HEAVY, BIN_HEAVY2, BIN_HUGE,                    // HEAVY / HUGE: column-bitmap blocks
  NUM_BINS
};
__host__ __device__ constexpr int bin_class(int b) {
  return b == BIN_SINGLE ? CLS_SINGLE
       : b <= BIN_T32   ? CLS_TINY
       : b <= BIN_L256  ? CLS_LIGHT
       : b <= BIN_M2048 ? CLS_MEDIUM
       : b <= BIN_HEAVY2 ? CLS_HEAVY : CLS_HUGE;
}
__host__ __device__ constexpr int class_first_bin(int c) {
  return c == CLS_SINGLE ? BIN_SINGLE
       : c == CLS_TINY   ? BIN_T4
       : c == CLS_LIGHT  ? BIN_L64
       : c == CLS_MEDIUM ? BIN_M512
       : c == CLS_HEAVY  ? BIN_HEAVY : BIN_HUGE;
}
__host__ __device__ constexpr bool bin_is_bitmap(int b) { return b >= BIN_HEAVY; }

// Class-kernel geometry.
constexpr int TINY_MAX = 32;          // one product per lane of a 4/8/16/32-lane group
constexpr int LIGHT_CAP = 256;        // warp merge, per-warp shared memory
constexpr int LIGHT_WARPS = 7;        // warps per block in the light kernel (4 blocks / SM fit in smem)
constexpr int MED1_NT = 128;          // MEDIUM rows f <= 1024: 128-thread blocks
constexpr int MEDIUM_NT = 256;        // MEDIUM rows f <= 2048: 256-thread blocks (occupancy)
constexpr int MED1_CAP = 1024;        // MEDIUM rows split by shared-memory footprint
constexpr int MEDIUM_CAP = 2048;
constexpr int HEAVY_CAP = 8192;       // largest f of the register-cached bitmap mode
constexpr int HEAVY1_CAP = 4096;      // HEAVY rows up to this f run as 512-thread blocks, 2 per SM
constexpr int BMP_NT = 1024;          // bitmap kernel block size for HEAVY2 / HUGE (one block per SM)
constexpr int BMP_NT_S = 512;         // ... for HEAVY (two blocks per SM)
constexpr int MERGE_VT_MAX = 14;      // outputs per thread per merge round: min(ceil(f / G), 14) | 1

// Shared-memory bytes a merge of f products (nr <= f runs) needs: values x2, keys x2, seg.
template <typename V>
__host__ __device__ constexpr int merge_smem_bytes(int cap) {
  return cap * (int)(2 * sizeof(V) + 2 * sizeof(int)) + (cap + 1) * (int)sizeof(int);
}

__device__ __forceinline__ unsigned lanemask_lt() {
  unsigned m;
  asm("mov.u32 %0, %%lanemask_lt;" : "=r"(m));
  return m;
}
__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }

template <typename T>
__device__ __forceinline__ T warp_incl_scan(T v) {
  int lane = lane_id();
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    T o = __shfl_up_sync(FULL, v, d);
    if (lane >= d) v += o;
  }
  return v;
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
  for (int d = 16; d > 0; d >>= 1) v += __shfl_xor_sync(FULL, v, d);
  return v;
}

// Group = one warp (G == 32) or the whole block (G == blockDim.x).
template <int G>
struct Group {
  static_assert(G == 32 || (G % 32 == 0 && G <= 1024), "group size");
  int rank;
  int* scratch;  // block groups: >= G/32 + 1 ints of shared memory
  __device__ __forceinline__ void sync() const {
    if constexpr (G == 32) __syncwarp(); else __syncthreads();
  }
  // Exclusive scan of v over the group; *total = group sum.  All G threads must call.
  __device__ __forceinline__ int excl_scan(int v, int& total) const {
    int incl = warp_incl_scan(v);
    if constexpr (G == 32) {
      total = __shfl_sync(FULL, incl, 31);
      return incl - v;
    } else {
      constexpr int NW = G / 32;
      int w = rank >> 5, lane = rank & 31;
      if (lane == 31) scratch[w] = incl;
      __syncthreads();
      if (w == 0) {
        int x = lane < NW ? scratch[lane] : 0;
        int xi = warp_incl_scan(x);
        if (lane < NW) scratch[lane] = xi - x;
        if (lane == NW - 1) scratch[NW] = xi;
      }
      __syncthreads();
      int r = incl - v + scratch[w];
      total = scratch[NW];
      __syncthreads();
      return r;
    }
  }
  __device__ __forceinline__ int max(int v) const {
    v = __reduce_max_sync(FULL, v);
    if constexpr (G == 32) {
      return v;
    } else {
      constexpr int NW = G / 32;
      __shared__ int redm[NW + 1];
      if ((rank & 31) == 0) redm[rank >> 5] = v;
      __syncthreads();
      if (rank < 32) {
        int x = rank < NW ? redm[rank] : INT_MIN;
        x = __reduce_max_sync(FULL, x);
        if (rank == 0) redm[NW] = x;
      }
      __syncthreads();
      return redm[NW];
    }
  }
  __device__ __forceinline__ long long sum(long long v) const {
    v = warp_sum(v);
    if constexpr (G == 32) {
      return v;
    } else {
      constexpr int NW = G / 32;
      __shared__ long long red[NW + 1];
      if ((rank & 31) == 0) red[rank >> 5] = v;
      __syncthreads();
      if (rank < 32) {
        long long x = rank < NW ? red[rank] : 0;
        x = warp_sum(x);
        if (rank == 0) red[NW] = x;
      }
      __syncthreads();
      return red[NW];
    }
  }
};

// Largest r in [0, n) with a[r] <= x, given a non-decreasing and a[0] <= x.
__device__ __forceinline__ int upper_idx(const int* a, int n, int x) {
  int lo = 0, hi = n - 1;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (a[mid] <= x) lo = mid; else hi = mid - 1;
  }
  return lo;
}

}  // namespace spg
