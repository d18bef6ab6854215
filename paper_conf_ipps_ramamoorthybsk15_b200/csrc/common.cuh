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

// Kernel paths ("bins").  TINY/LIGHT/MEDIUM rows all take the light (tile) kernel; HEAVY rows
// the register-cached bitmap kernel (512 threads when f <= HEAVY1_CAP, else 1024); HUGE rows
// (and rows the light kernel hands over) the uncached bitmap kernel.
enum : int { BIN_HEAVY = 0, BIN_HEAVY2, BIN_HUGE, NUM_BINS };
// Row lists: the bitmap bins, then the warp-per-row rows (f <= warp_max, k_warp.cu).
constexpr int BIN_WARP = NUM_BINS;
constexpr int NUM_LISTS = NUM_BINS + 1;
constexpr int WARP_MAX_CAP = 256;      // largest f of the warp-per-row symbolic kernel
constexpr int WARP_MAX_DEFAULT = 0;  // off: measured slower than the tiles (k_warp.cu header)

// Per-row path code stored in the cls[] array (low 3 bits = class, bit 3 = light path).
constexpr uint8_t CLS_LIGHT_PATH = 8;

// Light (tile) kernel geometry.
constexpr int TINY_MAX = 32;          // class boundaries for statistics only (same kernel)
constexpr int LIGHTC_MAX = 256;
constexpr int TILE_PMAX = 4096;       // products per tile: tile capacity + light threshold <= this
constexpr int TILE_CAP_DEFAULT = 3072;
constexpr int LIGHT_MAX_DEFAULT = 1024;
constexpr int TILE_NT = 512;          // threads per tile block
constexpr int TILE_RM = 512;          // light rows per batch
#ifndef SPG_TILE_BK
#define SPG_TILE_BK 2
#endif
constexpr int TILE_BK = SPG_TILE_BK;   // expected products per bucket
constexpr int TILE_NBMAX = TILE_PMAX / TILE_BK + TILE_RM;  // buckets per batch (ceil per row)
// Heavy (bitmap) kernel geometry.
constexpr int HEAVY_CAP = 8192;       // largest f of the register-cached bitmap mode (1024 threads)
#ifndef SPG_HEAVY1_CAP
#define SPG_HEAVY1_CAP 4096
#endif
constexpr int HEAVY1_CAP = SPG_HEAVY1_CAP;  // ... 512-thread blocks, two per SM
constexpr int BMP_NT = 1024;
constexpr int BMP_NT_S = 512;

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

// Predicated global loads that the compiler may not sink below later branches: a run of them is
// issued back to back, so their latencies overlap (plain loads used only under a data-dependent
// branch get moved under it, serialising R -> B-value -> B-column round trips).
__device__ __forceinline__ int ldp_s32(const int* p, bool pred, int dflt = 0) {
  int v = dflt;
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q ld.global.nc.b32 %0, [%1]; }" : "+r"(v) : "l"(p), "r"((int)pred));
  return v;
}
__device__ __forceinline__ unsigned ldp_u32_stream(const unsigned* p, bool pred, unsigned dflt = 0) {
  unsigned v = dflt;
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q ld.global.nc.L1::no_allocate.b32 %0, [%1]; }"
               : "+r"(v) : "l"(p), "r"((int)pred));
  return v;
}
__device__ __forceinline__ double ldp_val(const double* p, bool pred) {
  double v = 0.0;
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q ld.global.nc.f64 %0, [%1]; }" : "+d"(v) : "l"(p), "r"((int)pred));
  return v;
}
__device__ __forceinline__ float ldp_val(const float* p, bool pred) {
  float v = 0.f;
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %2, 0; @q ld.global.nc.f32 %0, [%1]; }" : "+f"(v) : "l"(p), "r"((int)pred));
  return v;
}

__device__ __forceinline__ int4 ldp_v4(const int4* p, bool pred) {
  int4 v = make_int4(0, 0, 0, 0);
  asm volatile("{ .reg .pred q; setp.ne.b32 q, %4, 0; @q ld.global.nc.v4.s32 {%0, %1, %2, %3}, [%5]; }"
               : "+r"(v.x), "+r"(v.y), "+r"(v.z), "+r"(v.w) : "r"((int)pred), "l"(p));
  return v;
}

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
