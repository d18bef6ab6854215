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

// Heavy-row kernel bins (k_heavy.cu): HEAVY rows are register-cached in 512-thread blocks,
// HEAVY2 in 1024-thread blocks, HUGE rows are re-gathered per pass.
enum : int { BIN_HEAVY = 0, BIN_HEAVY2, BIN_HUGE, NUM_BINS };

// Per-row flags in the cls[] byte: low 3 bits = class, plus
constexpr uint8_t CLS_HEAVY_PATH = 8;   // the row is its own item (bitmap symbolic, row item in numeric)
constexpr uint8_t CLS_WIDE = 16;        // heavy row whose plan entries take two words (A row or a
                                        // referenced B row longer than 65535 entries)
constexpr uint8_t CLS_SOLO = 32;        // tile row that is a tile of its own (the next row starts one)

// Flags k_row_flops stores next to the run count (bits 0-1) in nz[]
constexpr uint8_t NZ_LONGB = 0x10;      // a referenced B row has more than 65535 entries
constexpr uint8_t NZ_ALEN64K = 0x20;    // the A row has more than 65535 entries
constexpr uint8_t NZ_ALEN512 = 0x40;    // ... more than 512 (one 512-thread bitmap gather chunk)
constexpr uint8_t NZ_ALEN1K = 0x80;     // ... more than 1024

// Tiles (k_light.cu, k_numeric.cu): runs of consecutive non-heavy rows.
constexpr int TINY_MAX = 32;          // class boundaries for statistics only (same kernel)
constexpr int LIGHTC_MAX = 256;
constexpr int TILE_PMAX = 4096;       // products per tile: tile capacity + light threshold <= this
constexpr int TILE_CAP_DEFAULT = 2048;
constexpr int LIGHT_MAX_DEFAULT = 2048;
constexpr int TILE_EC = 1024;         // entries: a tile never crosses a multiple of TILE_EC in A's
                                      // entry space, so with rows of <= TILE_EC entries it has
                                      // < 2 * TILE_EC entries
constexpr int TILE_RM = 256;          // rows per tile (tiles never cross a multiple of TILE_RM)
constexpr int TILE_NT = 512;          // threads per symbolic tile block
constexpr int TILE_BK = 2;            // expected products per bucket
// Heavy (bitmap) kernel geometry.
constexpr int HEAVY_CAP = 8192;       // largest f of the register-cached bitmap mode (1024 threads)
constexpr int HEAVY1_CAP = 4096;      // ... 512-thread blocks, two per SM
constexpr int BMP_NT = 1024;
constexpr int BMP_NT_S = 512;

// The plan (symbolic -> numeric contract).  For an item (a tile of rows, or one heavy row) with
// plan region [P0, P0 + products) — a prefix over rows of their product counts — the first
// c entries describe the item's outputs in C order (output P0 + o -> C offset crow_item + o) and
// the remaining products - c entries are its repeated products ("dups"), in any order.  An entry
// is {e_rel: A entry relative to the item's first A entry, qoff: offset within that entry's B
// row}, packed e_rel | qoff << 16 in one word (two words, e_rel then qoff, for CLS_WIDE rows).
__host__ __device__ __forceinline__ unsigned plan_pack(unsigned e_rel, unsigned qoff) { return e_rel | (qoff << 16); }

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
  // Exclusive scan of v over the group; *total = group sum.  All G threads must call.  TRAIL =
  // false drops the closing barrier that protects the scratch words from the next scan: only for
  // call sites followed by a barrier of their own before the group scans again.
  template <bool TRAIL = true>
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
      if constexpr (TRAIL) __syncthreads();
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
