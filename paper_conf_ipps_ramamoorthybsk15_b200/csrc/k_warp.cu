// k_warp.cu — symbolic phase of the smallest light rows (f_i <= SPG_OPT_WARP_MAX_FLOPS, default
// 256): one warp per row, everything in registers and a few KB of warp-private shared memory, no
// block barriers.  The paper's A_L rows are "numerous subproblems of small computational
// intensity"; at this size a warp is the right processor (L33, L261).
//
//   expand  the row's A entries, 32 at a time: run lengths len_B, a warp scan gives each run's
//           product offset; the run table (offset, B start, A entry) goes to shared memory
//   keys    product p (p < f <= 256) of lane l, slot s: p = PT·l + s; its run by binary search in
//           the run table; key = column << 8 | p, {A entry, B entry} parked in shared memory
//   sort    bitonic network over the warp's 32·PT keys (PT = 1, 2, 4, 8 per lane: the smallest
//           power of two with 32·PT >= f): in-lane compare-exchanges, then shuffles
//   ranks   a key is a head when its column differs from the previous key's; rank = heads before
//           it (warp scan of per-lane head counts); heads write the gather plan EQ[Ro_i + rank],
//           the others the dup list (slots reserved once per row: f_i - c_i); c_i = heads
// (Phase IV "sort by (r,c), mark, scan, compact" of PAPER.md L154-156, per row in registers.)
//
// Measured on webbase1m (B200): with every light row of f <= 256 here (224k rows, 8.4M products)
// this kernel takes 746 us against the 219 us it saves the tile kernel — a warp per row waits on
// five dependent global round trips (row list, row pointers, A columns, B row pointers, B
// columns) per ~40 products, where a tile amortises them over ~4000.  So it is off by default
// (SPG_OPT_WARP_MAX_FLOPS = 0) and kept as an option and a tested alternative path.  Rows with
// f <= 32 go four per warp (group_rows): +0.7% on citpatents, +1% on webgoogle, -2% on webbase1m.
#include "kernels.cuh"

namespace spg {

constexpr int WARP_NT = 256;                 // 8 warps per block
constexpr int WARP_RT = 256;                 // run-table entries per warp (f <= 256 non-empty runs)
constexpr unsigned long long KEY_PAD = ~0ull;

struct WarpSmem {
  int off[WARP_RT + 1];   // run -> first product
  int bs[WARP_RT];        // run -> B start
  int ae[WARP_RT];        // run -> A entry
  int2 eq[WARP_MAX_CAP];  // product -> {A entry, B entry}
};

__device__ __forceinline__ unsigned long long shfl_xor64(unsigned long long v, int m) {
  const unsigned lo = __shfl_xor_sync(FULL, (unsigned)v, m), hi = __shfl_xor_sync(FULL, (unsigned)(v >> 32), m);
  return ((unsigned long long)hi << 32) | lo;
}
__device__ __forceinline__ unsigned long long shfl_up64(unsigned long long v, int d) {
  const unsigned lo = __shfl_up_sync(FULL, (unsigned)v, d), hi = __shfl_up_sync(FULL, (unsigned)(v >> 32), d);
  return ((unsigned long long)hi << 32) | lo;
}

// Ascending bitonic sort of the warp's 32·PT keys, element i = PT·lane + s held in k[s].
template <int PT>
__device__ __forceinline__ void warp_bitonic(unsigned long long (&k)[PT]) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int size = 2; size <= 32 * PT; size <<= 1) {
#pragma unroll
    for (int j = size >> 1; j > 0; j >>= 1) {
      if (j >= PT) {  // partner in lane ^ (j / PT), same slot
        const int lm = j / PT;
#pragma unroll
        for (int s = 0; s < PT; ++s) {
          const int i = PT * lane + s;
          const unsigned long long o = shfl_xor64(k[s], lm);
          const bool up = (i & size) == 0, low = (i & j) == 0;
          const bool take_min = up == low;
          k[s] = take_min ? (o < k[s] ? o : k[s]) : (o > k[s] ? o : k[s]);
        }
      } else {  // partner in the same lane
#pragma unroll
        for (int s = 0; s < PT; ++s) {
          if ((s & j) == 0) {
            const int i = PT * lane + s;
            const bool up = (i & size) == 0;
            const unsigned long long a = k[s], b = k[s + j];
            const bool sw = up ? (a > b) : (a < b);
            k[s] = sw ? b : a;
            k[s + j] = sw ? a : b;
          }
        }
      }
    }
  }
}

template <int PT>
__device__ __forceinline__ void warp_row(const SymProb& P, WarpSmem& W, int li, int f, int nruns) {
  const int lane = threadIdx.x & 31;
  unsigned long long k[PT];
  // keys: run of product p by binary search in the run table (off[] ascending, off[0] = 0)
#pragma unroll
  for (int s = 0; s < PT; ++s) {
    const int p = PT * lane + s;
    k[s] = KEY_PAD;
    if (p < f) {
      const int r = upper_idx(W.off, nruns, p);
      const int q = W.bs[r] + (p - W.off[r]);
      W.eq[p] = make_int2(W.ae[r], q);
      k[s] = ((unsigned long long)(unsigned)__ldg(P.colB + q) << 8) | (unsigned)p;
    }
  }
  __syncwarp();  // W.eq is read back by other lanes after the sort
  warp_bitonic<PT>(k);
  // heads, ranks
  unsigned long long prev = shfl_up64(k[PT - 1], 1);
  int nh = 0;
  bool head[PT];
#pragma unroll
  for (int s = 0; s < PT; ++s) {
    const unsigned long long pk = s == 0 ? prev : k[s - 1];
    const bool valid = k[s] != KEY_PAD;
    head[s] = valid && ((PT * lane + s) == 0 || (pk >> 8) != (k[s] >> 8));
    nh += head[s];
  }
  int incl = nh;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int o = __shfl_up_sync(FULL, incl, d);
    if (lane >= d) incl += o;
  }
  const int c = __shfl_sync(FULL, incl, 31);
  int rank = incl - nh - 1;  // rank of the last head before this lane's first slot
  // dup slots of the row: f - c, one reservation per row; per-lane offsets by a warp scan
  const int nd_lane = [&] {
    int n = 0;
#pragma unroll
    for (int s = 0; s < PT; ++s) n += (k[s] != KEY_PAD) && !head[s];
    return n;
  }();
  int dincl = nd_lane;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int o = __shfl_up_sync(FULL, dincl, d);
    if (lane >= d) dincl += o;
  }
  unsigned long long dbase = 0;
  if (lane == 0 && f > c) dbase = atomicAdd(P.dupn, (unsigned long long)(f - c));
  dbase = __shfl_sync(FULL, dbase, 0) + (unsigned long long)(dincl - nd_lane);
  int2* EQrow = P.EQ + P.Ro[li];
#pragma unroll
  for (int s = 0; s < PT; ++s) {
    if (k[s] == KEY_PAD) continue;
    const int2 eq = W.eq[(int)(k[s] & 0xff)];
    if (head[s]) {
      ++rank;
      EQrow[rank] = eq;
    } else {
      if ((long long)dbase < P.dupcap) P.dup[dbase] = make_int4(li, rank, eq.x, eq.y);
      ++dbase;
    }
  }
  if (lane == 0) P.crow[li + 1] = c;
}

// Four tiny rows (f <= 32) per warp, one per 8-lane group (4 keys per lane): a warp per row would
// leave most lanes idle and pay the row set-up latency once per ~17 products.  Same steps as
// warp_row; every shuffle is warp-wide with width 8, loops run to the warp's longest row.
constexpr int G_LANES = 8, G_PT = 4, G_CAP = G_LANES * G_PT;  // 32 products per group
__device__ __forceinline__ unsigned long long gshfl_xor64(unsigned long long v, int m) {
  const unsigned lo = __shfl_xor_sync(FULL, (unsigned)v, m, G_LANES);
  const unsigned hi = __shfl_xor_sync(FULL, (unsigned)(v >> 32), m, G_LANES);
  return ((unsigned long long)hi << 32) | lo;
}
__device__ __forceinline__ int gscan(int v, int gl) {  // inclusive scan within the 8-lane group
#pragma unroll
  for (int d = 1; d < G_LANES; d <<= 1) {
    const int o = __shfl_up_sync(FULL, v, d, G_LANES);
    if (gl >= d) v += o;
  }
  return v;
}

__device__ __forceinline__ void group_rows(const SymProb& P, WarpSmem& W, bool active, int li) {
  const int lane = threadIdx.x & 31, g = lane >> 3, gl = lane & 7;
  int* off = W.off + 64 * g;
  int* bsr = W.bs + 64 * g;
  int* aer = W.ae + 64 * g;
  int2* eqs = W.eq + 64 * g;
  int pa0 = 0, pa1 = 0, f = 0;
  if (active) {
    const int i = P.row_begin + li;
    pa0 = P.rpA[i];
    pa1 = P.rpA[i + 1];
    f = P.frow[i];
  }
  // run table, 8 A entries per step (trip count of the warp's longest row)
  const int steps = __reduce_max_sync(FULL, (unsigned)((pa1 - pa0 + G_LANES - 1) / G_LANES));
  int nruns = 0, poff = 0;
  for (int st = 0; st < steps; ++st) {
    const int e = pa0 + st * G_LANES + gl;
    int L = 0, bs = 0;
    if (e < pa1) {
      const int kk = P.colA[e];
      bs = P.rpB[kk];
      L = P.rpB[kk + 1] - bs;
    }
    const unsigned gm = (__ballot_sync(FULL, L > 0) >> (8 * g)) & 0xffu;
    const int incl = gscan(L, gl);
    if (L > 0) {
      const int r = nruns + __popc(gm & ((1u << gl) - 1u));
      off[r] = poff + incl - L;
      bsr[r] = bs;
      aer[r] = e;
    }
    nruns += __popc(gm);
    poff += __shfl_sync(FULL, incl, G_LANES - 1, G_LANES);
  }
  if (gl == 0) off[nruns] = poff;
  __syncwarp();
  unsigned long long k[G_PT];
#pragma unroll
  for (int s = 0; s < G_PT; ++s) {
    const int p = G_PT * gl + s;
    k[s] = KEY_PAD;
    if (p < f) {
      const int r = upper_idx(off, nruns, p);
      const int q = bsr[r] + (p - off[r]);
      eqs[p] = make_int2(aer[r], q);
      k[s] = ((unsigned long long)(unsigned)__ldg(P.colB + q) << 8) | (unsigned)p;
    }
  }
  __syncwarp();
  // bitonic sort of the group's 32 keys, element i = 4·gl + s
#pragma unroll
  for (int size = 2; size <= G_CAP; size <<= 1) {
#pragma unroll
    for (int j = size >> 1; j > 0; j >>= 1) {
      if (j >= G_PT) {
#pragma unroll
        for (int s = 0; s < G_PT; ++s) {
          const int i = G_PT * gl + s;
          const unsigned long long o = gshfl_xor64(k[s], j / G_PT);
          const bool take_min = ((i & size) == 0) == ((i & j) == 0);
          k[s] = take_min ? (o < k[s] ? o : k[s]) : (o > k[s] ? o : k[s]);
        }
      } else {
#pragma unroll
        for (int s = 0; s < G_PT; ++s) {
          if ((s & j) == 0) {
            const int i = G_PT * gl + s;
            const bool up = (i & size) == 0;
            const unsigned long long a = k[s], b = k[s + j];
            const bool sw = up ? (a > b) : (a < b);
            k[s] = sw ? b : a;
            k[s + j] = sw ? a : b;
          }
        }
      }
    }
  }
  const unsigned plo = __shfl_up_sync(FULL, (unsigned)k[G_PT - 1], 1, G_LANES);
  const unsigned phi = __shfl_up_sync(FULL, (unsigned)(k[G_PT - 1] >> 32), 1, G_LANES);
  const unsigned long long prev = ((unsigned long long)phi << 32) | plo;
  bool head[G_PT];
  int nh = 0, ndl = 0;
#pragma unroll
  for (int s = 0; s < G_PT; ++s) {
    const unsigned long long pk = s == 0 ? prev : k[s - 1];
    const bool valid = k[s] != KEY_PAD;
    head[s] = valid && ((G_PT * gl + s) == 0 || (pk >> 8) != (k[s] >> 8));
    nh += head[s];
    ndl += valid && !head[s];
  }
  const int incl = gscan(nh, gl);
  const int c = __shfl_sync(FULL, incl, G_LANES - 1, G_LANES);
  int rank = incl - nh - 1;
  const int dincl = gscan(ndl, gl);
  unsigned long long dbase = 0;
  if (gl == 0 && active && f > c) dbase = atomicAdd(P.dupn, (unsigned long long)(f - c));
  const unsigned blo = __shfl_sync(FULL, (unsigned)dbase, 0, G_LANES);
  const unsigned bhi = __shfl_sync(FULL, (unsigned)(dbase >> 32), 0, G_LANES);
  dbase = (((unsigned long long)bhi << 32) | blo) + (unsigned long long)(dincl - ndl);
  if (active) {
    int2* EQrow = P.EQ + P.Ro[li];
#pragma unroll
    for (int s = 0; s < G_PT; ++s) {
      if (k[s] == KEY_PAD) continue;
      const int2 eq = eqs[(int)(k[s] & 0xff)];
      if (head[s]) {
        ++rank;
        EQrow[rank] = eq;
      } else {
        if ((long long)dbase < P.dupcap) P.dup[dbase] = make_int4(li, rank, eq.x, eq.y);
        ++dbase;
      }
    }
    if (gl == 0) P.crow[li + 1] = c;
  }
}

__global__ void __launch_bounds__(WARP_NT, 4) k_warp_rank(SymProb P, const int* __restrict__ list,
                                                       const int* __restrict__ count) {
  __shared__ WarpSmem s_w[WARP_NT / 32];
  if (*P.heavy_total > P.r_cap) return;  // the plan's heavy region (which holds these rows) must fit
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  WarpSmem& W = s_w[warp];
  const int n = *count;
  // quads of list entries: four tiny rows at once when all four have f <= 32, else one by one
  for (int t4 = 4 * (blockIdx.x * (WARP_NT / 32) + warp); t4 < n; t4 += 4 * gridDim.x * (WARP_NT / 32)) {
    const int tg = t4 + (lane >> 3);
    const bool act = tg < n;
    const int lg = act ? list[tg] : 0;
    const int fg = act ? P.frow[P.row_begin + lg] : 0;
    if (__all_sync(FULL, fg <= G_CAP)) {
      group_rows(P, W, act, lg);
      __syncwarp();
      continue;
    }
    for (int t = t4; t < min(n, t4 + 4); ++t) {
    const int li = list[t];
    const int i = P.row_begin + li;
    const int pa0 = P.rpA[i], pa1 = P.rpA[i + 1];
    const int f = P.frow[i];
    // run table: non-empty runs of the row's A entries, 32 entries per step
    int nruns = 0, poff = 0;
    for (int e0 = pa0; e0 < pa1; e0 += 32) {
      const int e = e0 + lane;
      int L = 0, bs = 0;
      if (e < pa1) {
        const int kk = P.colA[e];
        bs = P.rpB[kk];
        L = P.rpB[kk + 1] - bs;
      }
      const unsigned m = __ballot_sync(FULL, L > 0);
      int incl = L;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const int o = __shfl_up_sync(FULL, incl, d);
        if (lane >= d) incl += o;
      }
      if (L > 0) {
        const int r = nruns + __popc(m & lanemask_lt());
        W.off[r] = poff + incl - L;
        W.bs[r] = bs;
        W.ae[r] = e;
      }
      nruns += __popc(m);
      poff += __shfl_sync(FULL, incl, 31);
    }
    if (lane == 0) W.off[nruns] = poff;
    __syncwarp();
    if (f <= 32) warp_row<1>(P, W, li, f, nruns);
    else if (f <= 64) warp_row<2>(P, W, li, f, nruns);
    else if (f <= 128) warp_row<4>(P, W, li, f, nruns);
    else warp_row<8>(P, W, li, f, nruns);
    __syncwarp();
    }
  }
}

int warp_occupancy() {
  int nb = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_warp_rank, WARP_NT, 0);
  return nb < 1 ? 1 : nb;
}

cudaError_t launch_warp_rank(cudaStream_t st, int grid, const SymProb& P, const int* list, const int* count) {
  k_warp_rank<<<grid, WARP_NT, 0, st>>>(P, list, count);
  return cudaGetLastError();
}

}  // namespace spg
