// k_small.cu — light rows (the paper's A_L: "numerous subproblems of small computational
// intensity ... assigned to individual threads of the GPU"):
//
//   SINGLE  one non-empty B row referenced: C(i,:) = a * B(k,:).  A warp takes 32 rows,
//           loads their headers lane-parallel, and copies all their products as one flat,
//           4x-unrolled stream (many independent loads in flight).
//   TINY    f <= W (W = 4, 8, 16, 32): a W-lane group per row, one product per lane, bitonic
//           sort by shuffles inside the group, segmented sum of equal columns, compacted
//           write.  32/W rows per warp.
//   LIGHT   f <= 256: one warp per row, run merge in a per-warp shared-memory slice
//           (merge.cuh).
#include "merge.cuh"

namespace spg {

// ================================ SINGLE (numeric only) =========================================
template <typename V>
__global__ void __launch_bounds__(256) k_single(Prob<V> P, const int* __restrict__ list, const int* __restrict__ count) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n = *count;
  for (int t0 = (blockIdx.x * 8 + warp) * 32; t0 < n; t0 += gridDim.x * 8 * 32) {
    const int t = t0 + lane;
    int L = 0, bs = 0;
    long long base = 0;
    V a = V(0);
    if (t < n) {
      const int i = list[t];
      const int p = P.sp[i];
      const int k = P.colA[p];
      bs = P.rpB[k];
      L = P.rpB[k + 1] - bs;
      a = P.valA[p];
      base = P.crow[i - P.row_begin];
    }
    const int incl = warp_incl_scan(L);
    const int off = incl - L;
    const int tot = __shfl_sync(FULL, incl, 31);
    constexpr int U = 4;
    for (int e0 = 0; e0 < tot; e0 += 32 * U) {
      int q[U];
      long long o[U];
      V s[U];
      bool ok[U];
#pragma unroll
      for (int u = 0; u < U; ++u) {
        const int e = e0 + u * 32 + lane;
        int r = 0;  // largest row r with off_r <= e (binary lifting over lanes)
#pragma unroll
        for (int sft = 16; sft > 0; sft >>= 1) {
          const int c = r + sft;
          if (__shfl_sync(FULL, off, c) <= e && c < 32) r = c;
        }
        const int offr = __shfl_sync(FULL, off, r);
        q[u] = __shfl_sync(FULL, bs, r) + (e - offr);
        o[u] = __shfl_sync(FULL, base, r) + (e - offr);
        s[u] = __shfl_sync(FULL, a, r);
        ok[u] = e < tot;
      }
      int cc[U];
      V vv[U];
#pragma unroll
      for (int u = 0; u < U; ++u)
        if (ok[u]) { cc[u] = P.colB[q[u]]; vv[u] = P.valB[q[u]]; }
#pragma unroll
      for (int u = 0; u < U; ++u)
        if (ok[u]) { P.ccol[o[u]] = cc[u]; P.cval[o[u]] = s[u] * vv[u]; }
    }
  }
}

// ================================ TINY (W-lane groups) ==========================================
template <int W, bool NUM, typename V>
__global__ void __launch_bounds__(256) k_tiny(Prob<V> P, const int* __restrict__ list, const int* __restrict__ count) {
  constexpr int WPB = 8, GPW = 32 / W;
  __shared__ int s_bs[WPB][32];
  __shared__ int s_len[WPB][32];
  __shared__ V s_a[WPB][32];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int grp = lane / W, gl = lane % W, sb = grp * W;
  const unsigned gmask = W == 32 ? FULL : (((1u << W) - 1) << sb);
  const unsigned below = (1u << gl) - 1;  // group-relative lanes below me
  const int n = *count;
  for (int t0 = (blockIdx.x * WPB + warp) * GPW; t0 < n; t0 += gridDim.x * WPB * GPW) {
    const int t = t0 + grp;
    if (t >= n) continue;  // group-uniform
    const int i = list[t];
    const int pa0 = P.rpA[i], pa1 = P.rpA[i + 1];
    int nr = 0;
    for (int p0 = pa0; p0 < pa1; p0 += W) {
      const int p = p0 + gl;
      int L = 0, bs = 0;
      V a = V(0);
      if (p < pa1) {
        const int k = P.colA[p];
        bs = P.rpB[k];
        L = P.rpB[k + 1] - bs;
        if (NUM) a = P.valA[p];
      }
      const unsigned m = (__ballot_sync(gmask, L > 0) >> sb);
      if (L > 0) {
        const int slot = sb + nr + __popc(m & below);  // < sb + W because f <= W
        s_bs[warp][slot] = bs;
        s_len[warp][slot] = L;
        if (NUM) s_a[warp][slot] = a;
      }
      nr += __popc(m);
    }
    __syncwarp(gmask);
    const int myL = gl < nr ? s_len[warp][sb + gl] : 0;
    int incl = myL;
#pragma unroll
    for (int d = 1; d < W; d <<= 1) {
      const int o = __shfl_up_sync(gmask, incl, d, W);
      if (gl >= d) incl += o;
    }
    const int off = incl - myL;
    const int f = __shfl_sync(gmask, incl, W - 1, W);
    int r = 0;  // run of product gl: largest r < nr with off_r <= gl
#pragma unroll
    for (int sft = W / 2; sft > 0; sft >>= 1) {
      const int c = r + sft;
      const int oc = __shfl_sync(gmask, off, c & (W - 1), W);
      if (c < nr && oc <= gl) r = c;
    }
    const int offr = __shfl_sync(gmask, off, r, W);
    int key = KEY_INF;
    V val = V(0);
    if (gl < f) {
      const int q = s_bs[warp][sb + r] + (gl - offr);
      key = P.colB[q];
      if (NUM) val = s_a[warp][sb + r] * P.valB[q];
    }
    __syncwarp(gmask);
    // bitonic sort of (key, val) across the W lanes of the group, ascending
#pragma unroll
    for (int k = 2; k <= W; k <<= 1) {
#pragma unroll
      for (int j = k >> 1; j > 0; j >>= 1) {
        const int ok = __shfl_xor_sync(gmask, key, j, W);
        V ov = V(0);
        if (NUM) ov = __shfl_xor_sync(gmask, val, j, W);
        const bool up = (gl & k) == 0;
        const bool lower = (gl & j) == 0;
        const bool take = (lower == up) ? (ok < key) : (ok > key);
        if (take) {
          key = ok;
          if (NUM) val = ov;
        }
      }
    }
    const int prev = __shfl_up_sync(gmask, key, 1, W);
    const bool bnd = gl == 0 || prev != key;   // segment starts (incl. the INF tail)
    const bool head = bnd && key != KEY_INF;
    const unsigned hm = __ballot_sync(gmask, head) >> sb;
    if (!NUM) {
      if (gl == 0) P.crow[i - P.row_begin + 1] = __popc(hm);
    } else {
      const unsigned bm = __ballot_sync(gmask, bnd) >> sb;
      V v = val;
#pragma unroll
      for (int d = 1; d < W; d <<= 1) {  // segmented suffix sum: heads get their segment total
        const V o = __shfl_down_sync(gmask, v, d, W);
        if (gl + d < W && !(bm & (((1u << d) - 1) << (gl + 1)))) v += o;
      }
      if (head) {
        const long long pos = P.crow[i - P.row_begin] + __popc(hm & below);
        P.ccol[pos] = key;
        P.cval[pos] = v;
      }
    }
  }
}

// ================================ LIGHT (warp merge) ============================================
template <int CAP, bool NUM, typename V>
__global__ void __launch_bounds__(LIGHT_WARPS * 32) k_light(Prob<V> P, const int* __restrict__ list,
                                                           const int* __restrict__ count) {
  extern __shared__ __align__(16) char smem[];
  constexpr int PER = NUM ? esc2_smem_aligned<V, CAP>() : msmem_aligned<V, NUM>(CAP);
  const int warp = threadIdx.x >> 5;
  const Group<32> g{lane_id(), nullptr};
  char* my = smem + warp * PER;
  const int n = *count;
  for (int t = blockIdx.x * LIGHT_WARPS + warp; t < n; t += gridDim.x * LIGHT_WARPS)
    if constexpr (NUM) esc2_row<32, CAP, V>(P, list[t], g, my);
    else esc_row<32, CAP, NUM, V>(P, list[t], g, my);
}

// ================================ MEDIUM (block merge) ==========================================
template <int NT, int CAP, bool NUM, typename V>
__global__ void __launch_bounds__(NT) k_block(Prob<V> P, const int* __restrict__ list, const int* __restrict__ count) {
  extern __shared__ __align__(16) char smem[];
  __shared__ int scratch[NT / 32 + 1];
  const Group<NT> g{(int)threadIdx.x, scratch};
  const int n = *count;
  for (int t = blockIdx.x; t < n; t += gridDim.x) {
    if constexpr (NUM) esc2_row<NT, CAP, V>(P, list[t], g, smem);
    else esc_row<NT, CAP, NUM, V>(P, list[t], g, smem);
  }
}

// ================================ hash-set symbolic (LIGHT, MEDIUM) ==============================
// Symbolic only needs c_i = |distinct columns|: insert each product's column into an
// open-addressing set in shared memory (2f..4f slots, key = col + 1, ATOMS.CAS — native on
// sm_100a, half the STS rate) and count the successful claims.  No merge, no sort.
template <int G, int TCAP>
__device__ __forceinline__ void hash_count_row(const Prob<double>& P0, const int* __restrict__ rpA,
                                               const int* __restrict__ colA, const int* __restrict__ rpB,
                                               const int* __restrict__ colB, int i, int f, const Group<G>& g,
                                               unsigned* table, int* seg, int* sbs, long long* crow, int row_begin) {
  (void)P0;
  int lt = 1;
  while ((1 << lt) < 2 * f) ++lt;  // table size 2^lt >= 2f
  const int T = 1 << lt;
  for (int x = g.rank; x < T; x += G) table[x] = 0u;
  const int pa0 = rpA[i], pa1 = rpA[i + 1];
  int nr = 0, tot = 0;
  for (int p0 = pa0; p0 < pa1; p0 += G) {
    const int p = p0 + g.rank;
    int L = 0, bs = 0;
    if (p < pa1) {
      const int k = colA[p];
      bs = rpB[k];
      L = rpB[k + 1] - bs;
    }
    int t2;
    const int ex = g.excl_scan((L << 16) | (L > 0 ? 1 : 0), t2);  // f <= 2048, G <= 128
    if (L > 0) {
      seg[nr + (ex & 0xffff)] = tot + (ex >> 16);
      sbs[nr + (ex & 0xffff)] = bs;
    }
    nr += t2 & 0xffff;
    tot += t2 >> 16;
  }
  if (g.rank == 0) seg[nr] = tot;
  g.sync();
  int cnt = 0;
  for (int j = g.rank; j < tot; j += G) {
    const int r = upper_idx(seg, nr, j);
    const unsigned key = (unsigned)colB[sbs[r] + (j - seg[r])] + 1u;
    unsigned h = (key * 0x9E3779B1u) >> (32 - lt);
    while (true) {
      const unsigned old = atomicCAS(&table[h], 0u, key);
      if (old == 0u) { ++cnt; break; }
      if (old == key) break;
      h = (h + 1) & (T - 1);
    }
  }
  const long long c = g.sum(cnt);
  if (g.rank == 0) crow[i - row_begin + 1] = c;
  g.sync();
}

template <typename V, int TCAP>
__global__ void __launch_bounds__(LIGHT_WARPS * 32) k_hsym_warp(Prob<V> P, const int* __restrict__ list,
                                                               const int* __restrict__ count) {
  __shared__ unsigned s_table[LIGHT_WARPS][TCAP];
  __shared__ int s_seg[LIGHT_WARPS][TCAP / 2 + 1];
  __shared__ int s_bs[LIGHT_WARPS][TCAP / 2];
  const int warp = threadIdx.x >> 5;
  const Group<32> g{lane_id(), nullptr};
  const int n = *count;
  for (int t = blockIdx.x * LIGHT_WARPS + warp; t < n; t += gridDim.x * LIGHT_WARPS) {
    const int i = list[t];
    hash_count_row<32, TCAP>(Prob<double>{}, P.rpA, P.colA, P.rpB, P.colB, i, P.frow[i], g, s_table[warp],
                             s_seg[warp], s_bs[warp], P.crow, P.row_begin);
  }
}

template <typename V, int NT, int TCAP>
__global__ void __launch_bounds__(NT) k_hsym_block(Prob<V> P, const int* __restrict__ list,
                                                  const int* __restrict__ count) {
  __shared__ unsigned s_table[TCAP];
  __shared__ int s_seg[TCAP / 2 + 1];
  __shared__ int s_bs[TCAP / 2];
  __shared__ int scratch[NT / 32 + 1];
  const Group<NT> g{(int)threadIdx.x, scratch};
  const int n = *count;
  for (int t = blockIdx.x; t < n; t += gridDim.x) {
    const int i = list[t];
    hash_count_row<NT, TCAP>(Prob<double>{}, P.rpA, P.colA, P.rpB, P.colB, i, P.frow[i], g, s_table, s_seg, s_bs,
                             P.crow, P.row_begin);
  }
}

// ================================ launch glue ====================================================
// Merge-class geometry per bin: (threads per row, capacity); warp bins run LIGHT_WARPS rows per block.
__host__ __device__ constexpr int merge_cap(int bin) {
  return bin == BIN_L64 ? 64 : bin == BIN_L128 ? 128 : bin == BIN_L256 ? 256
       : bin == BIN_M512 ? 512 : bin == BIN_M1024 ? 1024 : 2048;
}
constexpr int M512_NT = 64;

template <typename V>
size_t small_smem(int bin, bool numeric) {
  if (!numeric && bin >= BIN_L64 && bin <= BIN_M2048) return 0;  // hash symbolic: static shared memory
  switch (bin) {
    case BIN_HEAVY: return esc2_smem_aligned<V, HEAVY1_CAP>();  // numeric HEAVY through ESC2
    case BIN_L64: return (size_t)LIGHT_WARPS * esc2_smem_aligned<V, 64>();
    case BIN_L128: return (size_t)LIGHT_WARPS * esc2_smem_aligned<V, 128>();
    case BIN_L256: return (size_t)LIGHT_WARPS * esc2_smem_aligned<V, 256>();
    case BIN_M512: return esc2_smem_aligned<V, 512>();
    case BIN_M1024: return esc2_smem_aligned<V, 1024>();
    case BIN_M2048: return esc2_smem_aligned<V, 2048>();
  }
  return 0;
}

template <typename V>
int small_threads(int bin) {
  return bin == BIN_M512 ? M512_NT : bin == BIN_M1024 ? MED1_NT : (bin == BIN_M2048 || bin == BIN_HEAVY) ? MEDIUM_NT
       : (bin >= BIN_L64 && bin <= BIN_L256) ? LIGHT_WARPS * 32 : 256;
}

template <typename V>
int small_rows_per_block(int bin) {
  switch (bin) {
    case BIN_SINGLE: return 8 * 32;
    case BIN_T4: return 8 * 8;
    case BIN_T8: return 8 * 4;
    case BIN_T16: return 8 * 2;
    case BIN_T32: return 8;
    case BIN_L64: case BIN_L128: case BIN_L256: return LIGHT_WARPS;
    default: return 1;
  }
}

template <typename V>
static const void* small_kernel(int bin, bool numeric) {
  switch (bin) {
    case BIN_SINGLE: return (const void*)k_single<V>;
    case BIN_T4: return numeric ? (const void*)k_tiny<4, true, V> : (const void*)k_tiny<4, false, V>;
    case BIN_T8: return numeric ? (const void*)k_tiny<8, true, V> : (const void*)k_tiny<8, false, V>;
    case BIN_T16: return numeric ? (const void*)k_tiny<16, true, V> : (const void*)k_tiny<16, false, V>;
    case BIN_T32: return numeric ? (const void*)k_tiny<32, true, V> : (const void*)k_tiny<32, false, V>;
    case BIN_L64: return numeric ? (const void*)k_light<64, true, V> : (const void*)k_hsym_warp<V, 128>;
    case BIN_L128: return numeric ? (const void*)k_light<128, true, V> : (const void*)k_hsym_warp<V, 256>;
    case BIN_L256: return numeric ? (const void*)k_light<256, true, V> : (const void*)k_hsym_warp<V, 512>;
    case BIN_M512:
      return numeric ? (const void*)k_block<M512_NT, 512, true, V> : (const void*)k_hsym_block<V, M512_NT, 1024>;
    case BIN_M1024:
      return numeric ? (const void*)k_block<MED1_NT, 1024, true, V> : (const void*)k_hsym_block<V, MED1_NT, 2048>;
    case BIN_M2048:
      return numeric ? (const void*)k_block<MEDIUM_NT, 2048, true, V> : (const void*)k_hsym_block<V, MEDIUM_NT, 4096>;
    case BIN_HEAVY:  // numeric only (symbolic HEAVY runs on the bitmap tier)
      return (const void*)k_block<MEDIUM_NT, HEAVY1_CAP, true, V>;
  }
  return nullptr;
}

template <typename V>
cudaError_t small_configure() {
  for (int bin : {BIN_L64, BIN_L128, BIN_L256, BIN_M512, BIN_M1024, BIN_M2048, BIN_HEAVY}) {
    cudaError_t e = cudaFuncSetAttribute(small_kernel<V>(bin, true), cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)small_smem<V>(bin, true));
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

template <typename V>
int small_occupancy(int bin, bool numeric) {
  int nb = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, small_kernel<V>(bin, numeric), small_threads<V>(bin),
                                                small_smem<V>(bin, numeric));
  return nb < 1 ? 1 : nb;
}

template <typename V>
cudaError_t small_launch(int bin, cudaStream_t st, int grid, bool numeric, const Prob<V>& P, const int* list,
                         const int* count) {
  void* args[] = {(void*)&P, (void*)&list, (void*)&count};
  if (bin == BIN_SINGLE && !numeric) return cudaSuccess;
  return cudaLaunchKernel(small_kernel<V>(bin, numeric), dim3(grid), dim3(small_threads<V>(bin)), args,
                          small_smem<V>(bin, numeric), st);
}

#define INST(V)                                                                                        \
  template size_t small_smem<V>(int, bool);                                                            \
  template int small_threads<V>(int);                                                                  \
  template int small_rows_per_block<V>(int);                                                           \
  template cudaError_t small_configure<V>();                                                           \
  template int small_occupancy<V>(int, bool);                                                          \
  template cudaError_t small_launch<V>(int, cudaStream_t, int, bool, const Prob<V>&, const int*, const int*);
INST(double)
INST(float)
#undef INST

}  // namespace spg
