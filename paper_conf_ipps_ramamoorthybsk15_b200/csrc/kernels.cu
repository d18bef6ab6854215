// kernels.cu — symbolic and numeric class kernels (Phases II/III + the fused Phase IV of
// PAPER.md Algorithm 1, recast for one GPU).
//
// Every row of C is C(i,:) = sum_k A(i,k) B(k,:) (Row-Row formulation).  The
// products of row i are the union of the B rows its A entries select ("runs"); each run is
// already sorted by column (B canonical).  Instead of hashing products and sorting the
// result, the light/medium/heavy kernels MERGE the sorted runs pairwise in shared memory
// (log2(#runs) rounds of merge-path merges), then add like-tuples (equal adjacent columns)
// and write the compacted, sorted row straight into CSR — the paper's Phase IV merge
// (sort by (r,c), mark, scan, one master thread adds, compact; L154-156) done per row in
// shared memory, with no tuples crossing a device boundary.
//
//   TINY   (f <= 32)          one warp per row; products in registers, bitonic sort by shuffles
//   LIGHT  (f <= 256)         one warp per row; run merge in a per-warp shared-memory slice
//   MEDIUM (f <= 2048)        256-thread block per row; run merge in shared memory
//   HEAVY  (f <= 8192)        512-thread block per row; run merge in shared memory
//   HUGE   (f >  8192)        1024-thread block per row; dense accumulator PartialOutput[N]
//                             plus a touched-column bitmap (the [13] Alg. 1 data structures
//                             of PAPER.md L86-88), read back in column order
//   SINGLE (one non-empty run) scaled copy of that B row (c_i = f_i, no symbolic work)
#include "kernels.cuh"

namespace spg {

template <typename V, bool NUM>
__host__ __device__ constexpr int msmem(int cap) {
  return (NUM ? cap * (int)(2 * sizeof(V)) : 0) + cap * 2 * (int)sizeof(int) + (cap + 1) * (int)sizeof(int);
}
template <typename V, bool NUM>
__host__ __device__ constexpr int msmem_aligned(int cap) {
  return (msmem<V, NUM>(cap) + 15) & ~15;
}

// ================================ TINY =========================================================
template <bool NUM, typename V>
__global__ void __launch_bounds__(256) k_tiny(Prob<V> P, const int* __restrict__ list, const int* __restrict__ count) {
  constexpr int WPB = 8;
  __shared__ int s_bs[WPB][32];
  __shared__ int s_len[WPB][32];
  __shared__ V s_a[WPB][32];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n = *count;
  for (int t = blockIdx.x * WPB + warp; t < n; t += gridDim.x * WPB) {
    const int i = list[t];
    const int pa0 = P.rpA[i], pa1 = P.rpA[i + 1];
    int nr = 0;
    for (int p0 = pa0; p0 < pa1; p0 += 32) {
      const int p = p0 + lane;
      int L = 0, bs = 0;
      V a = V(0);
      if (p < pa1) {
        const int k = P.colA[p];
        bs = P.rpB[k];
        L = P.rpB[k + 1] - bs;
        if (NUM) a = P.valA[p];
      }
      const unsigned m = __ballot_sync(FULL, L > 0);
      if (L > 0) {
        const int slot = nr + __popc(m & lanemask_lt());  // < 32 because f <= 32
        s_bs[warp][slot] = bs;
        s_len[warp][slot] = L;
        if (NUM) s_a[warp][slot] = a;
      }
      nr += __popc(m);
    }
    __syncwarp();
    const int myL = lane < nr ? s_len[warp][lane] : 0;
    const int incl = warp_incl_scan(myL);
    const int off = incl - myL;
    const int f = __shfl_sync(FULL, incl, 31);
    // run of product `lane`: largest r < nr with off_r <= lane (binary lifting over lanes)
    int r = 0;
#pragma unroll
    for (int s = 16; s > 0; s >>= 1) {
      const int cand = r + s;
      const int oc = __shfl_sync(FULL, off, cand & 31);
      if (cand < nr && oc <= lane) r = cand;
    }
    const int offr = __shfl_sync(FULL, off, r);
    int key = KEY_INF;
    V val = V(0);
    if (lane < f) {
      const int q = s_bs[warp][r] + (lane - offr);
      key = P.colB[q];
      if (NUM) val = s_a[warp][r] * P.valB[q];
    }
    __syncwarp();
    // bitonic sort of (key, val) across the 32 lanes, ascending
#pragma unroll
    for (int k = 2; k <= 32; k <<= 1) {
#pragma unroll
      for (int j = k >> 1; j > 0; j >>= 1) {
        const int ok = __shfl_xor_sync(FULL, key, j);
        V ov = V(0);
        if (NUM) ov = __shfl_xor_sync(FULL, val, j);
        const bool up = (lane & k) == 0;
        const bool lower = (lane & j) == 0;
        const bool take = (lower == up) ? (ok < key) : (ok > key);
        if (take) {
          key = ok;
          if (NUM) val = ov;
        }
      }
    }
    const int prev = __shfl_up_sync(FULL, key, 1);
    const bool bnd = lane == 0 || prev != key;       // segment starts (incl. the INF tail)
    const bool head = bnd && key != KEY_INF;
    const unsigned hm = __ballot_sync(FULL, head);
    if (!NUM) {
      if (lane == 0) P.crow[i - P.row_begin + 1] = __popc(hm);
    } else {
      const unsigned bm = __ballot_sync(FULL, bnd);
      V v = val;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {   // segmented suffix sum: heads get their segment total
        const V o = __shfl_down_sync(FULL, v, d);
        if (lane + d < 32 && !(bm & (((1u << d) - 1) << (lane + 1)))) v += o;
      }
      if (head) {
        const long long pos = P.crow[i - P.row_begin] + __popc(hm & lanemask_lt());
        P.ccol[pos] = key;
        P.cval[pos] = v;
      }
    }
  }
}

// ================================ run merge (LIGHT / MEDIUM / HEAVY) ===========================
// Shared-memory layout for capacity CAP (bytes = msmem<V,NUM>(CAP)):
//   valX[CAP] valY[CAP] (numeric only) | keyX[CAP] keyY[CAP] | seg[CAP+1]
template <int G, int CAP, bool NUM, typename V>
__device__ __forceinline__ void merge_row(const Prob<V>& P, const int i, const Group<G>& g, char* smem) {
  V* valX = reinterpret_cast<V*>(smem);
  V* valY = valX + CAP;
  int* keyX = reinterpret_cast<int*>(smem + (NUM ? 2 * CAP * sizeof(V) : 0));
  int* keyY = keyX + CAP;
  int* seg = keyY + CAP;
  const int pa0 = P.rpA[i], pa1 = P.rpA[i + 1];

  // 1. runs: compact the non-empty B rows this A row selects; seg = run offsets.
  //    (run start bs stashed in keyY, scale a in valY — both free until the first round)
  int nr = 0, f = 0;
  for (int p0 = pa0; p0 < pa1; p0 += G) {
    const int p = p0 + g.rank;
    int L = 0, bs = 0;
    V a = V(0);
    if (p < pa1) {
      const int k = P.colA[p];
      bs = P.rpB[k];
      L = P.rpB[k + 1] - bs;
      if (NUM) a = P.valA[p];
    }
    // pack (length, non-empty flag): f <= CAP <= 8192 and G <= 1024 keep the fields apart
    int tot;
    const int ex = g.excl_scan((L << 16) | (L > 0 ? 1 : 0), tot);
    if (L > 0) {
      const int slot = nr + (ex & 0xffff);
      seg[slot] = f + (ex >> 16);
      keyY[slot] = bs;
      if (NUM) valY[slot] = a;
    }
    nr += tot & 0xffff;
    f += tot >> 16;
  }
  if (g.rank == 0) seg[nr] = f;
  g.sync();

  // 2. expand: product j of run r -> keyX[j] = colB, valX[j] = a_r * valB (coalesced per run)
  for (int j = g.rank; j < f; j += G) {
    const int r = upper_idx(seg, nr, j);
    const int q = keyY[r] + (j - seg[r]);
    keyX[j] = P.colB[q];
    if (NUM) valX[j] = valY[r] * P.valB[q];
  }
  g.sync();

  // 3. pairwise merge rounds (merge path; ties take the left run first => stable)
  int* sk = keyX;
  int* dk = keyY;
  V* sv = valX;
  V* dv = valY;
  const int vt = (f + G - 1) / G;
  for (int w = 1; w < nr; w <<= 1) {
    const int npairs = (nr + 2 * w - 1) / (2 * w);
    int o = g.rank * vt;
    const int oend = min(o + vt, f);
    if (o < oend) {
      int lo = 0, hi = npairs - 1;
      while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (seg[2 * mid * w] <= o) lo = mid; else hi = mid - 1;
      }
      int m = lo;
      while (o < oend) {
        const int ra = 2 * m * w, rb = min(ra + w, nr), rc = min(ra + 2 * w, nr);
        const int a0 = seg[ra], a1 = seg[rb], a2 = seg[rc];
        const int n = min(oend, a2) - o;
        const int d = o - a0, La = a1 - a0, Lb = a2 - a1;
        int x0 = max(0, d - Lb), x1 = min(d, La);
        while (x0 < x1) {
          const int mid = (x0 + x1) >> 1;
          if (sk[a0 + mid] <= sk[a1 + d - 1 - mid]) x0 = mid + 1; else x1 = mid;
        }
        int ia = a0 + x0, ib = a1 + (d - x0);
        int ka = ia < a1 ? sk[ia] : KEY_INF;
        int kb = ib < a2 ? sk[ib] : KEY_INF;
        for (int t = 0; t < n; ++t) {
          if (ka <= kb) {
            dk[o + t] = ka;
            if (NUM) dv[o + t] = sv[ia];
            ++ia;
            ka = ia < a1 ? sk[ia] : KEY_INF;
          } else {
            dk[o + t] = kb;
            if (NUM) dv[o + t] = sv[ib];
            ++ib;
            kb = ib < a2 ? sk[ib] : KEY_INF;
          }
        }
        o += n;
        ++m;
      }
    }
    g.sync();
    int* tk = sk; sk = dk; dk = tk;
    V* tv = sv; sv = dv; dv = tv;
  }

  // 4. like-tuples: head = first of each equal-column group; heads add their group and write
  const long long rowoff = NUM ? P.crow[i - P.row_begin] : 0;
  int base = 0;
  for (int j0 = 0; j0 < f; j0 += G) {
    const int j = j0 + g.rank;
    const int kj = j < f ? sk[j] : KEY_INF;
    const bool head = j < f && (j == 0 || sk[j - 1] != kj);
    int tot;
    const int pos = g.excl_scan(head ? 1 : 0, tot);
    if (NUM && head) {
      V s = sv[j];
      for (int t = j + 1; t < f && sk[t] == kj; ++t) s += sv[t];
      P.ccol[rowoff + base + pos] = kj;
      P.cval[rowoff + base + pos] = s;
    }
    base += tot;
  }
  if (!NUM && g.rank == 0) P.crow[i - P.row_begin + 1] = base;
  g.sync();
}

template <bool NUM, typename V>
__global__ void __launch_bounds__(LIGHT_WARPS * 32) k_light(Prob<V> P, const int* __restrict__ list,
                                                           const int* __restrict__ count) {
  extern __shared__ __align__(16) char smem[];
  constexpr int PER = msmem_aligned<V, NUM>(LIGHT_CAP);
  const int warp = threadIdx.x >> 5;
  const Group<32> g{lane_id(), nullptr};
  char* my = smem + warp * PER;
  const int n = *count;
  for (int t = blockIdx.x * LIGHT_WARPS + warp; t < n; t += gridDim.x * LIGHT_WARPS)
    merge_row<32, LIGHT_CAP, NUM, V>(P, list[t], g, my);
}

template <int NT, int CAP, bool NUM, typename V>
__global__ void __launch_bounds__(NT) k_block(Prob<V> P, const int* __restrict__ list, const int* __restrict__ count) {
  extern __shared__ __align__(16) char smem[];
  __shared__ int scratch[NT / 32 + 1];
  const Group<NT> g{(int)threadIdx.x, scratch};
  const int n = *count;
  for (int t = blockIdx.x; t < n; t += gridDim.x) merge_row<NT, CAP, NUM, V>(P, list[t], g, smem);
}

// ================================ SINGLE (numeric only) =========================================
template <typename V>
__global__ void __launch_bounds__(256) k_single(Prob<V> P, const int* __restrict__ list, const int* __restrict__ count) {
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n = *count;
  for (int t = blockIdx.x * 8 + warp; t < n; t += gridDim.x * 8) {
    const int i = list[t];
    const int pa0 = P.rpA[i], pa1 = P.rpA[i + 1];
    int bs = 0, L = 0;
    V a = V(0);
    for (int p0 = pa0; p0 < pa1; p0 += 32) {
      const int p = p0 + lane;
      int Lp = 0, bsp = 0;
      if (p < pa1) {
        const int k = P.colA[p];
        bsp = P.rpB[k];
        Lp = P.rpB[k + 1] - bsp;
      }
      const unsigned m = __ballot_sync(FULL, Lp > 0);
      if (m) {
        const int src = __ffs(m) - 1;
        bs = __shfl_sync(FULL, bsp, src);
        L = __shfl_sync(FULL, Lp, src);
        a = P.valA[p0 + src];
        break;
      }
    }
    const long long base = P.crow[i - P.row_begin];
    for (int q = lane; q < L; q += 32) {
      P.ccol[base + q] = P.colB[bs + q];
      P.cval[base + q] = a * P.valB[bs + q];
    }
  }
}

// ================================ HUGE ===========================================================
// Dense accumulator PartialOutput[N] + touched bitmap per resident block (the
// [13] Alg. 1 arrays; "NonZeroIndices" becomes a bitmap whose in-order scan yields the sorted
// column list directly).  A level-1 summary bit per bitmap word lives in shared memory so the
// read-back only visits touched words.
template <bool NUM, typename V>
__global__ void __launch_bounds__(HUGE_NT, 1) k_huge(Prob<V> P, const int* __restrict__ list,
                                                    const int* __restrict__ count, HugeWs<V> ws) {
  extern __shared__ unsigned L1[];
  __shared__ int s_seg[HUGE_NT + 1];
  __shared__ int s_bs[HUGE_NT];
  __shared__ V s_a[HUGE_NT];
  __shared__ int scratch[HUGE_NT / 32 + 1];
  const Group<HUGE_NT> g{(int)threadIdx.x, scratch};
  unsigned* bm = ws.bm + (long long)blockIdx.x * ws.nbw;
  V* acc = NUM ? ws.acc + (long long)blockIdx.x * ws.N : nullptr;
  for (int u = threadIdx.x; u < ws.nl1; u += HUGE_NT) L1[u] = 0;
  __syncthreads();
  const int n = *count;
  for (int t = blockIdx.x; t < n; t += gridDim.x) {
    const int i = list[t];
    const int pa0 = P.rpA[i], pa1 = P.rpA[i + 1];
    long long cnt = 0;
    for (int p0 = pa0; p0 < pa1; p0 += HUGE_NT) {
      const int p = p0 + threadIdx.x;
      int L = 0, bs = 0;
      V a = V(0);
      if (p < pa1) {
        const int k = P.colA[p];
        bs = P.rpB[k];
        L = P.rpB[k + 1] - bs;
        if (NUM) a = P.valA[p];
      }
      int nz, Lt;
      const int rk = g.excl_scan(L > 0 ? 1 : 0, nz);
      const int off = g.excl_scan(L, Lt);  // f_i < 2^31 (checked in analysis)
      if (L > 0) {
        s_seg[rk] = off;
        s_bs[rk] = bs;
        if (NUM) s_a[rk] = a;
      }
      if (threadIdx.x == 0) s_seg[nz] = Lt;
      __syncthreads();
      for (int j = threadIdx.x; j < Lt; j += HUGE_NT) {
        const int r = upper_idx(s_seg, nz, j);
        const int q = s_bs[r] + (j - s_seg[r]);
        const int col = P.colB[q];
        const int w = col >> 5;
        const unsigned b = 1u << (col & 31);
        const unsigned old = atomicOr(&bm[w], b);
        if (!(old & b)) {
          ++cnt;
          if (old == 0) atomicOr(&L1[w >> 5], 1u << (w & 31));
        }
        if (NUM) atomicAdd(&acc[col], s_a[r] * P.valB[q]);
      }
      __syncthreads();
    }
    if (!NUM) {
      const long long c = g.sum(cnt);
      if (threadIdx.x == 0) P.crow[i - P.row_begin + 1] = c;
      for (int u = threadIdx.x; u < ws.nl1; u += HUGE_NT) {
        unsigned x = L1[u];
        if (x) {
          L1[u] = 0;
          while (x) {
            const int b = __ffs(x) - 1;
            x &= x - 1;
            bm[(long long)u * 32 + b] = 0;
          }
        }
      }
      __threadfence();
      __syncthreads();
    } else {
      __threadfence();
      __syncthreads();
      const long long rowoff = P.crow[i - P.row_begin];
      int carry = 0;
      for (int u0 = 0; u0 < ws.nl1; u0 += HUGE_NT) {
        const int u = u0 + threadIdx.x;
        const unsigned x = u < ws.nl1 ? L1[u] : 0u;
        int mine = 0;
        for (unsigned y = x; y; y &= y - 1)
          mine += __popc(__ldcg(&bm[(long long)u * 32 + (__ffs(y) - 1)]));
        int tot;
        int pos = carry + g.excl_scan(mine, tot);
        for (unsigned y = x; y; y &= y - 1) {
          const long long wi = (long long)u * 32 + (__ffs(y) - 1);
          unsigned wv = __ldcg(&bm[wi]);
          bm[wi] = 0;
          while (wv) {
            const int bit = __ffs(wv) - 1;
            wv &= wv - 1;
            P.ccol[rowoff + pos++] = (int)(wi * 32 + bit);
          }
        }
        if (x) L1[u] = 0;
        carry += tot;
      }
      __threadfence();
      __syncthreads();
      for (int j = threadIdx.x; j < carry; j += HUGE_NT) {
        const int col = __ldcg(&P.ccol[rowoff + j]);
        P.cval[rowoff + j] = __ldcg(&acc[col]);
        acc[col] = V(0);
      }
      __threadfence();
      __syncthreads();
    }
  }
}

// ================================ launchers =======================================================
template <typename K>
static cudaError_t set_smem(K kern, int bytes) {
  return cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
}

template <typename V>
cudaError_t ClassLaunch<V>::configure() {
  cudaError_t e;
  if ((e = set_smem(k_light<false, V>, LIGHT_WARPS * msmem_aligned<V, false>(LIGHT_CAP))) != cudaSuccess) return e;
  if ((e = set_smem(k_light<true, V>, LIGHT_WARPS * msmem_aligned<V, true>(LIGHT_CAP))) != cudaSuccess) return e;
  if ((e = set_smem(k_block<MEDIUM_NT, MEDIUM_CAP, false, V>, msmem_aligned<V, false>(MEDIUM_CAP))) != cudaSuccess) return e;
  if ((e = set_smem(k_block<MEDIUM_NT, MEDIUM_CAP, true, V>, msmem_aligned<V, true>(MEDIUM_CAP))) != cudaSuccess) return e;
  if ((e = set_smem(k_block<HEAVY_NT, HEAVY_CAP, false, V>, msmem_aligned<V, false>(HEAVY_CAP))) != cudaSuccess) return e;
  if ((e = set_smem(k_block<HEAVY_NT, HEAVY_CAP, true, V>, msmem_aligned<V, true>(HEAVY_CAP))) != cudaSuccess) return e;
  if ((e = set_smem(k_huge<false, V>, 128 * 1024)) != cudaSuccess) return e;
  if ((e = set_smem(k_huge<true, V>, 128 * 1024)) != cudaSuccess) return e;
  return cudaSuccess;
}

template <typename V>
size_t ClassLaunch<V>::huge_smem(int nl1) { return (size_t)nl1 * sizeof(unsigned); }

template <typename V>
int ClassLaunch<V>::max_blocks_per_sm(int cls, bool numeric) {
  int nb = 1;
  switch (cls) {
    case CLS_SINGLE: cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_single<V>, 256, 0); break;
    case CLS_TINY:
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, numeric ? k_tiny<true, V> : k_tiny<false, V>, 256, 0);
      break;
    case CLS_LIGHT:
      if (numeric) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_light<true, V>, LIGHT_WARPS * 32,
                                                                 LIGHT_WARPS * msmem_aligned<V, true>(LIGHT_CAP));
      else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_light<false, V>, LIGHT_WARPS * 32,
                                                         LIGHT_WARPS * msmem_aligned<V, false>(LIGHT_CAP));
      break;
    case CLS_MEDIUM:
      if (numeric) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_block<MEDIUM_NT, MEDIUM_CAP, true, V>,
                                                                 MEDIUM_NT, msmem_aligned<V, true>(MEDIUM_CAP));
      else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_block<MEDIUM_NT, MEDIUM_CAP, false, V>, MEDIUM_NT,
                                                         msmem_aligned<V, false>(MEDIUM_CAP));
      break;
    case CLS_HEAVY:
      if (numeric) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_block<HEAVY_NT, HEAVY_CAP, true, V>,
                                                                 HEAVY_NT, msmem_aligned<V, true>(HEAVY_CAP));
      else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_block<HEAVY_NT, HEAVY_CAP, false, V>, HEAVY_NT,
                                                         msmem_aligned<V, false>(HEAVY_CAP));
      break;
    default: nb = 1;
  }
  return nb < 1 ? 1 : nb;
}

template <typename V>
cudaError_t ClassLaunch<V>::tiny(cudaStream_t st, int grid, bool numeric, const Prob<V>& P, const int* list,
                                 const int* count) {
  if (numeric) k_tiny<true, V><<<grid, 256, 0, st>>>(P, list, count);
  else k_tiny<false, V><<<grid, 256, 0, st>>>(P, list, count);
  return cudaGetLastError();
}
template <typename V>
cudaError_t ClassLaunch<V>::light(cudaStream_t st, int grid, bool numeric, const Prob<V>& P, const int* list,
                                  const int* count) {
  if (numeric)
    k_light<true, V><<<grid, LIGHT_WARPS * 32, LIGHT_WARPS * msmem_aligned<V, true>(LIGHT_CAP), st>>>(P, list, count);
  else
    k_light<false, V><<<grid, LIGHT_WARPS * 32, LIGHT_WARPS * msmem_aligned<V, false>(LIGHT_CAP), st>>>(P, list, count);
  return cudaGetLastError();
}
template <typename V>
cudaError_t ClassLaunch<V>::medium(cudaStream_t st, int grid, bool numeric, const Prob<V>& P, const int* list,
                                   const int* count) {
  if (numeric)
    k_block<MEDIUM_NT, MEDIUM_CAP, true, V><<<grid, MEDIUM_NT, msmem_aligned<V, true>(MEDIUM_CAP), st>>>(P, list, count);
  else
    k_block<MEDIUM_NT, MEDIUM_CAP, false, V><<<grid, MEDIUM_NT, msmem_aligned<V, false>(MEDIUM_CAP), st>>>(P, list, count);
  return cudaGetLastError();
}
template <typename V>
cudaError_t ClassLaunch<V>::heavy(cudaStream_t st, int grid, bool numeric, const Prob<V>& P, const int* list,
                                  const int* count) {
  if (numeric)
    k_block<HEAVY_NT, HEAVY_CAP, true, V><<<grid, HEAVY_NT, msmem_aligned<V, true>(HEAVY_CAP), st>>>(P, list, count);
  else
    k_block<HEAVY_NT, HEAVY_CAP, false, V><<<grid, HEAVY_NT, msmem_aligned<V, false>(HEAVY_CAP), st>>>(P, list, count);
  return cudaGetLastError();
}
template <typename V>
cudaError_t ClassLaunch<V>::single(cudaStream_t st, int grid, const Prob<V>& P, const int* list, const int* count) {
  k_single<V><<<grid, 256, 0, st>>>(P, list, count);
  return cudaGetLastError();
}
template <typename V>
cudaError_t ClassLaunch<V>::huge(cudaStream_t st, int grid, bool numeric, const Prob<V>& P, const int* list,
                                 const int* count, const HugeWs<V>& ws) {
  const size_t sm = huge_smem(ws.nl1);
  if (numeric) k_huge<true, V><<<grid, HUGE_NT, sm, st>>>(P, list, count, ws);
  else k_huge<false, V><<<grid, HUGE_NT, sm, st>>>(P, list, count, ws);
  return cudaGetLastError();
}

template struct ClassLaunch<double>;
template struct ClassLaunch<float>;

}  // namespace spg
