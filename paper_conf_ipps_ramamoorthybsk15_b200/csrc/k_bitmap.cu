// k_bitmap.cu — heavy rows (the paper's A_H: "good cache blocking techniques can be used when
// multiplying A_H with B_H"): one 1024-thread block per row, a column-tile
// bitmap in shared memory.
//
// The dense accumulator of [13] Alg. 1 (PartialOutput[N] + NonZeroIndices)
// becomes a bitmap over a column tile of width Wt (TR_b of L88): products are claimed with
// ATOMS.OR — on sm_100a as fast as a plain STS (tools/microbench_atomics.cu) — and a scan of
// the bitmap in column order yields the row's columns already sorted, so no sort is ever run.
// A level-1 summary bit per bitmap word lets every scan visit only touched words.
//
//   symbolic  pass 1 only: c_i = number of bits claimed.
//   numeric   pass 1  claim bits; the first claimer of a column sets its product's flag bit;
//             build   rank prefix per 1024-column superblock; C_col written in column order;
//             pass 2  rank(col) = prefix(superblock) + popc of the touched words below it +
//                     popc(bits below) -> first claimers store a*b into val[rank] (shared);
//             pass 3  duplicates (~7% of products) add with a shared atomic after a barrier,
//                     so no fp64 CAS loop races a first store; val is written out coalesced.
// Products are visited as work items (<= 64 consecutive products of one B row, one warp), so
// loads are coalesced and the run lookup is done once per item.  The tile width is the largest
// power of two whose structures plus expected values fit (2^20 columns for webbase-sized N, so
// these rows take a single tile); a tile whose distinct columns overflow the value slots falls
// back to RED.ADD into C_val in L2 (correct, slower).
#include "kernels.cuh"

namespace spg {

constexpr int BMP_RCAP = 1024;       // runs gathered per chunk (one per thread)
constexpr int BMP_CTCAP = 2048;      // 32-product windows per chunk with a precomputed run index
constexpr int BMP_SLOTS = 8;         // products per lane cached in registers across passes
constexpr int MODE_SYM = 0, MODE_NUM = 1;

__host__ __device__ constexpr int al16(int x) { return (x + 15) & ~15; }

template <typename V>
__host__ __device__ constexpr int bmp_fixed_bytes() {
  return 2 * al16((BMP_RCAP + 1) * 4) + al16(BMP_RCAP * (int)sizeof(V)) + al16(BMP_CTCAP * 2);
}
constexpr int BMP_SMEM = 226 * 1024;  // dynamic shared memory per block (1 block / SM; static on top)

// Region bytes for a 2^lw column tile: bitmap, level-1 summary (one bit per bitmap word), the
// rank prefixes (int per 1024 columns, u16 per 256 columns relative to its 1024) and — numeric —
// first-claim flags (f bits).
__device__ __forceinline__ int bmp_struct(int lw, int f, bool numeric, bool flags) {
  const int words = 1 << (lw - 5), nl1 = 1 << (lw - 10);
  int need = 4 * words + 4 * nl1;
  if (numeric) need += 4 * nl1 + 8 * nl1 + (flags ? 4 * ((f + 31) >> 5) : 0) + 16;
  return need;
}

template <int MODE, typename V>
__global__ void __launch_bounds__(BMP_NT, 1) k_bitmap(Prob<V> P, const int* __restrict__ list,
                                                     const int* __restrict__ count, int lwmax, int N) {
  constexpr bool NUM = MODE == MODE_NUM;
  extern __shared__ __align__(16) unsigned char sm[];
  int* seg = reinterpret_cast<int*>(sm);                                   // run -> product offset
  int* sbs = reinterpret_cast<int*>(sm + al16((BMP_RCAP + 1) * 4));        // run -> B row start
  V* sa = reinterpret_cast<V*>(sm + 2 * al16((BMP_RCAP + 1) * 4));         // run -> A value
  unsigned short* ctab = reinterpret_cast<unsigned short*>(sm + 2 * al16((BMP_RCAP + 1) * 4) +
                                                           al16(BMP_RCAP * (int)sizeof(V)));  // window -> run
  unsigned char* region = sm + bmp_fixed_bytes<V>();
  constexpr int REGION = BMP_SMEM - bmp_fixed_bytes<V>();
  __shared__ int scratch[BMP_NT / 32 + 1];
  const Group<BMP_NT> g{(int)threadIdx.x, scratch};
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const unsigned upto = (2u << lane) - 1u;  // lanes <= me

  // invariant between rows: the whole region is zero
  for (int x = tid; x < REGION / 4; x += BMP_NT) reinterpret_cast<unsigned*>(region)[x] = 0;
  __syncthreads();

  const int n = *count;
  for (int t = blockIdx.x; t < n; t += gridDim.x) {
    const int i = list[t];
    const int pa0 = P.rpA[i], pa1 = P.rpA[i + 1];
    const int f = P.frow[i];
    // Column tile: the widest one whose structures fit (one tile for N <= 2^20).  Values are
    // staged in shared memory when the tile's distinct columns fit the remaining space, else
    // they are added into C_val in L2 (rows with tens of thousands of distinct columns).
    const bool useflags = NUM && f <= 32 * BMP_NT * 4;
    int lw = lwmax;
    while (lw > 10 && bmp_struct(lw, f, NUM, useflags) > REGION) --lw;
    const int Wt = 1 << lw, words = Wt >> 5, nl1 = 1 << (lw - 10);
    unsigned* bm = reinterpret_cast<unsigned*>(region);
    unsigned* l1 = bm + words;
    int* sbp = reinterpret_cast<int*>(l1 + nl1);                          // rank prefix / 1024 columns
    unsigned short* sbq = reinterpret_cast<unsigned short*>(sbp + (NUM ? nl1 : 0));  // .. / 256 columns
    unsigned* flags = reinterpret_cast<unsigned*>(sbq + (NUM ? 4 * nl1 : 0));
    const int nfw = useflags ? (f + 31) >> 5 : 0;
    const int voff = (4 * (words + (NUM ? 4 : 1) * nl1 + nfw) + 15) & ~15;
    V* val = reinterpret_cast<V*>(region + voff);
    const int vcap = useflags ? (REGION - voff) / (int)sizeof(V) : 0;
    const int ntiles = (int)(((long long)N + Wt - 1) >> lw);
    const int nchunks = (pa1 - pa0 + BMP_RCAP - 1) / BMP_RCAP;
    const long long rowoff = NUM ? P.crow[i - P.row_begin] : 0;
    long long cnt = 0;
    int out = 0;
    int nz = 0, Lt = 0;  // current chunk: runs, products
    // register cache of this lane's products (B position, column, run) for single-chunk rows
    const bool cached = NUM && pa1 - pa0 <= BMP_RCAP && f <= BMP_SLOTS * BMP_NT;
    int cq[BMP_SLOTS], cc[BMP_SLOTS], cr[BMP_SLOTS];

    auto gather = [&](int c) {
      const int p = pa0 + c * BMP_RCAP + tid;
      const int pend = min(pa1, pa0 + (c + 1) * BMP_RCAP);
      int L = 0, bs = 0;
      V a = V(0);
      if (tid < BMP_RCAP && p < pend) {
        const int k = P.colA[p];
        bs = P.rpB[k];
        L = P.rpB[k + 1] - bs;
        if (NUM) a = P.valA[p];
      }
      const int rk = g.excl_scan(L > 0 ? 1 : 0, nz);
      const int off = g.excl_scan(L, Lt);  // f_i < 2^31 (checked in analysis)
      if (L > 0) {
        seg[rk] = off;
        sbs[rk] = bs;
        if (NUM) sa[rk] = a;
      }
      if (tid == 0) seg[nz] = Lt;
      __syncthreads();
      for (int x = tid; x < min((Lt + 31) >> 5, BMP_CTCAP); x += BMP_NT) ctab[x] = (unsigned short)upper_idx(seg, nz, x << 5);
      __syncthreads();
    };

    // product window [j0, j0+32): run of each lane (runs starting inside the window form a
    // bitmask, REDUX.OR; a lane's run = the window's first run + popcount of starts <= it)
    auto lane_run = [&](int j0) {
      const int rb = (j0 >> 5) < BMP_CTCAP ? (int)ctab[j0 >> 5] : upper_idx(seg, nz, j0);
      const int rs = rb + 1 + lane;
      const int d = rs <= nz ? seg[rs] - j0 : 32;
      const unsigned M = __reduce_or_sync(FULL, (d >= 1 && d <= 31) ? (1u << d) : 0u);
      return rb + __popc(M & upto);
    };

    // Visit the products of the current chunk that fall in [lo, lo+Wt).  Each warp takes 32
    // consecutive products (coalesced within a B row): one binary search finds the run of the
    // first; the runs starting inside the window form a bitmask (REDUX.OR) and each lane's run is
    // the first run + popcount of the starts at or below it.
    auto for_products = [&](int lo, auto&& fn) {
      if (cached) {
#pragma unroll
        for (int s = 0; s < BMP_SLOTS; ++s) {
          const int j = warp * 32 + s * BMP_NT + lane;
          const unsigned lc = (unsigned)(cc[s] - lo);
          if (j < Lt && lc < (unsigned)Wt) fn(j, cq[s], lc, cr[s]);
        }
        return;
      }
      for (int j0 = warp * 32; j0 < Lt; j0 += BMP_NT) {
        const int r = lane_run(j0);
        const int j = j0 + lane;
        if (j < Lt) {
          const int q = sbs[r] + (j - seg[r]);
          const unsigned lc = (unsigned)(P.colB[q] - lo);
          if (lc < (unsigned)Wt) fn(j, q, lc, r);
        }
      }
    };
    auto fill_cache = [&]() {
#pragma unroll
      for (int s = 0; s < BMP_SLOTS; ++s) {
        const int j0 = warp * 32 + s * BMP_NT;
        cq[s] = 0; cr[s] = 0; cc[s] = -1;
        if (j0 < Lt) {
          const int r = lane_run(j0);
          if (j0 + lane < Lt) {
            cr[s] = r;
            cq[s] = sbs[r] + (j0 + lane - seg[r]);
            cc[s] = P.colB[cq[s]];
          }
        }
      }
    };

    // rank of a tile-local column among the tile's claimed columns: prefix of its 1024- and
    // 256-column blocks + popcounts of the (<= 8) words of its 256-column block below it
    auto rank_of = [&](unsigned lc) {
      const int w = lc >> 5, v = w >> 3, k = w & 7;
      const uint4 a = reinterpret_cast<const uint4*>(bm)[2 * v];
      const uint4 b = reinterpret_cast<const uint4*>(bm)[2 * v + 1];
      const unsigned wd[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
      int r = sbp[w >> 5] + sbq[v];
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        const unsigned m = q < k ? 0xffffffffu : (q == k ? (1u << (lc & 31)) - 1 : 0u);
        r += __popc(wd[q] & m);
      }
      return r;
    };

    for (int tile = 0; tile < ntiles; ++tile) {
      const int lo = tile << lw;
      // ---- pass 1: claim bits -------------------------------------------------------------------
      int cbase = 0, inprod = 0;
      for (int c = 0; c < nchunks; ++c) {
        if (nchunks > 1 || tile == 0) {
          gather(c);
          if (cached) fill_cache();
        }
        for_products(lo, [&](int j, int q, unsigned lc, int r) {
          const int w = lc >> 5;
          const unsigned b = 1u << (lc & 31);
          const unsigned old = atomicOr(&bm[w], b);
          if (!(old & b)) {
            if (!NUM) ++cnt;
            else if (useflags) atomicOr(&flags[(cbase + j) >> 5], 1u << ((cbase + j) & 31));
          }
          if (old == 0) atomicOr(&l1[w >> 5], 1u << (w & 31));
          ++inprod;
        });
        cbase += Lt;
        __syncthreads();
      }
      if (NUM) {
        // ---- build: superblock rank prefixes and the columns of C in order --------------------
        int pcarry = 0;
        for (int u0 = 0; u0 < nl1; u0 += BMP_NT) {
          const int u = u0 + tid;
          const unsigned x = u < nl1 ? l1[u] : 0u;
          int pc = 0;
          for (unsigned y = x; y; y &= y - 1) pc += __popc(bm[(u << 5) + __ffs(y) - 1]);
          int ptot;
          int pp = pcarry + g.excl_scan(pc, ptot);
          if (x) sbp[u] = pp;  // only touched superblocks are ever queried (and cleared)
          const int p0 = pp;
          int qdone = 0;
          for (unsigned y = x; y; y &= y - 1) {
            const int wl = __ffs(y) - 1, w = (u << 5) + wl;
            while (qdone <= (wl >> 3)) sbq[4 * u + qdone++] = (unsigned short)(pp - p0);
            for (unsigned z = bm[w]; z; z &= z - 1) P.ccol[rowoff + out + pp++] = lo + (w << 5) + (__ffs(z) - 1);
          }
          if (x) while (qdone < 4) sbq[4 * u + qdone++] = (unsigned short)(pp - p0);
          pcarry += ptot;
        }
        const int ctile = pcarry;
        const bool sv = ctile <= vcap;                 // values staged in shared memory this tile
        const int ndup = (int)g.sum(inprod) - ctile;   // block-uniform
        if (!sv) {
          for (int r = tid; r < ctile; r += BMP_NT) P.cval[rowoff + out + r] = V(0);
          __threadfence();
        }
        __syncthreads();
        // ---- pass 2: first claimers store (smem) / every product adds (L2) ------------------------
        cbase = 0;
        for (int c = 0; c < nchunks; ++c) {
          if (nchunks > 1) gather(c);
          for_products(lo, [&](int j, int q, unsigned lc, int r) {
            if (sv) {
              if (flags[(cbase + j) >> 5] & (1u << ((cbase + j) & 31))) val[rank_of(lc)] = sa[r] * P.valB[q];
            } else {
              atomicAdd(&P.cval[rowoff + out + rank_of(lc)], sa[r] * P.valB[q]);
            }
          });
          cbase += Lt;
          __syncthreads();
        }
        if (sv) {
          // ---- pass 3: duplicates, after the first claimers' stores ------------------------------
          if (ndup > 0) {
            cbase = 0;
            for (int c = 0; c < nchunks; ++c) {
              if (nchunks > 1) gather(c);
              for_products(lo, [&](int j, int q, unsigned lc, int r) {
                if (!(flags[(cbase + j) >> 5] & (1u << ((cbase + j) & 31))))
                  atomicAdd(&val[rank_of(lc)], sa[r] * P.valB[q]);
              });
              cbase += Lt;
              __syncthreads();
            }
          }
          for (int r = tid; r < ctile; r += BMP_NT) {
            P.cval[rowoff + out + r] = val[r];
            val[r] = V(0);
          }
        }
        for (int x = tid; x < nfw; x += BMP_NT) flags[x] = 0;
        out += ctile;
      }
      // ---- restore the zero invariant: touched bitmap words, summary, prefixes -----------------
      for (int u = tid; u < nl1; u += BMP_NT) {
        unsigned x = l1[u];
        if (x) {
          l1[u] = 0;
          if (NUM) {
            sbp[u] = 0;
            reinterpret_cast<unsigned long long*>(sbq)[u] = 0ull;
          }
          while (x) {
            const int b = __ffs(x) - 1;
            x &= x - 1;
            bm[(u << 5) + b] = 0;
          }
        }
      }
      __syncthreads();
    }
    if (!NUM) {
      const long long c = g.sum(cnt);
      if (tid == 0) P.crow[i - P.row_begin + 1] = c;
    }
  }
}

// ================================ launch glue ====================================================
template <typename V>
static const void* bitmap_kernel(int, bool numeric) {
  return numeric ? (const void*)k_bitmap<MODE_NUM, V> : (const void*)k_bitmap<MODE_SYM, V>;
}

template <typename V>
cudaError_t bitmap_configure() {
  for (const void* k : {(const void*)k_bitmap<MODE_SYM, V>, (const void*)k_bitmap<MODE_NUM, V>}) {
    cudaError_t e = cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, BMP_SMEM);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

template <typename V>
cudaError_t bitmap_launch(int bin, cudaStream_t st, int grid, bool numeric, const Prob<V>& P, const int* list,
                          const int* count, long long N) {
  int lwmax = 10;
  while (lwmax < 20 && ((long long)1 << lwmax) < N) ++lwmax;
  int n32 = (int)N;
  void* args[] = {(void*)&P, (void*)&list, (void*)&count, (void*)&lwmax, (void*)&n32};
  return cudaLaunchKernel(bitmap_kernel<V>(bin, numeric), dim3(grid), dim3(BMP_NT), args, BMP_SMEM, st);
}

template cudaError_t bitmap_configure<double>();
template cudaError_t bitmap_configure<float>();
template cudaError_t bitmap_launch<double>(int, cudaStream_t, int, bool, const Prob<double>&, const int*, const int*,
                                           long long);
template cudaError_t bitmap_launch<float>(int, cudaStream_t, int, bool, const Prob<float>&, const int*, const int*,
                                          long long);

}  // namespace spg
