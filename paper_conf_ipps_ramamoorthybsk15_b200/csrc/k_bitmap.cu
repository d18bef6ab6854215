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
#include <type_traits>

#include "kernels.cuh"

namespace spg {

constexpr int BMP_CTCAP = 2048;      // 32-product windows per chunk with a precomputed run index
constexpr int BMP_SLOTS = 8;         // products per lane cached in registers (HEAVY: f <= 8192)
constexpr int MODE_SYM = 0, MODE_HEAVY = 1, MODE_HUGE = 2;
#ifndef SPG_HEAVY_SMALL
#define SPG_HEAVY_SMALL 1  // HEAVY rows (f <= 4096): 512-thread / 112 KB blocks that co-reside
#endif

__host__ __device__ constexpr int al16(int x) { return (x + 15) & ~15; }

// runs gathered per chunk = one per thread (NT); dynamic shared memory per block SMEM
template <typename V, int NT>
__host__ __device__ constexpr int bmp_fixed_bytes() {
  return 2 * al16((NT + 1) * 4) + al16(NT * (int)sizeof(V)) + al16(BMP_CTCAP * 2);
}
constexpr int BMP_SMEM_L = 226 * 1024;  // 1024-thread blocks, one per SM (static smem on top)
constexpr int BMP_SMEM_S = 112 * 1024;  // 512-thread blocks, two per SM

// Region bytes of a 2^lw column tile: bitmap, level-1 summary (one bit per bitmap word) and —
// numeric — rank prefixes (int per 1024 columns, u16 per 256 columns relative to its 1024),
// first-claim flags (f bits, HEAVY) and, HEAVY, `nv` staged (value, column) slots.
template <int MODE, typename V>
__device__ __forceinline__ int bmp_need(int lw, int f, int nv) {
  const int words = 1 << (lw - 5), nl1 = 1 << (lw - 10);
  int need = 4 * words + 4 * nl1;
  if (MODE != MODE_SYM) need += 12 * nl1 + 16;
  if (MODE == MODE_HEAVY) need += 4 * ((f + 31) >> 5) + ((int)sizeof(V) + 4) * nv + 16;
  return need;
}

template <int MODE, typename V, int BMP_NT, int BMP_SMEM>
__global__ void __launch_bounds__(BMP_NT, BMP_SMEM > 120 * 1024 ? 1 : 2) k_bitmap(Prob<V> P, const int* __restrict__ list,
                                                                                 const int* __restrict__ count,
                                                                                 int lwmax, int N) {
  constexpr int BMP_RCAP = BMP_NT;
  constexpr bool NUM = MODE != MODE_SYM;
  constexpr bool HEAVY = MODE == MODE_HEAVY;
  extern __shared__ __align__(16) unsigned char sm[];
  int* seg = reinterpret_cast<int*>(sm);                                   // run -> product offset
  int* sbs = reinterpret_cast<int*>(sm + al16((BMP_RCAP + 1) * 4));        // run -> B row start
  V* sa = reinterpret_cast<V*>(sm + 2 * al16((BMP_RCAP + 1) * 4));         // run -> A value
  unsigned short* ctab = reinterpret_cast<unsigned short*>(sm + 2 * al16((BMP_RCAP + 1) * 4) +
                                                           al16(BMP_RCAP * (int)sizeof(V)));  // window -> run
  unsigned char* region = sm + bmp_fixed_bytes<V, BMP_NT>();
  constexpr int REGION = BMP_SMEM - bmp_fixed_bytes<V, BMP_NT>();
  __shared__ int scratch[BMP_NT / 32 + 1];
  const Group<BMP_NT> g{(int)threadIdx.x, scratch};
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const unsigned upto = (2u << lane) - 1u;  // lanes <= me

  // invariant between rows: the whole region is zero
  for (int x = tid; x < REGION / 4; x += BMP_NT) reinterpret_cast<unsigned*>(region)[x] = 0;
  __syncthreads();

  // Rows are taken from a dynamic queue (one atomic per row): the bin's rows differ in size by
  // up to an order of magnitude, so static striding would leave a long tail — the paper's work
  // queue in its intra-GPU form.  count[0] = rows, count[16] = queue head.
  const int n = count[0];
  __shared__ int s_next;
  for (;;) {
    if (tid == 0) s_next = atomicAdd(const_cast<int*>(count) + 16, 1);
    __syncthreads();
    const int t = s_next;
    __syncthreads();
    if (t >= n) break;
    const int i = list[t];
    const int pa0 = P.rpA[i], pa1 = P.rpA[i + 1];
    const int f = P.frow[i];
    // Column tile.  HEAVY: the widest tile whose structures AND a (value, column) slot for every
    // column it can hold (min(f, Wt)) fit — never overflows.  SYM / HUGE: the widest tile whose
    // structures fit (one tile for N <= 2^20); HUGE adds values into C_val in L2.
    int lw = lwmax;
    while (lw > 10 && bmp_need<MODE, V>(lw, f, HEAVY ? min(f, 1 << lw) : 0) > REGION) --lw;
    const int Wt = 1 << lw, words = Wt >> 5, nl1 = 1 << (lw - 10);
    unsigned* bm = reinterpret_cast<unsigned*>(region);
    unsigned* l1 = bm + words;
    int* sbp = reinterpret_cast<int*>(l1 + nl1);                          // rank prefix / 1024 columns
    unsigned short* sbq = reinterpret_cast<unsigned short*>(sbp + (NUM ? nl1 : 0));  // .. / 256 columns
    unsigned* flags = reinterpret_cast<unsigned*>(sbq + (NUM ? 4 * nl1 : 0));
    const int nfw = HEAVY ? (f + 31) >> 5 : 0;
    const int voff = (4 * (words + (NUM ? 4 : 1) * nl1 + nfw) + 15) & ~15;
    V* val = reinterpret_cast<V*>(region + voff);
    const int nv = HEAVY ? min(f, Wt) : 0;
    int* colbuf = reinterpret_cast<int*>(val + nv);
    const int ntiles = (int)(((long long)N + Wt - 1) >> lw);
    const int nchunks = (pa1 - pa0 + BMP_RCAP - 1) / BMP_RCAP;
    const long long rowoff = NUM ? P.crow[i - P.row_begin] : 0;
    long long cnt = 0;
    int out = 0;
    int nz = 0, Lt = 0;  // current chunk: runs, products
    int cc[BMP_SLOTS];   // HEAVY: this lane's products (column, a*b), cached in registers
    V cv[BMP_SLOTS];

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

    // Visit the products of the current chunk in [lo, lo+Wt): fn(j, lc, v) with j the product
    // index, lc the tile-local column, v = a*b (when VALS).  HEAVY: from the register cache.
    // Otherwise each warp takes 32-product windows (coalesced within a B row), BATCH windows'
    // loads issued together.
    constexpr int BATCH = 4;
    auto for_products = [&](int lo, auto vals_tag, auto&& fn) {
      constexpr bool VALS = decltype(vals_tag)::value;
      if constexpr (HEAVY) {
#pragma unroll
        for (int s = 0; s < BMP_SLOTS; ++s) {
          const int j = warp * 32 + s * BMP_NT + lane;
          const unsigned lc = (unsigned)(cc[s] - lo);
          if (j < Lt && lc < (unsigned)Wt) fn(j, lc, cv[s]);
        }
      } else {
        for (int j00 = warp * 32; j00 < Lt; j00 += BATCH * BMP_NT) {
          int q[BATCH], col[BATCH], r[BATCH];
          V b[BATCH];
#pragma unroll
          for (int u = 0; u < BATCH; ++u) {
            const int j0 = j00 + u * BMP_NT;
            q[u] = -1;
            r[u] = 0;
            if (j0 < Lt) {
              r[u] = lane_run(j0);
              if (j0 + lane < Lt) q[u] = sbs[r[u]] + (j0 + lane - seg[r[u]]);
            }
          }
#pragma unroll
          for (int u = 0; u < BATCH; ++u) {
            col[u] = q[u] >= 0 ? P.colB[q[u]] : -1;
            if (VALS) b[u] = q[u] >= 0 ? P.valB[q[u]] : V(0);
          }
#pragma unroll
          for (int u = 0; u < BATCH; ++u) {
            const unsigned lc = (unsigned)(col[u] - lo);
            if (q[u] >= 0 && lc < (unsigned)Wt) fn(j00 + u * BMP_NT + lane, lc, VALS ? sa[r[u]] * b[u] : V(0));
          }
        }
      }
    };
    auto fill_cache = [&]() {
      int q[BMP_SLOTS], r[BMP_SLOTS];
#pragma unroll
      for (int s = 0; s < BMP_SLOTS; ++s) {
        const int j0 = warp * 32 + s * BMP_NT;
        q[s] = -1;
        r[s] = 0;
        if (j0 < Lt) {
          r[s] = lane_run(j0);
          if (j0 + lane < Lt) q[s] = sbs[r[s]] + (j0 + lane - seg[r[s]]);
        }
      }
#pragma unroll
      for (int s = 0; s < BMP_SLOTS; ++s) {
        cc[s] = q[s] >= 0 ? P.colB[q[s]] : -1;
        cv[s] = q[s] >= 0 ? P.valB[q[s]] : V(0);
      }
#pragma unroll
      for (int s = 0; s < BMP_SLOTS; ++s) cv[s] *= sa[r[s]];
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
          if constexpr (HEAVY) fill_cache();
        }
        if constexpr (HEAVY) {
          // cached windows start at multiples of 32: one ballot word of first-claim flags each
#pragma unroll
          for (int s = 0; s < BMP_SLOTS; ++s) {
            const int j0 = warp * 32 + s * BMP_NT;
            const unsigned lc = (unsigned)(cc[s] - lo);
            bool first = false;
            if (j0 + lane < Lt && lc < (unsigned)Wt) {
              const int w = lc >> 5;
              const unsigned b = 1u << (lc & 31);
              const unsigned old = atomicOr(&bm[w], b);
              first = !(old & b);
              if (old == 0) atomicOr(&l1[w >> 5], 1u << (w & 31));
              ++inprod;
            }
            const unsigned fm = __ballot_sync(FULL, first);
            if (lane == 0 && j0 < Lt) flags[j0 >> 5] = fm;
          }
        } else {
          for_products(lo, std::false_type{}, [&](int j, unsigned lc, V) {
            const int w = lc >> 5;
            const unsigned b = 1u << (lc & 31);
            const unsigned old = atomicOr(&bm[w], b);
            if (!NUM && !(old & b)) ++cnt;
            if (old == 0) atomicOr(&l1[w >> 5], 1u << (w & 31));
            ++inprod;
          });
        }
        cbase += Lt;
        __syncthreads();
      }
      if constexpr (NUM) {
        // ---- build: rank prefixes per 1024- and 256-column block (HEAVY: dense and uniform;
        //      HUGE: only touched words, and C_col written here in column order) --------------
        int pcarry = 0;
        for (int u0 = 0; u0 < nl1; u0 += BMP_NT) {
          const int u = u0 + tid;
          const unsigned x = u < nl1 ? l1[u] : 0u;
          int pc = 0;
          unsigned short q4[4] = {0, 0, 0, 0};
          if constexpr (HEAVY) {
            if (x) {
              // all 32 words of the superblock; the 16-byte reads are rotated by lane so a warp's
              // loads spread over all banks (a straight walk would be a 32-way conflict)
              int sub[4] = {0, 0, 0, 0};
#pragma unroll
              for (int k = 0; k < 8; ++k) {
                const int m = (k + tid) & 7;
                const uint4 a = reinterpret_cast<const uint4*>(bm)[8 * u + m];
                const int c4 = __popc(a.x) + __popc(a.y) + __popc(a.z) + __popc(a.w);
#pragma unroll
                for (int h = 0; h < 4; ++h) sub[h] += (m >> 1) == h ? c4 : 0;
              }
              q4[0] = 0;
              q4[1] = (unsigned short)sub[0];
              q4[2] = (unsigned short)(sub[0] + sub[1]);
              q4[3] = (unsigned short)(sub[0] + sub[1] + sub[2]);
              pc = sub[0] + sub[1] + sub[2] + sub[3];
            }
          } else {
            for (unsigned y = x; y; y &= y - 1) pc += __popc(bm[(u << 5) + __ffs(y) - 1]);
          }
          int ptot;
          int pp = pcarry + g.excl_scan(pc, ptot);
          if (x) {  // only touched superblocks are ever queried (and cleared)
            sbp[u] = pp;
            if constexpr (HEAVY) {
              reinterpret_cast<unsigned long long*>(sbq)[u] =
                  (unsigned long long)q4[0] | ((unsigned long long)q4[1] << 16) |
                  ((unsigned long long)q4[2] << 32) | ((unsigned long long)q4[3] << 48);
            } else {
              const int p0 = pp;
              int qdone = 0;
              for (unsigned y = x; y; y &= y - 1) {
                const int wl = __ffs(y) - 1, w = (u << 5) + wl;
                while (qdone <= (wl >> 3)) sbq[4 * u + qdone++] = (unsigned short)(pp - p0);
                for (unsigned z = bm[w]; z; z &= z - 1) P.ccol[rowoff + out + pp++] = lo + (w << 5) + (__ffs(z) - 1);
              }
              while (qdone < 4) sbq[4 * u + qdone++] = (unsigned short)(pp - p0);
            }
          }
          pcarry += ptot;
        }
        const int ctile = pcarry;
        if constexpr (!HEAVY) {
          for (int r = tid; r < ctile; r += BMP_NT) P.cval[rowoff + out + r] = V(0);
          __threadfence();
        }
        __syncthreads();
        // ---- pass 2: first claimers stage (value, column) in shared memory (HEAVY) / every
        //      product adds into C_val in L2 (HUGE) -------------------------------------------------
        cbase = 0;
        int ndup = 0;
        for (int c = 0; c < nchunks; ++c) {
          if (nchunks > 1) gather(c);
          for_products(lo, std::true_type{}, [&](int j, unsigned lc, V v) {
            if constexpr (HEAVY) {
              if (flags[(cbase + j) >> 5] & (1u << ((cbase + j) & 31))) {
                const int r = rank_of(lc);
                val[r] = v;
                colbuf[r] = lo + (int)lc;
              } else {
                ++ndup;
              }
            } else {
              atomicAdd(&P.cval[rowoff + out + rank_of(lc)], v);
            }
          });
          cbase += Lt;
          __syncthreads();
        }
        if constexpr (HEAVY) {
          // ---- pass 3: duplicates, after the first claimers' stores ------------------------------
          if (__syncthreads_or(ndup)) {
            for_products(lo, std::true_type{}, [&](int j, unsigned lc, V v) {
              if (!(flags[j >> 5] & (1u << (j & 31)))) atomicAdd(&val[rank_of(lc)], v);
            });
            __syncthreads();
          }
          for (int r = tid; r < ctile; r += BMP_NT) {
            P.ccol[rowoff + out + r] = colbuf[r];
            P.cval[rowoff + out + r] = val[r];
            val[r] = V(0);
            colbuf[r] = 0;
          }
          for (int x = tid; x < nfw; x += BMP_NT) flags[x] = 0;
        }
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
static const void* bitmap_kernel(int bin, bool numeric) {
  if (bin == BIN_HEAVY && SPG_HEAVY_SMALL)
    return numeric ? (const void*)k_bitmap<MODE_HEAVY, V, BMP_NT_S, BMP_SMEM_S>
                   : (const void*)k_bitmap<MODE_SYM, V, BMP_NT_S, BMP_SMEM_S>;
  if (!numeric) return (const void*)k_bitmap<MODE_SYM, V, BMP_NT, BMP_SMEM_L>;
  return bin == BIN_HUGE ? (const void*)k_bitmap<MODE_HUGE, V, BMP_NT, BMP_SMEM_L>
                         : (const void*)k_bitmap<MODE_HEAVY, V, BMP_NT, BMP_SMEM_L>;
}
static int bitmap_threads(int bin) { return bin == BIN_HEAVY && SPG_HEAVY_SMALL ? BMP_NT_S : BMP_NT; }
static int bitmap_smem(int bin) { return bin == BIN_HEAVY && SPG_HEAVY_SMALL ? BMP_SMEM_S : BMP_SMEM_L; }

template <typename V>
cudaError_t bitmap_configure() {
  for (int bin : {BIN_HEAVY, BIN_HEAVY2, BIN_HUGE})
    for (int num = 0; num < 2; ++num) {
      cudaError_t e = cudaFuncSetAttribute(bitmap_kernel<V>(bin, num), cudaFuncAttributeMaxDynamicSharedMemorySize,
                                           bitmap_smem(bin));
      if (e != cudaSuccess) return e;
    }
  return cudaSuccess;
}

template <typename V>
int bitmap_occupancy(int bin, bool numeric) {
  int nb = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, bitmap_kernel<V>(bin, numeric), bitmap_threads(bin),
                                                bitmap_smem(bin));
  return nb < 1 ? 1 : nb;
}

template <typename V>
cudaError_t bitmap_launch(int bin, cudaStream_t st, int grid, bool numeric, const Prob<V>& P, const int* list,
                          const int* count, long long N) {
  int lwmax = 10;
  while (lwmax < 20 && ((long long)1 << lwmax) < N) ++lwmax;
  int n32 = (int)N;
  void* args[] = {(void*)&P, (void*)&list, (void*)&count, (void*)&lwmax, (void*)&n32};
  return cudaLaunchKernel(bitmap_kernel<V>(bin, numeric), dim3(grid), dim3(bitmap_threads(bin)), args,
                          bitmap_smem(bin), st);
}

#define INST(V)                                                                                                   \
  template cudaError_t bitmap_configure<V>();                                                                     \
  template int bitmap_occupancy<V>(int, bool);                                                                    \
  template cudaError_t bitmap_launch<V>(int, cudaStream_t, int, bool, const Prob<V>&, const int*, const int*, long long);
INST(double)
INST(float)
#undef INST

}  // namespace spg
