// k_numeric.cu — numeric phase: C(i,j) = sum_k A(i,k)·B(k,j) (Row-Row
// formulation) written as sorted, compacted CSR.
//
// The symbolic phase left, for every intermediate product, its rank among the distinct
// columns of its row of C and a first-occurrence flag (R).  Numeric therefore never sorts: the
// output C is cut into windows of NUM_W consecutive entries; one block per window enumerates the
// products of the rows overlapping the window (A entries of those rows, B rows coalesced, runs
// looked up from a REDUX.OR run-start mask), reads each product's R, and scatters a·b into the
// window's shared-memory image at crow_i + rank: first occurrences store (column, value), the
// rest are queued and added after a barrier (Phase IV "add like-tuples").  The
// window is then written out with coalesced streaming stores.  Rows whose products all land in
// distinct, already ordered positions (SINGLE: one B row) have no R: rank = in-row offset.
//
// HBM traffic per window: its share of R (4 B per product), A (row, offset, column, value of
// each entry), and the C window itself (12 B per entry, fp64); B is gathered from L2.
#include "kernels.cuh"

namespace spg {

constexpr int NUM_DUPCAP = 1024;   // queued non-first products per window (else a second pass)
constexpr int NUM_CTCAP = 1024;    // 32-product windows per chunk with a precomputed run index
constexpr int NUM_BATCH = 4;       // 32-product windows per warp per step

template <typename V, int W>
struct NumSmem {
  static constexpr int val = 0;                                          // V[W]
  static constexpr int col = val + W * (int)sizeof(V);                   // int[W]
  static constexpr int dval = col + W * 4;                               // V[DUPCAP]
  static constexpr int dpos = dval + NUM_DUPCAP * (int)sizeof(V);        // int[DUPCAP]
  static constexpr int sg = dpos + NUM_DUPCAP * 4;                       // long long[NT]  R index of run start (-1: identity)
  static constexpr int sa = sg + NUM_NT * 8;                             // V[NT]          A value
  static constexpr int seg = sa + NUM_NT * (int)sizeof(V);               // int[NT+1]      product offset
  static constexpr int sbs = seg + (NUM_NT + 1) * 4;                     // int[NT]        B index of run start
  static constexpr int sbase = sbs + NUM_NT * 4;                         // int[NT]        window position of rank 0
  static constexpr int ctab = sbase + NUM_NT * 4;                        // u16[CTCAP]
  static constexpr int bytes = (ctab + NUM_CTCAP * 2 + 15) & ~15;
};

__device__ __forceinline__ long long block_excl_scan_ll(long long v, long long& total, long long* scratch) {
  constexpr int NW = NUM_NT / 32;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const long long incl = warp_incl_scan(v);
  if (lane == 31) scratch[w] = incl;
  __syncthreads();
  if (w == 0) {
    const long long x = lane < NW ? scratch[lane] : 0;
    const long long xi = warp_incl_scan(x);
    if (lane < NW) scratch[lane] = xi - x;
    if (lane == NW - 1) scratch[NW] = xi;
  }
  __syncthreads();
  const long long r = incl - v + scratch[w];
  total = scratch[NW];
  __syncthreads();
  return r;
}

template <typename V, int W>
__global__ void __launch_bounds__(NUM_NT) k_numeric(NumProb<V> P) {
  using S = NumSmem<V, W>;
  extern __shared__ __align__(16) unsigned char sm[];
  V* s_val = reinterpret_cast<V*>(sm + S::val);
  int* s_col = reinterpret_cast<int*>(sm + S::col);
  V* s_dval = reinterpret_cast<V*>(sm + S::dval);
  int* s_dpos = reinterpret_cast<int*>(sm + S::dpos);
  long long* sg = reinterpret_cast<long long*>(sm + S::sg);
  V* sa = reinterpret_cast<V*>(sm + S::sa);
  int* seg = reinterpret_cast<int*>(sm + S::seg);
  int* sbs = reinterpret_cast<int*>(sm + S::sbs);
  int* sbase = reinterpret_cast<int*>(sm + S::sbase);
  unsigned short* ctab = reinterpret_cast<unsigned short*>(sm + S::ctab);
  __shared__ long long scratch[NUM_NT / 32 + 1];
  __shared__ int s_ndup;
  constexpr int NT = NUM_NT;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const unsigned upto = (2u << lane) - 1u;

  const int w = blockIdx.x;
  const long long ws = (long long)w * W;
  const int wl = (int)min((long long)W, P.nnzC - ws);
  const int i0 = P.wrow[w];
  int i1 = P.mloc - 1;
  if (w + 1 < P.nwin) {
    i1 = P.wrow[w + 1];
    if (P.crow[i1] >= ws + wl) --i1;  // that row starts at the next window
  }
  const int ea = P.rpA[P.row_begin + i0], eb = P.rpA[P.row_begin + i1 + 1];
  if (tid == 0) s_ndup = 0;

  // One pass over the window's products.  pass 0: first occurrences store, the others are
  // queued; pass 1 (queue overflow only): the others add straight into the image.
  auto run_pass = [&](int pass) {
    for (int c0 = ea; c0 < eb; c0 += NT) {
      const int e = c0 + tid;
      long long L = 0, g0 = -1;
      int bs = 0, base = 0;
      V a = V(0);
      if (e < eb) {
        const int r = P.rowA[e] - P.row_begin;
        const int k = P.colA[e];
        bs = P.rpB[k];
        int Li = P.rpB[k + 1] - bs;
        a = P.valA[e];
        base = (int)(P.crow[r] - ws);
        const long long ro = P.Ro[r];
        const int pe = P.Pe[e];
        if (ro >= 0) {
          g0 = ro + pe;
        } else {  // identity row: ranks pe + [0, L) — clip to the window
          const int lo = max(0, -base - pe), hi = min(Li, wl - base - pe);
          if (hi <= lo) {
            Li = 0;
          } else {
            bs += lo;
            Li = hi - lo;
            base += pe + lo;
          }
        }
        L = Li;
      }
      long long tot;
      const long long ex = block_excl_scan_ll((L << 16) | (L > 0 ? 1 : 0), tot, scratch);
      const int slot = (int)(ex & 0xffff), nr = (int)(tot & 0xffff);
      const int Lt = (int)(tot >> 16);  // products of this chunk (< 2^31: see DESIGN.md)
      if (L > 0) {
        seg[slot] = (int)(ex >> 16);
        sbs[slot] = bs;
        sa[slot] = a;
        sg[slot] = g0;
        sbase[slot] = base;
      }
      if (tid == 0) seg[nr] = Lt;
      __syncthreads();
      for (int x = tid; x < min((Lt + 31) >> 5, NUM_CTCAP); x += NT) ctab[x] = (unsigned short)upper_idx(seg, nr, x << 5);
      __syncthreads();
      for (int j00 = warp * 32; j00 < Lt; j00 += NUM_BATCH * NT) {
        int q[NUM_BATCH], rr[NUM_BATCH], off[NUM_BATCH];
#pragma unroll
        for (int u = 0; u < NUM_BATCH; ++u) {
          const int j0 = j00 + u * NT;
          q[u] = -1;
          rr[u] = 0;
          off[u] = 0;
          if (j0 < Lt) {
            const int rb = (j0 >> 5) < NUM_CTCAP ? (int)ctab[j0 >> 5] : upper_idx(seg, nr, j0);
            const int rs = rb + 1 + lane;
            const int d = rs <= nr ? seg[rs] - j0 : 32;
            const unsigned M = __reduce_or_sync(FULL, (d >= 1 && d <= 31) ? (1u << d) : 0u);
            const int r = rb + __popc(M & upto);
            rr[u] = r;
            if (j0 + lane < Lt) {
              off[u] = j0 + lane - seg[r];
              q[u] = sbs[r] + off[u];
            }
          }
        }
        unsigned rv[NUM_BATCH];
#pragma unroll
        for (int u = 0; u < NUM_BATCH; ++u) {
          rv[u] = (unsigned)off[u] | RFLAG;
          if (q[u] >= 0) {
            const long long gg = sg[rr[u]];
            if (gg >= 0) rv[u] = __ldcs(P.R + gg + off[u]);
          }
        }
        int pos[NUM_BATCH];
#pragma unroll
        for (int u = 0; u < NUM_BATCH; ++u) {
          pos[u] = sbase[rr[u]] + (int)(rv[u] & ~RFLAG);
          if (q[u] >= 0 && (unsigned)pos[u] >= (unsigned)wl) q[u] = -1;
        }
        int col[NUM_BATCH];
        V bv[NUM_BATCH];
#pragma unroll
        for (int u = 0; u < NUM_BATCH; ++u) {
          col[u] = q[u] >= 0 ? P.colB[q[u]] : 0;
          bv[u] = q[u] >= 0 ? P.valB[q[u]] : V(0);
        }
#pragma unroll
        for (int u = 0; u < NUM_BATCH; ++u) {
          if (q[u] < 0) continue;
          const V v = sa[rr[u]] * bv[u];
          const bool first = rv[u] & RFLAG;
          if (pass == 0) {
            if (first) {
              s_col[pos[u]] = col[u];
              s_val[pos[u]] = v;
            } else {
              const int d = atomicAdd(&s_ndup, 1);
              if (d < NUM_DUPCAP) {
                s_dpos[d] = pos[u];
                s_dval[d] = v;
              }
            }
          } else if (!first) {
            atomicAdd(&s_val[pos[u]], v);
          }
        }
      }
      __syncthreads();
    }
  };

  run_pass(0);
  const int nd = s_ndup;
  if (nd <= NUM_DUPCAP) {
    for (int d = tid; d < nd; d += NT) atomicAdd(&s_val[s_dpos[d]], s_dval[d]);
  } else {
    run_pass(1);
  }
  __syncthreads();
  int* ccol = P.ccol + ws;
  V* cval = P.cval + ws;
  for (int x = tid; x < wl; x += NT) {
    __stcs(ccol + x, s_col[x]);
    __stcs(cval + x, s_val[x]);
  }
}

// wrow[w] = the local row holding output position w·NUM_W (rows with c_i = 0 hold none).
__global__ void k_window_rows(const long long* __restrict__ crow, int mloc, int* __restrict__ wrow) {
  for (long long li = blockIdx.x * (long long)blockDim.x + threadIdx.x; li < mloc;
       li += (long long)gridDim.x * blockDim.x) {
    const long long a = crow[li], b = crow[li + 1];
    for (long long x = (a + NUM_W - 1) / NUM_W; x * NUM_W < b; ++x) wrow[x] = (int)li;
  }
}

template <typename V>
cudaError_t numeric_configure() {
  return cudaFuncSetAttribute(k_numeric<V, NUM_W>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                              NumSmem<V, NUM_W>::bytes);
}

cudaError_t launch_window_rows(cudaStream_t st, const long long* crow, int mloc, int* wrow, int nwin) {
  if (mloc <= 0 || nwin <= 0) return cudaSuccess;
  long long g = (mloc + 255) / 256;
  if (g > 8192) g = 8192;
  k_window_rows<<<(int)g, 256, 0, st>>>(crow, mloc, wrow);
  return cudaGetLastError();
}

template <typename V>
cudaError_t launch_numeric(cudaStream_t st, const NumProb<V>& P) {
  if (P.nwin <= 0) return cudaSuccess;
  k_numeric<V, NUM_W><<<P.nwin, NUM_NT, NumSmem<V, NUM_W>::bytes, st>>>(P);
  return cudaGetLastError();
}

template cudaError_t numeric_configure<double>();
template cudaError_t numeric_configure<float>();
template cudaError_t launch_numeric<double>(cudaStream_t, const NumProb<double>&);
template cudaError_t launch_numeric<float>(cudaStream_t, const NumProb<float>&);

}  // namespace spg
