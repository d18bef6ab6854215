// k_numeric.cu — numeric phase: C(i,j) = sum_k A(i,k)·B(k,j) (Row-Row
// formulation) written as sorted, compacted CSR.
//
// The symbolic phase sorted every row's products by column and left a gather plan: for output
// r of row i (r-th distinct column), EQ[Ro_i + r] = {e, q}, the A entry and B entry of the
// column's first product; every further product of the column is a dup entry {i, r, e, q}.
// Rows whose products are all distinct and already ordered (SINGLE: one non-empty B row) have
// no plan: output r is B entry bs + r times their one A entry.
//
// So numeric is a stream in output order (Phase IV of PAPER.md L154-156, "add like-tuples and
// compact", with the sort done once in symbolic):
//   k_numeric      a block takes a chunk of NUM_CH consecutive outputs of C; the rows starting
//                  inside the chunk mark their first slot, a max-scan gives every slot its row;
//                  then per output: {e, q} = EQ[o + nd_row] (coalesced), C_col[o] = colB[q],
//                  C_val[o] = valA[e]·valB[q] (B and A gathers hit L2; B rows are read in
//                  ascending order, so sectors are reused through L1), coalesced streaming stores.
//   k_numeric_dup  C_val[crow_i + r] += valA[e]·valB[q] for the dup list (native RED.ADD.F64/F32;
//                  ~7% of the products on webbase1m), after k_numeric on the same stream.
//
// HBM traffic per output: 8 B of EQ read + 12 B (fp64) of C written; A and B mostly from L2.
#include "kernels.cuh"

#ifndef SPG_NUM_MINB
#define SPG_NUM_MINB 5  // k_numeric blocks per SM the register budget is cut for
#endif
#ifndef SPG_EQ_LOAD
#define SPG_EQ_LOAD 0  // plan loads: 0 streaming (ld.global.cs), 1 read-only path, 2 plain
#endif

namespace spg {

// ---- plan (end of symbolic) ---------------------------------------------------------------------
// Per local row li with c_i > 0: nd = Ro_i - crow_i (plan rows) or bs - crow_i with ne = the A
// entry whose B row is the only non-empty one (SINGLE rows); chunk_row[ch] = the row holding
// output ch·NUM_CH.
__global__ void __launch_bounds__(256) k_plan(const long long* __restrict__ crow, int mloc,
                                              const int* __restrict__ rpA, const int* __restrict__ colA,
                                              const int* __restrict__ rpB, const uint8_t* __restrict__ cls,
                                              const long long* __restrict__ Ro, int rb, long long* __restrict__ nd,
                                              int* __restrict__ ne, int* __restrict__ chunk_row, int chcap,
                                              Small* __restrict__ sm) {
  if (!sm->r_ok) return;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    const long long nnz = crow[mloc];
    sm->nch_need = (int)((nnz + NUM_CH - 1) / NUM_CH) + 1;
  }
  for (long long li = blockIdx.x * (long long)blockDim.x + threadIdx.x; li < mloc;
       li += (long long)gridDim.x * blockDim.x) {
    const long long a = crow[li], b = crow[li + 1];
    if (b <= a) continue;
    long long d;
    int e = -1;
    if ((cls[li] & 7) == CLS_SINGLE && Ro[li] < 0) {
      const int i = rb + (int)li;
      int p = rpA[i], bs = 0;
      for (const int pe = rpA[i + 1]; p < pe; ++p) {
        const int k = colA[p];
        bs = rpB[k];
        if (rpB[k + 1] > bs) break;
      }
      e = p;
      d = (long long)bs - a;
    } else {
      d = Ro[li] - a;
    }
    nd[li] = d;
    ne[li] = e;
    for (long long ch = (a + NUM_CH - 1) / NUM_CH; ch * NUM_CH < b; ++ch)
      if (ch < chcap) chunk_row[ch] = (int)li;
  }
}

cudaError_t launch_plan(cudaStream_t st, int sms, const long long* crow, int mloc, const int* rpA, const int* colA,
                        const int* rpB, const uint8_t* cls, const long long* Ro, int rb, long long* nd, int* ne,
                        int* chunk_row, int chcap, Small* small) {
  if (mloc <= 0) return cudaSuccess;
  long long g = (mloc + 255) / 256;
  if (g > sms * 8) g = sms * 8;
  k_plan<<<(int)g, 256, 0, st>>>(crow, mloc, rpA, colA, rpB, cls, Ro, rb, nd, ne, chunk_row, chcap, small);
  return cudaGetLastError();
}

// ---- numeric ------------------------------------------------------------------------------------
constexpr int NUM_PT = NUM_CH / NUM_NT;  // outputs per thread and chunk
static_assert(NUM_PT == 8, "slot ownership below assumes 8 slots per thread");

// Packed B entry: column and value in one 16-byte (fp64) or 8-byte (fp32) word, so the gather of
// an output's B entry is one load instead of two.
template <typename V> struct PackB;
template <> struct PackB<double> { using T = int4; };
template <> struct PackB<float> { using T = int2; };
template <typename V>
__device__ __forceinline__ typename PackB<V>::T pack_b(int c, V v);
template <>
__device__ __forceinline__ int4 pack_b<double>(int c, double v) {
  const long long b = __double_as_longlong(v);
  return make_int4(c, 0, (int)(unsigned)(b & 0xffffffffLL), (int)(b >> 32));
}
template <>
__device__ __forceinline__ int2 pack_b<float>(int c, float v) { return make_int2(c, __float_as_int(v)); }
__device__ __forceinline__ double unpack_v(const int4& t, double) {
  return __longlong_as_double(((long long)t.w << 32) | (unsigned)t.z);
}
__device__ __forceinline__ float unpack_v(const int2& t, float) { return __int_as_float(t.y); }

template <typename V>
__global__ void __launch_bounds__(256) k_pack_b(const int* __restrict__ colB, const V* __restrict__ valB, long long n,
                                                typename PackB<V>::T* __restrict__ out) {
  for (long long x = blockIdx.x * (long long)blockDim.x + threadIdx.x; x < n; x += (long long)gridDim.x * blockDim.x)
    out[x] = pack_b<V>(colB[x], valB[x]);
}

#ifndef SPG_C_STORE
#define SPG_C_STORE 0  // C stores: 0 streaming (st.global.cs), 1 plain
#endif
#ifndef SPG_NUM_PIPE
#define SPG_NUM_PIPE 0  // 1: software-pipelined chunks (next chunk's row heads + plan loads overlap the gathers)
#endif

// Row heads of chunk ch in shared memory: s_head[slot] = 1 + slot of its row's first output.
// Returns false for a chunk inside one row (nd1/ne1 set; no shared memory, no barrier).
__device__ __forceinline__ bool num_setup(const long long* __restrict__ crow, const long long* __restrict__ ndv,
                                          const int* __restrict__ nev, const int* __restrict__ chunk_row, int nch,
                                          int mloc, int ch, long long base, int* s_head, long long* s_nd, int* s_ne,
                                          int* s_wmax, long long& nd1, int& ne1) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int r0 = chunk_row[ch];
  const int r1 = ch + 1 < nch ? chunk_row[ch + 1] : mloc - 1;
  if (r0 == r1) {
    nd1 = ndv[r0];
    ne1 = nev[r0];
    return false;
  }
  {
    int4* h4 = reinterpret_cast<int4*>(s_head);
    h4[2 * tid] = make_int4(0, 0, 0, 0);
    h4[2 * tid + 1] = make_int4(0, 0, 0, 0);
  }
  __syncthreads();
  if (tid == 0) {
    s_head[0] = 1;
    s_nd[0] = ndv[r0];
    s_ne[0] = nev[r0];
  }
  // rows starting inside the chunk (every row is visited by exactly one chunk: O(M) in total)
  for (int r = r0 + 1 + tid; r <= r1; r += NUM_NT) {
    const long long a = crow[r], b = crow[r + 1];
    const long long s = a - base;
    if (b > a && s < NUM_CH) {
      s_head[s] = (int)s + 1;
      s_nd[s] = ndv[r];
      s_ne[s] = nev[r];
    }
  }
  __syncthreads();
  // fill forward: slot -> its row's head slot (max scan over 8 slots per thread, then warps)
  int4* h4 = reinterpret_cast<int4*>(s_head);
  int4 x = h4[2 * tid], y = h4[2 * tid + 1];
  x.y = max(x.y, x.x); x.z = max(x.z, x.y); x.w = max(x.w, x.z);
  y.x = max(y.x, x.w); y.y = max(y.y, y.x); y.z = max(y.z, y.y); y.w = max(y.w, y.z);
  int m = y.w;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int o = __shfl_up_sync(FULL, m, d);
    if (lane >= d) m = max(m, o);
  }
  if (lane == 31) s_wmax[warp] = m;
  int carry = __shfl_up_sync(FULL, m, 1);
  if (lane == 0) carry = 0;
  __syncthreads();
  for (int w = 0; w < warp; ++w) carry = max(carry, s_wmax[w]);
  x.x = max(x.x, carry); x.y = max(x.y, carry); x.z = max(x.z, carry); x.w = max(x.w, carry);
  y.x = max(y.x, carry); y.y = max(y.y, carry); y.z = max(y.z, carry); y.w = max(y.w, carry);
  h4[2 * tid] = x;
  h4[2 * tid + 1] = y;
  __syncthreads();
  return true;
}

// Plan loads of the chunk: output slot s = k·NUM_NT + tid gets {A entry e, B entry q}; e = -1 past
// the chunk's end.
__device__ __forceinline__ void num_plan_loads(const int2* __restrict__ EQ, long long base, int n, bool one,
                                               long long nd1, int ne1, const int* s_head, const long long* s_nd,
                                               const int* s_ne, int* e, int* q) {
  const int tid = threadIdx.x;
#pragma unroll
  for (int k = 0; k < NUM_PT; ++k) {
    const int s = k * NUM_NT + tid;
    const bool ok = s < n;
    long long d = nd1;
    int es = ne1;
    if (!one) {
      const int h = ok ? s_head[s] - 1 : 0;
      d = s_nd[h];
      es = s_ne[h];
    }
    const long long src = base + s + d;
    const bool plan = ok && es < 0;
#if SPG_EQ_LOAD == 1
    const int2 eq = plan ? __ldg(EQ + src) : make_int2(es, (int)src);
#elif SPG_EQ_LOAD == 2
    const int2 eq = plan ? EQ[src] : make_int2(es, (int)src);
#else
    const int2 eq = plan ? __ldcs(EQ + src) : make_int2(es, (int)src);
#endif
    e[k] = ok ? eq.x : -1;
    q[k] = eq.y;
  }
}

template <typename V, bool PACK>
__device__ __forceinline__ void num_gathers(const NumProb<V>& P, const int* e, const int* q, int* col, V* va, V* vb) {
#pragma unroll
  for (int k = 0; k < NUM_PT; ++k) {
    const bool ok = e[k] >= 0;
    if constexpr (PACK) {
      using T = typename PackB<V>::T;
      const T t = ok ? __ldg(reinterpret_cast<const T*>(P.packB) + q[k]) : T{};
      col[k] = t.x;
      vb[k] = unpack_v(t, V(0));
    } else {
      col[k] = ok ? __ldg(P.colB + q[k]) : 0;
      vb[k] = ok ? __ldg(P.valB + q[k]) : V(0);
    }
    va[k] = ok ? __ldg(P.valA + e[k]) : V(0);
  }
}

template <typename V>
__device__ __forceinline__ void num_stores(const NumProb<V>& P, long long base, int n, const int* col, const V* va,
                                           const V* vb) {
  const int tid = threadIdx.x;
#pragma unroll
  for (int k = 0; k < NUM_PT; ++k) {
    const int s = k * NUM_NT + tid;
    if (s < n) {
#if SPG_C_STORE == 1
      P.ccol[base + s] = col[k];
      P.cval[base + s] = va[k] * vb[k];
#else
      __stcs(P.ccol + base + s, col[k]);
      __stcs(P.cval + base + s, va[k] * vb[k]);
#endif
    }
  }
}

template <typename V, bool PACK>
__global__ void __launch_bounds__(NUM_NT, SPG_NUM_MINB) k_numeric(NumProb<V> P) {
  __shared__ __align__(16) int s_head[NUM_CH];   // slot -> 1 + slot of its row's first output in the chunk
  __shared__ long long s_nd[NUM_CH];             // head slot -> nd of its row
  __shared__ int s_ne[NUM_CH];                   // head slot -> ne of its row
  __shared__ int s_wmax[NUM_NT / 32];
  auto chunk_n = [&](int ch) { return (int)min((long long)NUM_CH, P.nnz - (long long)ch * NUM_CH); };
#if SPG_NUM_PIPE
  // Software pipeline over this block's chunks: the gathers of chunk ch are in flight while the
  // row heads and plan loads of the next chunk are computed; the stores of ch come last.
  int ch = blockIdx.x;
  if (ch >= P.nch) return;
  int e[NUM_PT], q[NUM_PT];
  {
    long long nd1 = 0;
    int ne1 = 0;
    const long long base = (long long)ch * NUM_CH;
    const bool multi = num_setup(P.crow, P.nd, P.ne, P.chunk_row, P.nch, P.mloc, ch, base, s_head, s_nd, s_ne,
                                 s_wmax, nd1, ne1);
    num_plan_loads(P.EQ, base, chunk_n(ch), !multi, nd1, ne1, s_head, s_nd, s_ne, e, q);
  }
  for (; ch < P.nch; ch += gridDim.x) {
    int col[NUM_PT];
    V va[NUM_PT], vb[NUM_PT];
    num_gathers<V, PACK>(P, e, q, col, va, vb);
    const int nx = ch + gridDim.x;
    if (nx < P.nch) {
      __syncthreads();  // every thread's plan loads of ch read s_head before it is rebuilt
      long long nd1 = 0;
      int ne1 = 0;
      const long long base = (long long)nx * NUM_CH;
      const bool multi = num_setup(P.crow, P.nd, P.ne, P.chunk_row, P.nch, P.mloc, nx, base, s_head, s_nd, s_ne,
                                   s_wmax, nd1, ne1);
      num_plan_loads(P.EQ, base, chunk_n(nx), !multi, nd1, ne1, s_head, s_nd, s_ne, e, q);
    }
    num_stores<V>(P, (long long)ch * NUM_CH, chunk_n(ch), col, va, vb);
  }
#else
  for (int ch = blockIdx.x; ch < P.nch; ch += gridDim.x) {
    const long long base = (long long)ch * NUM_CH;
    long long nd1 = 0;
    int ne1 = 0;
    // a chunk inside one row (half of webbase1m's chunks: heavy rows) needs no row heads, no
    // shared memory and no barrier
    const bool multi = num_setup(P.crow, P.nd, P.ne, P.chunk_row, P.nch, P.mloc, ch, base, s_head, s_nd, s_ne,
                                 s_wmax, nd1, ne1);
    // outputs o = base + k·NUM_NT + tid: plan loads, then gathers, then stores (all batched)
    int e[NUM_PT], q[NUM_PT];
    num_plan_loads(P.EQ, base, chunk_n(ch), !multi, nd1, ne1, s_head, s_nd, s_ne, e, q);
    int col[NUM_PT];
    V va[NUM_PT], vb[NUM_PT];
    num_gathers<V, PACK>(P, e, q, col, va, vb);
    num_stores<V>(P, base, chunk_n(ch), col, va, vb);
    if (multi) __syncthreads();
  }
#endif
}

template <typename V>
__global__ void __launch_bounds__(256) k_numeric_dup(NumProb<V> P) {
  for (long long d = blockIdx.x * (long long)blockDim.x + threadIdx.x; d < P.ndup;
       d += (long long)gridDim.x * blockDim.x) {
    const int4 t = __ldcs(P.dup + d);
    const long long pos = P.crow[t.x] + t.y;
    atomicAdd(P.cval + pos, __ldg(P.valA + t.z) * __ldg(P.valB + t.w));
  }
}

template <typename V>
cudaError_t numeric_configure() {
  cudaError_t e = cudaFuncSetAttribute(k_numeric<V, false>, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(k_numeric<V, true>, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
  return e;
}

template <typename V>
int numeric_occupancy() {
  int nb = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_numeric<V, false>, NUM_NT, 0);
  return nb < 1 ? 1 : nb;
}

template <typename V>
cudaError_t launch_numeric(cudaStream_t st, int grid, const NumProb<V>& P) {
  if (P.packB) {
    long long g = (P.nB + 255) / 256;
    if (g > 148LL * 16) g = 148LL * 16;
    if (P.nB > 0) k_pack_b<V><<<(int)g, 256, 0, st>>>(P.colB, P.valB, P.nB, reinterpret_cast<typename PackB<V>::T*>(P.packB));
    if (P.nch > 0 && grid > 0) k_numeric<V, true><<<grid, NUM_NT, 0, st>>>(P);
  } else if (P.nch > 0 && grid > 0) {
    k_numeric<V, false><<<grid, NUM_NT, 0, st>>>(P);
  }
  if (P.ndup > 0) {
    long long g = (P.ndup + 255) / 256;
    if (g > 148LL * 16) g = 148LL * 16;
    k_numeric_dup<V><<<(int)g, 256, 0, st>>>(P);
  }
  return cudaGetLastError();
}

#define INST(V)                                                \
  template cudaError_t numeric_configure<V>();                 \
  template int numeric_occupancy<V>();                         \
  template cudaError_t launch_numeric<V>(cudaStream_t, int, const NumProb<V>&);
INST(double)
INST(float)
#undef INST

}  // namespace spg
