// k_numeric.cu — numeric phase: C(i,j) = sum_k A(i,k)·B(k,j) (Row-Row
// formulation) written as sorted, compacted CSR.
//
// The symbolic phase left, for every intermediate product, its rank among the distinct
// columns of its row of C and a first-occurrence flag (R).  Numeric therefore never sorts: a
// block takes a window of consecutive outputs of C, enumerates the products of the window's
// rows (A entries of those rows, B rows coalesced, the run of each lane from a REDUX.OR mask of
// run starts), reads each product's R, and scatters a·b into the window's shared-memory image at
// crow_i + rank: first occurrences store (column, value), the others are queued and added after
// a barrier (Phase IV "add like-tuples").  The image is then written out with
// coalesced streaming stores.  Rows whose products are all distinct and already ordered
// (SINGLE: one B row) have no R: rank = in-row offset.
//
// Work units are row-aligned, so a product is visited once: rows with c_i <= NUM_CS are grouped
// into windows (cut where a row's output range crosses a multiple of NUM_WS - NUM_CS), rows with
// NUM_CS < c_i <= NUM_WS are a window each (k_num_windows); longer rows are units of k_num_large,
// which stages NUM_LS outputs per pass; a row longer than that is enumerated once per pass, but
// every run, and every work item of a long run, whose rank range misses the pass is skipped
// (ranks increase along a run: B rows are sorted).
//
// B-side split of the products (the A_H/A_L x B_H/B_L product classes of
// PAPER.md L104-106, L138): a run with >= NUM_LONG products is cut into work items that one warp
// walks with warp-uniform run data and coalesced loads; shorter runs are flattened across the
// lanes (run of each lane from a REDUX.OR mask of run starts).  Both kernels are persistent: each
// thread prefetches its A entry's run record (precomputed at the end of symbolic by k_records)
// for the NEXT chunk while the current chunk's products are processed.
//
// HBM traffic per output: its share of R (4 B per product), of A (row, offset, column, value of
// each entry) and the C entry itself (12 B fp64); B is gathered from L2.
#include "kernels.cuh"

namespace spg {


// ---- plan (end of symbolic): units and per-entry run records ----------------------------------
// Cuts (window starts) of row li (c_i > 0): small rows one cut at their start when their output
// range crosses a multiple of W = NUM_WS - NUM_CS (or starts on one); other rows a cut at each end
// (the window between them is the row itself: a window unit when c_i <= NUM_WS, else a unit of
// the large-row kernel).
__global__ void k_cut_count(const long long* __restrict__ crow, int mloc, const int* __restrict__ rpA, int rb,
                            int* __restrict__ cnt, Unit* __restrict__ lunits, int lcap, Small* __restrict__ sm) {
  constexpr int W = NUM_WS - NUM_CS;
  if (!sm->r_ok) return;
  const int lane = threadIdx.x & 31;
  const int ea0 = rpA[rb];
  if (blockIdx.x == 0 && threadIdx.x == 0) sm->ea0 = ea0;
  const long long nup = ((long long)mloc + 31) & ~31LL;
  for (long long li = blockIdx.x * (long long)blockDim.x + threadIdx.x; li < nup;
       li += (long long)gridDim.x * blockDim.x) {
    int nseg = 0;
    long long a = 0, c = 0;
    if (li < mloc) {
      a = crow[li];
      c = crow[li + 1] - a;
      int n = 0;
      if (c > NUM_CS) {
        n = 2;
        if (c > NUM_WS) nseg = 1;
      } else if (c > 0) {
        n = (a % W == 0) || (a / W != (a + c - 1) / W);
      }
      cnt[li] = n;
    }
    const unsigned m = __ballot_sync(FULL, nseg > 0);
    if (m) {
      int base = 0;
      if (lane == 0) base = atomicAdd(&sm->nlunits, __popc(m));
      base = __shfl_sync(FULL, base, 0) + __popc(m & lanemask_lt());
      if (nseg > 0 && base < lcap) lunits[base] = Unit{a, rpA[rb + li] - ea0, rpA[rb + li + 1] - ea0, (int)c, 0};
    }
  }
}

__global__ void k_cut_write(const long long* __restrict__ crow, int mloc, const long long* __restrict__ coff,
                            Cut* __restrict__ cuts, const Small* __restrict__ sm) {
  if (!sm->r_ok) return;
  if (blockIdx.x == 0 && threadIdx.x == 0) cuts[coff[mloc]] = Cut{crow[mloc], mloc, 0};
  for (long long li = blockIdx.x * (long long)blockDim.x + threadIdx.x; li < mloc;
       li += (long long)gridDim.x * blockDim.x) {
    const long long o = coff[li], n = coff[li + 1] - o;
    if (n == 0) continue;
    cuts[o] = Cut{crow[li], (int)li, 0};
    if (n == 2) cuts[o + 1] = Cut{crow[li + 1], (int)li + 1, 0};
  }
}

// Window units: cut w covers outputs [cuts[w].pos, cuts[w+1].pos) of rows [cuts[w].row, end) (end =
// the next cut's row, or row + 1 when both cuts share a row); empty windows and long rows drop out.
__global__ void k_units(const Cut* __restrict__ cuts, const long long* __restrict__ coff, int mloc,
                        const int* __restrict__ rpA, int rb, Unit* __restrict__ wunits, Small* __restrict__ sm) {
  if (!sm->r_ok) return;
  const int lane = threadIdx.x & 31;
  const long long ncut = coff[mloc];
  const int ea0 = rpA[rb];
  const long long nup = (ncut + 31) & ~31LL;
  for (long long w = blockIdx.x * (long long)blockDim.x + threadIdx.x; w < nup; w += (long long)gridDim.x * blockDim.x) {
    bool ok = false;
    Unit u{};
    if (w < ncut) {
      const Cut c0 = cuts[w], c1 = cuts[w + 1];
      const long long wl = c1.pos - c0.pos;
      if (wl > 0 && wl <= NUM_WS) {
        const int re = c1.row == c0.row ? c0.row + 1 : c1.row;
        u = Unit{c0.pos, rpA[rb + c0.row] - ea0, rpA[rb + re] - ea0, (int)wl, 0};
        ok = true;
      }
    }
    const unsigned m = __ballot_sync(FULL, ok);
    if (m) {
      int base = 0;
      if (lane == 0) base = atomicAdd(&sm->nwunits, __popc(m));
      base = __shfl_sync(FULL, base, 0);
      if (ok) wunits[base + __popc(m & lanemask_lt())] = u;
    }
  }
}

// Run record of every local A entry e: rec0 = {B row start, length, R index of its first product
// (lo, hi; -(in-row offset) - 1 for rows without R, whose rank = offset)}, rec1 = {C offset of its
// row (lo, hi), rank of its first product, rank of its last product}.
__global__ void k_records(const int* __restrict__ rpA, const int* __restrict__ colA, const int* __restrict__ rpB,
                          const int* __restrict__ rowA, const int* __restrict__ Pe, const long long* __restrict__ Ro,
                          const unsigned* __restrict__ R, const long long* __restrict__ crow, int rb, int re,
                          int4* __restrict__ rec0, int4* __restrict__ rec1, const Small* __restrict__ sm) {
  if (!sm->r_ok) return;
  const int ea0 = rpA[rb], n = rpA[re] - ea0;
  for (long long x = blockIdx.x * (long long)blockDim.x + threadIdx.x; x < n; x += (long long)gridDim.x * blockDim.x) {
    const int e = ea0 + (int)x;
    const int r = rowA[e] - rb;
    const int k = colA[e];
    const int bs = rpB[k], L = rpB[k + 1] - bs;
    const long long ro = Ro[r];
    const int pe = Pe[e];
    const long long g = ro >= 0 ? ro + pe : -(long long)pe - 1;
    int rlo = pe, rhi = pe + L - 1;
    if (ro >= 0 && L > 0) {
      rlo = (int)(R[g] & ~RFLAG);
      rhi = (int)(R[g + L - 1] & ~RFLAG);
    }
    const long long cr = crow[r];
    rec0[x] = make_int4(bs, L, (int)(unsigned)(g & 0xffffffffLL), (int)(g >> 32));
    rec1[x] = make_int4((int)(unsigned)(cr & 0xffffffffLL), (int)(cr >> 32), rlo, rhi);
  }
}

// ---- numeric core ----------------------------------------------------------------------------
constexpr int NUM_LONG = 64;     // runs with at least this many products become work items
constexpr int NUM_ITEM = 256;    // products per work item
constexpr int NUM_CTCAP = 1024;  // 32-product windows per chunk with a precomputed run index

template <typename V, int NT, int WS, int DUPCAP>
struct NumSmem {
  static constexpr int val = 0;                                    // V[WS]     image values
  static constexpr int col = val + WS * (int)sizeof(V);            // int[WS]   image columns
  static constexpr int dval = col + WS * 4;                        // V[DUPCAP] queued duplicates
  static constexpr int dpos = dval + DUPCAP * (int)sizeof(V);      // int[DUPCAP]
  static constexpr int rg = (dpos + DUPCAP * 4 + 15) & ~15;        // long long[NT] short run: R index of its start (-1: none)
  static constexpr int ra = rg + NT * 8;                           // V[NT]     short run: A value
  static constexpr int rec = (ra + NT * (int)sizeof(V) + 15) & ~15;  // int4[NT] short run: {offset, B start, image pos of rank 0, -}
  static constexpr int lrg = rec + NT * 16;                        // long long[NT] long run: R index
  static constexpr int lra = lrg + NT * 8;                         // V[NT]     long run: A value
  static constexpr int lrec = (lra + NT * (int)sizeof(V) + 15) & ~15;  // int4[NT] long run: {B start, image pos, L, -}
  static constexpr int libase = lrec + NT * 16;                    // int[NT+1] long run: first work item
  static constexpr int seg = libase + (NT + 1) * 4;                // int[NT+1] short run: product offset
  static constexpr int ctab = seg + (NT + 1) * 4;                  // u16[CTCAP] short-run index of each 32-product window
  static constexpr int bytes = (ctab + NUM_CTCAP * 2 + 15) & ~15;
};

template <int NT>
__device__ __forceinline__ unsigned long long block_excl_scan_u64(unsigned long long v, unsigned long long& total,
                                                                  unsigned long long* scratch) {
  constexpr int NW = NT / 32;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const unsigned long long incl = warp_incl_scan(v);
  if (lane == 31) scratch[w] = incl;
  __syncthreads();
  if (w == 0) {
    const unsigned long long x = lane < NW ? scratch[lane] : 0;
    const unsigned long long xi = warp_incl_scan(x);
    if (lane < NW) scratch[lane] = xi - x;
    if (lane == NW - 1) scratch[NW] = xi;
  }
  __syncthreads();
  const unsigned long long r = incl - v + scratch[w];
  total = scratch[NW];
  __syncthreads();
  return r;
}

struct ChunkShape {
  int Ls, ns;   // short runs: products, runs
  int nl, nit;  // long runs: runs, work items
};

// A thread's prefetched A entry: its run records and its value.
template <typename V>
struct Pref {
  int4 r0, r1;
  V a;
};

// Issue the loads of local A entry e (< eb) now; they are consumed a chunk later.
template <typename V>
__device__ __forceinline__ Pref<V> pref_load(const NumProb<V>& P, int e, int eb, int ea0) {
  const bool ok = e < eb;
  Pref<V> f;
  f.r0 = ldp_v4(P.rec0 + e, ok);  // length 0 when !ok
  f.r1 = ldp_v4(P.rec1 + e, ok);
  f.a = ldp_val(P.valA + ea0 + e, ok);
  return f;
}

// Run tables of one chunk (one prefetched A entry per thread) for the outputs [lo, lo + wl).
template <typename V, int NT, int WS, int DUPCAP>
__device__ __forceinline__ ChunkShape num_chunk_table(unsigned char* sm, unsigned long long* scratch, const Pref<V>& pf,
                                                      long long lo, int wl) {
  using S = NumSmem<V, NT, WS, DUPCAP>;
  const int tid = threadIdx.x;
  int bs = pf.r0.x, L = pf.r0.y;
  long long g0 = ((long long)pf.r0.w << 32) | (unsigned)pf.r0.z;
  int base = (int)((((long long)pf.r1.y << 32) | (unsigned)pf.r1.x) - lo);
  const V a = pf.a;
  if (L > 0 && (base + pf.r1.w < 0 || base + pf.r1.z >= wl)) L = 0;  // rank range misses the pass
  if (L > 0 && g0 < 0) {  // identity row: ranks pe + [0, L) — clip to the pass
    const int pe = (int)(-g0 - 1);
    g0 = -1;
    const int l0 = max(0, -base - pe), l1 = min(L, wl - base - pe);
    bs += l0;
    L = l1 - l0;
    base += pe + l0;
  }
  const bool lg = L >= NUM_LONG, sh = L > 0 && !lg;
  const unsigned long long items = lg ? (unsigned long long)((L + NUM_ITEM - 1) / NUM_ITEM) : 0ull;
  // fields: short products [0,16) | short runs [16,26) | long runs [26,36) | items [36,64)
  const unsigned long long pk = (sh ? (unsigned long long)L : 0ull) | ((unsigned long long)sh << 16) |
                                ((unsigned long long)lg << 26) | (items << 36);
  unsigned long long tot;
  const unsigned long long ex = block_excl_scan_u64<NT>(pk, tot, scratch);
  ChunkShape cs;
  cs.Ls = (int)(tot & 0xffff);
  cs.ns = (int)((tot >> 16) & 0x3ff);
  cs.nl = (int)((tot >> 26) & 0x3ff);
  cs.nit = (int)(tot >> 36);
  if (sh) {
    const int slot = (int)((ex >> 16) & 0x3ff), off = (int)(ex & 0xffff);
    reinterpret_cast<int*>(sm + S::seg)[slot] = off;
    reinterpret_cast<int4*>(sm + S::rec)[slot] = make_int4(off, bs, base, 0);
    reinterpret_cast<long long*>(sm + S::rg)[slot] = g0;
    reinterpret_cast<V*>(sm + S::ra)[slot] = a;
  } else if (lg) {
    const int slot = (int)((ex >> 26) & 0x3ff), ib = (int)(ex >> 36);
    reinterpret_cast<int*>(sm + S::libase)[slot] = ib;
    reinterpret_cast<int4*>(sm + S::lrec)[slot] = make_int4(bs, base, L, 0);
    reinterpret_cast<long long*>(sm + S::lrg)[slot] = g0;
    reinterpret_cast<V*>(sm + S::lra)[slot] = a;
  }
  if (tid == 0) {
    reinterpret_cast<int*>(sm + S::seg)[cs.ns] = cs.Ls;
    reinterpret_cast<int*>(sm + S::libase)[cs.nl] = cs.nit;
  }
  __syncthreads();
  const int* seg = reinterpret_cast<const int*>(sm + S::seg);
  unsigned short* ctab = reinterpret_cast<unsigned short*>(sm + S::ctab);
  for (int x = tid; x < min((cs.Ls + 31) >> 5, NUM_CTCAP); x += NT) ctab[x] = (unsigned short)upper_idx(seg, cs.ns, x << 5);
  __syncthreads();
  return cs;
}

// Global overflow queue of non-first products (large rows: a block's own region).
template <typename V>
struct GQueue {
  int* pos;
  V* val;
  int cap;
};

// One product per lane.  PASS 0 stores first occurrences into the image and queues the others
// (shared queue, then the block's global overflow queue); PASS 1 (both queues full) adds them
// directly.
template <typename V, int NT, int WS, int DUPCAP, int PASS>
__device__ __forceinline__ void num_emit(unsigned char* sm, int* s_ndup, const GQueue<V>& gq, bool in, bool first, int pos,
                                         int col, V v) {
  using S = NumSmem<V, NT, WS, DUPCAP>;
  const int lane = threadIdx.x & 31;
  V* s_val = reinterpret_cast<V*>(sm + S::val);
  if (PASS == 0) {
    if (in && first) {
      reinterpret_cast<int*>(sm + S::col)[pos] = col;
      s_val[pos] = v;
    }
    const bool dup = in && !first;
    const unsigned dm = __ballot_sync(FULL, dup);
    if (dm) {
      const int leader = __ffs(dm) - 1;
      int d0 = 0;
      if (lane == leader) d0 = atomicAdd(s_ndup, __popc(dm));
      d0 = __shfl_sync(FULL, d0, leader) + __popc(dm & lanemask_lt());
      if (dup) {
        if (d0 < DUPCAP) {
          reinterpret_cast<int*>(sm + S::dpos)[d0] = pos;
          reinterpret_cast<V*>(sm + S::dval)[d0] = v;
        } else if (d0 - DUPCAP < gq.cap) {
          gq.pos[d0 - DUPCAP] = pos;
          gq.val[d0 - DUPCAP] = v;
        }
      }
    }
  } else if (in && !first) {
    atomicAdd(&s_val[pos], v);
  }
}

template <typename V, int NT, int WS, int DUPCAP, int PASS>
__device__ __forceinline__ void num_chunk_products(const NumProb<V>& P, unsigned char* sm, int* s_ndup,
                                                   const GQueue<V>& gq, const ChunkShape& cs, int wl) {
  using S = NumSmem<V, NT, WS, DUPCAP>;
  constexpr int NW = NT / 32;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const unsigned upto = (2u << lane) - 1u;
  // ---- long runs: one warp per work item, run data warp-uniform --------------------------------
  {
    const int4* lrec = reinterpret_cast<const int4*>(sm + S::lrec);
    const long long* lrg = reinterpret_cast<const long long*>(sm + S::lrg);
    const V* lra = reinterpret_cast<const V*>(sm + S::lra);
    const int* libase = reinterpret_cast<const int*>(sm + S::libase);
    for (int t = warp; t < cs.nit; t += NW) {
      const int lr = upper_idx(libase, cs.nl, t);
      const int4 lc = lrec[lr];
      const long long g = lrg[lr];
      const V a = lra[lr];
      const int o0 = (t - libase[lr]) * NUM_ITEM, o1 = min(o0 + NUM_ITEM, lc.z);
      const bool hasR = g >= 0;
      const unsigned* rr = P.R + (hasR ? g : 0);
      if (hasR && WS > NUM_WS) {  // multi-pass rows: skip an item whose rank range misses the pass
        const int rf = (int)(rr[o0] & ~RFLAG), rl = (int)(rr[o1 - 1] & ~RFLAG);
        if (lc.y + rl < 0 || lc.y + rf >= wl) continue;
      }
      const int* cb = P.colB + lc.x;
      const V* vb = P.valB + lc.x;
      constexpr int U = NT >= 1024 ? 2 : 4;
      for (int ob = o0; ob < o1; ob += 32 * U) {
        unsigned rv[U];
        int cB[U];
        V bB[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int off = ob + u * 32 + lane;
          const bool ok = off < o1;
          rv[u] = ldp_u32_stream(rr + off, ok && hasR, (unsigned)off | RFLAG);
          cB[u] = ldp_s32(cb + off, ok && PASS == 0);
          bB[u] = ldp_val(vb + off, ok);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
          const int off = ob + u * 32 + lane;
          const int pos = lc.y + (int)(rv[u] & ~RFLAG);
          const bool in = off < o1 && (unsigned)pos < (unsigned)wl;
          num_emit<V, NT, WS, DUPCAP, PASS>(sm, s_ndup, gq, in, rv[u] & RFLAG, pos, cB[u], a * bB[u]);
        }
      }
    }
  }
  // ---- short runs: flattened across lanes ------------------------------------------------------
  const long long* rg = reinterpret_cast<const long long*>(sm + S::rg);
  const V* ra = reinterpret_cast<const V*>(sm + S::ra);
  const int4* rec = reinterpret_cast<const int4*>(sm + S::rec);
  const int* seg = reinterpret_cast<const int*>(sm + S::seg);
  const unsigned short* ctab = reinterpret_cast<const unsigned short*>(sm + S::ctab);
  const int Lt = cs.Ls, nr = cs.ns;
  constexpr int U = 2;
  for (int jb = warp * 32; jb < Lt; jb += U * NT) {
    int r[U], off[U], q[U];
    long long g[U];
    bool ok[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int j0 = jb + u * NT;
      r[u] = 0;
      ok[u] = false;
      if (j0 < Lt) {  // warp-uniform
        const int rb = (j0 >> 5) < NUM_CTCAP ? (int)ctab[j0 >> 5] : upper_idx(seg, nr, j0);
        const int rs = rb + 1 + lane;
        const int d = rs <= nr ? seg[rs] - j0 : 32;
        const unsigned M = __reduce_or_sync(FULL, (unsigned)(d - 1) < 31u ? (1u << d) : 0u);
        r[u] = rb + __popc(M & upto);
        ok[u] = j0 + lane < Lt;
      }
      const int4 rc = rec[r[u]];
      off[u] = j0 + lane - rc.x;
      q[u] = rc.y + off[u];
      g[u] = rg[r[u]];
    }
    unsigned rv[U];
    int cB[U];
    V bB[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      rv[u] = ldp_u32_stream(P.R + (g[u] + off[u]), ok[u] && g[u] >= 0, (unsigned)off[u] | RFLAG);
      cB[u] = ldp_s32(P.colB + q[u], ok[u] && PASS == 0);
      bB[u] = ldp_val(P.valB + q[u], ok[u]);
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int pos = rec[r[u]].z + (int)(rv[u] & ~RFLAG);
      const bool in = ok[u] && (unsigned)pos < (unsigned)wl;
      num_emit<V, NT, WS, DUPCAP, PASS>(sm, s_ndup, gq, in, rv[u] & RFLAG, pos, cB[u], ra[r[u]] * bB[u]);
    }
  }
}

// One pass of a unit: outputs [lo, lo + wl) from local A entries [ea, eb).  pf holds the first
// chunk's records on entry and the records of (ne, neb) — the next chunk of this block's
// sequence — on exit.
template <typename V, int NT, int WS, int DUPCAP>
__device__ __forceinline__ void num_pass(const NumProb<V>& P, unsigned char* sm, unsigned long long* scratch,
                                         int* s_ndup, const GQueue<V>& gq, Pref<V>& pf, int ea, int eb, long long lo,
                                         int wl, int ne, int neb, int ea0) {
  using S = NumSmem<V, NT, WS, DUPCAP>;
  V* s_val = reinterpret_cast<V*>(sm + S::val);
  const int* s_col = reinterpret_cast<const int*>(sm + S::col);
  const int tid = threadIdx.x;
  if (tid == 0) *s_ndup = 0;
  for (int c0 = ea; c0 < eb; c0 += NT) {
    const ChunkShape cs = num_chunk_table<V, NT, WS, DUPCAP>(sm, scratch, pf, lo, wl);
    if (c0 + NT < eb) pf = pref_load(P, c0 + NT + tid, eb, ea0);
    else pf = pref_load(P, ne + tid, neb, ea0);
    num_chunk_products<V, NT, WS, DUPCAP, 0>(P, sm, s_ndup, gq, cs, wl);
    __syncthreads();
  }
  const int nd = *s_ndup;
  if (nd <= DUPCAP + gq.cap) {
    const int* s_dpos = reinterpret_cast<const int*>(sm + S::dpos);
    const V* s_dval = reinterpret_cast<const V*>(sm + S::dval);
    for (int d = tid; d < min(nd, DUPCAP); d += NT) atomicAdd(&s_val[s_dpos[d]], s_dval[d]);
    for (int d = DUPCAP + tid; d < nd; d += NT) atomicAdd(&s_val[gq.pos[d - DUPCAP]], gq.val[d - DUPCAP]);
  } else {  // both queues full: re-enumerate, every duplicate adds directly (first occurrences are stored)
    for (int c0 = ea; c0 < eb; c0 += NT) {
      const Pref<V> pq = pref_load(P, c0 + tid, eb, ea0);
      const ChunkShape cs = num_chunk_table<V, NT, WS, DUPCAP>(sm, scratch, pq, lo, wl);
      num_chunk_products<V, NT, WS, DUPCAP, 1>(P, sm, s_ndup, gq, cs, wl);
      __syncthreads();
    }
  }
  __syncthreads();
  int* ccol = P.ccol + lo;
  V* cval = P.cval + lo;
  for (int x = tid; x < wl; x += NT) {
    __stcs(ccol + x, s_col[x]);
    __stcs(cval + x, s_val[x]);
  }
  __syncthreads();
}

// Window units (c <= NUM_WS, one pass each), static striding; the next unit's first records are
// prefetched during the last chunk of the current one.
template <typename V>
__global__ void __launch_bounds__(NUM_NT, 4) k_num_windows(NumProb<V> P) {
  extern __shared__ __align__(16) unsigned char sm[];
  __shared__ unsigned long long scratch[NUM_NT / 32 + 1];
  __shared__ int s_ndup;
  const int n = P.small->nwunits;
  int u = blockIdx.x;
  if (u >= n) return;
  const int ea0 = P.small->ea0;
  const GQueue<V> gq{nullptr, nullptr, 0};
  Unit cur = P.wunits[u];
  Pref<V> pf = pref_load(P, cur.ea + (int)threadIdx.x, cur.eb, ea0);
  for (;;) {
    const int un = u + gridDim.x;
    const Unit nxt = un < n ? P.wunits[un] : Unit{0, 0, 0, 0, 0};
    num_pass<V, NUM_NT, NUM_WS, NUM_WDUP>(P, sm, scratch, &s_ndup, gq, pf, cur.ea, cur.eb, cur.lo, cur.c, nxt.ea,
                                          nxt.eb, ea0);
    if (un >= n) break;
    u = un;
    cur = nxt;
  }
}

// Long rows (c > NUM_WS): one block per row from a dynamic queue, NUM_LS outputs per pass.
template <typename V, int NT, int LS, int MINB>
__global__ void __launch_bounds__(NT, MINB) k_num_large(NumProb<V> P) {
  extern __shared__ __align__(16) unsigned char sm[];
  __shared__ unsigned long long scratch[NT / 32 + 1];
  __shared__ int s_ndup, s_next;
  const int n = P.small->nlunits;
  const int ea0 = P.small->ea0;
  const GQueue<V> gq{P.gq_pos + (size_t)blockIdx.x * NUM_GDUP, P.gq_val + (size_t)blockIdx.x * NUM_GDUP, NUM_GDUP};
  if (threadIdx.x == 0) s_next = atomicAdd(P.lqhead, 1);
  __syncthreads();
  int t = s_next;
  __syncthreads();
  if (t >= n) return;
  Unit cur = P.lunits[t];
  Pref<V> pf = pref_load(P, cur.ea + (int)threadIdx.x, cur.eb, ea0);
  for (;;) {
    if (threadIdx.x == 0) s_next = atomicAdd(P.lqhead, 1);
    __syncthreads();
    const int tn = s_next;
    const Unit nxt = tn < n ? P.lunits[tn] : Unit{0, 0, 0, 0, 0};
    for (int s0 = 0; s0 < cur.c; s0 += LS) {
      const bool lastpass = s0 + LS >= cur.c;
      num_pass<V, NT, LS, NUM_LDUP>(P, sm, scratch, &s_ndup, gq, pf, cur.ea, cur.eb, cur.lo + s0,
                                    min(LS, cur.c - s0), lastpass ? nxt.ea : cur.ea, lastpass ? nxt.eb : cur.eb, ea0);
    }
    if (tn >= n) break;
    cur = nxt;
  }
}

// Large-row kernel configurations: A = one 512-thread block per SM staging NUM_LS_A outputs;
// B = two per SM staging NUM_LS_B (more rows in flight, more multi-pass rows).
// C = one 1024-thread block per SM staging NUM_LS_A outputs.
constexpr int NUM_LS_A = 12288, NUM_LS_B = 5120;
#define NUM_LARGE_A k_num_large<V, 512, NUM_LS_A, 1>
#define NUM_LARGE_B k_num_large<V, 512, NUM_LS_B, 2>
#define NUM_LARGE_C k_num_large<V, 1024, NUM_LS_A, 1>
template <typename V>
constexpr int large_smem(int cfg) {
  return cfg == 1 ? NumSmem<V, 512, NUM_LS_B, NUM_LDUP>::bytes
                  : cfg == 2 ? NumSmem<V, 1024, NUM_LS_A, NUM_LDUP>::bytes : NumSmem<V, 512, NUM_LS_A, NUM_LDUP>::bytes;
}
static_assert(NumSmem<double, 1024, NUM_LS_A, NUM_LDUP>::bytes + 2048 <= 227 * 1024, "large-row kernel C");

static_assert(NumSmem<double, 512, NUM_LS_A, NUM_LDUP>::bytes + 1024 <= 227 * 1024, "large-row kernel A");
static_assert(2 * (NumSmem<double, 512, NUM_LS_B, NUM_LDUP>::bytes + 1024) <= 228 * 1024, "large-row kernel B");
static_assert(NumSmem<double, NUM_NT, NUM_WS, NUM_WDUP>::bytes * 4 <= 227 * 1024, "window kernel: 4 blocks per SM");

// ---- launch glue ---------------------------------------------------------------------------
static int grid_n(long long n, int cap) { return (int)(n < 1 ? 1 : (n > cap ? cap : n)); }

cudaError_t launch_plan(cudaStream_t st, int sms, const long long* crow, int mloc, const int* rpA, const int* colA,
                        const int* rpB, const int* rowA, const int* Pe, const long long* Ro, const unsigned* R, int rb,
                        int re, long long nnzA_upper, int* cnt, long long* coff, long long* scan_tmp, Cut* cuts,
                        Unit* wunits, Unit* lunits, int lcap, int4* rec0, int4* rec1, Small* small) {
  if (mloc <= 0) return cudaSuccess;
  k_cut_count<<<grid_n((mloc + 255) / 256, sms * 8), 256, 0, st>>>(crow, mloc, rpA, rb, cnt, lunits, lcap, small);
  cudaError_t e = cudaMemsetAsync(coff, 0, sizeof(long long), st);
  if (e != cudaSuccess) return e;
  e = launch_incl_scan<int>(st, cnt, coff + 1, mloc, scan_tmp);
  if (e != cudaSuccess) return e;
  k_cut_write<<<grid_n((mloc + 255) / 256, sms * 8), 256, 0, st>>>(crow, mloc, coff, cuts, small);
  k_units<<<grid_n((2LL * mloc + 2 + 255) / 256, sms * 8), 256, 0, st>>>(cuts, coff, mloc, rpA, rb, wunits, small);
  k_records<<<grid_n((nnzA_upper + 255) / 256, sms * 16), 256, 0, st>>>(rpA, colA, rpB, rowA, Pe, Ro, R, crow, rb, re,
                                                                        rec0, rec1, small);
  return cudaGetLastError();
}

int plan_launches(long long mloc) { return mloc <= 0 ? 0 : 4 + scan_launches(mloc); }

template <typename V>
cudaError_t numeric_configure() {
  cudaError_t e = cudaFuncSetAttribute(k_num_windows<V>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       NumSmem<V, NUM_NT, NUM_WS, NUM_WDUP>::bytes);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(NUM_LARGE_A, cudaFuncAttributeMaxDynamicSharedMemorySize, large_smem<V>(0));
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(NUM_LARGE_B, cudaFuncAttributeMaxDynamicSharedMemorySize, large_smem<V>(1));
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(NUM_LARGE_C, cudaFuncAttributeMaxDynamicSharedMemorySize, large_smem<V>(2));
  return e;
}

template <typename V>
int numeric_occupancy(int which) {
  int nb = 1;
  if (which == 0)
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_num_windows<V>, NUM_NT, NumSmem<V, NUM_NT, NUM_WS, NUM_WDUP>::bytes);
  else if (which == 1)
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, NUM_LARGE_A, 512, large_smem<V>(0));
  else if (which == 2)
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, NUM_LARGE_B, 512, large_smem<V>(1));
  else
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, NUM_LARGE_C, 1024, large_smem<V>(2));
  return nb < 1 ? 1 : nb;
}

template <typename V>
cudaError_t launch_num_windows(cudaStream_t st, int grid, const NumProb<V>& P) {
  if (grid <= 0) return cudaSuccess;
  k_num_windows<V><<<grid, NUM_NT, NumSmem<V, NUM_NT, NUM_WS, NUM_WDUP>::bytes, st>>>(P);
  return cudaGetLastError();
}

template <typename V>
cudaError_t launch_num_large(cudaStream_t st, int grid, int cfg, const NumProb<V>& P) {
  if (grid <= 0) return cudaSuccess;
  if (cfg == 1) NUM_LARGE_B<<<grid, 512, large_smem<V>(1), st>>>(P);
  else if (cfg == 2) NUM_LARGE_C<<<grid, 1024, large_smem<V>(2), st>>>(P);
  else NUM_LARGE_A<<<grid, 512, large_smem<V>(0), st>>>(P);
  return cudaGetLastError();
}

#define INST(V)                                                                              \
  template cudaError_t numeric_configure<V>();                                               \
  template int numeric_occupancy<V>(int);                                                    \
  template cudaError_t launch_num_windows<V>(cudaStream_t, int, const NumProb<V>&);          \
  template cudaError_t launch_num_large<V>(cudaStream_t, int, int, const NumProb<V>&);
INST(double)
INST(float)
#undef INST

}  // namespace spg
