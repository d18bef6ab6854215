// merge.cuh — in-row run merge for LIGHT (warp) and MEDIUM (block) rows.
//
// The products of row i are the union of the B rows its A entries select ("runs"), each
// already sorted by column (B canonical).  The row is produced by merging the runs pairwise
// in shared memory (merge path, stable), then adding like-tuples (equal adjacent columns) and
// writing the compacted, sorted row straight into CSR: the Phase IV merge of PAPER.md
// L154-156 (sort by (r,c), mark, scan, one master thread adds, compact) done per row.
//
// Scale-free rows are skewed: one long B row (a hub) usually carries most of the products
// (DESIGN.md §4).  The longest run is therefore moved to the end and
// merged last, so the log2(#runs) rounds only touch the short runs' products and the hub's
// products move once.  Each thread emits ceil(round size / threads) outputs per round (odd,
// <= 15), so every lane works and the merge-path search is amortised on long rounds.
#pragma once
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

// Merge the segment pairs of one round: segments are groups of `w` consecutive runs (run r
// spans [seg[r], seg[r+1])), pairs (2m, 2m+1) over runs [0, nr); output elements [0, fr).
template <int G, bool NUM, typename V>
__device__ __forceinline__ void merge_round(const int* sk, int* dk, const V* sv, V* dv, const int* seg, int nr, int w,
                                            int fr, int rank) {
  const int lw2 = 31 - __clz(2 * w);
  const int npairs = (nr + 2 * w - 1) >> lw2;
  // odd: each thread writes vt consecutive outputs, so an even vt would put lanes on the same
  // shared-memory banks (vt = 16 is a 16-way conflict)
  // (and as small as covers the round with every thread: idle lanes still pay each instruction)
  const int vt = min(MERGE_VT_MAX, (fr + G - 1) / G) | 1;
  for (int o0 = rank * vt; o0 < fr; o0 += G * vt) {
    int o = o0;
    const int oend = min(o0 + vt, fr);
    int lo = 0, hi = npairs - 1;
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (seg[mid << lw2] <= o) lo = mid; else hi = mid - 1;
    }
    int m = lo;
    while (o < oend) {
      const int ra = m << lw2, rb = min(ra + w, nr), rc = min(ra + 2 * w, nr);
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
      for (int t = 0; t < n; ++t) {  // branchless: one key load per output
        const bool ta = ka <= kb;
        const int src = ta ? ia : ib;
        dk[o + t] = ta ? ka : kb;
        if (NUM) dv[o + t] = sv[src];
        const int nx = src + 1, lim = ta ? a1 : a2;
        const int kn = nx < lim ? sk[nx] : KEY_INF;
        ia += ta;
        ib += !ta;
        ka = ta ? kn : ka;
        kb = ta ? kb : kn;
      }
      o += n;
      ++m;
    }
  }
}

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

  // 1. runs: compact the non-empty B rows this A row selects; seg = run offsets; track the
  //    longest run.  (run start bs stashed in keyY, scale a in valY — free until round 1)
  int nr = 0, f = 0, best = -1;
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
    const int slot = nr + (ex & 0xffff);
    if (L > 0) {
      seg[slot] = f + (ex >> 16);
      keyY[slot] = bs;
      if (NUM) valY[slot] = a;
    }
    best = max(best, L > 0 ? (L << 13) | slot : -1);  // L <= 8192, slot < 8192
    nr += tot & 0xffff;
    f += tot >> 16;
  }
  best = g.max(best);
  if (g.rank == 0) seg[nr] = f;
  g.sync();

  // 2. hub last: swap the longest run into the last slot (only the seg entries between the
  //    two slots move) when that saves element moves.
  const int Lbest = best >> 13, m = best & 8191;
  bool hub = nr >= 3 && 4 * Lbest >= f;
  if (hub && m != nr - 1) {
    const int Llast = seg[nr] - seg[nr - 1];
    const int sh = Llast - Lbest;
    int bsm = 0, bsl = 0;
    V am = V(0), al = V(0);
    if (g.rank == 0) { bsm = keyY[m]; bsl = keyY[nr - 1]; if (NUM) { am = valY[m]; al = valY[nr - 1]; } }
    g.sync();
    for (int r = m + 1 + g.rank; r <= nr - 1; r += G) seg[r] += sh;
    if (g.rank == 0) {
      keyY[m] = bsl; keyY[nr - 1] = bsm;
      if (NUM) { valY[m] = al; valY[nr - 1] = am; }
    }
    g.sync();
  }

  // 3. expand: product j of run r -> keyX[j] = colB, valX[j] = a_r * valB (coalesced per run).
  //    EU products per thread per step: run lookups first, then all loads, then the stores, so
  //    one L2 round trip covers EU products.
  constexpr int EU = 8;
  for (int j0 = g.rank; j0 < f; j0 += G * EU) {
    int q[EU], r[EU];
#pragma unroll
    for (int u = 0; u < EU; ++u) {
      const int j = j0 + u * G;
      r[u] = 0;
      q[u] = -1;
      if (j < f) {
        r[u] = upper_idx(seg, nr, j);
        q[u] = keyY[r[u]] + (j - seg[r[u]]);
      }
    }
    int kk[EU];
    V bb[EU];
#pragma unroll
    for (int u = 0; u < EU; ++u) {
      kk[u] = q[u] >= 0 ? P.colB[q[u]] : 0;
      if (NUM) bb[u] = q[u] >= 0 ? P.valB[q[u]] : V(0);
    }
#pragma unroll
    for (int u = 0; u < EU; ++u) {
      const int j = j0 + u * G;
      if (j < f) {
        keyX[j] = kk[u];
        if (NUM) valX[j] = valY[r[u]] * bb[u];
      }
    }
  }
  g.sync();
  const int nrs = hub ? nr - 1 : nr;
  const int fs = seg[nrs];
  if (hub) {  // the hub's products never move during the short-run rounds: mirror them once
    for (int j = fs + g.rank; j < f; j += G) {
      keyY[j] = keyX[j];
      if (NUM) valY[j] = valX[j];
    }
    g.sync();
  }

  // 4. pairwise rounds over the short runs (all runs when there is no hub), then the hub
  int* sk = keyX;
  int* dk = keyY;
  V* sv = valX;
  V* dv = valY;
  for (int w = 1; w < nrs; w <<= 1) {
    merge_round<G, NUM, V>(sk, dk, sv, dv, seg, nrs, w, fs, g.rank);
    g.sync();
    int* tk = sk; sk = dk; dk = tk;
    V* tv = sv; sv = dv; dv = tv;
  }
  if (hub) {
    // two segments [0, fs) and [fs, f): the round reads seg[0], seg[1], seg[2]
    g.sync();
    if (g.rank == 0) { seg[1] = fs; seg[2] = f; }
    g.sync();
    merge_round<G, NUM, V>(sk, dk, sv, dv, seg, 2, 1, f, g.rank);
    g.sync();
    int* tk = sk; sk = dk; dk = tk;
    V* tv = sv; sv = dv; dv = tv;
  }

  // 5. like-tuples: head = first of each equal-column group; each thread owns a contiguous
  //    segment, counts its heads, one group scan gives output positions, heads add their group.
  const long long rowoff = NUM ? P.crow[i - P.row_begin] : 0;
  const int vo = (f + G - 1) / G;
  const int s0 = min(g.rank * vo, f), s1 = min(s0 + vo, f);
  int heads = 0;
  for (int j = s0; j < s1; ++j) heads += (j == 0 || sk[j - 1] != sk[j]);
  int tot;
  int pos = g.excl_scan(heads, tot);
  if (NUM) {
    for (int j = s0; j < s1; ++j) {
      const int kj = sk[j];
      if (j > 0 && sk[j - 1] == kj) continue;
      V s = sv[j];
      for (int t2 = j + 1; t2 < f && sk[t2] == kj; ++t2) s += sv[t2];
      P.ccol[rowoff + pos] = kj;
      P.cval[rowoff + pos] = s;
      ++pos;
    }
  }
  if (!NUM && g.rank == 0) P.crow[i - P.row_begin + 1] = tot;
  g.sync();
}

// Bucketed ESC for one row (LIGHT / MEDIUM): expand the products, histogram them by the column's
// high bits into NB buckets (ATOMS.ADD returns each product's slot), scan, scatter into bucket
// order, then every thread insertion-sorts its own few buckets (random columns: ~CAP/NB
// products per bucket), counts heads and writes the compacted row.  A fixed number of barriers
// per row — no log2(#runs) merge rounds.  Rows whose buckets turn out skewed (clustered
// columns, > MAXB in one bucket) fall back to merge_row.  Same shared-memory footprint as
// merge_row: the run table's space (seg) holds the slots and bucket counts after the expand.
template <int G, int CAP, bool NUM, typename V>
__device__ __forceinline__ void esc_row(const Prob<V>& P, const int i, const Group<G>& g, char* smem) {
  constexpr int NB = CAP / 4, MAXB = 48;
  V* valX = reinterpret_cast<V*>(smem);
  V* valY = valX + CAP;
  int* keyX = reinterpret_cast<int*>(smem + (NUM ? 2 * CAP * sizeof(V) : 0));
  int* keyY = keyX + CAP;
  int* seg = keyY + CAP;
  const int pa0 = P.rpA[i], pa1 = P.rpA[i + 1];
  // runs (no hub handling needed)
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
    int tot;
    const int ex = g.excl_scan((L << 16) | (L > 0 ? 1 : 0), tot);
    const int slot = nr + (ex & 0xffff);
    if (L > 0) {
      seg[slot] = f + (ex >> 16);
      keyY[slot] = bs;
      if (NUM) valY[slot] = a;
    }
    nr += tot & 0xffff;
    f += tot >> 16;
  }
  if (g.rank == 0) seg[nr] = f;
  g.sync();
  constexpr int EU = 8;
  for (int j0 = g.rank; j0 < f; j0 += G * EU) {
    int q[EU], r[EU];
#pragma unroll
    for (int u = 0; u < EU; ++u) {
      const int j = j0 + u * G;
      r[u] = 0;
      q[u] = -1;
      if (j < f) {
        r[u] = upper_idx(seg, nr, j);
        q[u] = keyY[r[u]] + (j - seg[r[u]]);
      }
    }
    int kk[EU];
    V bb[EU];
#pragma unroll
    for (int u = 0; u < EU; ++u) {
      kk[u] = q[u] >= 0 ? P.colB[q[u]] : 0;
      if (NUM) bb[u] = q[u] >= 0 ? P.valB[q[u]] : V(0);
    }
#pragma unroll
    for (int u = 0; u < EU; ++u) {
      const int j = j0 + u * G;
      if (j < f) {
        keyX[j] = kk[u];
        if (NUM) valX[j] = valY[r[u]] * bb[u];
      }
    }
  }
  g.sync();
  // histogram (seg area reused: cnt[NB + 1] then 16-bit slots)
  int* cnt = seg;
  unsigned short* slot = reinterpret_cast<unsigned short*>(seg + NB + 1);
  const int lgNB = 31 - __clz(NB);
  const int shift = P.lgN > lgNB ? P.lgN - lgNB : 0;
  for (int b = g.rank; b <= NB; b += G) cnt[b] = 0;
  g.sync();
  for (int j = g.rank; j < f; j += G) slot[j] = (unsigned short)atomicAdd(&cnt[keyX[j] >> shift], 1);
  g.sync();
  // exclusive scan of the bucket counts, NB / G contiguous buckets per thread
  constexpr int BPT = NB / G > 0 ? NB / G : 1;
  int mine = 0, mx = 0;
  int c8[BPT];
#pragma unroll
  for (int k = 0; k < BPT; ++k) {
    const int b = g.rank * BPT + k;
    c8[k] = b < NB ? cnt[b] : 0;
    mine += c8[k];
    mx = max(mx, c8[k]);
  }
  int tot;
  int run = g.excl_scan(mine, tot);
  const int mxall = g.max(mx);
  if (mxall > MAXB) {  // clustered columns: merge instead (re-gathers the runs)
    merge_row<G, CAP, NUM, V>(P, i, g, smem);
    return;
  }
#pragma unroll
  for (int k = 0; k < BPT; ++k) {
    const int b = g.rank * BPT + k;
    if (b < NB) cnt[b] = run;
    run += c8[k];
  }
  if (g.rank == 0) cnt[NB] = f;
  g.sync();
  for (int j = g.rank; j < f; j += G) {
    const int d = cnt[keyX[j] >> shift] + slot[j];
    keyY[d] = keyX[j];
    if (NUM) valY[d] = valX[j];
  }
  g.sync();
  // sort each of my buckets (insertion sort), count heads
  int heads = 0;
#pragma unroll
  for (int k = 0; k < BPT; ++k) {
    const int b = g.rank * BPT + k;
    if (b >= NB) break;
    const int s0 = cnt[b], s1 = cnt[b + 1];
    for (int x = s0 + 1; x < s1; ++x) {
      const int kx = keyY[x];
      V vx = V(0);
      if (NUM) vx = valY[x];
      int y = x - 1;
      while (y >= s0 && keyY[y] > kx) {
        keyY[y + 1] = keyY[y];
        if (NUM) valY[y + 1] = valY[y];
        --y;
      }
      keyY[y + 1] = kx;
      if (NUM) valY[y + 1] = vx;
    }
    for (int x = s0; x < s1; ++x) heads += (x == s0 || keyY[x - 1] != keyY[x]);
  }
  int htot;
  int pos = g.excl_scan(heads, htot);
  if (NUM) {
    const long long rowoff = P.crow[i - P.row_begin];
#pragma unroll
    for (int k = 0; k < BPT; ++k) {
      const int b = g.rank * BPT + k;
      if (b >= NB) break;
      const int s0 = cnt[b], s1 = cnt[b + 1];
      for (int x = s0; x < s1;) {
        const int kx = keyY[x];
        V s = valY[x];
        int y = x + 1;
        for (; y < s1 && keyY[y] == kx; ++y) s += valY[y];
        P.ccol[rowoff + pos] = kx;
        P.cval[rowoff + pos] = s;
        ++pos;
        x = y;
      }
    }
  } else if (g.rank == 0) {
    P.crow[i - P.row_begin + 1] = htot;
  }
  g.sync();
}

// ESC2 (numeric, LIGHT / MEDIUM): the bucketed ESC of esc_row with ~17 bytes of shared memory
// per product instead of 28, so twice the rows are in flight per SM.  The runs go to a small
// table (<= CAP/4 runs); the products are enumerated twice — a histogram pass, then a pass that
// scatters (key, a*b) straight into its bucket slot (atomicAdd cursor) — so no expand buffer.
// Rows with more runs or skewed buckets are appended to the fallback list (processed afterwards
// by the general HUGE-tier kernel) and nothing of them is written here.
template <int CAP>
__host__ __device__ constexpr int esc2_rcap() { return CAP / 4; }
template <typename V, int CAP>
__host__ __device__ constexpr int esc2_smem() {
  return CAP * (int)(sizeof(V) + 4) + (CAP / 4 + 1) * 4 + (esc2_rcap<CAP>() + 1) * 4 + esc2_rcap<CAP>() * 4 +
         esc2_rcap<CAP>() * (int)sizeof(V) + 32;
}
template <typename V, int CAP>
__host__ __device__ constexpr int esc2_smem_aligned() { return (esc2_smem<V, CAP>() + 15) & ~15; }

// Run of product j for a window of 32 consecutive products starting at jw (warp-uniform): one
// binary search for the window, then each lane's run = first run + popcount of the run starts
// inside the window at or below it (REDUX.OR bitmask).  All 32 lanes must call.
__device__ __forceinline__ int window_run(const int* seg, int nr, int jw) {
  const int lane = lane_id();
  const int rb = upper_idx(seg, nr, jw);
  const int rs = rb + 1 + lane;
  const int d = rs <= nr ? seg[rs] - jw : 32;
  const unsigned M = __reduce_or_sync(FULL, (d >= 1 && d <= 31) ? (1u << d) : 0u);
  return rb + __popc(M & ((2u << lane) - 1u));
}

// Run of product jw + lane for a window starting inside run rb (warp-uniform); advances rb to
// the run holding jw + 32.  All 32 lanes must call.
__device__ __forceinline__ int esc2_walk(const int* seg, int nr, int jw, int& rb) {
  const int lane = lane_id();
  const int rs = rb + 1 + lane;
  const int d = rs <= nr ? seg[rs] - jw : 64;
  const unsigned M = __reduce_or_sync(FULL, (d >= 1 && d <= 31) ? (1u << d) : 0u);
  const int r = rb + __popc(M & ((2u << lane) - 1u));
  rb += __popc(M) + (__ballot_sync(FULL, d == 32) != 0u);
  return r;
}

template <int G, int CAP, typename V>
__device__ __forceinline__ void esc2_row(const Prob<V>& P, const int i, const Group<G>& g, char* smem) {
  constexpr int NB = CAP / 4, MAXB = 48, RC = esc2_rcap<CAP>();
  V* vals = reinterpret_cast<V*>(smem);
  int* keys = reinterpret_cast<int*>(smem + CAP * sizeof(V));
  int* cnt = keys + CAP;                 // NB + 1
  int* seg = cnt + NB + 1;               // RC + 1
  int* sbs = seg + RC + 1;               // RC
  V* sa = reinterpret_cast<V*>(reinterpret_cast<uintptr_t>(sbs + RC + 1) & ~(uintptr_t)7);  // RC (8-aligned)
  const int pa0 = P.rpA[i], pa1 = P.rpA[i + 1];
  int nr = 0, f = 0;
  for (int p0 = pa0; p0 < pa1; p0 += G) {
    const int p = p0 + g.rank;
    int L = 0, bs = 0;
    V a = V(0);
    if (p < pa1) {
      const int k = P.colA[p];
      bs = P.rpB[k];
      L = P.rpB[k + 1] - bs;
      a = P.valA[p];
    }
    int tot;
    const int ex = g.excl_scan((L << 16) | (L > 0 ? 1 : 0), tot);
    const int slot = nr + (ex & 0xffff);
    if (L > 0 && slot < RC) {
      seg[slot] = f + (ex >> 16);
      sbs[slot] = bs;
      sa[slot] = a;
    }
    nr += tot & 0xffff;
    f += tot >> 16;
  }
  if (nr > RC) {  // too many runs for the table: general kernel
    if (g.rank == 0) P.fb_list[atomicAdd(P.fb_count, 1)] = i;
    g.sync();
    return;
  }
  if (g.rank == 0) seg[nr] = f;
  const int lgNB = 31 - __clz(NB);
  const int shift = P.lgN > lgNB ? P.lgN - lgNB : 0;
  for (int b = g.rank; b <= NB; b += G) cnt[b] = 0;
  g.sync();
  // Each warp enumerates one contiguous chunk of products in windows of 32; the run of every
  // lane comes from the run-start bitmask of the window (REDUX.OR), and the first run of the
  // next window from the current one (no search after the first window).
  constexpr int EU = 8, NW = G / 32;
  const int lane = lane_id(), w = g.rank >> 5;
  const int chunk = (f + NW * 32 - 1) / (NW * 32) * 32;
  const int jbeg = min(f, w * chunk), jend = min(f, jbeg + chunk);
  const int rb0 = jbeg < jend ? upper_idx(seg, nr, jbeg) : 0;
  // pass A: histogram of bucket sizes (columns only)
  int rb = rb0;
  for (int j0 = jbeg; j0 < jend; j0 += 32 * EU) {
    int q[EU];
#pragma unroll
    for (int u = 0; u < EU; ++u) {
      const int jw = j0 + u * 32, j = jw + lane;
      q[u] = -1;
      if (jw < jend) {
        const int r = esc2_walk(seg, nr, jw, rb);
        if (j < jend) q[u] = sbs[r] + (j - seg[r]);
      }
    }
    int kk[EU];
#pragma unroll
    for (int u = 0; u < EU; ++u) kk[u] = q[u] >= 0 ? P.colB[q[u]] : 0;
#pragma unroll
    for (int u = 0; u < EU; ++u)
      if (q[u] >= 0) atomicAdd(&cnt[kk[u] >> shift], 1);
  }
  g.sync();
  // exclusive scan of the bucket sizes (NB / G contiguous buckets per thread) -> bucket bases
  constexpr int BPT = NB / G > 0 ? NB / G : 1;
  int mine = 0, mx = 0;
  int c8[BPT];
#pragma unroll
  for (int k = 0; k < BPT; ++k) {
    const int b = g.rank * BPT + k;
    c8[k] = b < NB ? cnt[b] : 0;
    mine += c8[k];
    mx = max(mx, c8[k]);
  }
  int tot;
  int run = g.excl_scan(mine, tot);
  if (g.max(mx) > MAXB) {  // clustered columns: general kernel
    if (g.rank == 0) P.fb_list[atomicAdd(P.fb_count, 1)] = i;
    g.sync();
    return;
  }
#pragma unroll
  for (int k = 0; k < BPT; ++k) {
    const int b = g.rank * BPT + k;
    if (b < NB) cnt[b] = run;
    run += c8[k];
  }
  g.sync();
  // pass B: scatter (key, a*b) into bucket slots; afterwards cnt[b] = end of bucket b
  rb = rb0;
  for (int j0 = jbeg; j0 < jend; j0 += 32 * EU) {
    int q[EU], r[EU];
#pragma unroll
    for (int u = 0; u < EU; ++u) {
      const int jw = j0 + u * 32, j = jw + lane;
      q[u] = -1;
      r[u] = 0;
      if (jw < jend) {
        r[u] = esc2_walk(seg, nr, jw, rb);
        if (j < jend) q[u] = sbs[r[u]] + (j - seg[r[u]]);
      }
    }
    int kk[EU];
    V bb[EU];
#pragma unroll
    for (int u = 0; u < EU; ++u) {
      kk[u] = q[u] >= 0 ? P.colB[q[u]] : 0;
      bb[u] = q[u] >= 0 ? P.valB[q[u]] : V(0);
    }
#pragma unroll
    for (int u = 0; u < EU; ++u)
      if (q[u] >= 0) {
        const int d = atomicAdd(&cnt[kk[u] >> shift], 1);
        keys[d] = kk[u];
        vals[d] = sa[r[u]] * bb[u];
      }
  }
  g.sync();
  // Per product x in bucket b: x is the head of its column if no earlier slot of b holds the
  // same column (later duplicates get the sign bit); hc[b] counts the distinct columns of b.
  int* hc = sbs;  // the run table is dead after pass B
  for (int b = g.rank; b < NB; b += G) hc[b] = 0;
  g.sync();
  for (int x = g.rank; x < f; x += G) {
    const int kx = keys[x], b = kx >> shift;
    const int s0 = b ? cnt[b - 1] : 0;
    bool head = true;
    for (int y = s0; y < x; ++y)
      if ((keys[y] & 0x7fffffff) == kx) { head = false; break; }
    if (head) atomicAdd(&hc[b], 1);
    else keys[x] = kx | int(0x80000000);
  }
  g.sync();
  {  // bucket output bases (same contiguous ownership as the size scan)
    int h8[BPT], hm = 0;
#pragma unroll
    for (int k = 0; k < BPT; ++k) {
      const int b = g.rank * BPT + k;
      h8[k] = b < NB ? hc[b] : 0;
      hm += h8[k];
    }
    int ht;
    int hr = g.excl_scan(hm, ht);
#pragma unroll
    for (int k = 0; k < BPT; ++k) {
      const int b = g.rank * BPT + k;
      if (b < NB) hc[b] = hr;
      hr += h8[k];
    }
  }
  g.sync();
  // each head: output slot = bucket base + number of distinct smaller columns in the bucket;
  // value = sum of its column's products in slot order
  const long long rowoff = P.crow[i - P.row_begin];
  for (int x = g.rank; x < f; x += G) {
    const int kx = keys[x];
    if (kx < 0) continue;
    const int b = kx >> shift;
    const int s0 = b ? cnt[b - 1] : 0, s1 = cnt[b];
    int u = 0;
    V s = V(0);
    for (int y = s0; y < s1; ++y) {
      const int ky = keys[y];
      u += (ky >= 0 && ky < kx);
      if ((ky & 0x7fffffff) == kx) s += vals[y];
    }
    P.ccol[rowoff + hc[b] + u] = kx;
    P.cval[rowoff + hc[b] + u] = s;
  }
  g.sync();
}

}  // namespace spg
