// analysis.cu — Phase I of the method: per-row intermediate-product
// counts, classification of rows into light/heavy classes (the paper's Boolean H/L array,
// generalised to a few classes and bins), the log2 flop histogram, and the scans / split
// points the symbolic phase and the multi-GPU partitioner need.
//
// No 64-bit shared-memory atomics anywhere: on sm_100a they compile to ATOMS.CAST.SPIN.64
// CAS loops that serialise under contention (hub rows, 7-way class counters).  Sums are
// pre-reduced per warp — per-row sums by a segmented warp scan (k_row_flops), class counters by
// MATCH.ANY + REDUX in 16-bit halves (k_classify) — and accumulated with native 32-bit ATOMS.
#include "kernels.cuh"

namespace spg {

// f_i = sum over stored A(i,k) of len_B(k); nz_i = #entries with len_B(k) > 0 (capped at 2), plus
// the NZ_* size flags (A row longer than 512 / 1024 / 65535 entries, a B row longer than 65535).  One block owns ROWS
// consecutive rows; its threads stride over the rows' A entries (coalesced) and find the owning row
// by binary search in the cached row_ptr tile; rows are non-decreasing across a warp's lanes, so
// a segmented warp scan (5 shuffles of one 64-bit word: products in
// the low 40 bits, non-empty runs above) leaves each row's sums in its last lane, which adds
// them into 32-bit shared accumulators.
template <int ROWS>
__global__ void __launch_bounds__(ROWS) k_row_flops(int M, const int* __restrict__ rpA, const int* __restrict__ colA,
                                                    int K, const int* __restrict__ rpB, int* __restrict__ f_out,
                                                    uint8_t* __restrict__ nz_out, int* __restrict__ Tb,
                                                    int* __restrict__ Tl, unsigned long long* __restrict__ hist,
                                                    int* __restrict__ err, int* __restrict__ amax) {
  __shared__ int s_rp[ROWS + 1];
  __shared__ unsigned s_f[ROWS];
  __shared__ int s_nz[ROWS];
  __shared__ int s_lb[ROWS];
  __shared__ unsigned s_hist[65];
  __shared__ int s_amax;
  const int t = threadIdx.x, lane = t & 31;
  const int r0 = blockIdx.x * ROWS;
  const int nr = min(ROWS, M - r0);
  if (t <= nr) s_rp[t] = rpA[r0 + t];
  if (t == 0 && nr == ROWS) s_rp[ROWS] = rpA[r0 + ROWS];
  s_f[t] = 0;
  s_nz[t] = 0;
  s_lb[t] = 0;
  if (t < 65) s_hist[t] = 0;
  if (t == 0) s_amax = 0;
  __syncthreads();
  const int e0 = s_rp[0], e1 = s_rp[nr];
  int bad = 0;
  // 64-bit loop index: base + ROWS may pass INT_MAX when nnz(A) is within ROWS of 2^31.  The
  // next iteration's column is loaded one iteration ahead (its latency overlaps this iteration's
  // B-row-pointer gathers).
  int kn = (long long)e0 + t < e1 ? __ldg(colA + e0 + t) : 0;
  for (long long base = e0; base < e1; base += ROWS) {  // uniform trip count: warp collectives below
    const int e = (int)(base + t);
    const bool act = base + t < e1;
    const int k = kn;
    kn = base + ROWS + t < e1 ? __ldg(colA + (base + ROWS + t)) : 0;
    int L = 0, r = -1;
    if (act) {
      r = upper_idx(s_rp, nr, e);
      int bs = 0;
      if ((unsigned)k >= (unsigned)K) bad |= 1;
      else { bs = rpB[k]; L = rpB[k + 1] - bs; }
      Tb[e] = bs;
      Tl[e] = L;
      if (L > 65535) atomicOr(&s_lb[r], 1);
    }
    // segmented inclusive scan over the lanes of each row (inactive lanes, r = -1, come last)
    const int rprev = __shfl_up_sync(FULL, r, 1);
    const unsigned heads = __ballot_sync(FULL, lane == 0 || r != rprev);
    const int sstart = 31 - __clz(heads & ((2u << lane) - 1u));
    unsigned long long v = act ? (unsigned long long)(unsigned)L + (L > 0 ? (1ull << 40) : 0ull) : 0ull;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const unsigned long long o = __shfl_up_sync(FULL, v, d);
      if (lane - d >= sstart) v += o;
    }
    const bool last = lane == 31 || ((heads >> (lane + 1)) & 1u);
    if (act && last) {
      const unsigned long long tot = v & ((1ull << 40) - 1);
      if (tot > (unsigned long long)INT_MAX) {
        bad |= 2;
      } else {
        const unsigned old = atomicAdd(&s_f[r], (unsigned)tot);
        if ((unsigned long long)old + tot > (unsigned long long)INT_MAX) bad |= 2;
      }
      atomicAdd(&s_nz[r], (int)(v >> 40));
    }
  }
  __syncthreads();
  if (t < nr) {
    unsigned f = s_f[t];
    if (f > (unsigned)INT_MAX) f = INT_MAX;
    f_out[r0 + t] = (int)f;
    // size flags: the A row has more entries than a 512- / 1024-thread bitmap block gathers in one
    // chunk (register-cached HEAVY kernels need single-chunk rows; TILE_EC = 1024 bounds tiles),
    // or than a 16-bit plan field holds; a referenced B row longer than 65535 (16-bit offset)
    const int alen = s_rp[t + 1] - s_rp[t];
    nz_out[r0 + t] = (uint8_t)(min(s_nz[t], 2) | (alen > BMP_NT_S ? NZ_ALEN512 : 0) | (alen > BMP_NT ? NZ_ALEN1K : 0) |
                               (alen > 65535 ? NZ_ALEN64K : 0) | (s_lb[t] ? NZ_LONGB : 0));
    const int b = f == 0 ? 0 : 1 + (f == 1 ? 0 : 32 - __clz((int)f - 1));
    atomicAdd(&s_hist[b], 1u);
    atomicMax(&s_amax, alen);
  }
  if (bad) atomicOr(err, bad);
  __syncthreads();
  if (t < 65 && s_hist[t]) atomicAdd(&hist[t], (unsigned long long)s_hist[t]);
  if (t == 0) atomicMax(amax, s_amax);
}

// Row path.  Returns the class (CLS_*); heavy: the row is an item of its own on the bitmap path
// (bin = its bitmap bin), else it belongs to a tile.
static_assert(TILE_EC == BMP_NT, "NZ_ALEN1K marks rows too long for a tile");
__device__ __forceinline__ int classify_row(int f, int nz, const ClassParams& p, int& bin, bool& heavy) {
  bin = -1;
  heavy = false;
  if (f == 0) return CLS_EMPTY;
  const bool long1 = nz & NZ_ALEN512, long2 = nz & NZ_ALEN1K;
  const int runs = nz & 3;
  int c;
  if (p.force < 0 && runs == 1 && p.single_ok) {
    c = CLS_SINGLE;  // one non-empty B row: c_i = f_i, no sort
    if (f <= p.light_max && !long2) return c;
  } else {
    if (f <= p.light_max && p.force < CLS_HEAVY && !long2)
      return f <= TINY_MAX ? CLS_TINY : (f <= LIGHTC_MAX ? CLS_LIGHT : CLS_MEDIUM);
    c = -1;
  }
  heavy = true;
  const int hm = min(p.heavy_max, HEAVY_CAP);
  if (c == CLS_SINGLE || p.force == CLS_HUGE || f > hm) bin = BIN_HUGE;
  else if (f <= HEAVY1_CAP && !long1) bin = BIN_HEAVY;
  else if (!long2) bin = BIN_HEAVY2;
  else bin = BIN_HUGE;
  return c >= 0 ? c : (bin == BIN_HUGE ? CLS_HUGE : CLS_HEAVY);
}

// Classify this rank's rows [rb, re) (local index li = i - rb): cls[li] = class | path flags;
// pw[li] = plan words of the row (f_i, 2 f_i for wide heavy rows; scanned into Ro).  Heavy rows
// are appended to their bitmap bin's list.  Per-class statistics are pre-reduced per warp
// (MATCH.ANY + REDUX, 16-bit halves) and flushed once per block.
constexpr int CL_NT = 256;

__global__ void __launch_bounds__(CL_NT) k_classify(const int* __restrict__ f, const uint8_t* __restrict__ nz, int rb,
                                                    int re, ClassParams prm, uint8_t* __restrict__ cls,
                                                    int* __restrict__ pw, HeavyLists lists, Small* __restrict__ sm) {
  __shared__ unsigned s_rows[NUM_CLS], s_flo[NUM_CLS], s_fhi[NUM_CLS], s_fmax;
  const int tid = threadIdx.x, lane = tid & 31;
  if (tid < NUM_CLS) { s_rows[tid] = 0; s_flo[tid] = 0; s_fhi[tid] = 0; }
  if (tid == 0) s_fmax = 0;
  __syncthreads();
  const long long n = (long long)re - rb;
  const long long nup = (n + 31) & ~31LL;  // warp-uniform trip count
  int bad = 0;
  for (long long li = (long long)blockIdx.x * CL_NT + tid; li < nup; li += (long long)gridDim.x * CL_NT) {
    const bool act = li < n;
    int fi = 0, bin = -1, c = -1;
    bool heavy = false;
    if (act) {
      fi = f[rb + li];
      const int z = nz[rb + li];
      c = classify_row(fi, z, prm, bin, heavy);
      const bool wide = heavy && (z & (NZ_LONGB | NZ_ALEN64K));
      const bool solo = !heavy && (fi > TILE_PMAX - prm.tile_cap || (z & NZ_ALEN1K));
      cls[li] = (uint8_t)(c | (heavy ? CLS_HEAVY_PATH : 0) | (wide ? CLS_WIDE : 0) | (solo ? CLS_SOLO : 0));
      if (wide && fi >= (1 << 30)) bad = 2;
      pw[li] = wide ? 2 * fi : fi;
    }
    const unsigned gc = __match_any_sync(FULL, c);
    if (act) {
      const unsigned lo = __reduce_add_sync(gc, (unsigned)fi & 0xffffu);
      const unsigned hi = __reduce_add_sync(gc, (unsigned)fi >> 16);
      if (lane == __ffs(gc) - 1) {
        atomicAdd(&s_rows[c], (unsigned)__popc(gc));
        atomicAdd(&s_flo[c], lo);
        atomicAdd(&s_fhi[c], hi);
      }
    }
    const unsigned fm = __reduce_max_sync(FULL, (unsigned)fi);
    if (lane == 0 && fm) atomicMax(&s_fmax, fm);
    // heavy rows: list append (rare: one warp-level atomic per bin when present)
    if (__ballot_sync(FULL, bin >= 0)) {
      const unsigned gb = __match_any_sync(FULL, bin);
      if (bin >= 0) {
        const int leader = __ffs(gb) - 1;
        int pos = 0;
        if (lane == leader) pos = atomicAdd(&sm->counts[bin], __popc(gb));
        pos = __shfl_sync(gb, pos, leader) + __popc(gb & lanemask_lt());
        lists.rows[bin][pos] = (int)li;
      }
    }
  }
  if (bad) atomicOr(&sm->err, bad);
  __syncthreads();
  if (tid < NUM_CLS) {
    const unsigned long long fl2 = ((unsigned long long)s_fhi[tid] << 16) + s_flo[tid];
    if (s_rows[tid]) atomicAdd(&sm->cstats[tid], (unsigned long long)s_rows[tid]);
    if (fl2) atomicAdd(&sm->cstats[NUM_CLS + tid], fl2);
  }
  if (tid == 0 && s_fmax) atomicMax(&sm->cstats[2 * NUM_CLS], (unsigned long long)s_fmax);
}

// Item starts.  A heavy row is an item; a non-heavy row starts a tile when the row before it is
// heavy or solo, when it is solo itself, when its index is a multiple of TILE_RM, or when its plan
// range [Ro_i, Ro_i + f_i) contains a multiple of `cap` or its A entry range a multiple of TILE_EC.
// So a tile holds <= TILE_RM rows, < cap + f_first <= TILE_PMAX products and < 2 TILE_EC A
// entries (rows longer than TILE_EC are heavy, or solo when f = 0).
__global__ void __launch_bounds__(256) k_tile_flags(const int* __restrict__ f, const int* __restrict__ rpA, int rb,
                                                    int re, int cap, const uint8_t* __restrict__ cls,
                                                    const long long* __restrict__ Ro, int* __restrict__ tflag) {
  const long long n = (long long)re - rb;
  for (long long li = (long long)blockIdx.x * blockDim.x + threadIdx.x; li < n; li += (long long)gridDim.x * blockDim.x) {
    // every load issued up front (independent), then the tests
    const int c = cls[li];
    const int cp = li > 0 ? cls[li - 1] : 0;
    const long long fi = f[rb + li];
    const long long pl = Ro[li];
    const long long ea = rpA[rb + li], al = rpA[rb + li + 1] - ea;
    bool start = (c & CLS_HEAVY_PATH) || (c & CLS_SOLO) || li == 0 || (li % TILE_RM) == 0 ||
                 (cp & CLS_HEAVY_PATH) || (cp & CLS_SOLO);
    if (fi > 0) start = start || (pl % cap == 0) || (pl / cap != (pl + fi - 1) / cap);
    if (al > 0) start = start || (ea % TILE_EC == 0) || (ea / TILE_EC != (ea + al - 1) / TILE_EC);
    tflag[li] = start ? 1 : 0;
  }
}

// items[k] = the k-th item start (tscan = inclusive scan of the start flags); items[n] = Mloc.
__global__ void __launch_bounds__(256) k_items(const int* __restrict__ tflag, const long long* __restrict__ tscan,
                                               int mloc, int* __restrict__ items, Small* __restrict__ sm) {
  for (long long li = (long long)blockIdx.x * blockDim.x + threadIdx.x; li < mloc; li += (long long)gridDim.x * blockDim.x)
    if (tflag[li]) items[tscan[li] - 1] = (int)li;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    const int n = mloc > 0 ? (int)tscan[mloc - 1] : 0;
    items[n] = mloc;
    sm->nitems = n;
  }
}

// Numeric work units per item t: ceil(c_t / NUM_SH).
__global__ void __launch_bounds__(256) k_unit_count(const int* __restrict__ items, const long long* __restrict__ crow,
                                                    int n, int* __restrict__ ucnt) {
  for (long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x; t < n; t += (long long)gridDim.x * blockDim.x)
    ucnt[t] = (int)((crow[items[t + 1]] - crow[items[t]] + NUM_SH - 1) / NUM_SH);
}

__global__ void __launch_bounds__(256) k_unit_fill(const int* __restrict__ ucnt, const long long* __restrict__ uscan,
                                                   int n, NumUnit* __restrict__ units, Small* __restrict__ sm,
                                                   const int* __restrict__ items, const long long* __restrict__ crow,
                                                   const long long* __restrict__ Ro, const uint8_t* __restrict__ cls,
                                                   const int* __restrict__ rpA, int rb,
                                                   const long long* __restrict__ dub) {
  for (long long t = (long long)blockIdx.x * blockDim.x + threadIdx.x; t < n; t += (long long)gridDim.x * blockDim.x) {
    const int u = ucnt[t];
    const long long b = uscan[t] - u;
    const int r = items[t], r2 = items[t + 1];
    const long long o0 = crow[r], c = crow[r2] - o0, P0 = Ro[r];
    const bool wide = (cls[r] & CLS_HEAVY_PATH) && (cls[r] & CLS_WIDE);
    const int sw = wide ? 2 : 1;
    const long long f = (Ro[r2] - P0) / sw;
    const int e0 = rpA[rb + r];
    const long long* db = dub + dub_index(P0, t);
    const bool rep = f > c;
    for (int k = 0; k < u; ++k) {
      NumUnit v;
      v.pw = P0 + (long long)k * NUM_SH * sw;
      v.oc = o0 + (long long)k * NUM_SH;
      v.dw = rep ? db[k] : 0;
      v.d = rep ? (int)(db[k + 1] - db[k]) : 0;
      v.n = (int)min((long long)NUM_SH, c - (long long)k * NUM_SH);
      v.e0 = e0;
      v.ob = k * NUM_SH | (wide ? UNIT_WIDE : 0);
      units[b + k] = v;
    }
  }
  if (blockIdx.x == 0 && threadIdx.x == 0) sm->nunits = n > 0 ? uscan[n - 1] : 0;
}

// ---- inclusive scan to int64: one pass with decoupled look-back ----------------------------------
// Tiles of SCAN_TILE elements take their index from a counter in launch order; a tile publishes
// its aggregate (flag A), then — once its predecessors' prefix is known — its inclusive prefix
// (flag P), each as one 64-bit word {flag:2, value:62}.  Warp 0 of a tile looks back over the
// 32 preceding words at a time: it stops at the nearest P, summing the A values in between.  A
// tile only waits on tiles with smaller indices, which were started before it, so the scan
// cannot deadlock.  In place is allowed (a tile reads its whole input before writing).
constexpr int SCAN_NT = 256, SCAN_IPT = 8, SCAN_TILE = SCAN_NT * SCAN_IPT;
constexpr unsigned long long SCAN_FA = 1ull << 62, SCAN_FP = 2ull << 62, SCAN_VAL = SCAN_FA - 1;

template <typename Tin>
__global__ void __launch_bounds__(SCAN_NT) k_scan_lb(const Tin* __restrict__ in, long long* __restrict__ out,
                                                     long long n, unsigned long long* __restrict__ st,
                                                     int* __restrict__ ctr) {
  __shared__ long long s_w[SCAN_NT / 32];
  __shared__ long long s_pre;
  __shared__ int s_tile;
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) s_tile = atomicAdd(ctr, 1);
  __syncthreads();
  const int tile = s_tile;
  const long long base = (long long)tile * SCAN_TILE + (long long)threadIdx.x * SCAN_IPT;
  long long v[SCAN_IPT];
  long long run = 0;
#pragma unroll
  for (int k = 0; k < SCAN_IPT; ++k) {
    const long long x = base + k < n ? (long long)in[base + k] : 0;
    run += x;
    v[k] = run;
  }
  const long long incl = warp_incl_scan(run);
  if (lane == 31) s_w[w] = incl;
  __syncthreads();
  if (w == 0) {
    const long long x = lane < SCAN_NT / 32 ? s_w[lane] : 0;
    const long long xi = warp_incl_scan(x);
    if (lane < SCAN_NT / 32) s_w[lane] = xi - x;
    const long long agg = __shfl_sync(FULL, xi, SCAN_NT / 32 - 1);
    volatile unsigned long long* vst = st;
    if (tile == 0) {
      if (lane == 0) {
        vst[0] = SCAN_FP | (unsigned long long)agg;
        s_pre = 0;
      }
    } else {
      if (lane == 0) vst[tile] = SCAN_FA | (unsigned long long)agg;
      long long pre = 0;
      int p = tile - 1;  // lane k inspects tile p - k
      for (;;) {
        unsigned long long wd = SCAN_FP;  // below tile 0: a zero prefix
        if (p - lane >= 0) {
          do { wd = vst[p - lane]; } while ((wd >> 62) == 0);
        }
        const unsigned pm = __ballot_sync(FULL, (wd & SCAN_FP) != 0);
        // the nearest P (lowest lane) ends the look-back; 64-bit sum of the lanes up to it
        const int stop = pm ? __ffs(pm) - 1 : 31;
        long long val = lane <= stop ? (long long)(wd & SCAN_VAL) : 0;
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) val += __shfl_xor_sync(FULL, val, d);
        pre += val;
        if (pm) break;
        p -= 32;
      }
      if (lane == 0) {
        vst[tile] = SCAN_FP | (unsigned long long)(pre + agg);
        s_pre = pre;
      }
    }
  }
  __syncthreads();
  const long long off = incl - run + s_w[w] + s_pre;
#pragma unroll
  for (int k = 0; k < SCAN_IPT; ++k)
    if (base + k < n) out[base + k] = v[k] + off;
}

// s_0 = 0, s_P = M, s_r = min{ i : Pf[i]*P >= r*F }.  Pf = int64[M+1].
__global__ void k_split_points(const long long* __restrict__ Pf, int M, int P, int* __restrict__ s) {
  const int r = threadIdx.x + blockIdx.x * blockDim.x;
  if (r > P) return;
  if (r == 0) { s[0] = 0; return; }
  if (r == P) { s[P] = M; return; }
  const __int128 F = Pf[M];
  const __int128 target = (__int128)r * F;
  int lo = 0, hi = M;  // smallest i in [0, M] with Pf[i]*P >= target (Pf[M]*P >= target holds)
  while (lo < hi) {
    int mid = lo + ((hi - lo) >> 1);
    if ((__int128)Pf[mid] * P >= target) hi = mid; else lo = mid + 1;
  }
  s[r] = lo;
}

// SPG_OPT_VALIDATE: err |= 4 malformed row_ptr, 8 column out of range, 16 row not strictly ascending.
__global__ void k_validate(int M, const int* __restrict__ rp, const int* __restrict__ ci, int ncols, long long nnz,
                           int check_sorted, int* __restrict__ err) {
  int bad = 0;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < M; i += (long long)gridDim.x * blockDim.x) {
    const int s = rp[i], e = rp[i + 1];
    if (s > e || s < 0 || (long long)e > nnz) { bad |= 4; continue; }
    if (i == 0 && s != 0) bad |= 4;
    if (i == M - 1 && (long long)e != nnz) bad |= 4;
    int prev = -1;
    for (int p = s; p < e; ++p) {
      const int c = ci[p];
      if (c < 0 || c >= ncols) bad |= 8;
      if (check_sorted && c <= prev) bad |= 16;
      prev = c;
    }
  }
  if (M == 0 && nnz != 0 && blockIdx.x == 0 && threadIdx.x == 0) bad |= 4;
  if (bad) atomicOr(err, bad);
}

// row_ptr_full[i] += off[r] for the rank r owning row i; row_ptr_full[M] = off[P].
__global__ void k_rebase(long long* __restrict__ rp, int M, int P, const int* __restrict__ sp,
                         const long long* __restrict__ off) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i <= M; i += (long long)gridDim.x * blockDim.x) {
    if (i == M) { rp[M] = off[P]; continue; }
    int lo = 0, hi = P - 1;  // largest r with sp[r] <= i
    while (lo < hi) { int mid = (lo + hi + 1) >> 1; if (sp[mid] <= i) lo = mid; else hi = mid - 1; }
    rp[i] += off[lo];
  }
}

// Scatter of A's row blocks: rp[i] -= rp[0] (a received block's row offsets start at 0), and the
// per-rank row / entry counts of a split: out[r] = s[r+1]-s[r], out[P+r] = rpA[s[r+1]]-rpA[s[r]].
__global__ void k_rebase32(int* __restrict__ rp, long long n, const int* __restrict__ first) {
  const int b = *first;
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    rp[i] -= b;
}
__global__ void k_split_sizes(const int* __restrict__ s, const int* __restrict__ rpA, int P, long long* __restrict__ out) {
  for (int r = threadIdx.x; r < P; r += blockDim.x) {
    out[r] = s[r + 1] - s[r];
    out[P + r] = (long long)rpA[s[r + 1]] - rpA[s[r]];
    out[2 * P + r] = rpA[s[r]];
  }
}

// Canonicalisation helpers (SPG_OPT_INPUT_CANONICAL = 0): iota, constant fill, narrowing copy.
__global__ void k_iota(int* __restrict__ p, long long n) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    p[i] = (int)i;
}
template <typename V>
__global__ void k_fill(V* __restrict__ p, long long n, V v) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    p[i] = v;
}
__global__ void k_narrow(const long long* __restrict__ in, int* __restrict__ out, long long n) {
  for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x)
    out[i] = (int)in[i];
}

// ---- host launchers ------------------------------------------------------------------------
cudaError_t launch_row_flops(cudaStream_t st, int M, const int* rpA, const int* colA, int K, const int* rpB,
                             int* f, uint8_t* nz, int* Tb, int* Tl, unsigned long long* hist, int* err, int* amax) {
  if (M <= 0) return cudaSuccess;
  constexpr int ROWS = 256;
  k_row_flops<ROWS><<<(M + ROWS - 1) / ROWS, ROWS, 0, st>>>(M, rpA, colA, K, rpB, f, nz, Tb, Tl, hist, err, amax);
  return cudaGetLastError();
}

cudaError_t launch_classify(cudaStream_t st, int sms, const int* f, const uint8_t* nz, int rb, int re,
                            const ClassParams& prm, uint8_t* cls, int* pw, const HeavyLists& lists, Small* small) {
  const long long n = (long long)re - rb;
  if (n <= 0) return cudaSuccess;
  long long blocks = (n + CL_NT - 1) / CL_NT;
  if (blocks > (long long)sms * 8) blocks = (long long)sms * 8;
  k_classify<<<(int)blocks, CL_NT, 0, st>>>(f, nz, rb, re, prm, cls, pw, lists, small);
  return cudaGetLastError();
}

static int grid_for_rows(long long n, int sms) {
  long long g = (n + 255) / 256;
  if (g > (long long)sms * 8) g = (long long)sms * 8;
  return (int)(g < 1 ? 1 : g);
}

cudaError_t launch_tile_flags(cudaStream_t st, int sms, const int* f, const int* rpA, int rb, int re, int tile_cap,
                              const uint8_t* cls, const long long* Ro, int* tflag) {
  const long long n = (long long)re - rb;
  if (n <= 0) return cudaSuccess;
  k_tile_flags<<<grid_for_rows(n, sms), 256, 0, st>>>(f, rpA, rb, re, tile_cap, cls, Ro, tflag);
  return cudaGetLastError();
}

cudaError_t launch_unit_count(cudaStream_t st, int sms, const int* items, const long long* crow, int n, int* ucnt) {
  if (n <= 0) return cudaSuccess;
  k_unit_count<<<grid_for_rows(n, sms), 256, 0, st>>>(items, crow, n, ucnt);
  return cudaGetLastError();
}

cudaError_t launch_unit_fill(cudaStream_t st, int sms, const int* ucnt, const long long* uscan, int n,
                             NumUnit* units, Small* small, const int* items, const long long* crow,
                             const long long* Ro, const uint8_t* cls, const int* rpA, int rb, const long long* dub) {
  k_unit_fill<<<grid_for_rows(n, sms), 256, 0, st>>>(ucnt, uscan, n, units, small, items, crow, Ro, cls, rpA, rb,
                                                     dub);
  return cudaGetLastError();
}

cudaError_t launch_items(cudaStream_t st, int sms, const int* tflag, const long long* tscan, int mloc, int* items,
                         Small* small) {
  k_items<<<grid_for_rows(mloc, sms), 256, 0, st>>>(tflag, tscan, mloc, items, small);
  return cudaGetLastError();
}

// Largest rows first: a bitmap bin's row list is put in descending f_i order (approximately: 8
// classes per octave, order inside a class arbitrary — a one-block counting sort, the rows held
// in shared memory when they fit, else through a scratch copy).  Launched on the bin's own
// stream, just before its kernel.  The bins' blocks take rows from a dynamic queue, so this is
// longest-processing-time-first scheduling: the biggest HUGE rows (up to ~9x the bin average on
// webbase1m) start first instead of forming the kernel's tail.
constexpr int ORD_NT = 1024, ORD_CAP = 4096, ORD_KEYS = 256;
__global__ void __launch_bounds__(ORD_NT) k_order_list(HeavyLists lists, int b, const int* __restrict__ f, int rb,
                                                      const Small* __restrict__ sm, int* __restrict__ tmp) {
  __shared__ int hist[ORD_KEYS];
  __shared__ int s_li[ORD_CAP];
  const int n = sm->counts[b];
  if (n <= 1) return;
  int* list = lists.rows[b];
  const bool insm = n <= ORD_CAP;
  const int tid = threadIdx.x;
  if (tid < ORD_KEYS) hist[tid] = 0;
  __syncthreads();
  auto key = [&](int li) {  // ascending key = descending f: exponent and 3 bits below the leading one
    const unsigned v = (unsigned)max(f[rb + li], 1);
    const int ex = 31 - __clz(v);
    const unsigned m = ex >= 3 ? (v >> (ex - 3)) & 7u : (v << (3 - ex)) & 7u;
    return ORD_KEYS - 1 - (ex * 8 + (int)m);
  };
  for (int x = tid; x < n; x += ORD_NT) {
    const int li = list[x];
    if (insm) s_li[x] = li;
    atomicAdd(&hist[key(li)], 1);
  }
  __syncthreads();
  if (tid < 32) {  // exclusive scan of the counters: 8 per lane
    int c[ORD_KEYS / 32], sum = 0;
#pragma unroll
    for (int k = 0; k < ORD_KEYS / 32; ++k) {
      c[k] = hist[tid * (ORD_KEYS / 32) + k];
      sum += c[k];
    }
    int run = warp_incl_scan(sum) - sum;
#pragma unroll
    for (int k = 0; k < ORD_KEYS / 32; ++k) {
      hist[tid * (ORD_KEYS / 32) + k] = run;
      run += c[k];
    }
  }
  __syncthreads();
  for (int x = tid; x < n; x += ORD_NT) {
    const int li = insm ? s_li[x] : list[x];
    const int pos = atomicAdd(&hist[key(li)], 1);
    if (insm) list[pos] = li;
    else tmp[pos] = li;
  }
  if (insm) return;
  __syncthreads();
  for (int x = tid; x < n; x += ORD_NT) list[x] = tmp[x];
}

cudaError_t launch_sort_list(cudaStream_t st, const HeavyLists& lists, int bin, const int* f, int rb,
                             const Small* small, int* tmp) {
  k_order_list<<<1, ORD_NT, 0, st>>>(lists, bin, f, rb, small, tmp);
  return cudaGetLastError();
}

size_t scan_tmp_elems(long long n) { return (size_t)((n + SCAN_TILE - 1) / SCAN_TILE) + 2; }
int scan_launches(long long n) { return n <= 0 ? 0 : 1; }

// tmp: scan_tmp_elems(n) words — the tiles' status words, then the tile counter
template <typename Tin>
cudaError_t launch_incl_scan(cudaStream_t st, const Tin* in, long long* out, long long n, long long* tmp) {
  if (n <= 0) return cudaSuccess;
  const int ntiles = (int)((n + SCAN_TILE - 1) / SCAN_TILE);
  cudaError_t e = cudaMemsetAsync(tmp, 0, (size_t)(ntiles + 1) * sizeof(long long), st);
  if (e != cudaSuccess) return e;
  k_scan_lb<Tin><<<ntiles, SCAN_NT, 0, st>>>(in, out, n, reinterpret_cast<unsigned long long*>(tmp),
                                            reinterpret_cast<int*>(tmp + ntiles));
  return cudaGetLastError();
}
template cudaError_t launch_incl_scan<int>(cudaStream_t, const int*, long long*, long long, long long*);
template cudaError_t launch_incl_scan<long long>(cudaStream_t, const long long*, long long*, long long, long long*);

cudaError_t launch_validate(cudaStream_t st, int sms, int M, const int* rp, const int* ci, int ncols, long long nnz,
                            int check_sorted, int* err) {
  int grid = (M + 255) / 256;
  if (grid > sms * 8) grid = sms * 8;
  if (grid < 1) grid = 1;
  k_validate<<<grid, 256, 0, st>>>(M, rp, ci, ncols, nnz, check_sorted, err);
  return cudaGetLastError();
}

cudaError_t launch_rebase(cudaStream_t st, long long* rp_full, int M, int P, const int* splits, const long long* off) {
  int grid = (M + 1 + 255) / 256;
  if (grid > 4096) grid = 4096;
  k_rebase<<<grid, 256, 0, st>>>(rp_full, M, P, splits, off);
  return cudaGetLastError();
}

static int grid_for(long long n) { long long g = (n + 255) / 256; return (int)(g < 1 ? 1 : (g > 4096 ? 4096 : g)); }
cudaError_t launch_rebase32(cudaStream_t st, int* rp, long long n, const int* first) {
  if (n > 0) k_rebase32<<<grid_for(n), 256, 0, st>>>(rp, n, first);
  return cudaGetLastError();
}
cudaError_t launch_split_sizes(cudaStream_t st, const int* s, const int* rpA, int P, long long* out) {
  k_split_sizes<<<1, 256, 0, st>>>(s, rpA, P, out);
  return cudaGetLastError();
}
cudaError_t launch_iota(cudaStream_t st, int* p, long long n) {
  if (n > 0) k_iota<<<grid_for(n), 256, 0, st>>>(p, n);
  return cudaGetLastError();
}
template <typename V>
cudaError_t launch_fill(cudaStream_t st, V* p, long long n, V v) {
  if (n > 0) k_fill<V><<<grid_for(n), 256, 0, st>>>(p, n, v);
  return cudaGetLastError();
}
template cudaError_t launch_fill<double>(cudaStream_t, double*, long long, double);
template cudaError_t launch_fill<float>(cudaStream_t, float*, long long, float);
cudaError_t launch_narrow(cudaStream_t st, const long long* in, int* out, long long n) {
  if (n > 0) k_narrow<<<grid_for(n), 256, 0, st>>>(in, out, n);
  return cudaGetLastError();
}

cudaError_t launch_split_points(cudaStream_t st, const long long* Pf, int M, int P, int* s) {
  k_split_points<<<(P + 1 + 127) / 128, 128, 0, st>>>(Pf, M, P, s);
  return cudaGetLastError();
}

}  // namespace spg
