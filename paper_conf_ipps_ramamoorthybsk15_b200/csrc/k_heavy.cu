// k_heavy.cu — symbolic phase of the heavy rows (the paper's A_H: "good cache blocking
// techniques can be used when multiplying A_H with B_H"): one 512- or 1024-thread
// block per row, a column-tile bitmap in shared memory.
//
// The dense accumulator of [13] Alg. 1 (PartialOutput[N] + NonZeroIndices)
// becomes a bitmap over a column tile of width Wt (TR_b of L88):
//   pass 1  every product claims its column's bit with ATOMS.OR (on sm_100a as fast as a plain
//           STS, tools/microbench_atomics.cu); the claimer that found the bit clear is the
//           column's head.  A level-1 summary bit per bitmap word keeps every later step
//           proportional to the touched words.
//   build   rank prefixes: an int per 1024 columns and a u16 per 256 columns.
//   pass 2  rank(col) = prefix + popcount of the <= 8 bitmap words below it in its 256-column
//           block; the head writes its plan word {e_rel, qoff} at Ro_i + rank (C order), every
//           other product at the end of the row's plan region (the row's dups, each with its
//           output in D at the same word).
//   c_i     = claimed bits (summed over column tiles).
// HEAVY rows (f <= 8192, one gather chunk) keep their products (column) in registers across
// the passes and their head flags in a shared bit array, and write their repeats as R records
// {B entry, A entry, output} bucketed by numeric unit at the end of the row; HUGE rows re-gather
// columns per pass, keep the flag in a global byte per product (fl8) between pass 1 and pass 2,
// and park their repeats at the end of the plan region with the outputs in D, then turn them into
// R records bucketed by numeric unit at the end of the row.  Products are
// visited in 32-product warp windows (coalesced within a B row); the run of each lane comes from
// a REDUX.OR mask of run starts.  SINGLE rows (one non-empty B row) only copy their run.
#include "kernels.cuh"

namespace spg {

constexpr int BMP_CTCAP = 2048;      // 32-product windows per chunk with a precomputed run index
constexpr int BMP_SLOTS = 8;         // products per lane cached in registers
constexpr int MODE_CACHED = 0, MODE_PLAIN = 1;

__host__ __device__ constexpr int al16(int x) { return (x + 15) & ~15; }

template <int NT>
__host__ __device__ constexpr int bmp_fixed_bytes() {
  return 3 * al16((NT + 1) * 4) + al16(BMP_CTCAP * 2);
}
constexpr int BMP_SMEM_L = 226 * 1024;  // 1024-thread blocks, one per SM (static smem on top)
constexpr int BMP_SMEM_S = 112 * 1024;  // 512-thread blocks, two per SM

// Region bytes of a 2^lw column tile: bitmap, level-1 summary (one bit per bitmap word), rank
// prefixes (int per 1024 columns, u16 per 256 columns) and — cached mode — f first-claim bits.
template <int MODE>
__device__ __forceinline__ int bmp_need(int lw, int f) {
  const int words = 1 << (lw - 5), nl1 = 1 << (lw - 10);
  int need = 4 * words + 4 * nl1 + 12 * nl1 + 16;
  if (MODE == MODE_CACHED) need += 4 * ((f + 31) >> 5) + 16;
  return need;
}

template <int MODE, int NT, int SMEM>
__global__ void __launch_bounds__(NT, SMEM > 120 * 1024 ? 1 : 2) k_bitmap_rank(SymProb P, const int* __restrict__ list,
                                                                              const int* __restrict__ count, int lwmax,
                                                                              int N) {
  constexpr int RCAP = NT;
  constexpr bool CACHED = MODE == MODE_CACHED;
  extern __shared__ __align__(16) unsigned char sm[];
  int* seg = reinterpret_cast<int*>(sm);                                   // run -> product offset
  int* sbs = reinterpret_cast<int*>(sm + al16((RCAP + 1) * 4));            // run -> B row start
  int* sae = reinterpret_cast<int*>(sm + 2 * al16((RCAP + 1) * 4));      // run -> A entry
  unsigned short* ctab = reinterpret_cast<unsigned short*>(sm + 3 * al16((RCAP + 1) * 4));  // window -> run
  unsigned char* region = sm + bmp_fixed_bytes<NT>();
  constexpr int REGION = SMEM - bmp_fixed_bytes<NT>();
  static_assert(CACHED || (DUP_SORT_UNITS + 1) * 4 <= REGION, "HUGE rows' unit counters fit the region");
  __shared__ int scratch[NT / 32 + 1];
  const Group<NT> g{(int)threadIdx.x, scratch};
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const unsigned upto = (2u << lane) - 1u;  // lanes <= me
  if (P.Ro[P.row_end - P.row_begin] > P.r_cap) return;  // plan too small: the host grows it and reruns

  // invariant between rows: the whole region is zero
  for (int x = tid; x < REGION / 4; x += NT) reinterpret_cast<unsigned*>(region)[x] = 0;
  __syncthreads();

  // Rows are taken from a dynamic queue (one atomic per row): the bin's rows differ in size by
  // up to an order of magnitude, so static striding would leave a long tail — the paper's work
  // queue in its intra-GPU form.  count[0] = rows, count[8] = queue head.
  const int n = count[0];
  // dual-ended queue: the PLAIN (HUGE) kernel is the front consumer, the 1024-thread cached
  // (HEAVY2) kernel the back consumer; the 512-thread HEAVY bin keeps its own queue
  constexpr bool FRONT = !CACHED, BACK = CACHED && NT == BMP_NT;
  const bool dual = P.dual && (FRONT || BACK);
  const int ndq = dual ? *P.dq_nh + *P.dq_n2 : 0;
  __shared__ int s_next;
  __shared__ int s_dcnt, s_single;
  __shared__ int s_uc[HEAVY_CAP / NUM_SH + 2];  // cached rows: repeats per numeric unit
  __shared__ long long s_rbase;
  for (;;) {
    if (tid == 0) {
      if (!dual) {
        const int t = atomicAdd(const_cast<int*>(count) + 8, 1);
        s_next = t < n ? list[t] : -1;
      } else {
        int li = -1;
        const int nh = *P.dq_nh;
        if (FRONT) {  // dense end: the next index nobody has claimed yet
          for (;;) {
            const int t = atomicAdd(P.dq_front, 1);
            if (t >= ndq) break;
            if (atomicMax(P.dq_claim + t, P.dq_gen) < P.dq_gen) {
              li = t < nh ? P.dq_lh[t] : P.dq_l2[t - nh];
              break;
            }
          }
        } else {  // sparse end: HEAVY2 rows only; stop where the front has been
          const int t = ndq - 1 - atomicAdd(P.dq_back, 1);
          if (t >= nh && atomicMax(P.dq_claim + t, P.dq_gen) < P.dq_gen) li = P.dq_l2[t - nh];
        }
        s_next = li;
      }
    }
    __syncthreads();
    const int li = s_next;
    __syncthreads();
    if (li < 0) break;
    const int i = P.row_begin + li;
    const int pa0 = P.rpA[i], pa1 = P.rpA[i + 1];
    const int f = P.frow[i];
    const long long ro = P.Ro[li];
    const uint8_t rc = P.cls[li];
    unsigned* prow = P.plan + ro;
    uint8_t* frow8 = P.fl8 + ro;
    const bool wide = rc & CLS_WIDE;
    // plan word(s) of output / dup position pos
    auto put = [&](int pos, int e_rel, int qoff) {
      if (wide) {
        prow[2 * (long long)pos] = (unsigned)e_rel;
        prow[2 * (long long)pos + 1] = (unsigned)qoff;
      } else {
        prow[pos] = plan_pack((unsigned)e_rel, (unsigned)qoff);
      }
    };
    // a repeated product: plan entry from the end of the region, its output o in D at the same word
    auto put_dup = [&](int o, int e_rel, int qoff) {
      const int pos = f - 1 - atomicAdd(&s_dcnt, 1);
      put(pos, e_rel, qoff);
      P.D[ro + (wide ? 2 * (long long)pos : (long long)pos)] = (unsigned)o;
    };
    if (tid == 0) s_dcnt = 0;
    if ((rc & 7) == CLS_SINGLE) {  // one non-empty B row (B canonical): output t = its entry t
      for (int p = pa0 + tid; p < pa1; p += NT)
        if (P.Tl[p] > 0) s_single = p - pa0;
      __syncthreads();
      const int er = s_single;
      for (int t2 = tid; t2 < f; t2 += NT) put(t2, er, t2);
      if (tid == 0) P.crow[li + 1] = f;
      __syncthreads();
      continue;
    }
    // Column tile: the widest whose structures (and, cached, the flag bits) fit.
    int lw = lwmax;
    while (lw > 10 && bmp_need<MODE>(lw, f) > REGION) --lw;
    const int Wt = 1 << lw, words = Wt >> 5, nl1 = 1 << (lw - 10);
    unsigned* bm = reinterpret_cast<unsigned*>(region);
    unsigned* l1 = bm + words;
    int* sbp = reinterpret_cast<int*>(l1 + nl1);                           // rank prefix / 1024 columns
    unsigned short* sbq = reinterpret_cast<unsigned short*>(sbp + nl1);   // .. / 256 columns (4 per 1024)
    unsigned* flags = reinterpret_cast<unsigned*>(sbq + 4 * nl1);
    const int nfw = CACHED ? (f + 31) >> 5 : 0;
    // HUGE rows whose products fit the region after the bitmap structures keep every product's
    // column there (filled by the first claim pass): later passes and column tiles read it instead
    // of gathering B again.  Zeroed at the end of the row (the region's zero invariant).
    int* ccache = nullptr;
    if constexpr (!CACHED) {
      const int off = (bmp_need<MODE>(lw, f) + 15) & ~15;
      if (f <= (REGION - off) / 4) ccache = reinterpret_cast<int*>(region + off);
    }
    int cmode = 0;  // for_products: 0 gather B, 1 gather B and fill ccache, 2 read ccache
    int cbase = 0;  // row product index of the current chunk's first product
    int ntiles = (int)(((long long)N + Wt - 1) >> lw);
    const int nchunks = (pa1 - pa0 + RCAP - 1) / RCAP;
    int lo0 = 0;  // first column of tile 0
    int out = 0;
    int nz = 0, Lt = 0;  // current chunk: runs, products
    int cc[BMP_SLOTS];   // cached mode: this lane's product columns
    int oo[BMP_SLOTS];   // ... and the outputs of those that repeat a column (bit s of dmask)
    unsigned dmask = 0;

    auto gather = [&](int c) {
      const int p = pa0 + c * RCAP + tid;
      const int pend = min(pa1, pa0 + (c + 1) * RCAP);
      int L = 0, bs = 0;
      if (p < pend) {
        bs = P.Tb[p];
        L = P.Tl[p];
      }
      const int rk = g.excl_scan(L > 0 ? 1 : 0, nz);
      const int off = g.excl_scan(L, Lt);  // f_i < 2^31 (checked in analysis)
      if (L > 0) {
        seg[rk] = off;
        sbs[rk] = bs;
        sae[rk] = p;
      }
      if (tid == 0) seg[nz] = Lt;
      __syncthreads();
      for (int x = tid; x < min((Lt + 31) >> 5, BMP_CTCAP); x += NT) ctab[x] = (unsigned short)upper_idx(seg, nz, x << 5);
      __syncthreads();
    };

    // product window [j0, j0+32): run of each lane (runs starting inside the window form a
    // bitmask, REDUX.OR; a lane's run = the window's first run + popcount of starts <= it)
    // B-side classes (the paper's B_H / B_L split): a window inside one
    // long B row (B_H: in a heavy row the longest B row holds ~80% of the products) is that row
    // for every lane; only windows over short B rows (B_L) pay for the run-start mask.
    auto lane_run = [&](int j0) {
      const int rb = (j0 >> 5) < BMP_CTCAP ? (int)ctab[j0 >> 5] : upper_idx(seg, nz, j0);
      if (seg[rb + 1] >= j0 + 32) return rb;  // warp-uniform
      const int rs = rb + 1 + lane;
      const int d = rs <= nz ? seg[rs] - j0 : 32;
      const unsigned M = __reduce_or_sync(FULL, (d >= 1 && d <= 31) ? (1u << d) : 0u);
      return rb + __popc(M & upto);
    };

    // Visit the products of the current chunk: fn(j, col) with j the chunk product index.
    // Cached: from the register cache.  Otherwise each warp takes 32-product windows, BATCH
    // windows' loads issued together.
    constexpr int BATCH = 4;
    auto for_products = [&](auto&& fn) {
      if constexpr (CACHED) {
#pragma unroll
        for (int s = 0; s < BMP_SLOTS; ++s) {
          const int j = warp * 32 + s * NT + lane;
          if (j < Lt) fn(j, cc[s]);
        }
      } else {
        for (int j00 = warp * 32; j00 < Lt; j00 += BATCH * NT) {
          int q[BATCH], col[BATCH];
#pragma unroll
          for (int u = 0; u < BATCH; ++u) {
            const int j0 = j00 + u * NT;
            q[u] = -1;
            if (j0 < Lt) {
              const int r = lane_run(j0);
              if (j0 + lane < Lt) q[u] = sbs[r] + (j0 + lane - seg[r]);
            }
          }
#pragma unroll
          for (int u = 0; u < BATCH; ++u)
            col[u] = q[u] < 0 ? -1 : (cmode == 2 ? ccache[cbase + j00 + u * NT + lane] : P.colB[q[u]]);
          if (cmode == 1) {
#pragma unroll
            for (int u = 0; u < BATCH; ++u)
              if (q[u] >= 0) ccache[cbase + j00 + u * NT + lane] = col[u];
          }
#pragma unroll
          for (int u = 0; u < BATCH; ++u)
            if (q[u] >= 0) fn(j00 + u * NT + lane, col[u]);
        }
      }
    };
    auto fill_cache = [&]() {
      int q[BMP_SLOTS];
#pragma unroll
      for (int s = 0; s < BMP_SLOTS; ++s) {
        const int j0 = warp * 32 + s * NT;
        q[s] = -1;
        if (j0 < Lt) {
          const int r = lane_run(j0);
          if (j0 + lane < Lt) q[s] = sbs[r] + (j0 + lane - seg[r]);
        }
      }
#pragma unroll
      for (int s = 0; s < BMP_SLOTS; ++s) cc[s] = q[s] >= 0 ? P.colB[q[s]] : -1;
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
      const int lo = lo0 + (tile << lw);
      // ---- pass 1: claim bits; first claimers flagged -----------------------------------------
      cbase = 0;
      cmode = ccache ? (tile == 0 ? 1 : 2) : 0;
      for (int c = 0; c < nchunks; ++c) {
        if (nchunks > 1 || tile == 0) {
          gather(c);
          if constexpr (CACHED) fill_cache();
        }
        if constexpr (CACHED) {
          // cached windows start at multiples of 32: one ballot word of first-claim flags each
#pragma unroll
          for (int s = 0; s < BMP_SLOTS; ++s) {
            const int j0 = warp * 32 + s * NT;
            const unsigned lc = (unsigned)(cc[s] - lo);
            bool first = false;
            if (j0 + lane < Lt && lc < (unsigned)Wt) {
              const int w = lc >> 5;
              const unsigned b = 1u << (lc & 31);
              const unsigned old = atomicOr(&bm[w], b);
              first = !(old & b);
              if (old == 0) atomicOr(&l1[w >> 5], 1u << (w & 31));
            }
            const unsigned fm = __ballot_sync(FULL, first);
            if (lane == 0 && j0 < Lt) flags[j0 >> 5] = fm;
          }
        } else {
          for_products([&](int j, int col) {
            const unsigned lc = (unsigned)(col - lo);
            if (lc < (unsigned)Wt) {
              const int w = lc >> 5;
              const unsigned b = 1u << (lc & 31);
              const unsigned old = atomicOr(&bm[w], b);
              if (old == 0) atomicOr(&l1[w >> 5], 1u << (w & 31));
              frow8[cbase + j] = (old & b) ? 0 : 1;
            }
          });
        }
        cbase += Lt;
        __syncthreads();
      }
      // ---- build: rank prefixes per 1024- and 256-column block (touched superblocks only) -----
      int pcarry = 0;
      for (int u0 = 0; u0 < nl1; u0 += NT) {
        const int u = u0 + tid;
        const unsigned x = u < nl1 ? l1[u] : 0u;
        int pc = 0;
        unsigned short q4[4] = {0, 0, 0, 0};
        if (x && __popc(x) <= 8) {
          // sparse superblock (the common case: a heavy row touches ~3 of its 32 words): count
          // the touched words only; per 256-column block a 16-bit field of one 64-bit sum
          unsigned long long acc = 0;
          for (unsigned y = x; y; y &= y - 1) {
            const int b = __ffs(y) - 1;
            acc += (unsigned long long)__popc(bm[(u << 5) + b]) << (16 * (b >> 3));
          }
          const int s0 = (int)(acc & 0xffff), s1 = (int)((acc >> 16) & 0xffff), s2 = (int)((acc >> 32) & 0xffff);
          q4[1] = (unsigned short)s0;
          q4[2] = (unsigned short)(s0 + s1);
          q4[3] = (unsigned short)(s0 + s1 + s2);
          pc = s0 + s1 + s2 + (int)(acc >> 48);
        } else if (x) {
          // dense superblock: all 32 words; the 16-byte reads are rotated by lane so a warp's
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
          q4[1] = (unsigned short)sub[0];
          q4[2] = (unsigned short)(sub[0] + sub[1]);
          q4[3] = (unsigned short)(sub[0] + sub[1] + sub[2]);
          pc = sub[0] + sub[1] + sub[2] + sub[3];
        }
        int ptot;
        const int pp = pcarry + g.excl_scan(pc, ptot);
        if (x) {  // only touched superblocks are ever queried (and cleared)
          sbp[u] = pp;
          reinterpret_cast<unsigned long long*>(sbq)[u] =
              (unsigned long long)q4[0] | ((unsigned long long)q4[1] << 16) | ((unsigned long long)q4[2] << 32) |
              ((unsigned long long)q4[3] << 48);
        }
        pcarry += ptot;
      }
      const int ctile = pcarry;
      __syncthreads();
      // ---- pass 2: ranks -> gather plan (first claimers) and dup list (the others) ---------------
      cbase = 0;
      for (int c = 0; c < nchunks; ++c) {
        if (nchunks > 1) gather(c);
        if constexpr (CACHED) {
#pragma unroll
          for (int s = 0; s < BMP_SLOTS; ++s) {
            const int j0 = warp * 32 + s * NT;
            if (j0 < Lt) {  // warp-uniform
              const int r = lane_run(j0);
              const int j = j0 + lane;
              const unsigned lc = (unsigned)(cc[s] - lo);
              const bool in = j < Lt && lc < (unsigned)Wt;
              if (in) {
                const bool first = (flags[j >> 5] >> (j & 31)) & 1u;
                const int o = out + rank_of(lc);
                if (first) {
                  put(o, sae[r] - pa0, j - seg[r]);
                } else {  // placed after the row's outputs once c_i is known (below)
                  oo[s] = o;
                  dmask |= 1u << s;
                }
              }
            }
          }
        } else {
          for (int j00 = warp * 32; j00 < Lt; j00 += BATCH * NT) {
            int q[BATCH], col[BATCH], rr[BATCH];
#pragma unroll
            for (int u = 0; u < BATCH; ++u) {
              const int j0 = j00 + u * NT;
              q[u] = -1;
              rr[u] = 0;
              if (j0 < Lt) {
                rr[u] = lane_run(j0);
                if (j0 + lane < Lt) q[u] = j0 + lane - seg[rr[u]];
              }
            }
            uint8_t fb[BATCH];
#pragma unroll
            for (int u = 0; u < BATCH; ++u) {
              col[u] = q[u] < 0 ? -1 : (ccache ? ccache[cbase + j00 + u * NT + lane] : P.colB[sbs[rr[u]] + q[u]]);
              fb[u] = q[u] >= 0 ? frow8[cbase + j00 + u * NT + lane] : 0;
            }
#pragma unroll
            for (int u = 0; u < BATCH; ++u) {
              const unsigned lc = (unsigned)(col[u] - lo);
              if (q[u] >= 0 && lc < (unsigned)Wt) {
                const int o = out + rank_of(lc);
                if (fb[u]) put(o, sae[rr[u]] - pa0, q[u]);
                else put_dup(o, sae[rr[u]] - pa0, q[u]);
              }
            }
          }
        }
        cbase += Lt;
        __syncthreads();
      }
      out += ctile;
      // ---- restore the zero invariant: touched bitmap words, summary, prefixes, flags ------------
      for (int u = tid; u < nl1; u += NT) {
        unsigned x = l1[u];
        if (x) {
          l1[u] = 0;
          sbp[u] = 0;
          reinterpret_cast<unsigned long long*>(sbq)[u] = 0ull;
          while (x) {
            const int b = __ffs(x) - 1;
            x &= x - 1;
            bm[(u << 5) + b] = 0;
          }
        }
      }
      if (CACHED)
        for (int x = tid; x < nfw; x += NT) flags[x] = 0;
      __syncthreads();
    }
    if (ccache) {  // the zero invariant of the region
      for (int x = tid; x < f; x += NT) ccache[x] = 0;
      __syncthreads();
    }
    if constexpr (CACHED) {
      if (f > out) {  // repeats after the outputs, bucketed by the numeric unit owning their output
        const int hs = (out + NUM_SH - 1) / NUM_SH;
        if (tid <= hs) s_uc[tid] = 0;
        __syncthreads();
#pragma unroll
        for (int s = 0; s < BMP_SLOTS; ++s)
          if (dmask >> s & 1u) atomicAdd(&s_uc[oo[s] / NUM_SH], 1);
        __syncthreads();
        if (tid == 0) {  // R records, first one per numeric unit in dub
          long long base = (long long)atomicAdd(reinterpret_cast<unsigned long long*>(P.dups), (unsigned long long)(f - out));
          if (base + (f - out) > P.r_dcap) base = -1;  // too small: the host grows R and reruns
          s_rbase = base;
          long long* db = P.dub + dub_index(ro, P.tscan[li] - 1);
          int run = 0;
          for (int k = 0; k < hs; ++k) {
            const int v = s_uc[k];
            s_uc[k] = run;
            db[k] = base + run;
            run += v;
          }
          db[hs] = base + run;
        }
        __syncthreads();
        const long long rbase = s_rbase;
#pragma unroll
        for (int s = 0; s < BMP_SLOTS; ++s) {
          const int j0 = warp * 32 + s * NT;
          if (j0 < Lt) {  // warp-uniform
            const int r = lane_run(j0);
            if ((dmask >> s & 1u) && rbase >= 0) {
              const int pos = atomicAdd(&s_uc[oo[s] / NUM_SH], 1);
              const int qo = j0 + lane - seg[r];
              P.R[rbase + pos] = make_int2(sbs[r] + qo, rec_meta(sae[r] - pa0, oo[s]));
            }
          }
        }
      }
    }
    if constexpr (!CACHED) {
      // HUGE rows: the repeats parked at the end of the plan region (outputs in D) become R
      // records bucketed by numeric unit — a counting sort on o / NUM_SH with the counters in the
      // (now zero) region, while the row's plan words and D are still in L2
      if (f > out) {
        const int d = f - out;
        const int hs = (out + NUM_SH - 1) / NUM_SH;
        const int sw = wide ? 2 : 1;
        int* ucnt = reinterpret_cast<int*>(region);
        const unsigned* Drow = P.D + ro;
        if (hs <= DUP_SORT_UNITS) {
          for (int j = tid; j < d; j += NT) atomicAdd(&ucnt[Drow[(long long)(out + j) * sw] / NUM_SH], 1);
          if (tid == 0) {
            long long base = (long long)atomicAdd(reinterpret_cast<unsigned long long*>(P.dups), (unsigned long long)d);
            if (base + d > P.r_dcap) base = -1;  // too small: the host grows R and reruns
            s_rbase = base;
          }
          __syncthreads();
          const long long rbase = s_rbase;
          long long* db = P.dub + dub_index(ro, P.tscan[li] - 1);
          {  // exclusive scan of the unit counters (contiguous ownership); db[k] = first record of unit k
            const int per = (hs + NT) / NT;
            int mine = 0;
            for (int x = 0; x < per; ++x) {
              const int k = tid * per + x;
              if (k < hs) mine += ucnt[k];
            }
            int tot;
            int run = g.excl_scan(mine, tot);
            for (int x = 0; x < per; ++x) {
              const int k = tid * per + x;
              if (k < hs) {
                const int v = ucnt[k];
                ucnt[k] = run;
                db[k] = rbase + run;
                run += v;
              }
            }
            if (tid == 0) db[hs] = rbase + tot;
          }
          __syncthreads();
          if (rbase >= 0)
            for (int j = tid; j < d; j += NT) {
              const long long x = (long long)(out + j) * sw;
              const unsigned o = Drow[x];
              unsigned er, qo;
              if (wide) {
                er = prow[x];
                qo = prow[x + 1];
              } else {
                const unsigned w = prow[x];
                er = w & 0xffffu;
                qo = w >> 16;
              }
              const int e = pa0 + (int)er;
              const int pos = atomicAdd(&ucnt[o / NUM_SH], 1);
              if (er >= (1u << REC_EBITS)) atomicOr(P.err, 32);  // beyond the record's A-entry field
              P.R[rbase + pos] = make_int2(P.Tb[e] + (int)qo, rec_meta((int)er, (int)o));
            }
          __syncthreads();
          for (int k = tid; k <= hs; k += NT) ucnt[k] = 0;  // the zero invariant (next row's barrier orders it)
        } else if (tid == 0) {
          atomicOr(P.err, 4);  // more numeric units than counters: the host reports NOT_SUPPORTED
        }
      }
    }
    if (tid == 0) {
      P.crow[li + 1] = out;
      if (f > out) atomicAdd(reinterpret_cast<unsigned long long*>(P.dups_all), (unsigned long long)(f - out));
    }
    __syncthreads();
  }
}

// ================================ launch glue ====================================================
static const void* bitmap_kernel(int bin) {
  switch (bin) {
    case BIN_HEAVY: return (const void*)k_bitmap_rank<MODE_CACHED, BMP_NT_S, BMP_SMEM_S>;
    case BIN_HEAVY2: return (const void*)k_bitmap_rank<MODE_CACHED, BMP_NT, BMP_SMEM_L>;
    default: return (const void*)k_bitmap_rank<MODE_PLAIN, BMP_NT, BMP_SMEM_L>;
  }
}
static int bitmap_threads(int bin) { return bin == BIN_HEAVY ? BMP_NT_S : BMP_NT; }
static int bitmap_smem(int bin) { return bin == BIN_HEAVY ? BMP_SMEM_S : BMP_SMEM_L; }

cudaError_t heavy_configure() {
  for (int bin : {BIN_HEAVY, BIN_HEAVY2, BIN_HUGE}) {
    cudaError_t e = cudaFuncSetAttribute(bitmap_kernel(bin), cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         bitmap_smem(bin));
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

int heavy_occupancy(int bin) {
  int nb = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, bitmap_kernel(bin), bitmap_threads(bin), bitmap_smem(bin));
  return nb < 1 ? 1 : nb;
}

cudaError_t launch_heavy_rank(int bin, cudaStream_t st, int grid, const SymProb& P, const int* list,
                              const int* count, long long N) {
  int lwmax = 10;
  while (lwmax < 20 && ((long long)1 << lwmax) < N) ++lwmax;
  int n32 = (int)N;
  void* args[] = {(void*)&P, (void*)&list, (void*)&count, (void*)&lwmax, (void*)&n32};
  return cudaLaunchKernel(bitmap_kernel(bin), dim3(grid), dim3(bitmap_threads(bin)), args, bitmap_smem(bin), st);
}

}  // namespace spg
