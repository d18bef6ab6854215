// k_light.cu — symbolic phase of the tiles: runs of consecutive non-heavy rows (the paper's A_L,
// "numerous subproblems of small computational intensity"), many rows per block.
//
// A tile is an item of the ordered item list (k_tile_flags / k_items): <= TILE_RM consecutive
// rows, < TILE_PMAX products, < 2 TILE_EC A entries.  A block takes BATCH_NI consecutive items
// from a dynamic queue and packs the tiles among them (heavy rows are skipped: k_bitmap_rank)
// into batches of <= TILE_PMAX products and <= BATCH_RM rows, so a batch holds ~3-4k products
// even where heavy rows cut the tiles short.  It sorts all products of a batch at once with one
// bucketed counting sort, so the per-row cost of a row-per-warp design (barriers, scans, idle
// lanes) is paid once per batch instead:
//
//   1. rows      per row its tile, first A entry and product count; block scans give the batch's
//                A-entry and product offsets of every row.
//   2. expand    every product's column and plan word {e_rel, qoff} go to shared memory
//                (coalesced B-row loads; the run of each lane from a REDUX.OR run-start mask).
//                Each light row's column range [cmin, cmax] comes from the first and last entry
//                of its (sorted) B rows.
//   3. buckets   light row j gets NB_j = min(ceil(f_j / TILE_BK), range) equal buckets over its own
//                column range: bucket order is (row, column) order; sizes by ATOMS.ADD.
//   4. scatter   exclusive scan of the sizes; each product is placed in its bucket.
//   5. heads     a product is the head of its column when no earlier slot of its bucket holds the
//                same column; heads are counted per bucket and scanned; c_j = heads of the row.
//   6. offsets   block scan of c_j: the output offset of every row inside its tile.
//   7. ranks     rank = heads of the row's earlier buckets + distinct smaller columns in the own
//                bucket; a head writes its plan word at P0_tile + out_j + rank (C order), every
//                other product (a repeat) an R record {B entry, A entry, output out_j + rank},
//                bucketed by the numeric unit that owns that output.  SINGLE rows (one non-empty
//                B row, already sorted) write their products in order.
// This is Phase IV's "sort, mark like-tuples, scan, compact", done per batch
// in shared memory.  Every block scan here is followed by a barrier of its own before the next
// one, so the scans skip their closing barrier (excl_scan<false>).
#include "kernels.cuh"

namespace spg {

// Two instances of the kernel: tiles (batches of <= 4096 products, 512 threads, two blocks per SM)
// popped from the item list, and "big tiles" (<= 8192 products, 1024 threads, one block per SM)
// that sort the register-cached heavy rows (f <= 8192) popped from their bin lists — instead of
// the column bitmap, whose per-row cost grows with the column count (SPG_OPT_HEAVY_SORT).
template <int PMAX_, int NT_, bool LIST_>
struct TileCfg {
  static constexpr int PMAX = PMAX_;   // products per batch
  static constexpr int NT = NT_;       // threads
  static constexpr bool LIST = LIST_;  // pop heavy rows from the bin lists (else items)
  static constexpr int RM = NT_ < 512 ? NT_ : 512;  // rows per batch
  static constexpr int NI = 16;        // items per queue pop
  static constexpr int NB = PMAX / TILE_BK + RM;  // buckets per batch (ceil per row)
  static constexpr int NU = NI + PMAX / NUM_SH;   // numeric units of a batch's items
  static_assert(PMAX / NT <= 32, "head marks of a thread fit one 32-bit mask");
  static_assert(RM <= NT, "one row per thread in the row phases");
  static_assert(TILE_RM <= RM, "a tile fits a batch");
};
using TileSmall = TileCfg<TILE_PMAX, TILE_NT, false>;
using TileBig = TileCfg<HEAVY_CAP, 1024, true>;
constexpr int TILE_EU = 4;  // 32-product windows per warp per step (loads in flight)

// Run of product jw + lane for a window starting inside run rb (warp-uniform); advances rb to
// the run holding jw + 32.  All 32 lanes must call.  (No B_H fast path here: light rows' B rows
// are short, and the extra check measured -1.5% on citpatents / webgoogle / ab2m.)
__device__ __forceinline__ int walk_run(const int* seg, int nr, int jw, int& rb) {
  const int lane = lane_id();
  const int rs = rb + 1 + lane;
  const int d = rs <= nr ? seg[rs] - jw : 64;
  const unsigned M = __reduce_or_sync(FULL, (d >= 1 && d <= 31) ? (1u << d) : 0u);
  const int r = rb + __popc(M & ((2u << lane) - 1u));
  rb += __popc(M) + (__ballot_sync(FULL, d == 32) != 0u);
  return r;
}

// Shared-memory layout of one tile block (bytes).
template <class C>
struct TileSmem {
  static constexpr int keys = 0;                                    // int[PMAX]   idx -> column (expand), then
                                                                    //             slot -> column (sign: not head)
  static constexpr int pay = keys + C::PMAX * 4;                  // u32[PMAX]   idx -> plan word
  static constexpr int sidx = pay + C::PMAX * 4;                  // u16[PMAX]   slot -> product index
  static constexpr int sbk = sidx + C::PMAX * 2;                  // u16[PMAX]   slot -> bucket (repeats: output)
  static constexpr int exrow = sbk + C::PMAX * 2;                 // u16[PMAX]   idx -> batch row
  static constexpr int cnt = exrow + C::PMAX * 2;                 // int[NB+1]   sizes -> starts -> ends
  static constexpr int ae = (cnt + (C::NB + 1) * 4 + 15) & ~15;  // int[RM+1]   A-entry offset of the row
  static constexpr int pf = ae + (C::RM + 1) * 4;                // int[RM+1]   product offset of the row
  static constexpr int bb = pf + (C::RM + 1) * 4;                // int[RM+1]   bucket base
  static constexpr int out = bb + (C::RM + 1) * 4;               // int[RM+1]   output offset in the batch
  static constexpr int sf = out + (C::RM + 1) * 4;               // int[RM+1]   SINGLE-row products before the row
  static constexpr int rpa = sf + (C::RM + 1) * 4;               // int[RM]     first A entry of the row
  static constexpr int row = rpa + C::RM * 4;                    // int[RM]     local row index
  static constexpr int cmin = row + C::RM * 4;                   // int[RM]     column range of the row (later:
                                                                  //             heads before the row)
  static constexpr int cmax = cmin + C::RM * 4;                  // int[RM]
  static constexpr int mul = cmax + C::RM * 4;                   // u32[RM]     bucket scale (0: one column each)
  static constexpr int kind = mul + C::RM * 4;                   // u8[RM]      class of the row
  static constexpr int item = kind + C::RM;                      // u8[RM]      tile of the row (in the batch)
  static constexpr int seg = (item + C::RM + 15) & ~15;          // int[NT+1]   chunk run -> product offset
  static constexpr int sbs = seg + (C::NT + 1) * 4;               // int[NT]     chunk run -> B row start
  static constexpr int sae = sbs + C::NT * 4;                     // int[NT]     chunk run -> tile A entry
  static constexpr int srw = sae + C::NT * 4;                     // u16[NT]     chunk run -> batch row
  static constexpr int bytes = (srw + C::NT * 2 + 15) & ~15;
};

template <class C>
__global__ void __launch_bounds__(C::NT) k_tile_rank(SymProb P, const int* __restrict__ items,
                                                     const int* __restrict__ nitems, int* __restrict__ tqhead,
                                                     HeavyLists hl, const int* __restrict__ hcount) {
  using SM = TileSmem<C>;
  extern __shared__ __align__(16) unsigned char sm[];
  int* keys = reinterpret_cast<int*>(sm + SM::keys);
  unsigned* pay = reinterpret_cast<unsigned*>(sm + SM::pay);
  unsigned short* sidx = reinterpret_cast<unsigned short*>(sm + SM::sidx);
  unsigned short* sbk = reinterpret_cast<unsigned short*>(sm + SM::sbk);
  unsigned short* exrow = reinterpret_cast<unsigned short*>(sm + SM::exrow);
  int* cnt = reinterpret_cast<int*>(sm + SM::cnt);
  int* s_ae = reinterpret_cast<int*>(sm + SM::ae);
  int* s_pf = reinterpret_cast<int*>(sm + SM::pf);
  int* s_bb = reinterpret_cast<int*>(sm + SM::bb);
  int* s_out = reinterpret_cast<int*>(sm + SM::out);
  int* s_sf = reinterpret_cast<int*>(sm + SM::sf);
  int* s_rpa = reinterpret_cast<int*>(sm + SM::rpa);
  int* s_row = reinterpret_cast<int*>(sm + SM::row);
  int* s_cmin = reinterpret_cast<int*>(sm + SM::cmin);
  int* s_cmax = reinterpret_cast<int*>(sm + SM::cmax);
  unsigned* s_mul = reinterpret_cast<unsigned*>(sm + SM::mul);
  uint8_t* s_kind = reinterpret_cast<uint8_t*>(sm + SM::kind);
  uint8_t* s_item = reinterpret_cast<uint8_t*>(sm + SM::item);
  int* seg = reinterpret_cast<int*>(sm + SM::seg);
  int* sbs = reinterpret_cast<int*>(sm + SM::sbs);
  int* sae = reinterpret_cast<int*>(sm + SM::sae);
  unsigned short* srw = reinterpret_cast<unsigned short*>(sm + SM::srw);
  __shared__ int2 scratch2[C::NT / 32 + 1];
  __shared__ int scratch[C::NT / 32 + 1];
  // the popped items, and the tiles of the current batch
  __shared__ int s_t0, s_qr0[C::NI], s_qr1[C::NI], s_qskip[C::NI], s_qp[C::NI], s_qe0[C::NI], s_qt[C::NI];
  __shared__ long long s_qP0[C::NI];
  __shared__ int s_nb, s_bi[C::NI], s_irb[C::NI + 1], s_ie0[C::NI], s_iub[C::NI + 1], s_inext;
  __shared__ long long s_iP0[C::NI], s_idb[C::NI];
  __shared__ int s_uc[C::NU];
  __shared__ int s_htot;
  constexpr int NT = C::NT, NW = NT / 32;
  const Group<NT> g{(int)threadIdx.x, scratch};
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int mloc = P.row_end - P.row_begin;
  if (P.Ro[mloc] > P.r_cap) return;  // plan too small: the host grows it and reruns
  // the queue: consecutive items, or (LIST) the HEAVY then HEAVY2 bin lists
  const int n0 = C::LIST ? hcount[BIN_HEAVY] : 0;
  const int nt = C::LIST ? n0 + hcount[BIN_HEAVY2] : *nitems;

  for (;;) {
    // ---- pop NI consecutive items (their cost varies with their rows' shapes) ---------------------
    if (tid == 0) s_t0 = atomicAdd(tqhead, C::NI);
    __syncthreads();
    const int t0 = s_t0;
    if (t0 >= nt) break;
    const int nq = min(C::NI, nt - t0);
    if (tid < nq) {
      int r, r2, t, skip;
      if constexpr (C::LIST) {  // a heavy row is an item of its own
        const int x = t0 + tid;
        r = x < n0 ? hl.rows[BIN_HEAVY][x] : hl.rows[BIN_HEAVY2][x - n0];
        r2 = r + 1;
        t = (int)(P.tscan[r] - 1);
        skip = 0;
      } else {
        t = t0 + tid;
        r = items[t];
        r2 = items[t + 1];
        skip = (P.cls[r] & CLS_HEAVY_PATH) ? 1 : 0;  // heavy rows: k_bitmap_rank or the big tiles
      }
      s_qr0[tid] = r;
      s_qr1[tid] = r2;
      s_qt[tid] = t;
      s_qskip[tid] = skip;
      s_qP0[tid] = P.Ro[r];
      s_qp[tid] = (int)(P.Ro[r2] - P.Ro[r]);
      s_qe0[tid] = P.rpA[P.row_begin + r];
    }
    if (tid == 0) s_inext = 0;
    __syncthreads();
    for (;;) {
      // ---- the next batch: consecutive tiles of the pop, <= C::PMAX products, <= C::RM rows
      if (tid == 0) {
        int k = s_inext, nb = 0, rows = 0;
        long long prod = 0;
        s_irb[0] = 0;
        for (; k < nq; ++k) {
          if (s_qskip[k]) continue;
          const int nr = s_qr1[k] - s_qr0[k];
          const int p = s_qp[k];
          if (nb > 0 && (rows + nr > C::RM || prod + p > C::PMAX)) break;
          s_bi[nb] = k;
          s_iP0[nb] = s_qP0[k];
          s_ie0[nb] = s_qe0[k];
          rows += nr;
          prod += p;
          s_irb[++nb] = rows;
        }
        s_inext = k;
        s_nb = nb;
      }
      __syncthreads();
      const int NI = s_nb;
      if (NI == 0) break;
      const int NR = s_irb[NI];
      // the bucket counters of step 3, zeroed here (the barriers of steps 1-2 order it)
      for (int b = tid; b <= C::NB; b += NT) cnt[b] = 0;

      // ---- 1. rows: tile, first A entry, A entries and products (block scans) ------------------------
      int ii = 0, j_al = 0, j_f = 0, j_s = 0;
      if (tid < NR) {
        ii = upper_idx(s_irb, NI, tid);
        const int li = s_qr0[s_bi[ii]] + (tid - s_irb[ii]);
        const int i = P.row_begin + li;
        const int pa = P.rpA[i];
        j_al = P.rpA[i + 1] - pa;
        j_f = (int)(P.Ro[li + 1] - P.Ro[li]);
        s_row[tid] = li;
        s_rpa[tid] = pa;
        s_item[tid] = (uint8_t)ii;
        const int k1 = P.cls[li] & 7;
        s_kind[tid] = (uint8_t)k1;
        j_s = k1 == CLS_SINGLE ? j_f : 0;
        s_cmin[tid] = INT_MAX;
        s_cmax[tid] = -1;
      }
      {
        int2 tot;
        const int lane_ = tid & 31, w_ = tid >> 5;
        // exclusive scans of (A entries, products | SINGLE-row products << 16) over the batch rows
        // (both halves sum to <= PMAX < 2^16)
        int ia = j_al, ib = j_f | (j_s << 16);
#pragma unroll
        for (int d = 1; d < 32; d <<= 1) {
          const int oa = __shfl_up_sync(FULL, ia, d), ob = __shfl_up_sync(FULL, ib, d);
          if (lane_ >= d) { ia += oa; ib += ob; }
        }
        if (lane_ == 31) scratch2[w_] = make_int2(ia, ib);
        __syncthreads();
        if (w_ == 0) {
          int2 x = lane_ < NW ? scratch2[lane_] : make_int2(0, 0);
          int xa = x.x, xb = x.y;
#pragma unroll
          for (int d = 1; d < 32; d <<= 1) {
            const int oa = __shfl_up_sync(FULL, xa, d), ob = __shfl_up_sync(FULL, xb, d);
            if (lane_ >= d) { xa += oa; xb += ob; }
          }
          if (lane_ < NW) scratch2[lane_] = make_int2(xa - x.x, xb - x.y);
          if (lane_ == NW - 1) scratch2[NW] = make_int2(xa, xb);
        }
        __syncthreads();
        const int2 base = scratch2[w_];
        tot = scratch2[NW];
        if (tid < NR) {
          const int ex = base.y + ib - (j_f | (j_s << 16));
          s_ae[tid] = base.x + ia - j_al;
          s_pf[tid] = ex & 0xffff;
          s_sf[tid] = ex >> 16;
        }
        if (tid == 0) {
          s_ae[NR] = tot.x;
          s_pf[NR] = tot.y & 0xffff;
          s_sf[NR] = tot.y >> 16;
        }
      }
      __syncthreads();
      const int AE = s_ae[NR], PT = s_pf[NR];
      if (PT == 0) {  // only empty rows
        if (tid < NR) P.crow[s_row[tid] + 1] = 0;
        __syncthreads();
        continue;
      }

      // ---- 2. expand: columns and plan words of every product; column range per light row -------
      int pc = 0;  // products before this chunk
      for (int u0 = 0; u0 < AE; u0 += NT) {
        const int u = u0 + tid;
        int L = 0, bs = 0, j = 0, er = 0;
        if (u < AE) {
          j = upper_idx(s_ae, NR, u);
          const int e = s_rpa[j] + (u - s_ae[j]);
          er = e - s_ie0[s_item[j]];
          bs = P.Tb[e];
          L = P.Tl[e];
          if (L > 0 && s_kind[j] >= CLS_TINY) {  // B rows are sorted: first and last entry bound them
            atomicMin(&s_cmin[j], P.colB[bs]);
            atomicMax(&s_cmax[j], P.colB[bs + L - 1]);
          }
        }
        int tot;
        const int ex = g.template excl_scan<false>((L << 16) | (L > 0 ? 1 : 0), tot);  // L <= PT <= 2^12, runs <= NT
        const int slot = ex & 0xffff, nrun = tot & 0xffff, Lt = tot >> 16;
        if (L > 0) {
          seg[slot] = ex >> 16;
          sbs[slot] = bs;
          sae[slot] = er;
          srw[slot] = (unsigned short)j;
        }
        if (tid == 0) seg[nrun] = Lt;
        __syncthreads();
        // each warp walks one contiguous range of the chunk's products in 32-product windows
        const int chunk = (Lt + NW * 32 - 1) / (NW * 32) * 32;
        const int jbeg = min(Lt, warp * chunk), jend = min(Lt, jbeg + chunk);
        int rb = jbeg < jend ? upper_idx(seg, nrun, jbeg) : 0;
        for (int jw0 = jbeg; jw0 < jend; jw0 += 32 * TILE_EU) {
          int q[TILE_EU], rr[TILE_EU];
#pragma unroll
          for (int x = 0; x < TILE_EU; ++x) {
            const int jw = jw0 + x * 32, jj = jw + lane;
            q[x] = -1;
            rr[x] = 0;
            if (jw < jend) {
              rr[x] = walk_run(seg, nrun, jw, rb);
              if (jj < jend) q[x] = jj - seg[rr[x]];
            }
          }
          int col[TILE_EU];
#pragma unroll
          for (int x = 0; x < TILE_EU; ++x) col[x] = q[x] >= 0 ? P.colB[sbs[rr[x]] + q[x]] : 0;
#pragma unroll
          for (int x = 0; x < TILE_EU; ++x)
            if (q[x] >= 0) {
              const int idx = pc + jw0 + x * 32 + lane;
              keys[idx] = col[x];
              pay[idx] = plan_pack((unsigned)sae[rr[x]], (unsigned)q[x]);
              exrow[idx] = srw[rr[x]];
            }
        }
        pc += Lt;
        __syncthreads();
      }

      // ---- 3. buckets: the row's own column range cut into nb = min(ceil(f / TILE_BK), range)
      //         equal parts — bucket(col) = floor((col - cmin) * nb / range) as one __umulhi with a
      //         per-row 32-bit scale (monotonic in col, so bucket order is (row, column) order)
      {
        int nb = 0;
        if (tid < NR && s_kind[tid] >= CLS_TINY) {
          const int f = s_pf[tid + 1] - s_pf[tid];
          const unsigned span = (unsigned)(s_cmax[tid] - s_cmin[tid]);  // range - 1 (< 2^31)
          const unsigned want = (unsigned)((f + TILE_BK - 1) / TILE_BK);
          const unsigned nbu = want < span + 1u ? want : span + 1u;
          s_mul[tid] = nbu == span + 1u ? 0u : (unsigned)(((unsigned long long)nbu << 32) / (span + 1u));
          nb = (int)nbu;
        }
        int tot;
        const int ex = g.template excl_scan<false>(nb, tot);
        if (tid < NR) s_bb[tid] = ex;
        if (tid == 0) s_bb[NR] = tot;
      }
      __syncthreads();
      const int NBt = s_bb[NR];
      // bucket of product idx (light rows; -1: SINGLE row, no sort)
      auto bucket_of = [&](int idx) -> int {
        const int j = exrow[idx];
        if (s_kind[j] < CLS_TINY) return -1;
        const unsigned d = (unsigned)(keys[idx] - s_cmin[j]), m = s_mul[j];
        return s_bb[j] + (int)(m ? __umulhi(d, m) : d);
      };
      // every product's bucket and column in registers (thread tid owns products tid + u NT);
      // single: bit u set for a product of a SINGLE row (placed in order, no sort)
      constexpr int IPT = C::PMAX / C::NT;
      int bk[IPT], cl[IPT];
      unsigned single = 0;
#pragma unroll
      for (int u = 0; u < IPT; ++u) {
        const int idx = tid + u * NT;
        bk[u] = -1;
        cl[u] = 0;
        if (idx < PT) {
          bk[u] = bucket_of(idx);
          cl[u] = keys[idx];
          if (bk[u] >= 0) atomicAdd(&cnt[bk[u]], 1);
          else if (s_kind[exrow[idx]] == CLS_SINGLE) single |= 1u << u;
        }
      }
      __syncthreads();

      // ---- 4. bucket starts (exclusive scan, contiguous ownership), scatter ------------------------
      constexpr int BPT = (C::NB + NT - 1) / NT;
      {
        int c8[BPT], mine = 0;
#pragma unroll
        for (int k = 0; k < BPT; ++k) {
          const int b = tid * BPT + k;
          c8[k] = b < NBt ? cnt[b] : 0;
          mine += c8[k];
        }
        int tot;
        int run = g.template excl_scan<false>(mine, tot);
#pragma unroll
        for (int k = 0; k < BPT; ++k) {
          const int b = tid * BPT + k;
          if (b < NBt) cnt[b] = run;
          run += c8[k];
        }
      }
      __syncthreads();
      //      (the expand pass parked every product's column in keys[idx]; all of them are read into
      //      registers before the first slot is overwritten)
      {
#pragma unroll
        for (int u = 0; u < IPT; ++u) {
          const int b = bk[u];
          if (b < 0) continue;
          const int slot = atomicAdd(&cnt[b], 1);  // afterwards cnt[b] = end of bucket b
          keys[slot] = cl[u];
          sidx[slot] = (unsigned short)(tid + u * NT);
          sbk[slot] = (unsigned short)b;
        }
      }
      __syncthreads();
      const int Pg = NBt > 0 ? cnt[NBt - 1] : 0;

      // ---- 5. sort every bucket in place: slot x moves to s0 + #{y : (key, slot) of y < that of x}
      //         (buckets hold ~TILE_BK products; the permutation goes through registers)
      {
        static_assert(C::PMAX <= 65536, "slot and product index in 16 bits each");
        unsigned nps[IPT];  // new slot | product index << 16; ~0u: none
        int nkey[IPT];
#pragma unroll
        for (int u = 0; u < IPT; ++u) {
          const int x = tid + u * NT;
          nps[u] = ~0u;
          if (x < Pg) {
            const int bb = sbk[x];
            const int s0 = bb ? cnt[bb - 1] : 0, s1 = cnt[bb];
            const int kx = keys[x];
            int pos = x;
            if (s1 - s0 > 1) {
              pos = s0;
              for (int y = s0; y < s1; ++y) {
                const int ky = keys[y];
                pos += (ky < kx) || (ky == kx && y < x);
              }
            }
            nps[u] = (unsigned)pos | ((unsigned)sidx[x] << 16);
            nkey[u] = kx;
          }
        }
        __syncthreads();
#pragma unroll
        for (int u = 0; u < IPT; ++u) {
          const int pos = (int)(nps[u] & 0xffffu);
          if (nps[u] != ~0u && pos != tid + u * NT) {
            keys[pos] = nkey[u];
            sidx[pos] = (unsigned short)(nps[u] >> 16);
          }
        }
      }
      __syncthreads();

      // ---- 6. heads: the first slot of its bucket or a column unlike the previous slot's; a block
      //         scan of the head flags (slots are in (row, column) order) numbers the outputs:
      //         keys[x] = index of the column's head among the batch's heads, sign bit = repeat
      {
        unsigned hf = 0;
        int nh = 0;
#pragma unroll
        for (int k = 0; k < IPT; ++k) {
          const int x = tid * IPT + k;
          if (x < Pg) {
            const bool h = x == 0 || sbk[x] != sbk[x - 1] || keys[x] != keys[x - 1];
            hf |= (unsigned)h << k;
            nh += h;
          }
        }
        int tot;
        int run = g.template excl_scan<false>(nh, tot);  // (its barriers order the reads above before the writes below)
#pragma unroll
        for (int k = 0; k < IPT; ++k) {
          const int x = tid * IPT + k;
          if (x < Pg) {
            const bool h = hf >> k & 1u;
            run += h;
            keys[x] = (run - 1) | (h ? 0 : int(0x80000000));
          }
        }
        if (tid == 0) s_htot = tot;
      }
      __syncthreads();

      // ---- 7. output offsets of the rows (in the batch; a tile's outputs start at the offset of its
      //         first row) without a scan: heads before the row's first slot (that slot is a head;
      //         for a row without buckets, the next light row's) + SINGLE-row products before it;
      //         s_cmin[j] = the heads before row j -----------------------------------------------------
      if (tid < NR) {
        const int b0 = s_bb[tid];
        const int x0 = b0 ? cnt[b0 - 1] : 0;
        const int h = x0 < Pg ? keys[x0] & 0x7fffffff : s_htot;
        s_out[tid] = h + s_sf[tid];
        s_cmin[tid] = h;
      }
      if (tid == 0) s_out[NR] = s_htot + s_sf[NR];
      __syncthreads();
      if (tid < NR) P.crow[s_row[tid] + 1] = s_out[tid + 1] - s_out[tid];  // c_j
      const bool reps = PT != s_out[NR];  // the batch has repeated products (block-uniform)
      if (reps) {
        if (tid == 0) {  // per tile: repeats (statistics), numeric-unit bases of the repeat counters
          long long dups = 0;
          int ub = 0;
          for (int x = 0; x < NI; ++x) {
            const int C = s_out[s_irb[x + 1]] - s_out[s_irb[x]];
            dups += (s_pf[s_irb[x + 1]] - s_pf[s_irb[x]]) - C;
            s_iub[x] = ub;
            ub += (C + NUM_SH - 1) / NUM_SH;
          }
          s_iub[NI] = ub;
          if (dups) atomicAdd(reinterpret_cast<unsigned long long*>(P.dups_all), (unsigned long long)dups);
        }
        if (tid < C::NU) s_uc[tid] = 0;
        __syncthreads();
      }

      // ---- 8. plan: heads in C order; repeats after them, bucketed by numeric unit ----------------
      for (int x = tid; x < Pg; x += NT) {
        const int kx = keys[x];
        const int jr = exrow[sidx[x]];
        const int it = s_item[jr];
        // output of the product's column, relative to its tile
        const int o = s_out[jr] - s_out[s_irb[it]] + (kx & 0x7fffffff) - s_cmin[jr];
        if (kx >= 0) {
          P.plan[s_iP0[it] + o] = pay[sidx[x]];
        } else {  // a repeat: its output parked in sbk (own slot only)
          sbk[x] = (unsigned short)o;
          atomicAdd(&s_uc[s_iub[it] + o / NUM_SH], 1);
        }
      }
#pragma unroll
      for (int u = 0; u < IPT; ++u)  // SINGLE rows: products already in column order
        if (single >> u & 1u) {
          const int idx = tid + u * NT;
          const int j = exrow[idx];
          const int it = s_item[j];
          P.plan[s_iP0[it] + s_out[j] - s_out[s_irb[it]] + idx - s_pf[j]] = pay[idx];
        }
      __syncthreads();
      if (!reps) continue;  // no repeated product in the batch: no R records
      if (tid < NI) {  // R records of the tile's repeats, bucketed by numeric unit (dub: first record)
        const int x = tid;
        const int C = s_out[s_irb[x + 1]] - s_out[s_irb[x]];
        const int F = s_pf[s_irb[x + 1]] - s_pf[s_irb[x]];
        s_idb[x] = -1;
        if (F > C) {
          long long base = (long long)atomicAdd(reinterpret_cast<unsigned long long*>(P.dups), (unsigned long long)(F - C));
          if (base + (F - C) > P.r_dcap) base = -1;  // too small: the host grows R and reruns
          s_idb[x] = base;
          long long* db = P.dub + dub_index(s_iP0[x], s_qt[s_bi[x]]);
          const int hs = (C + NUM_SH - 1) / NUM_SH;
          int run = 0;
          for (int k = 0; k < hs; ++k) {
            const int v = s_uc[s_iub[x] + k];
            s_uc[s_iub[x] + k] = run;
            db[k] = base + run;
            run += v;
          }
          db[hs] = base + run;
        }
      }
      __syncthreads();
      for (int x = tid; x < Pg; x += NT)
        if (keys[x] < 0) {
          const int o = sbk[x], idx = sidx[x];
          const int it = s_item[exrow[idx]];
          if (s_idb[it] < 0) continue;
          const int pos = atomicAdd(&s_uc[s_iub[it] + o / NUM_SH], 1);
          const unsigned w = pay[idx];
          const int e = s_ie0[it] + (int)(w & 0xffffu);
          P.R[s_idb[it] + pos] = make_int2(P.Tb[e] + (int)(w >> 16), rec_meta((int)(w & 0xffffu), o));
        }
      __syncthreads();
    }
  }
}

cudaError_t tile_configure() {
  cudaError_t e = cudaFuncSetAttribute(k_tile_rank<TileSmall>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       TileSmem<TileSmall>::bytes);
  if (e == cudaSuccess)
    e = cudaFuncSetAttribute(k_tile_rank<TileBig>, cudaFuncAttributeMaxDynamicSharedMemorySize, TileSmem<TileBig>::bytes);
  return e;
}

int tile_occupancy(int big) {
  int nb = 1;
  if (big) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_tile_rank<TileBig>, TileBig::NT, TileSmem<TileBig>::bytes);
  else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_tile_rank<TileSmall>, TileSmall::NT, TileSmem<TileSmall>::bytes);
  return nb < 1 ? 1 : nb;
}

cudaError_t launch_tile_rank(cudaStream_t st, int grid, const SymProb& P, const int* items, const int* nitems,
                             int* tqhead) {
  HeavyLists none{};
  k_tile_rank<TileSmall><<<grid, TileSmall::NT, TileSmem<TileSmall>::bytes, st>>>(P, items, nitems, tqhead, none,
                                                                                  nullptr);
  return cudaGetLastError();
}

cudaError_t launch_tile_heavy(cudaStream_t st, int grid, const SymProb& P, const HeavyLists& lists, const int* counts,
                              int* qhead) {
  k_tile_rank<TileBig><<<grid, TileBig::NT, TileSmem<TileBig>::bytes, st>>>(P, nullptr, nullptr, qhead, lists, counts);
  return cudaGetLastError();
}

}  // namespace spg
