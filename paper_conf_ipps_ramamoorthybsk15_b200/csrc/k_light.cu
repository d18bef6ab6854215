// k_light.cu — symbolic phase of the tiles: runs of consecutive non-heavy rows (the paper's A_L,
// "numerous subproblems of small computational intensity"), many rows per block.
//
// A tile is an item of the ordered item list (k_tile_flags / k_items): <= TILE_RM consecutive
// rows, < TILE_PMAX products, < 2 TILE_EC A entries.  The block sorts all products of the tile at
// once with one bucketed counting sort, so the per-row cost of a row-per-warp design (barriers,
// scans, idle lanes) is paid once per ~3k products instead:
//
//   1. rows      per row its A-entry and product offsets inside the tile (from row_ptr and the
//                plan prefix Ro: no scan needed).
//   2. expand    every product's column and plan word {e_rel, qoff} go to shared memory
//                (coalesced B-row loads; the run of each lane from a REDUX.OR run-start mask).
//                Each light row's column range [cmin, cmax] comes from the first and last entry
//                of its (sorted) B rows.
//   3. buckets   light row j gets NB_j <= ceil(f_j / TILE_BK) buckets of 2^sh_j columns over its
//                own range: bucket order is (row, column) order; sizes by ATOMS.ADD.
//   4. scatter   exclusive scan of the sizes; each product is placed in its bucket.
//   5. heads     a product is the head of its column when no earlier slot of its bucket holds the
//                same column; heads are counted per bucket and scanned; c_j = heads of the row.
//   6. offsets   block scan of c_j: the output offset of every row inside the tile.
//   7. ranks     rank = heads of the row's earlier buckets + distinct smaller columns in the own
//                bucket; a head writes its plan word at P0 + out_j + rank (C order), every other
//                product after the tile's outputs (the dups, each with its output out_j + rank
//                in D at the same word), bucketed by the numeric unit that owns that output.
//                SINGLE rows (one non-empty B row, already sorted) write their products in order.
// This is Phase IV's "sort, mark like-tuples, scan, compact", done per tile in
// shared memory.
#include "kernels.cuh"

namespace spg {

static_assert(TILE_PMAX / TILE_NT <= 32, "head marks of a thread fit one 32-bit mask");
static_assert(TILE_RM <= TILE_NT, "one row per thread in the row phases");
constexpr int TILE_EU = 4;  // 32-product windows per warp per step (loads in flight)
constexpr unsigned short NOBUCKET = 0xffff;

// Run of product jw + lane for a window starting inside run rb (warp-uniform); advances rb to
// the run holding jw + 32.  All 32 lanes must call.
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
struct TileSmem {
  static constexpr int keys = 0;                                    // int[PMAX]   idx -> column (expand), then
                                                                    //             slot -> column (sign: not head)
  static constexpr int pay = keys + TILE_PMAX * 4;                  // u32[PMAX]   idx -> plan word
  static constexpr int sidx = pay + TILE_PMAX * 4;                  // u16[PMAX]   slot -> product index
  static constexpr int sbk = sidx + TILE_PMAX * 2;                  // u16[PMAX]   slot -> bucket
  static constexpr int exb = sbk + TILE_PMAX * 2;                   // u16[PMAX]   idx -> bucket
  static constexpr int exrow = exb + TILE_PMAX * 2;                 // u8[PMAX]    idx -> tile row
  static constexpr int cnt = exrow + TILE_PMAX;                     // int[NBMAX+1] sizes -> starts -> ends
  static constexpr int hc = cnt + (TILE_NBMAX + 1) * 4;             // int[NBMAX+1] heads -> head prefix
  static constexpr int brow = hc + (TILE_NBMAX + 1) * 4;            // u16[NBMAX]   bucket -> tile row
  static constexpr int ae = (brow + TILE_NBMAX * 2 + 15) & ~15;     // int[RM+1]    A-entry offset of the row
  static constexpr int pf = ae + (TILE_RM + 1) * 4;                 // int[RM+1]    product offset of the row
  static constexpr int bb = pf + (TILE_RM + 1) * 4;                 // int[RM+1]    bucket base
  static constexpr int out = bb + (TILE_RM + 1) * 4;                // int[RM+1]    output offset
  static constexpr int cmin = out + (TILE_RM + 1) * 4;              // int[RM]      column range of the row
  static constexpr int cmax = cmin + TILE_RM * 4;                   // int[RM]
  static constexpr int sh = cmax + TILE_RM * 4;                     // u8[RM]       bucket width log2
  static constexpr int kind = sh + TILE_RM;                         // u8[RM]       class of the row
  static constexpr int seg = (kind + TILE_RM + 15) & ~15;           // int[NT+1]    chunk run -> product offset
  static constexpr int sbs = seg + (TILE_NT + 1) * 4;               // int[NT]      chunk run -> B row start
  static constexpr int sae = sbs + TILE_NT * 4;                     // int[NT]      chunk run -> tile A entry
  static constexpr int srw = sae + TILE_NT * 4;                     // u8[NT]       chunk run -> tile row
  static constexpr int bytes = (srw + TILE_NT + 15) & ~15;
};

__global__ void __launch_bounds__(TILE_NT) k_tile_rank(SymProb P, const int* __restrict__ items,
                                                       const int* __restrict__ nitems, int* __restrict__ tqhead) {
  extern __shared__ __align__(16) unsigned char sm[];
  int* keys = reinterpret_cast<int*>(sm + TileSmem::keys);
  unsigned* pay = reinterpret_cast<unsigned*>(sm + TileSmem::pay);
  unsigned short* sidx = reinterpret_cast<unsigned short*>(sm + TileSmem::sidx);
  unsigned short* sbk = reinterpret_cast<unsigned short*>(sm + TileSmem::sbk);
  unsigned short* exb = reinterpret_cast<unsigned short*>(sm + TileSmem::exb);
  uint8_t* exrow = reinterpret_cast<uint8_t*>(sm + TileSmem::exrow);
  int* cnt = reinterpret_cast<int*>(sm + TileSmem::cnt);
  int* hc = reinterpret_cast<int*>(sm + TileSmem::hc);
  unsigned short* brow = reinterpret_cast<unsigned short*>(sm + TileSmem::brow);
  int* s_ae = reinterpret_cast<int*>(sm + TileSmem::ae);
  int* s_pf = reinterpret_cast<int*>(sm + TileSmem::pf);
  int* s_bb = reinterpret_cast<int*>(sm + TileSmem::bb);
  int* s_out = reinterpret_cast<int*>(sm + TileSmem::out);
  int* s_cmin = reinterpret_cast<int*>(sm + TileSmem::cmin);
  int* s_cmax = reinterpret_cast<int*>(sm + TileSmem::cmax);
  uint8_t* s_sh = reinterpret_cast<uint8_t*>(sm + TileSmem::sh);
  uint8_t* s_kind = reinterpret_cast<uint8_t*>(sm + TileSmem::kind);
  int* seg = reinterpret_cast<int*>(sm + TileSmem::seg);
  int* sbs = reinterpret_cast<int*>(sm + TileSmem::sbs);
  int* sae = reinterpret_cast<int*>(sm + TileSmem::sae);
  uint8_t* srw = reinterpret_cast<uint8_t*>(sm + TileSmem::srw);
  __shared__ int scratch[TILE_NT / 32 + 1];
  __shared__ int s_tile;
  constexpr int TU = TILE_PMAX / NUM_SH;  // numeric units of a tile
  __shared__ int s_uc[TU + 1], s_us[TU + 1];
  constexpr int NT = TILE_NT, NW = NT / 32;
  const Group<NT> g{(int)threadIdx.x, scratch};
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int mloc = P.row_end - P.row_begin;
  if (P.Ro[mloc] > P.r_cap) return;  // plan too small: the host grows it and reruns
  const int nt = *nitems;

  // tiles from a dynamic queue (their cost varies with their rows' shapes)
  for (;;) {
    if (tid == 0) s_tile = atomicAdd(tqhead, 1);
    __syncthreads();
    const int t = s_tile;
    __syncthreads();
    if (t >= nt) break;
    const int r0 = items[t];
    if (P.cls[r0] & CLS_HEAVY_PATH) continue;  // heavy rows: k_bitmap_rank
    const int nr = items[t + 1] - r0;
    const int e0 = P.rpA[P.row_begin + r0];
    const long long P0 = P.Ro[r0];

    // ---- 1. rows ---------------------------------------------------------------------------
    if (tid <= nr) {
      s_ae[tid] = P.rpA[P.row_begin + r0 + tid] - e0;
      s_pf[tid] = (int)(P.Ro[r0 + tid] - P0);
    }
    if (tid < nr) {
      s_kind[tid] = P.cls[r0 + tid] & 7;
      s_cmin[tid] = INT_MAX;
      s_cmax[tid] = -1;
    }
    __syncthreads();
    const int AE = s_ae[nr], PT = s_pf[nr];
    if (PT == 0) {  // only empty rows
      if (tid < nr) P.crow[r0 + tid + 1] = 0;
      __syncthreads();
      continue;
    }

    // ---- 2. expand: columns and plan words of every product; column range per light row -------
    int pc = 0;  // products before this chunk
    for (int u0 = 0; u0 < AE; u0 += NT) {
      const int u = u0 + tid;
      int L = 0, bs = 0, j = 0;
      if (u < AE) {
        j = upper_idx(s_ae, nr, u);
        bs = P.Tb[e0 + u];
        L = P.Tl[e0 + u];
        if (L > 0 && s_kind[j] >= CLS_TINY) {  // B rows are sorted: first and last entry bound them
          atomicMin(&s_cmin[j], P.colB[bs]);
          atomicMax(&s_cmax[j], P.colB[bs + L - 1]);
        }
      }
      int tot;
      const int ex = g.excl_scan((L << 16) | (L > 0 ? 1 : 0), tot);  // L <= PT < 2^12, runs <= NT
      const int slot = ex & 0xffff, nrun = tot & 0xffff, Lt = tot >> 16;
      if (L > 0) {
        seg[slot] = ex >> 16;
        sbs[slot] = bs;
        sae[slot] = u;
        srw[slot] = (uint8_t)j;
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

    // ---- 3. buckets: 2^sh columns each over the row's own column range --------------------------
    {
      int nb = 0;
      if (tid < nr && s_kind[tid] >= CLS_TINY) {
        const int f = s_pf[tid + 1] - s_pf[tid];
        const unsigned span = (unsigned)(s_cmax[tid] - s_cmin[tid]);  // range - 1
        const unsigned want = (unsigned)((f + TILE_BK - 1) / TILE_BK);
        int sh = 0;
        while ((span >> sh) >= want) ++sh;
        s_sh[tid] = (uint8_t)sh;
        nb = (int)(span >> sh) + 1;
      }
      int tot;
      const int ex = g.excl_scan(nb, tot);
      if (tid < nr) s_bb[tid] = ex;
      if (tid == 0) s_bb[nr] = tot;
    }
    __syncthreads();
    const int NBt = s_bb[nr];
    for (int b = tid; b <= NBt; b += NT) {
      cnt[b] = 0;
      hc[b] = 0;
      if (b < NBt) brow[b] = (unsigned short)upper_idx(s_bb, nr, b);
    }
    __syncthreads();
    for (int idx = tid; idx < PT; idx += NT) {
      const int j = exrow[idx];
      unsigned short b = NOBUCKET;
      if (s_kind[j] >= CLS_TINY) {
        b = (unsigned short)(s_bb[j] + ((keys[idx] - s_cmin[j]) >> s_sh[j]));
        atomicAdd(&cnt[b], 1);
      }
      exb[idx] = b;
    }
    __syncthreads();

    // ---- 4. bucket starts (exclusive scan, contiguous ownership), scatter ------------------------
    constexpr int BPT = (TILE_NBMAX + NT - 1) / NT;
    {
      int c8[BPT], mine = 0;
#pragma unroll
      for (int k = 0; k < BPT; ++k) {
        const int b = tid * BPT + k;
        c8[k] = b < NBt ? cnt[b] : 0;
        mine += c8[k];
      }
      int tot;
      int run = g.excl_scan(mine, tot);
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
    constexpr int IPT = TILE_PMAX / TILE_NT;
    {
      int bk[IPT], cl[IPT];
#pragma unroll
      for (int u = 0; u < IPT; ++u) {
        const int idx = tid + u * NT;
        bk[u] = idx < PT && exb[idx] != NOBUCKET ? (int)exb[idx] : -1;
        cl[u] = idx < PT ? keys[idx] : 0;
      }
      __syncthreads();
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

    // ---- 5. heads: first slot of its column within the bucket -----------------------------------
    //      (non-head marks are applied after a barrier, so no thread reads a key while another
    //      marks it)
    unsigned nonhead = 0;  // bit u: slot tid + u·NT is not a head
    for (int x = tid, u = 0; x < Pg; x += NT, ++u) {
      const int b = sbk[x];
      const int s0 = b ? cnt[b - 1] : 0;
      const int kx = keys[x];
      bool head = true;
      for (int y = s0; y < x; ++y)
        if (keys[y] == kx) { head = false; break; }
      if (head) atomicAdd(&hc[b], 1);
      else nonhead |= 1u << u;
    }
    __syncthreads();
    for (int x = tid, u = 0; x < Pg; x += NT, ++u)
      if (nonhead >> u & 1u) keys[x] |= int(0x80000000);
    {  // head prefix per bucket; hc[NBt] = total
      int c8[BPT], mine = 0;
#pragma unroll
      for (int k = 0; k < BPT; ++k) {
        const int b = tid * BPT + k;
        c8[k] = b < NBt ? hc[b] : 0;
        mine += c8[k];
      }
      int tot;
      int run = g.excl_scan(mine, tot);  // (its barriers also order the marks above)
#pragma unroll
      for (int k = 0; k < BPT; ++k) {
        const int b = tid * BPT + k;
        if (b < NBt) hc[b] = run;
        run += c8[k];
      }
      if (tid == 0) hc[NBt] = tot;
    }
    __syncthreads();

    // ---- 6. c_j and output offsets of the rows ----------------------------------------------------
    {
      int cj = 0;
      if (tid < nr) {
        const int k = s_kind[tid];
        cj = k >= CLS_TINY ? hc[s_bb[tid + 1]] - hc[s_bb[tid]] : (k == CLS_SINGLE ? s_pf[tid + 1] - s_pf[tid] : 0);
        P.crow[r0 + tid + 1] = cj;
      }
      int tot;
      const int ex = g.excl_scan(cj, tot);
      if (tid < nr) s_out[tid] = ex;
      if (tid == 0) {
        s_out[nr] = tot;
        if (PT > tot) atomicAdd(reinterpret_cast<unsigned long long*>(P.dups), (unsigned long long)(PT - tot));
      }
      if (tid <= TU) s_uc[tid] = 0;
    }
    __syncthreads();

    // ---- 7. ranks -> plan: heads in C order; repeats after them, bucketed by numeric unit --------
    unsigned* plan = P.plan + P0;
    for (int x = tid; x < Pg; x += NT) {
      const int b = sbk[x];
      const int s0 = b ? cnt[b - 1] : 0, s1 = cnt[b];
      const int kx = keys[x];
      const int k = kx & 0x7fffffff;
      int u = 0;
      for (int y = s0; y < s1; ++y) {
        const int ky = keys[y];
        u += (ky >= 0 && ky < k);
      }
      const int jr = brow[b];
      const int o = s_out[jr] + hc[b] - hc[s_bb[jr]] + u;  // output of the product's column
      if (kx >= 0) {
        plan[o] = pay[sidx[x]];
      } else {  // a repeat: its output parked in sbk (read above, own slot only)
        sbk[x] = (unsigned short)o;
        atomicAdd(&s_uc[o / NUM_SH], 1);
      }
    }
    const int Ct = s_out[nr];
    __syncthreads();
    if (PT > Ct) {
      if (tid == 0) {  // bucket starts, also for numeric (dub)
        int* db = P.dub + dub_index(P0, t);
        const int hs = (Ct + NUM_SH - 1) / NUM_SH;
        int run = 0;
        for (int k = 0; k < hs; ++k) {
          s_us[k] = run;
          db[k] = run;
          run += s_uc[k];
        }
        db[hs] = run;
      }
      __syncthreads();
      for (int x = tid; x < Pg; x += NT)
        if (keys[x] < 0) {
          const int o = sbk[x];
          const int pos = Ct + atomicAdd(&s_us[o / NUM_SH], 1);
          plan[pos] = pay[sidx[x]];
          P.D[P0 + pos] = (unsigned)o;
        }
    }
    for (int idx = tid; idx < PT; idx += NT)  // SINGLE rows: products already in column order
      if (exb[idx] == NOBUCKET) {
        const int j = exrow[idx];
        plan[s_out[j] + idx - s_pf[j]] = pay[idx];
      }
    __syncthreads();
  }
}

cudaError_t tile_configure() {
  return cudaFuncSetAttribute(k_tile_rank, cudaFuncAttributeMaxDynamicSharedMemorySize, TileSmem::bytes);
}

int tile_occupancy() {
  int nb = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_tile_rank, TILE_NT, TileSmem::bytes);
  return nb < 1 ? 1 : nb;
}

cudaError_t launch_tile_rank(cudaStream_t st, int grid, const SymProb& P, const int* items, const int* nitems,
                             int* tqhead) {
  k_tile_rank<<<grid, TILE_NT, TileSmem::bytes, st>>>(P, items, nitems, tqhead);
  return cudaGetLastError();
}

}  // namespace spg
