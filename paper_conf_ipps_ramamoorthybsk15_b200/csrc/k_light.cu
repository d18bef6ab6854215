// k_light.cu — symbolic phase of the light rows (the paper's A_L: "numerous subproblems of
// small computational intensity"), many rows per thread block.
//
// A tile is a run of light rows whose products form a contiguous range of the light-product
// prefix PL (< tile_cap + light_max products; cut points from k_tiles).  The block sorts all
// products of up to TILE_RM rows at once with one bucketed counting sort, so the per-row cost of
// a row-per-warp design (barriers, scans, idle lanes) is paid once per ~2k products instead:
//
//   1. rows      row j gets NB_j = ceil(f_j / TILE_BK) buckets; product (j, col) goes to bucket
//                bb_j + floor(col * NB_j / 2^lgN): buckets of a row are contiguous and ordered by
//                column, rows are ordered, so bucket order is (row, column) order.
//   2. expand    every product's column and bucket go to shared memory (coalesced B-row loads,
//                run of each lane from a REDUX.OR run-start mask); bucket sizes by ATOMS.ADD.
//   3. scatter   exclusive scan of the sizes; each product is placed in its bucket (ATOMS.ADD
//                cursor) with its product index.
//   4. heads     a product is the head (first occurrence) of its column when no earlier slot of
//                its bucket holds the same column; heads are counted per bucket and scanned.
//   5. ranks     rank = heads of the row's earlier buckets + distinct smaller columns in the own
//                bucket; a head writes its {A entry, B entry} to the gather plan at
//                EQ[Ro_j + rank], every other product goes to the dup list; c_j = heads of the
//                row's buckets (Phase IV "mark, scan, compact" of PAPER.md L154-156, done per
//                tile in shared memory).
//
// Rows whose columns cluster (a bucket above TILE_MAXB) are handed to the bitmap kernel (the
// fallback list); their plan and c are written there.
#include "kernels.cuh"

namespace spg {

// Phase timing (experiments only: nvcc -DSPG_PHASE_PROF): clock64 deltas per phase, thread 0 of
// every block, summed into spg_phase_clk.
#ifdef SPG_PHASE_PROF
__device__ unsigned long long spg_phase_clk[16];
#define SPG_PH(i)                                                               \
  do {                                                                          \
    if (threadIdx.x == 0) {                                                     \
      const long long now_ = clock64();                                         \
      if (ph_last_ >= 0) atomicAdd(&spg_phase_clk[ph_id_], (unsigned long long)(now_ - ph_last_)); \
      ph_last_ = now_;                                                          \
      ph_id_ = (i);                                                             \
    }                                                                           \
  } while (0)
#else
#define SPG_PH(i) do { } while (0)
#endif

constexpr int TILE_MAXB = 48;
static_assert(TILE_PMAX / TILE_NT <= 32, "head marks of a thread fit one 32-bit mask");
constexpr int TILE_EU = 4;  // 32-product windows per warp per step (loads in flight)

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

// Exclusive block scan of two ints at once; totals returned.  All threads must call.
template <int NT>
__device__ __forceinline__ int2 block_scan2(int a, int b, int2& tot, int2* scratch) {
  constexpr int NW = NT / 32;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  int ia = a, ib = b;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const int oa = __shfl_up_sync(FULL, ia, d), ob = __shfl_up_sync(FULL, ib, d);
    if (lane >= d) { ia += oa; ib += ob; }
  }
  if (lane == 31) scratch[w] = make_int2(ia, ib);
  __syncthreads();
  if (w == 0) {
    int2 x = lane < NW ? scratch[lane] : make_int2(0, 0);
    int xa = x.x, xb = x.y;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int oa = __shfl_up_sync(FULL, xa, d), ob = __shfl_up_sync(FULL, xb, d);
      if (lane >= d) { xa += oa; xb += ob; }
    }
    if (lane < NW) scratch[lane] = make_int2(xa - x.x, xb - x.y);
    if (lane == NW - 1) scratch[NW] = make_int2(xa, xb);
  }
  __syncthreads();
  const int2 base = scratch[w];
  tot = scratch[NW];
  __syncthreads();
  return make_int2(base.x + ia - a, base.y + ib - b);
}

// Shared-memory layout of one tile block (bytes).
struct LightSmem {
  static constexpr int keys = 0;                                   // int[PMAX]    idx -> column (expand), then
                                                                   //              slot -> column (sign: not head)
  static constexpr int sq = keys + TILE_PMAX * 4;                  // int[PMAX]    idx -> B entry
  static constexpr int se = sq + TILE_PMAX * 4;                    // u16[PMAX]    idx -> batch A entry
  static constexpr int sidx = se + TILE_PMAX * 2;                  // u16[PMAX]    slot -> product index
  static constexpr int sbk = sidx + TILE_PMAX * 2;                 // u16[PMAX]    slot -> bucket
  static constexpr int exb = sbk + TILE_PMAX * 2;                  // u16[PMAX]    idx -> bucket
  static constexpr int cnt = exb + TILE_PMAX * 2;                  // int[NBMAX+1] sizes -> starts -> ends
  static constexpr int hc = cnt + (TILE_NBMAX + 1) * 4;            // int[NBMAX+1] heads -> head prefix
  static constexpr int brow = hc + (TILE_NBMAX + 1) * 4;           // u16[NBMAX]   bucket -> batch row
  static constexpr int row = (brow + TILE_NBMAX * 2 + 15) & ~15;   // int[RM+1]    local row index
  static constexpr int ae = row + (TILE_RM + 1) * 4;               // int[RM+1]    A-entry prefix
  static constexpr int bb = ae + (TILE_RM + 1) * 4;                // int[RM+1]    bucket base
  static constexpr int rpa = bb + (TILE_RM + 1) * 4;               // int[RM]      first A entry
  static constexpr int ro = (rpa + TILE_RM * 4 + 15) & ~15;        // i64[RM]      EQ offset of the row
  static constexpr int sae = ro + TILE_RM * 8;                     // int[NT]      chunk run -> batch A entry
  static constexpr int seg = sae + TILE_NT * 4;                    // int[NT+1]    chunk run -> product offset
  static constexpr int sbs = seg + (TILE_NT + 1) * 4;              // int[NT]      chunk run -> B row start
  static constexpr int srw = sbs + TILE_NT * 4;                    // u16[NT]      chunk run -> batch row
  static constexpr int bad = srw + TILE_NT * 2;                    // u8[RM]
  static constexpr int bytes = (bad + TILE_RM + 15) & ~15;
};

__global__ void __launch_bounds__(TILE_NT) k_light_rank(SymProb P, const int* __restrict__ tiles,
                                                        const int* __restrict__ ntiles, int* __restrict__ tqhead,
                                                        const uint8_t* __restrict__ tflag,
                                                        const long long* __restrict__ PL, int* __restrict__ fb_list,
                                                        int* __restrict__ fb_count) {
  extern __shared__ __align__(16) unsigned char sm[];
  int* keys = reinterpret_cast<int*>(sm + LightSmem::keys);
  unsigned short* se = reinterpret_cast<unsigned short*>(sm + LightSmem::se);
  int* sq = reinterpret_cast<int*>(sm + LightSmem::sq);
  long long* s_ro = reinterpret_cast<long long*>(sm + LightSmem::ro);
  int* sae = reinterpret_cast<int*>(sm + LightSmem::sae);
  unsigned short* sidx = reinterpret_cast<unsigned short*>(sm + LightSmem::sidx);
  unsigned short* sbk = reinterpret_cast<unsigned short*>(sm + LightSmem::sbk);
  unsigned short* exb = reinterpret_cast<unsigned short*>(sm + LightSmem::exb);
  int* cnt = reinterpret_cast<int*>(sm + LightSmem::cnt);
  int* hc = reinterpret_cast<int*>(sm + LightSmem::hc);
  unsigned short* brow = reinterpret_cast<unsigned short*>(sm + LightSmem::brow);
  int* s_row = reinterpret_cast<int*>(sm + LightSmem::row);
  int* s_ae = reinterpret_cast<int*>(sm + LightSmem::ae);
  int* s_bb = reinterpret_cast<int*>(sm + LightSmem::bb);
  int* s_rpa = reinterpret_cast<int*>(sm + LightSmem::rpa);
  int* seg = reinterpret_cast<int*>(sm + LightSmem::seg);
  int* sbs = reinterpret_cast<int*>(sm + LightSmem::sbs);
  unsigned short* srw = reinterpret_cast<unsigned short*>(sm + LightSmem::srw);
  uint8_t* s_bad = reinterpret_cast<uint8_t*>(sm + LightSmem::bad);
  __shared__ int2 scratch2[TILE_NT / 32 + 1];
  __shared__ int scratch[TILE_NT / 32 + 1];
  __shared__ int s_misc[4];
  __shared__ unsigned long long s_dbase;
  __shared__ int s_dcnt;
  constexpr int NT = TILE_NT, NW = NT / 32;
  const Group<NT> g{(int)threadIdx.x, scratch};
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int nloc = P.row_end - P.row_begin;
  const int lgN = P.lgN;
  if (!*P.r_ok) return;
  const int nt = *ntiles;

#ifdef SPG_PHASE_PROF
  long long ph_last_ = -1;
  int ph_id_ = 0;
#endif
  // tiles from a dynamic queue (their cost varies with their rows' shapes; static striding left
  // a tail)
  __shared__ int s_tile;
  for (;;) {
    if (tid == 0) s_tile = atomicAdd(tqhead, 1);
    __syncthreads();
    const int t = s_tile;
    __syncthreads();
    if (t >= nt) break;
    const int s = tiles[t];
    int cur = s;
    bool done = false;
    while (!done) {
      SPG_PH(0);
      // ---- collect a batch: light rows from `cur` up to the next tile start, <= TILE_RM rows ----
      int nr = 0;
      for (;;) {
        const int li = cur + tid;
        const bool stop = li >= nloc || (li != s && tflag[li]);
        if (tid == 0) s_misc[0] = NT;
        __syncthreads();
        if (stop) atomicMin(&s_misc[0], tid);
        __syncthreads();
        const int fs = s_misc[0];
        const bool lt = tid < fs && (P.cls[li] & CLS_LIGHT_PATH);
        int tot;
        const int pos = g.excl_scan(lt ? 1 : 0, tot);
        if (lt && nr + pos < TILE_RM) s_row[nr + pos] = li;
        if (nr + tot > TILE_RM) {  // batch full: continue from the first light row left over
          if (lt && nr + pos == TILE_RM) s_misc[1] = li;
          __syncthreads();
          cur = s_misc[1];
          nr = TILE_RM;
          break;
        }
        nr += tot;
        if (fs < NT) { done = true; break; }
        cur += NT;
      }
      __syncthreads();
      if (nr == 0) break;

      SPG_PH(1);
      // ---- rows: A range, bucket count; prefixes over the batch ----------------------------
      int a0 = 0, a1 = 0, n0 = 0, n1 = 0;  // two rows per thread (TILE_RM = 2 * NT)
      {
        const int j0 = 2 * tid, j1 = 2 * tid + 1;
        if (j0 < nr) {
          const int i = P.row_begin + s_row[j0];
          const int pa = P.rpA[i];
          s_rpa[j0] = pa;
          s_ro[j0] = P.Ro[s_row[j0]];
          a0 = P.rpA[i + 1] - pa;
          n0 = (P.frow[i] + TILE_BK - 1) / TILE_BK;
        }
        if (j1 < nr) {
          const int i = P.row_begin + s_row[j1];
          const int pa = P.rpA[i];
          s_rpa[j1] = pa;
          s_ro[j1] = P.Ro[s_row[j1]];
          a1 = P.rpA[i + 1] - pa;
          n1 = (P.frow[i] + TILE_BK - 1) / TILE_BK;
        }
        int2 tot;
        const int2 ex = block_scan2<NT>(a0 + a1, n0 + n1, tot, scratch2);
        if (j0 < nr) { s_ae[j0] = ex.x; s_bb[j0] = ex.y; s_bad[j0] = 0; }
        if (j1 < nr) { s_ae[j1] = ex.x + a0; s_bb[j1] = ex.y + n0; s_bad[j1] = 0; }
        if (tid == 0) { s_ae[nr] = tot.x; s_bb[nr] = tot.y; }
      }
      __syncthreads();
      const int AE = s_ae[nr], NBt = s_bb[nr];
      if (AE > 65535) {  // batch A entries do not fit the u16 index: hand the rows to the bitmap kernel
        for (int j = tid; j < nr; j += NT) fb_list[atomicAdd(fb_count, 1)] = s_row[j];
        __syncthreads();
        continue;
      }
      for (int b = tid; b <= NBt; b += NT) {
        cnt[b] = 0;
        hc[b] = 0;
        if (b < NBt) brow[b] = (unsigned short)upper_idx(s_bb, nr, b);
      }
      __syncthreads();

      SPG_PH(2);
      // ---- pass 1: expand columns, bucket of every product, bucket sizes ---------------------
      int pc = 0;  // products before this chunk
      for (int u0 = 0; u0 < AE; u0 += NT) {
        const int u = u0 + tid;
        int L = 0, bs = 0, j = 0, e = 0;
        if (u < AE) {
          j = upper_idx(s_ae, nr, u);
          e = s_rpa[j] + (u - s_ae[j]);
          const int k = P.colA[e];
          bs = P.rpB[k];
          L = P.rpB[k + 1] - bs;
        }
        int tot;
        const int ex = g.excl_scan((L << 16) | (L > 0 ? 1 : 0), tot);  // L <= f <= TILE_PMAX
        const int slot = ex & 0xffff, nrun = tot & 0xffff, Lt = tot >> 16;
        if (L > 0) {
          seg[slot] = ex >> 16;
          sbs[slot] = bs;
          sae[slot] = u;
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
              if (jj < jend) q[x] = sbs[rr[x]] + (jj - seg[rr[x]]);
            }
          }
          int col[TILE_EU];
#pragma unroll
          for (int x = 0; x < TILE_EU; ++x) col[x] = q[x] >= 0 ? P.colB[q[x]] : 0;
#pragma unroll
          for (int x = 0; x < TILE_EU; ++x)
            if (q[x] >= 0) {
              const int jr = srw[rr[x]];
              const int b0 = s_bb[jr], nb = s_bb[jr + 1] - b0;
              const int b = b0 + (int)(((unsigned long long)(unsigned)col[x] * (unsigned)nb) >> lgN);
              const int idx = pc + jw0 + x * 32 + lane;
              keys[idx] = col[x];
              se[idx] = (unsigned short)sae[rr[x]];
              sq[idx] = q[x];
              exb[idx] = (unsigned short)b;
              atomicAdd(&cnt[b], 1);
            }
        }
        pc += Lt;
        __syncthreads();
      }
      const int Pb = pc;

      SPG_PH(3);
      // ---- clustered columns: hand the row to the bitmap kernel -----------------------------
      int badb = 0;
      for (int b = tid; b < NBt; b += NT)
        if (cnt[b] > TILE_MAXB) { s_bad[brow[b]] = 1; badb = 1; }
      if (__syncthreads_or(badb)) {
        for (int j = tid; j < nr; j += NT)
          if (s_bad[j]) {
            fb_list[atomicAdd(fb_count, 1)] = s_row[j];
            for (int b = s_bb[j]; b < s_bb[j + 1]; ++b) cnt[b] = 0;
          }
        __syncthreads();
      }

      SPG_PH(4);
      // ---- bucket starts (exclusive scan, contiguous ownership) ------------------------------
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

      SPG_PH(5);
      // ---- pass 2: scatter into buckets; afterwards cnt[b] = end of bucket b -----------------
      //      (the expand pass parked every product's column in keys[idx]; all of them are read
      //      into registers before the first slot is overwritten)
      constexpr int IPT = TILE_PMAX / TILE_NT;
      int bk[IPT], cl[IPT];
#pragma unroll
      for (int u = 0; u < IPT; ++u) {
        const int idx = tid + u * NT;
        bk[u] = idx < Pb ? (int)exb[idx] : -1;
        cl[u] = idx < Pb ? keys[idx] : 0;
      }
      __syncthreads();
#pragma unroll
      for (int u = 0; u < IPT; ++u) {
        const int b = bk[u];
        if (b < 0 || s_bad[brow[b]]) continue;
        const int slot = atomicAdd(&cnt[b], 1);
        keys[slot] = cl[u];
        sidx[slot] = (unsigned short)(tid + u * NT);
        sbk[slot] = (unsigned short)b;
      }
      __syncthreads();
      const int Pg = NBt > 0 ? cnt[NBt - 1] : 0;

      SPG_PH(6);
      // ---- heads: first slot of its column within the bucket -------------------------------
      //      (non-head marks are applied after a barrier, so no thread reads a key while
      //      another marks it)
      unsigned nonhead = 0;  // bit u: slot tid + u·NT is not a head (<= TILE_PMAX / NT slots)
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
      __syncthreads();
      {  // head prefix per bucket; hc[NBt] = total
        int c8[BPT], mine = 0;
#pragma unroll
        for (int k = 0; k < BPT; ++k) {
          const int b = tid * BPT + k;
          c8[k] = b < NBt ? hc[b] : 0;
          mine += c8[k];
        }
        int tot;
        int run = g.excl_scan(mine, tot);
#pragma unroll
        for (int k = 0; k < BPT; ++k) {
          const int b = tid * BPT + k;
          if (b < NBt) hc[b] = run;
          run += c8[k];
        }
        if (tid == 0) {
          hc[NBt] = tot;
          // dup slots of the batch: products placed in buckets minus distinct columns
          const int nd = (NBt > 0 ? cnt[NBt - 1] : 0) - tot;
          s_dbase = nd > 0 ? atomicAdd(P.dupn, (unsigned long long)nd) : 0ull;
          s_dcnt = 0;
        }
      }
      __syncthreads();

      SPG_PH(7);
      // ---- ranks: heads of the row's earlier buckets + distinct smaller columns in the bucket;
      //      heads -> gather plan (slots are in (row, bucket) order: nearly coalesced), others
      //      -> dup list --------------------------------------------------------------------
      for (int x0 = warp * 32; x0 < Pg; x0 += NT) {  // warp-uniform trips (dup_push)
        const int x = x0 + lane;
        bool head = false, dup = false;
        int rank = 0, jr = 0, idx = 0;
        if (x < Pg) {
          const int b = sbk[x];
          const int s0 = b ? cnt[b - 1] : 0, s1 = cnt[b];
          const int kx = keys[x];
          const int k = kx & 0x7fffffff;
          int u = 0;
          for (int y = s0; y < s1; ++y) {
            const int ky = keys[y];
            u += (ky >= 0 && ky < k);
          }
          jr = brow[b];
          rank = hc[b] - hc[s_bb[jr]] + u;
          idx = sidx[x];
          head = kx >= 0;
          dup = !head;
        }
        const int e = s_rpa[jr] + ((int)se[idx] - s_ae[jr]), q = sq[idx];
        if (head) P.EQ[s_ro[jr] + rank] = make_int2(e, q);
        dup_push(P, dup, s_row[jr], rank, e, q, s_dbase, &s_dcnt);
      }
      for (int j = tid; j < nr; j += NT)
        if (!s_bad[j]) P.crow[s_row[j] + 1] = hc[s_bb[j + 1]] - hc[s_bb[j]];
      __syncthreads();
      SPG_PH(8);
    }
  }
}

cudaError_t light_configure() {
  return cudaFuncSetAttribute(k_light_rank, cudaFuncAttributeMaxDynamicSharedMemorySize, LightSmem::bytes);
}

int light_occupancy() {
  int nb = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_light_rank, TILE_NT, LightSmem::bytes);
  return nb < 1 ? 1 : nb;
}

cudaError_t launch_light_rank(cudaStream_t st, int grid, const SymProb& P, const int* tiles, const int* ntiles, int* tqhead,
                              const uint8_t* tflag, const long long* PL, int* fb_list, int* fb_count) {
  k_light_rank<<<grid, TILE_NT, LightSmem::bytes, st>>>(P, tiles, ntiles, tqhead, tflag, PL, fb_list, fb_count);
  return cudaGetLastError();
}

}  // namespace spg

#ifdef SPG_PHASE_PROF
extern "C" int spg_debug_phase_clk(unsigned long long* out, int reset) {
  cudaMemcpyFromSymbol(out, spg::spg_phase_clk, 16 * sizeof(unsigned long long));
  if (reset) {
    unsigned long long z[16] = {};
    cudaMemcpyToSymbol(spg::spg_phase_clk, z, sizeof z);
  }
  return 0;
}
#endif
