// kernels.cuh — declarations shared by the kernel translation units and the C-ABI layer.
//
// Pipeline:
//   analysis   k_row_flops: f_i, run count and size flags per row, log2 histogram
//   classify   k_classify: heavy rows (f_i > light_max, or long A rows) go to a bitmap bin list;
//              every other row belongs to a tile; plan words per row (scanned into Ro)
//   items      k_tile_flags + scan + k_items: the ordered list of items — a heavy row, or a tile
//              of consecutive non-heavy rows (<= TILE_RM rows, < TILE_PMAX products,
//              < 2 TILE_EC A entries)
//   symbolic   k_tile_rank (tiles) and k_bitmap_rank (heavy rows) sort every item's products by
//              (row, column), count c_i and write the plan: the item's outputs in C order as
//              {A entry, B offset} words, then its repeated products (dups)
//   units      k_unit_count + scan + k_unit_fill: numeric work units — segments of an item's
//              outputs
//   numeric    k_numeric: persistent warps take units from a queue — C(i, j) = valA[e]·valB[q]
//              streamed in C order (TMA-staged plan words, coalesced C write; A/B from L2); then
//              the unit adds the item's repeated products that land in its outputs with RED
//              (Phase IV of PAPER.md L154-156: the sort moved to symbolic, so numeric re-runs on
//              new values are a stream)
#pragma once
#include "common.cuh"

namespace spg {

struct ClassParams {
  int light_max;   // f <= light_max -> tile path
  int heavy_max;   // heavy rows with f <= heavy_max -> register-cached bitmap kernel, else HUGE
  int tile_cap;    // nominal products per tile; rows above TILE_PMAX - tile_cap are solo tiles
  int force;       // -1 or a class id >= CLS_TINY
  int single_ok;   // B rows canonical -> SINGLE (copy) shortcut allowed
};

struct HeavyLists {
  int* rows[NUM_BINS];
};

// Small per-call device scratch (zeroed at the start of every symbolic call).
struct Small {
  int counts[8];            // per bitmap bin: rows
  int qhead[8];             // per bitmap bin: dynamic row-queue heads (counts + 8)
  int nitems;               // items (tiles + heavy rows)
  int err;
  int amax;                 // longest row of A
  int tqhead;               // tiles: dynamic queue head
  long long dups;           // repeat records reserved (R entries)
  long long dups_all;       // repeated products (statistics)
  long long nunits;         // numeric work units
  unsigned long long hist[65];
  unsigned long long cstats[2 * NUM_CLS + 2];
};

// Problem view passed to the symbolic kernels.  Row indices in lists / cls / Ro / crow are
// local (i - row_begin).
struct SymProb {
  const int* __restrict__ rpA;
  const int* __restrict__ colA;
  const int* __restrict__ rpB;
  const int* __restrict__ colB;
  const int* __restrict__ Tb;   // per A entry: start of its B row (rpB[colA[e]])
  const int* __restrict__ Tl;   // per A entry: length of its B row
  const int* frow;          // f_i (global row index)
  const uint8_t* cls;       // class and path flags per local row
  const long long* Ro;      // plan word offset per local row (exclusive prefix, [Mloc + 1])
  unsigned* plan;           // the plan (capacity r_cap words)
  uint8_t* fl8;             // uncached bitmap rows: first-claim flag per product (Ro_i + offset)
  long long* crow;          // C row offsets (local); symbolic writes counts at [li + 1]
  const long long* tscan;   // inclusive scan of the item-start flags: item of row li = tscan[li] - 1
  unsigned* D;              // HUGE rows: item-relative output of the repeated product whose plan
                            // entry starts at the same word (written only for their repeats)
  long long* dub;           // repeats' first R record per numeric unit (dub_index(P0, t) + k)
  int2* R;                  // repeat records {B entry, rec_meta(A entry - item's first, output)}
  long long r_dcap;         // R capacity (records); beyond it nothing is written (host grows, reruns)
  long long* dups;          // R reservation counter
  long long* dups_all;      // repeated-product counter (statistics)
  int* err;                 // error bits (Small::err)
  long long r_cap;          // plan capacity (words); the kernels do nothing if Ro[Mloc] > r_cap
  int row_begin, row_end;
  // Dual-ended queue (SPG_OPT_HEAVY_DUAL, the paper's cpuOffset / gpuOffset work
  // queue): the virtual list [HUGE rows ; HEAVY2 rows], each part largest
  // first.  HUGE-kernel blocks (any row) take from the front, HEAVY2 (register-cached) blocks from
  // the back; a row is processed by whichever side claims it first (claim[t] raised to gen).
  int dual;                 // 1: on
  const int* dq_lh;         // HUGE list, count dq_nh[0]
  const int* dq_l2;         // HEAVY2 list, count dq_n2[0]
  const int* dq_nh;
  const int* dq_n2;
  int* dq_front;            // front cursor (Small::qhead[BIN_HUGE])
  int* dq_back;             // back cursor (Small::qhead[BIN_HEAVY2])
  int* dq_claim;            // per list index: generation of the last claim
  int dq_gen;               // this call's generation (> every earlier one)
};

// Numeric work units, in a list built in item order: item t has ceil(c_t / NUM_SH) units, unit k
// owning outputs [k NUM_SH, (k + 1) NUM_SH) of the item.  A unit stores its outputs, then adds
// the item's repeated products (d_t = f_t - c_t) that land in its own outputs: a warp only ever
// adds into outputs it stored itself, so no unit waits for another.  The repeats are 8-byte
// records (rec_meta below) in R, bucketed by unit (tiles: k_tile_rank;
// heavy rows: k_bitmap_rank at the end of the row); unit k's
// records start at R[dub[dub_index(P0, t) + k]].
constexpr int NUM_SH = 512;
constexpr int DUP_SORT_UNITS = 48 * 1024;   // HUGE rows' unit counters in k_bitmap_rank (rows up to 24M outputs)
__host__ __device__ __forceinline__ long long dub_index(long long P0, long long t) { return P0 / NUM_SH + 2 * t; }
// A repeat record is 8 bytes {B entry, e_rel | (o mod NUM_SH) << 23}: e_rel = its A entry minus the
// item's first A entry (< 2^23: A rows longer than that are rejected on the host), o mod NUM_SH =
// its output's offset inside the numeric unit that owns it (the unit adds it).
constexpr int REC_EBITS = 23;
static_assert(NUM_SH <= (1 << (32 - REC_EBITS)), "unit offset fits the record");
__host__ __device__ __forceinline__ int rec_meta(int e_rel, int o) {
  return (int)((unsigned)e_rel | ((unsigned)(o % NUM_SH) << REC_EBITS));
}
struct NumUnit {
  long long pw;   // plan word of the unit's first output
  long long oc;   // C offset (local) of the unit's first output
  long long dw;   // first R record of the unit's repeats
  int d;          // repeats landing in the unit's outputs
  int n;          // outputs of the unit
  int e0;         // first A entry of the item
  int ob;         // item-relative output of the unit's first output | UNIT_WIDE
};
constexpr int UNIT_WIDE = 1 << 30;   // two plan words per entry

// Numeric phase.
template <typename V>
struct NumProb {
  const int* __restrict__ rpA;
  const V* __restrict__ valA;
  const int* __restrict__ Tb;           // per A entry: start of its B row
  const int* __restrict__ colB;
  const V* __restrict__ valB;
  const void* __restrict__ Bp;          // packed {column, value} copy of B (one gather per output) or NULL
  const unsigned* __restrict__ plan;
  const long long* __restrict__ Ro;
  const long long* __restrict__ crow;   // C row offsets (local)
  const uint8_t* __restrict__ cls;
  const int* __restrict__ items;        // ordered item starts (local rows) + sentinel
  const NumUnit* __restrict__ units;
  const long long* __restrict__ nunits;
  const int2* __restrict__ R;           // repeat records {B entry, rec_meta(...)}
  int* ticket;                          // work-unit queue head (zeroed before the launch)
  int row_begin;
  int* ccol;
  V* cval;
};

// analysis.cu
cudaError_t launch_row_flops(cudaStream_t st, int M, const int* rpA, const int* colA, int K, const int* rpB, int* f,
                             uint8_t* nz, int* Tb, int* Tl, unsigned long long* hist, int* err, int* amax);
cudaError_t launch_unit_count(cudaStream_t st, int sms, const int* items, const long long* crow, int n, int* ucnt);
cudaError_t launch_unit_fill(cudaStream_t st, int sms, const int* ucnt, const long long* uscan, int n,
                             NumUnit* units, Small* small, const int* items, const long long* crow,
                             const long long* Ro, const uint8_t* cls, const int* rpA, int rb, const long long* dub);
cudaError_t launch_classify(cudaStream_t st, int sms, const int* f, const uint8_t* nz, int rb, int re,
                            const ClassParams& prm, uint8_t* cls, int* pw, const HeavyLists& lists, Small* small);
cudaError_t launch_tile_flags(cudaStream_t st, int sms, const int* f, const int* rpA, int rb, int re, int tile_cap,
                              const uint8_t* cls, const long long* Ro, int* tflag);
cudaError_t launch_items(cudaStream_t st, int sms, const int* tflag, const long long* tscan, int mloc, int* items,
                         Small* small);
cudaError_t launch_sort_list(cudaStream_t st, const HeavyLists& lists, int bin, const int* f, int rb,
                             const Small* small, int* tmp);
size_t scan_tmp_elems(long long n);
int scan_launches(long long n);
template <typename Tin>
cudaError_t launch_incl_scan(cudaStream_t st, const Tin* in, long long* out, long long n, long long* tmp);
cudaError_t launch_split_points(cudaStream_t st, const long long* Pf, int M, int P, int* s);
cudaError_t launch_validate(cudaStream_t st, int sms, int M, const int* rp, const int* ci, int ncols, long long nnz,
                            int check_sorted, int* err);
cudaError_t launch_rebase(cudaStream_t st, long long* rp_full, int M, int P, const int* splits, const long long* off);
cudaError_t launch_iota(cudaStream_t st, int* p, long long n);
cudaError_t launch_rebase32(cudaStream_t st, int* rp, long long n, const int* first);
cudaError_t launch_split_sizes(cudaStream_t st, const int* s, const int* rpA, int P, long long* out);
template <typename V>
cudaError_t launch_fill(cudaStream_t st, V* p, long long n, V v);
cudaError_t launch_narrow(cudaStream_t st, const long long* in, int* out, long long n);

// k_light.cu — symbolic sort of the tiles, one tile per block iteration.
cudaError_t tile_configure();
int tile_occupancy(int big);
cudaError_t launch_tile_rank(cudaStream_t st, int grid, const SymProb& P, const int* items, const int* nitems,
                             int* tqhead);
// big tiles: the HEAVY and HEAVY2 bins' rows (f <= 8192) sorted like tiles (SPG_OPT_HEAVY_SORT)
cudaError_t launch_tile_heavy(cudaStream_t st, int grid, const SymProb& P, const HeavyLists& lists, const int* counts,
                              int* qhead);

// k_heavy.cu — symbolic sort of the heavy rows (column bitmap), one row per block iteration.
cudaError_t heavy_configure();
int heavy_occupancy(int bin);
cudaError_t launch_heavy_rank(int bin, cudaStream_t st, int grid, const SymProb& P, const int* list,
                              const int* count, long long N);  // (P.dual: the HUGE and HEAVY2 bins share the dual queue)

// k_csrmm.cu — sparse x dense.
template <typename V>
cudaError_t launch_csrmm(cudaStream_t st, int sms, int M, const int* rpA, const int* colA, const void* valA,
                         const void* D, long long ldd, int n, void* C, long long ldc, int light_nnz, int* hlist,
                         int* hcount);

// k_numeric.cu — numeric phase.
template <typename V>
cudaError_t launch_numeric(cudaStream_t st, int sms, const NumProb<V>& P);
template <typename V>
cudaError_t launch_pack_b(cudaStream_t st, int sms, const int* colB, const V* valB, long long n, void* out);

}  // namespace spg
