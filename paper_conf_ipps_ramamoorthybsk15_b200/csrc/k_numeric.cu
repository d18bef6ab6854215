// k_numeric.cu — numeric phase: C(i,j) = sum_k A(i,k)·B(k,j) (Row-Row
// formulation) written as sorted, compacted CSR.
//
// The symbolic phase sorted every item's products by (row, column) and left the plan: for an
// item (a tile of consecutive rows, or one heavy row) with plan region [P0, P0 + f) and outputs
// [o0, o0 + c), plan word P0 + o describes output o0 + o — {e_rel, qoff}: the A entry e0 + e_rel
// and the offset of the B entry inside that entry's B row.  The item's repeated products (a
// product whose column another product of its row already produced) are 8-byte records
// {B entry, A entry - item's first | output - unit's first << 23} in R, bucketed by the numeric
// unit owning the output.
//
// So numeric is a stream in C order (Phase IV of PAPER.md L154-156, "add like-tuples and
// compact", with the sort done once in symbolic).  Persistent warps take work units (NUM_SH
// consecutive outputs of one item) from a queue built in item order at the end of symbolic;
// while a unit is processed, one lane has already put the next unit's plan words in flight into
// the warp's other shared-memory buffer with a TMA bulk copy (cp.async.bulk + mbarrier), so the
// plan stream from HBM is never on the dependent path:
//   outputs   per output one plan word (shared memory), the A entry's B-row start Tb[e] and value
//             valA[e] (the item's A entries: L1), the B gather (column and value, L2: B rows are
//             consumed in ascending order), one multiply, two coalesced streaming stores.
//   repeats   the unit's repeat records (8-byte {B entry, A entry, output}, bucketed by unit in
//             symbolic) add a·b into its own outputs with RED.ADD.F64/F32 — into lines it just
//             wrote (L2), ordered after its stores by __syncwarp; no unit ever waits for another.
// HBM traffic per output: 4 B of plan read + (4 + sizeof(V)) B of C written; A and B once.
#include "kernels.cuh"

namespace spg {

constexpr int NUM_NT = 128;            // threads per block: 4 independent warps
constexpr int NUM_W = NUM_NT / 32;
constexpr int NUM_U = 4;               // outputs per lane in flight
// Resident blocks per SM: the register budget of 7 blocks (72 registers) and the grid's cap.  More
// resident warps share L1 among more units and lose B-line hits (8 blocks: 0.355 vs 0.342 ms on
// webbase1m); letting the compiler pick its own budget gave 64 registers and a slower schedule
// with the 8-byte repeat records (0.360 ms), the 7-block bound 0.325 ms (profiles/experiments).
// With packed fp64 B (16-byte entries; B does not fit L2: citpatents, rmat23) 5 blocks (96
// registers) are best: citpatents 0.745 -> 0.707 ms, rmat23 50.2 -> 42.6 ms; packed fp32 B (8-byte
// entries, ab2m) keeps 7 (5 blocks: 0.361 -> 0.387 ms).  profiles/experiments/r02_numeric_blocks_ab.txt
constexpr int NUM_BLOCKS_SM = 7;
constexpr int NUM_BLOCKS_SM_PACKED64 = 5;
template <typename V, bool PACKED> constexpr int num_blocks_sm() {
  return PACKED && sizeof(V) == 8 ? NUM_BLOCKS_SM_PACKED64 : NUM_BLOCKS_SM;
}
constexpr int NUM_BUFW = NUM_SH + 8;   // plan words per staging buffer (16-byte alignment slack)

__device__ __forceinline__ void st_cs(int* p, int v) { __stcs(p, v); }
__device__ __forceinline__ void st_cs(double* p, double v) { __stcs(p, v); }
__device__ __forceinline__ void st_cs(float* p, float v) { __stcs(p, v); }


// ---- TMA (cp.async.bulk) staging of a unit's plan words with an mbarrier ------------------------
__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned long long* bar) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void tma_plan(unsigned* dst, const unsigned* src, unsigned bytes, unsigned long long* bar) {
  asm volatile(
      "fence.proxy.async.shared::cta;\n\t"  // earlier generic reads of dst before the async write
      "mbarrier.arrive.expect_tx.shared::cta.b64 _, [%3], %2;\n\t"
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* bar, unsigned phase) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(smem_u32(bar)),
      "r"(phase)
      : "memory");
}

// Packed B: {column, value} in one 16-byte (fp64) or 8-byte (fp32) record, so an output's B
// gather is one sector instead of two when B does not stay in L2 (rmat23's B is 1.6 GB).
template <typename V> struct PackB;
template <> struct PackB<double> {
  using T = int4;
  __device__ static T make(int c, double v) {
    return make_int4(c, 0, __double2loint(v), __double2hiint(v));
  }
  __device__ static int col(const T& t) { return t.x; }
  __device__ static double val(const T& t) { return __hiloint2double(t.w, t.z); }
};
template <> struct PackB<float> {
  using T = int2;
  __device__ static T make(int c, float v) { return make_int2(c, __float_as_int(v)); }
  __device__ static int col(const T& t) { return t.x; }
  __device__ static float val(const T& t) { return __int_as_float(t.y); }
};

template <typename V>
__global__ void __launch_bounds__(256) k_pack_b(const int* __restrict__ colB, const V* __restrict__ valB, long long n,
                                                typename PackB<V>::T* __restrict__ out) {
  for (long long x = blockIdx.x * (long long)blockDim.x + threadIdx.x; x < n; x += (long long)gridDim.x * blockDim.x)
    out[x] = PackB<V>::make(colB[x], valB[x]);
}

template <typename V, bool PACKED>
__global__ void __launch_bounds__(NUM_NT, (num_blocks_sm<V, PACKED>())) k_numeric(NumProb<V> P) {
  using PB = PackB<V>;
  const typename PB::T* __restrict__ Bp = reinterpret_cast<const typename PB::T*>(P.Bp);
  __shared__ __align__(16) unsigned s_buf[NUM_W][2][NUM_BUFW];
  __shared__ __align__(8) unsigned long long s_bar[NUM_W][2];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const long long nunits = *P.nunits;
  if (lane == 0) {
    mbar_init(&s_bar[w][0]);
    mbar_init(&s_bar[w][1]);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  auto grab = [&]() -> long long {
    long long u = 0;
    if (lane == 0) u = atomicAdd(P.ticket, 1);
    return __shfl_sync(FULL, u, 0);
  };
  // stage the plan words of unit x into buffer b (narrow units; wide ones read the plan
  // directly); returns the word offset of the unit's first word inside the buffer
  auto staged = [](const NumUnit& x) { return !(x.ob & UNIT_WIDE); };
  auto stage = [&](const NumUnit& x, int b) -> int {
    if (!staged(x)) return 0;
    const long long a0 = x.pw & ~3LL, a1 = (x.pw + x.n + 3) & ~3LL;
    if (lane == 0) tma_plan(s_buf[w][b], P.plan + a0, (unsigned)(a1 - a0) * 4u, &s_bar[w][b]);
    return (int)(x.pw - a0);
  };

  long long u = grab();
  if (u >= nunits) return;
  NumUnit cur = P.units[u];
  int cur_sh = stage(cur, 0);
  unsigned phases = 0u;  // bit b: parity of buffer b's next completion
  int cb = 0;
  for (;;) {
    // prefetch the next unit's plan while this one is processed
    const long long un = grab();
    const bool more = un < nunits;
    NumUnit nxt;
    int nxt_sh = 0;
    if (more) {
      nxt = P.units[un];
      nxt_sh = stage(nxt, cb ^ 1);
    }
    const bool wide = cur.ob & UNIT_WIDE;
    const int e0 = cur.e0, n = cur.n;
    // the first 32 repeat records: fetched now, used after the outputs
    int2 rec = make_int2(0, 0);
    if (lane < cur.d) rec = __ldg(P.R + cur.dw + lane);
    // ---- outputs in C order -----------------------------------------------------------------------
    int* __restrict__ ccol = P.ccol + cur.oc;
    V* __restrict__ cval = P.cval + cur.oc;
    const unsigned* pb = s_buf[w][cb] + cur_sh;
    if (!wide) {
      mbar_wait(&s_bar[w][cb], (phases >> cb) & 1u);
      phases ^= 1u << cb;
    }
    // one output: its A entry and B entry from the plan word(s), then the gathers
    auto gather = [&](unsigned er, unsigned qo, int& col, V& prod) {
      const int e = e0 + (int)er;
      const int q = __ldg(P.Tb + e) + (int)qo;
      const V a = __ldg(P.valA + e);
      V b;
      if constexpr (PACKED) {
        const typename PB::T t = __ldg(Bp + q);
        col = PB::col(t);
        b = PB::val(t);
      } else {
        col = __ldg(P.colB + q);
        b = __ldg(P.valB + q);
      }
      prod = a * b;
    };
    if (!wide) {
      // full iterations without predicates, then the ragged tail
      int o00 = lane;
      for (; o00 + 32 * (NUM_U - 1) < n; o00 += 32 * NUM_U) {
        unsigned wd[NUM_U];
#pragma unroll
        for (int x = 0; x < NUM_U; ++x) wd[x] = pb[o00 + 32 * x];
        int col[NUM_U];
        V prod[NUM_U];
#pragma unroll
        for (int x = 0; x < NUM_U; ++x) gather(wd[x] & 0xffffu, wd[x] >> 16, col[x], prod[x]);
#pragma unroll
        for (int x = 0; x < NUM_U; ++x) {
          st_cs(ccol + o00 + 32 * x, col[x]);
          st_cs(cval + o00 + 32 * x, prod[x]);
        }
      }
      if (o00 < n) {  // fewer than 32 NUM_U outputs left: one predicated pass
        int col[NUM_U];
        V prod[NUM_U];
#pragma unroll
        for (int x = 0; x < NUM_U; ++x)
          if (o00 + 32 * x < n) {
            const unsigned wd = pb[o00 + 32 * x];
            gather(wd & 0xffffu, wd >> 16, col[x], prod[x]);
          }
#pragma unroll
        for (int x = 0; x < NUM_U; ++x)
          if (o00 + 32 * x < n) {
            st_cs(ccol + o00 + 32 * x, col[x]);
            st_cs(cval + o00 + 32 * x, prod[x]);
          }
      }
    } else {
      const unsigned* __restrict__ pw = P.plan + cur.pw;
      for (int o = lane; o < n; o += 32) {
        int col;
        V prod;
        gather(__ldcs(pw + 2 * o), __ldcs(pw + 2 * o + 1), col, prod);
        st_cs(ccol + o, col);
        st_cs(cval + o, prod);
      }
    }
    __syncwarp();  // every lane is done with buffer cb, and its stores precede the adds below
    // ---- repeated products landing in this unit's outputs (R records: B entry, A entry relative to
    //      the item, output inside the unit) ------------------------------------------------------
    if (cur.d > 0) {
      constexpr unsigned EM = (1u << REC_EBITS) - 1u;
      auto bval = [&](int q) -> V {
        if constexpr (PACKED) return PB::val(__ldg(Bp + q));
        else return __ldg(P.valB + q);
      };
      if (lane < cur.d)
        atomicAdd(cval + ((unsigned)rec.y >> REC_EBITS), __ldg(P.valA + e0 + (int)((unsigned)rec.y & EM)) * bval(rec.x));
      for (int j = 32 + lane; j < cur.d; j += 32) {
        const int2 x = __ldg(P.R + cur.dw + j);
        atomicAdd(cval + ((unsigned)x.y >> REC_EBITS), __ldg(P.valA + e0 + (int)((unsigned)x.y & EM)) * bval(x.x));
      }
    }
    if (!more) break;
    cur = nxt;
    cur_sh = nxt_sh;
    if (staged(cur)) cb ^= 1;
  }
}

template <typename V>
cudaError_t launch_numeric(cudaStream_t st, int sms, const NumProb<V>& P) {
  // persistent grid: every block of the variant that fits at once
  static int occ[2] = {0, 0};
  const int v = P.Bp ? 1 : 0;
  if (!occ[v]) {
    int nb = 1;
    if (v) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_numeric<V, true>, NUM_NT, 0);
    else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_numeric<V, false>, NUM_NT, 0);
    const int cap = v ? num_blocks_sm<V, true>() : num_blocks_sm<V, false>();
    occ[v] = nb < 1 ? 1 : (nb > cap ? cap : nb);
  }
  const int grid = occ[v] * sms;
  if (v) k_numeric<V, true><<<grid, NUM_NT, 0, st>>>(P);
  else k_numeric<V, false><<<grid, NUM_NT, 0, st>>>(P);
  return cudaGetLastError();
}

template <typename V>
cudaError_t launch_pack_b(cudaStream_t st, int sms, const int* colB, const V* valB, long long n, void* out) {
  if (n <= 0) return cudaSuccess;
  long long g = (n + 255) / 256;
  if (g > (long long)sms * 16) g = (long long)sms * 16;
  k_pack_b<V><<<(int)g, 256, 0, st>>>(colB, valB, n, reinterpret_cast<typename PackB<V>::T*>(out));
  return cudaGetLastError();
}

template cudaError_t launch_numeric<double>(cudaStream_t, int, const NumProb<double>&);
template cudaError_t launch_numeric<float>(cudaStream_t, int, const NumProb<float>&);
template cudaError_t launch_pack_b<double>(cudaStream_t, int, const int*, const double*, long long, void*);
template cudaError_t launch_pack_b<float>(cudaStream_t, int, const int*, const float*, long long, void*);

}  // namespace spg
