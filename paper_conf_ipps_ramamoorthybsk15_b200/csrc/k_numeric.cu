// k_numeric.cu — numeric phase: C(i,j) = sum_k A(i,k)·B(k,j) (Row-Row
// formulation) written as sorted, compacted CSR.
//
// The symbolic phase sorted every item's products by (row, column) and left the plan: for an
// item (a tile of consecutive rows, or one heavy row) with plan region [P0, P0 + f) and outputs
// [o0, o0 + c), plan word P0 + o describes output o0 + o — {e_rel, qoff}: the A entry e0 + e_rel
// and the offset of the B entry inside that entry's B row — and the words from the end of the
// region backwards are the item's repeated products (dups), each with its output in D at the
// same word.
//
// So numeric is a stream in C order (Phase IV of PAPER.md L154-156, "add like-tuples and
// compact", with the sort done once in symbolic).  Persistent warps take work units (NUM_SH
// consecutive outputs of one item) from a queue built in item order at the end of symbolic:
//   outputs   per output one coalesced plan word, the A entry's B-row start Tb[e] and value
//             valA[e] (the item's A entries: L1), the B gather (column and value, L2: B rows are
//             consumed in ascending order), one multiply, two coalesced streaming stores; then
//             hd[t] += 1 (release).
//   repeats   the unit's share of the item's repeated products waits (relaxed polling, no L1
//             invalidation) until hd[t] says every unit of the item has stored — they were
//             dequeued no later than the item's last unit, so they are running or done — then
//             adds a·b into its output with RED.ADD.F64/F32 (the lines are still in L2).
// HBM traffic per output: 4 B of plan read + (4 + sizeof(V)) B of C written; A and B once.
#include "kernels.cuh"

namespace spg {

constexpr int NUM_NT = 256;            // threads per block (8 independent warps)
constexpr int NUM_U = 4;               // outputs per lane in flight

__device__ __forceinline__ void st_cs(int* p, int v) { __stcs(p, v); }
__device__ __forceinline__ void st_cs(double* p, double v) { __stcs(p, v); }
__device__ __forceinline__ void st_cs(float* p, float v) { __stcs(p, v); }

// Release increment: MEMBAR + RED (no L1 invalidation, unlike __threadfence()).
__device__ __forceinline__ void red_release(int* p, int v) {
  asm volatile("red.release.gpu.global.add.s32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ int ld_relaxed(const int* p) {
  int v;
  asm volatile("ld.relaxed.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

template <typename V>
__global__ void __launch_bounds__(NUM_NT) k_numeric(NumProb<V> P) {
  const int lane = threadIdx.x & 31;
  const long long nunits = *P.nunits;
  for (;;) {
    long long u = 0;
    if (lane == 0) u = atomicAdd(P.ticket, 1);
    u = __shfl_sync(FULL, u, 0);
    if (u >= nunits) break;
    const int2 un = P.units[u];
    const int t = un.x, k = un.y;
    // ---- the item ----------------------------------------------------------------------------
    const int r = P.items[t], r2 = P.items[t + 1];
    const long long o0 = P.crow[r];
    const int c = (int)(P.crow[r2] - o0);
    const long long P0 = P.Ro[r];
    const uint8_t cl = P.cls[r];
    const bool wide = (cl & CLS_HEAVY_PATH) && (cl & CLS_WIDE);
    const int e0 = P.rpA[P.row_begin + r];
    const unsigned* __restrict__ plan = P.plan + P0;
    // plan position x -> A entry e, B entry q
    auto decode = [&](long long x, int& e, int& q) {
      unsigned er, qo;
      if (wide) {
        er = __ldcs(plan + 2 * x);
        qo = __ldcs(plan + 2 * x + 1);
      } else {
        const unsigned w = __ldcs(plan + x);
        er = w & 0xffffu;
        qo = w >> 16;
      }
      e = e0 + (int)er;
      q = __ldg(P.Tb + e) + (int)qo;
    };
    int* __restrict__ ccol = P.ccol + o0;
    V* __restrict__ cval = P.cval + o0;

    // ---- outputs [k NUM_SH, ...) in C order ------------------------------------------------
    const int ob = k * NUM_SH, oe = min(c, ob + NUM_SH);
    for (int o00 = ob + lane; o00 < oe; o00 += 32 * NUM_U) {
      int e[NUM_U], q[NUM_U];
#pragma unroll
      for (int x = 0; x < NUM_U; ++x) {
        const int o = o00 + 32 * x;
        q[x] = -1;
        if (o < oe) decode(o, e[x], q[x]);
      }
      int col[NUM_U];
      V a[NUM_U], b[NUM_U];
#pragma unroll
      for (int x = 0; x < NUM_U; ++x)
        if (q[x] >= 0) {
          a[x] = __ldg(P.valA + e[x]);
          col[x] = __ldg(P.colB + q[x]);
          b[x] = __ldg(P.valB + q[x]);
        }
#pragma unroll
      for (int x = 0; x < NUM_U; ++x)
        if (q[x] >= 0) {
          const int o = o00 + 32 * x;
          st_cs(ccol + o, col[x]);
          st_cs(cval + o, a[x] * b[x]);
        }
    }
    // ---- this unit's share of the repeated products ---------------------------------------------
    const int f = (int)((P.Ro[r2] - P0) >> (wide ? 1 : 0));
    if (f > c) {
      const int hs = (c + NUM_SH - 1) / NUM_SH, d = f - c;
      const int jb = (int)((long long)d * k / hs), je = (int)((long long)d * (k + 1) / hs);
      __syncwarp();
      if (lane == 0) {
        red_release(P.hd + t, 1);  // this warp's outputs are in L2 before the count
        if (je > jb) {
          // The adds below are L2 atomics issued only after the loop exits (control dependency;
          // no speculative stores), so they land after every counted unit's outputs.
          const int need = P.epoch * hs;
          while (ld_relaxed(P.hd + t) < need) __nanosleep(100);
        }
      }
      __syncwarp();
      for (int j = jb + lane; j < je; j += 32) {
        const long long x = f - 1 - j;
        int e, q;
        decode(x, e, q);
        const V v = __ldg(P.valA + e) * __ldg(P.valB + q);
        const int o = (int)__ldcs(P.D + P0 + (wide ? 2 * x : x));
        atomicAdd(cval + o, v);
      }
    }
  }
}

template <typename V>
int numeric_occupancy() {
  int nb = 1;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_numeric<V>, NUM_NT, 0);
  return nb < 1 ? 1 : nb;
}

template <typename V>
cudaError_t launch_numeric(cudaStream_t st, int grid, const NumProb<V>& P) {
  if (grid <= 0) return cudaSuccess;
  k_numeric<V><<<grid, NUM_NT, 0, st>>>(P);
  return cudaGetLastError();
}

template int numeric_occupancy<double>();
template int numeric_occupancy<float>();
template cudaError_t launch_numeric<double>(cudaStream_t, int, const NumProb<double>&);
template cudaError_t launch_numeric<float>(cudaStream_t, int, const NumProb<float>&);

}  // namespace spg
