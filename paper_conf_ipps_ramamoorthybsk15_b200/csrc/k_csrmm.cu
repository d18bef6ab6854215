// k_csrmm.cu — sparse x dense C = A x D, the CSTMM / csrmm extension the paper names as future
// work (§VI), with the same "right work to the right processor" split as the
// SpGEMM: C(i,:) = sum_k A(i,k) D(k,:) (Row-Row).
//
//   light rows (<= light_nnz stored entries): one warp per row.  The warp loads 32 of the row's
//     entries at once (coalesced) and broadcasts them with shuffles; each lane owns columns
//     lane, lane + 32, ... of a 32·CSRMM_CPT-column chunk, so every D row is read coalesced.
//   heavy rows: one block per row (from a list the light kernel appends to).  Its warps split
//     the row's entries, each accumulates the chunk's columns, and the partial rows are summed
//     in shared memory — a long row no longer serialises on one warp.
// D and C are dense row-major (leading dimensions ldd, ldc).  HBM-bound when n is small, D-reuse
// (L2) bound when it is large; no tensor cores (a sparse left operand is not a dense contraction).
#include "kernels.cuh"

namespace spg {

constexpr int CSRMM_NT = 256;
constexpr int CSRMM_CPT = 4;   // columns per lane per chunk
constexpr int CSRMM_W = CSRMM_NT / 32;

template <typename V>
__global__ void __launch_bounds__(CSRMM_NT) k_csrmm_light(int M, const int* __restrict__ rpA,
                                                         const int* __restrict__ colA, const V* __restrict__ valA,
                                                         const V* __restrict__ D, long long ldd, int n,
                                                         V* __restrict__ C, long long ldc, int light_nnz,
                                                         int* __restrict__ hlist, int* __restrict__ hcount) {
  const int lane = threadIdx.x & 31;
  const long long nw = (long long)gridDim.x * CSRMM_W;
  for (long long i = (long long)blockIdx.x * CSRMM_W + (threadIdx.x >> 5); i < M; i += nw) {
    const int p0 = rpA[i], p1 = rpA[i + 1];
    if (p1 - p0 > light_nnz) {
      if (lane == 0) hlist[atomicAdd(hcount, 1)] = (int)i;
      continue;
    }
    for (int c0 = 0; c0 < n; c0 += 32 * CSRMM_CPT) {
      V acc[CSRMM_CPT];
#pragma unroll
      for (int x = 0; x < CSRMM_CPT; ++x) acc[x] = V(0);
      for (int pb = p0; pb < p1; pb += 32) {
        const int cnt = min(32, p1 - pb);
        int k = 0;
        V a = V(0);
        if (lane < cnt) {
          k = colA[pb + lane];
          a = valA[pb + lane];
        }
        for (int t = 0; t < cnt; ++t) {
          const long long kk = __shfl_sync(FULL, k, t);
          const V aa = __shfl_sync(FULL, a, t);
          const V* __restrict__ d = D + kk * ldd;
#pragma unroll
          for (int x = 0; x < CSRMM_CPT; ++x) {
            const int col = c0 + lane + 32 * x;
            if (col < n) acc[x] += aa * __ldg(d + col);
          }
        }
      }
#pragma unroll
      for (int x = 0; x < CSRMM_CPT; ++x) {
        const int col = c0 + lane + 32 * x;
        if (col < n) C[i * ldc + col] = acc[x];
      }
    }
  }
}

template <typename V>
__global__ void __launch_bounds__(CSRMM_NT) k_csrmm_heavy(const int* __restrict__ rpA, const int* __restrict__ colA,
                                                         const V* __restrict__ valA, const V* __restrict__ D,
                                                         long long ldd, int n, V* __restrict__ C, long long ldc,
                                                         const int* __restrict__ hlist, const int* __restrict__ hcount) {
  __shared__ V part[CSRMM_W][32 * CSRMM_CPT];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int nh = *hcount;
  for (int h = blockIdx.x; h < nh; h += gridDim.x) {
    const long long i = hlist[h];
    const int p0 = rpA[i], p1 = rpA[i + 1];
    for (int c0 = 0; c0 < n; c0 += 32 * CSRMM_CPT) {
      V acc[CSRMM_CPT];
#pragma unroll
      for (int x = 0; x < CSRMM_CPT; ++x) acc[x] = V(0);
      // warp w takes the 32-entry groups w, w + W, ... of the row
      for (int pb = p0 + 32 * w; pb < p1; pb += 32 * CSRMM_W) {
        const int cnt = min(32, p1 - pb);
        int k = 0;
        V a = V(0);
        if (lane < cnt) {
          k = colA[pb + lane];
          a = valA[pb + lane];
        }
        for (int t = 0; t < cnt; ++t) {
          const long long kk = __shfl_sync(FULL, k, t);
          const V aa = __shfl_sync(FULL, a, t);
          const V* __restrict__ d = D + kk * ldd;
#pragma unroll
          for (int x = 0; x < CSRMM_CPT; ++x) {
            const int col = c0 + lane + 32 * x;
            if (col < n) acc[x] += aa * __ldg(d + col);
          }
        }
      }
#pragma unroll
      for (int x = 0; x < CSRMM_CPT; ++x) part[w][lane + 32 * x] = acc[x];
      __syncthreads();
      for (int c = threadIdx.x; c < 32 * CSRMM_CPT; c += CSRMM_NT) {
        V s = V(0);
#pragma unroll
        for (int y = 0; y < CSRMM_W; ++y) s += part[y][c];
        if (c0 + c < n) C[i * ldc + c0 + c] = s;
      }
      __syncthreads();
    }
  }
}

template <typename V>
cudaError_t launch_csrmm(cudaStream_t st, int sms, int M, const int* rpA, const int* colA, const void* valA,
                         const void* D, long long ldd, int n, void* C, long long ldc, int light_nnz, int* hlist,
                         int* hcount) {
  if (M <= 0 || n <= 0) return cudaSuccess;
  cudaError_t e = cudaMemsetAsync(hcount, 0, sizeof(int), st);
  if (e != cudaSuccess) return e;
  long long g = ((long long)M + CSRMM_W - 1) / CSRMM_W;
  if (g > (long long)sms * 16) g = (long long)sms * 16;
  k_csrmm_light<V><<<(int)g, CSRMM_NT, 0, st>>>(M, rpA, colA, (const V*)valA, (const V*)D, ldd, n, (V*)C, ldc,
                                                light_nnz, hlist, hcount);
  k_csrmm_heavy<V><<<sms * 4, CSRMM_NT, 0, st>>>(rpA, colA, (const V*)valA, (const V*)D, ldd, n, (V*)C, ldc, hlist,
                                               hcount);
  return cudaGetLastError();
}

template cudaError_t launch_csrmm<double>(cudaStream_t, int, int, const int*, const int*, const void*, const void*,
                                          long long, int, void*, long long, int, int*, int*);
template cudaError_t launch_csrmm<float>(cudaStream_t, int, int, const int*, const int*, const void*, const void*,
                                         long long, int, void*, long long, int, int*, int*);

}  // namespace spg
