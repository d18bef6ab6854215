// tools/microbench_cstore.cu — how fast can a numeric SpGEMM kernel write C on the B200?
// Design input for the product-order numeric; not product code.
//
// Every variant writes nnz = 70M outputs (int32 column + fp64 value, 840 MB, like webbase1m's
// C) from warps that own windows of WIN consecutive outputs:
//   0 coalesced plain stores                       (the floor: pure write bandwidth)
//   1 plain stores, positions permuted within SPAN-output blocks (a row's products visited in
//     product order land at their ranks: scattered inside the row's C range)
//   2 zero-fill the window's values, __syncwarp, then RED.ADD.F64 at permuted positions
//     (dup-bearing rows: every product adds, no first/dup distinction)
//   3 as 2 with every output hit by two products (two REDs per output, half the values each)
//   4 plain stores permuted + a u16 plan read per output (coalesced) + a B gather from a
//     41 MB table (L2-resident): the whole numeric inner loop without the A side
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o build/mb_cstore tools/microbench_cstore.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int WIN = 2048;
constexpr int SPAN = 128;

__device__ __forceinline__ unsigned perm(unsigned i) {  // bijection on [0, SPAN)
  return (i * 37u + 11u) & (SPAN - 1);
}

template <int MODE>
__global__ void __launch_bounds__(256) k_store(int* __restrict__ col, double* __restrict__ val, long long n,
                                               const unsigned short* __restrict__ plan,
                                               const double* __restrict__ tab, int tabn) {
  const int lane = threadIdx.x & 31;
  const long long warp = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const long long nwarps = ((long long)gridDim.x * blockDim.x) >> 5;
  for (long long w0 = warp * WIN; w0 < n; w0 += nwarps * WIN) {
    const int len = (int)(n - w0 < WIN ? n - w0 : WIN);
    if (MODE == 2 || MODE == 3) {
      for (int i = lane; i < len; i += 32) val[w0 + i] = 0.0;
      __syncwarp();
    }
    const int reps = MODE == 3 ? 2 : 1;
    for (int r = 0; r < reps; ++r)
#pragma unroll 4
      for (int i = lane; i < len; i += 32) {
        long long p = w0 + i;
        if (MODE != 0 && len == WIN) p = w0 + (i & ~(SPAN - 1)) + perm(i & (SPAN - 1));
        double v = (double)(p & 1023);
        if (MODE == 4) {
          const unsigned pl = __ldcs(plan + w0 + i);
          v += __ldg(tab + ((p * 2654435761ull + pl) % (unsigned long long)tabn));
        }
        if (MODE == 2 || MODE == 3) {
          atomicAdd(val + p, MODE == 3 ? 0.5 * v : v);
          col[p] = (int)(p & 0x7fffffff);
        } else {
          __stcs(val + p, v);
          __stcs(col + p, (int)(p & 0x7fffffff));
        }
      }
  }
}

#define CK(x)                                                              \
  do {                                                                     \
    cudaError_t e = (x);                                                   \
    if (e != cudaSuccess) {                                                \
      printf("%s: %s\n", #x, cudaGetErrorString(e));                       \
      return 1;                                                            \
    }                                                                      \
  } while (0)

template <int MODE>
float run(int grid, int* col, double* val, long long n, const unsigned short* plan, const double* tab, int tabn,
          char* flush, size_t flush_bytes) {
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  float best = 1e30f;
  for (int it = 0; it < 6; ++it) {
    cudaMemset(flush, it, flush_bytes);  // evict C from L2 between repetitions
    cudaEventRecord(a);
    k_store<MODE><<<grid, 256>>>(col, val, n, plan, tab, tabn);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    if (it > 0 && ms < best) best = ms;
  }
  return best;
}

int main() {
  const long long n = 70000000;
  const int tabn = 41 * 1024 * 1024 / 8;
  int* col;
  double* val;
  unsigned short* plan;
  double* tab;
  char* flush;
  const size_t flush_bytes = 256u << 20;
  CK(cudaMalloc(&col, n * 4));
  CK(cudaMalloc(&val, n * 8));
  CK(cudaMalloc(&plan, n * 2));
  CK(cudaMalloc(&tab, (size_t)tabn * 8));
  CK(cudaMalloc(&flush, flush_bytes));
  CK(cudaMemset(plan, 1, n * 2));
  CK(cudaMemset(tab, 0, (size_t)tabn * 8));
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const double bytes = (double)n * 12.0;
  const char* names[] = {"coalesced stores", "permuted stores (128-span)", "zero-fill + RED permuted",
                         "zero-fill + 2x RED permuted", "permuted stores + u16 plan + L2 gather"};
  for (int occ : {4, 8}) {
    const int grid = sms * occ;
    float t[5];
    t[0] = run<0>(grid, col, val, n, plan, tab, tabn, flush, flush_bytes);
    t[1] = run<1>(grid, col, val, n, plan, tab, tabn, flush, flush_bytes);
    t[2] = run<2>(grid, col, val, n, plan, tab, tabn, flush, flush_bytes);
    t[3] = run<3>(grid, col, val, n, plan, tab, tabn, flush, flush_bytes);
    t[4] = run<4>(grid, col, val, n, plan, tab, tabn, flush, flush_bytes);
    for (int m = 0; m < 5; ++m)
      printf("grid %4d  %-42s %8.1f us  %7.0f GB/s (C bytes)\n", grid, names[m], t[m] * 1e3, bytes / (t[m] * 1e6));
  }
  CK(cudaGetLastError());
  return 0;
}
