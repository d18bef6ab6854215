// tools/microbench_atomics.cu — measures shared/global atomic and plain-access throughput on
// the B200 (design input for the SpGEMM accumulators).  Not product code.
// nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o build/mb_atomics tools/microbench_atomics.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int SMEM_WORDS = 8192;  // 32 KB
constexpr int ITERS = 4096;

__device__ __forceinline__ uint32_t hash32(uint32_t x) {
  x ^= x >> 16; x *= 0x7feb352d; x ^= x >> 15; x *= 0x846ca68b; x ^= x >> 16;
  return x;
}

template <int MODE>
__global__ void __launch_bounds__(1024) k_smem(unsigned long long* out) {
  __shared__ uint32_t s[SMEM_WORDS];
  for (int i = threadIdx.x; i < SMEM_WORDS; i += blockDim.x) s[i] = 0;
  __syncthreads();
  uint32_t h = hash32(threadIdx.x * 7919 + blockIdx.x * 104729);
  uint32_t acc = 0;
  double* sd = reinterpret_cast<double*>(s);
  for (int it = 0; it < ITERS; ++it) {
    h = h * 1664525u + 1013904223u;
    const uint32_t a = (h >> 8) & (SMEM_WORDS - 1);
    if (MODE == 0) { s[a] = h; }                                   // STS
    else if (MODE == 1) { acc += s[a]; }                            // LDS
    else if (MODE == 2) { acc += atomicOr(&s[a], 1u << (h & 31)); } // ATOMS.OR (ret)
    else if (MODE == 3) { atomicOr(&s[a], 1u << (h & 31)); }        // ATOMS.OR (no ret)
    else if (MODE == 4) { acc += atomicCAS(&s[a], 0u, h); }         // ATOMS.CAS
    else if (MODE == 5) { atomicAdd(&s[a], 1u); }                    // ATOMS.ADD
    else if (MODE == 6) { atomicAdd(&sd[a >> 1], 1.0); }             // fp64 add (CAS loop)
    else if (MODE == 7) { atomicAdd(reinterpret_cast<float*>(&s[a]), 1.0f); }  // fp32 add
  }
  __syncthreads();
  if (threadIdx.x == 0) out[blockIdx.x] = acc + s[0];
}

template <int MODE>
__global__ void __launch_bounds__(1024) k_gmem(uint32_t* g, double* gd, size_t words, unsigned long long* out) {
  uint32_t h = hash32(threadIdx.x * 7919 + blockIdx.x * 104729);
  uint32_t acc = 0;
  for (int it = 0; it < ITERS / 4; ++it) {
    h = h * 1664525u + 1013904223u;
    const size_t a = (size_t)(h % words);
    if (MODE == 0) { acc += atomicOr(&g[a], 1u << (h & 31)); }
    else if (MODE == 1) { atomicOr(&g[a], 1u << (h & 31)); }
    else if (MODE == 2) { atomicAdd(&gd[a >> 1], 1.0); }
    else if (MODE == 3) { g[a] = h; }
  }
  if (threadIdx.x == 0) out[blockIdx.x] = acc;
}

int main() {
  int sms;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk;
  cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  unsigned long long* out;
  cudaMalloc(&out, sizeof(unsigned long long) * 4096);
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  const char* sn[] = {"STS", "LDS", "ATOMS.OR ret", "ATOMS.OR noret", "ATOMS.CAS", "ATOMS.ADD", "smem fp64 add",
                      "smem fp32 add"};
  const int blocks = sms * 2;
  auto run = [&](auto kern, const char* name, double ops_per_thread) {
    kern<<<blocks, 1024>>>(out);
    cudaEventRecord(e0);
    kern<<<blocks, 1024>>>(out);
    cudaEventRecord(e1);
    cudaEventSynchronize(e1);
    float ms;
    cudaEventElapsedTime(&ms, e0, e1);
    double ops = (double)blocks * 1024 * ops_per_thread;
    double per_sm_cycle = ops / (ms * 1e-3) / sms / (clk * 1e3);
    printf("%-16s %8.3f ms  %8.2f Gop/s  %6.3f lanes/SM/cycle (at %d MHz nominal)\n", name, ms, ops / ms / 1e6,
           per_sm_cycle, clk / 1000);
  };
  run(k_smem<0>, sn[0], ITERS);
  run(k_smem<1>, sn[1], ITERS);
  run(k_smem<2>, sn[2], ITERS);
  run(k_smem<3>, sn[3], ITERS);
  run(k_smem<4>, sn[4], ITERS);
  run(k_smem<5>, sn[5], ITERS);
  run(k_smem<6>, sn[6], ITERS);
  run(k_smem<7>, sn[7], ITERS);
  for (size_t words : {(size_t)(4 << 20), (size_t)(512 << 20)}) {  // 16 MB (L2) and 2 GB (HBM)
    uint32_t* g;
    cudaMalloc(&g, words * 4);
    cudaMemset(g, 0, words * 4);
    const char* gn[] = {"ATOMG.OR ret", "RED.OR", "RED.ADD.F64", "STG"};
    auto grun = [&](auto kern, const char* name) {
      kern<<<blocks, 1024>>>(g, (double*)g, words, out);
      cudaEventRecord(e0);
      kern<<<blocks, 1024>>>(g, (double*)g, words, out);
      cudaEventRecord(e1);
      cudaEventSynchronize(e1);
      float ms;
      cudaEventElapsedTime(&ms, e0, e1);
      double ops = (double)blocks * 1024 * (ITERS / 4);
      printf("%-16s %5zu MB %8.3f ms  %8.2f Gop/s\n", name, words * 4 >> 20, ms, ops / ms / 1e6);
    };
    grun(k_gmem<0>, gn[0]);
    grun(k_gmem<1>, gn[1]);
    grun(k_gmem<2>, gn[2]);
    grun(k_gmem<3>, gn[3]);
    cudaFree(g);
  }
  cudaError_t e = cudaGetLastError();
  printf("status: %s\n", cudaGetErrorString(e));
  return 0;
}
