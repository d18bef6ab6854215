// bins.cu — one dispatcher over the class kernels (k_small.cu, k_bitmap.cu).
#include "kernels.cuh"

namespace spg {

template <typename V> size_t small_smem(int, bool);
template <typename V> int small_threads(int);
template <typename V> int small_rows_per_block(int);
template <typename V> cudaError_t small_configure();
template <typename V> int small_occupancy(int, bool);
template <typename V>
cudaError_t small_launch(int, cudaStream_t, int, bool, const Prob<V>&, const int*, const int*);
template <typename V> cudaError_t bitmap_configure();
template <typename V> int bitmap_occupancy(int, bool);
template <typename V>
cudaError_t bitmap_launch(int, cudaStream_t, int, bool, const Prob<V>&, const int*, const int*, long long);

// HEAVY rows (f <= 4096) take the ESC2 kernel for numeric, the bitmap tier for symbolic
static bool is_bitmap(int bin, bool numeric) { return bin_is_bitmap(bin) && !(numeric && bin == BIN_HEAVY); }

template <typename V>
cudaError_t BinLaunch<V>::launch(int bin, cudaStream_t st, int grid, bool numeric, const Prob<V>& P, const int* list,
                                 const int* count, long long N) {
  if (is_bitmap(bin, numeric)) return bitmap_launch<V>(bin, st, grid, numeric, P, list, count, N);
  return small_launch<V>(bin, st, grid, numeric, P, list, count);
}

template <typename V>
int BinLaunch<V>::rows_per_block(int bin) {
  return bin_is_bitmap(bin) ? 1 : small_rows_per_block<V>(bin);
}

template <typename V>
int BinLaunch<V>::max_blocks_per_sm(int bin, bool numeric) {
  return is_bitmap(bin, numeric) ? bitmap_occupancy<V>(bin, numeric) : small_occupancy<V>(bin, numeric);
}

template <typename V>
cudaError_t BinLaunch<V>::configure() {
  cudaError_t e = small_configure<V>();
  if (e != cudaSuccess) return e;
  return bitmap_configure<V>();
}

template <typename V>
cudaError_t BinLaunch<V>::launch_general(cudaStream_t st, int grid, const Prob<V>& P, const int* list,
                                         const int* count, long long N) {
  return bitmap_launch<V>(BIN_HUGE, st, grid, true, P, list, count, N);
}

template struct BinLaunch<double>;
template struct BinLaunch<float>;

}  // namespace spg
