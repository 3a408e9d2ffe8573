// Device-wide exclusive prefix sums (integer, so the result is order independent).
// Used for the row-pointer array of C ("A device-wide prefix sum over the row counts
// yields the row pointer array and C's memory requirement", §3.5), for
// the deterministic chunk-pool offsets, the dense chunk order and the merge packing.
// Three phases: tile sums, one-CTA scan of the tile sums, tile-local scan + offset.
#include "kernels.cuh"

namespace acs {

constexpr int SCAN_ITEMS = 8;
constexpr int SCAN_TILE = THREADS * SCAN_ITEMS;

int64_t scan_tmp_elems(int64_t n) { return (n + SCAN_TILE - 1) / SCAN_TILE + 2; }

template <typename In>
__global__ void __launch_bounds__(THREADS) k_tile_sums(const In* __restrict__ in, int64_t n, int64_t* __restrict__ tile_sum) {
  __shared__ int64_t scratch[THREADS / 32 + 1];
  const int64_t base = (int64_t)blockIdx.x * SCAN_TILE;
  int64_t s = 0;
#pragma unroll
  for (int i = 0; i < SCAN_ITEMS; ++i) {
    const int64_t idx = base + (int64_t)i * THREADS + threadIdx.x;
    if (idx < n) s += (int64_t)in[idx];
  }
  int64_t total;
  block_exclusive_sum<int64_t>(s, scratch, &total);
  if (threadIdx.x == 0) tile_sum[blockIdx.x] = total;
}

__global__ void __launch_bounds__(THREADS) k_scan_tiles(int64_t* __restrict__ tile_sum, int64_t ntiles,
                                                        int64_t* __restrict__ total_dev) {
  __shared__ int64_t scratch[THREADS / 32 + 1];
  int64_t carry = 0;
  for (int64_t base = 0; base < ntiles; base += THREADS) {
    const int64_t idx = base + threadIdx.x;
    const int64_t v = idx < ntiles ? tile_sum[idx] : 0;
    int64_t total;
    const int64_t ex = block_exclusive_sum<int64_t>(v, scratch, &total);
    if (idx < ntiles) tile_sum[idx] = carry + ex;
    carry += total;
  }
  if (threadIdx.x == 0 && total_dev) *total_dev = carry;
}

template <typename In, typename Out>
__global__ void __launch_bounds__(THREADS) k_scan_apply(const In* __restrict__ in, Out* __restrict__ out, int64_t n,
                                                        const int64_t* __restrict__ tile_off, const int64_t* __restrict__ total_dev,
                                                        bool write_total) {
  __shared__ int64_t scratch[THREADS / 32 + 1];
  const int64_t base = (int64_t)blockIdx.x * SCAN_TILE + (int64_t)threadIdx.x * SCAN_ITEMS;
  int64_t v[SCAN_ITEMS];
  int64_t s = 0;
#pragma unroll
  for (int i = 0; i < SCAN_ITEMS; ++i) {
    const int64_t idx = base + i;
    v[i] = idx < n ? (int64_t)in[idx] : 0;
    s += v[i];
  }
  int64_t total;
  int64_t run = tile_off[blockIdx.x] + block_exclusive_sum<int64_t>(s, scratch, &total);
#pragma unroll
  for (int i = 0; i < SCAN_ITEMS; ++i) {
    const int64_t idx = base + i;
    if (idx < n) out[idx] = (Out)run;
    run += v[i];
  }
  if (write_total && blockIdx.x == 0 && threadIdx.x == 0) out[n] = (Out)(*total_dev);
}

template <typename In, typename Out>
static void scan_impl(const In* in, Out* out, int64_t n, int64_t* total_dev, int64_t* tmp, bool write_total,
                      cudaStream_t st) {
  if (n <= 0) {
    cudaMemsetAsync(total_dev, 0, sizeof(int64_t), st);
    if (write_total) cudaMemsetAsync(out, 0, sizeof(Out), st);
    return;
  }
  const int64_t ntiles = (n + SCAN_TILE - 1) / SCAN_TILE;
  k_tile_sums<In><<<(unsigned)ntiles, THREADS, 0, st>>>(in, n, tmp);
  k_scan_tiles<<<1, THREADS, 0, st>>>(tmp, ntiles, total_dev);
  k_scan_apply<In, Out><<<(unsigned)ntiles, THREADS, 0, st>>>(in, out, n, tmp, total_dev, write_total);
}

void launch_scan_i64(const int64_t* in, int64_t* out, int64_t n, int64_t* total_dev, int64_t* tmp, cudaStream_t st) {
  scan_impl<int64_t, int64_t>(in, out, n, total_dev, tmp, false, st);
}
void launch_scan_i32(const int32_t* in, int64_t* out, int64_t n, int64_t* total_dev, int64_t* tmp, cudaStream_t st) {
  scan_impl<int32_t, int64_t>(in, out, n, total_dev, tmp, false, st);
}
void launch_scan_rowptr(const int32_t* in, int64_t* row_ptr, int64_t n, int64_t* total_dev, int64_t* tmp,
                        cudaStream_t st) {
  scan_impl<int32_t, int64_t>(in, row_ptr, n, total_dev, tmp, true, st);
}

}  // namespace acs
