// Device-wide exclusive prefix sums (integer, so the result is order independent).
// Used for the row-pointer array of C ("A device-wide prefix sum over the row counts
// yields the row pointer array and C's memory requirement", §3.5), for
// the deterministic chunk-pool offsets, the dense chunk order and the merge packing.
// One kernel per scan (decoupled look-back, below).
#include "kernels.cuh"

namespace acs {

constexpr int SCAN_ITEMS = 8;
constexpr int SCAN_TILE = THREADS * SCAN_ITEMS;

int64_t scan_tmp_elems(int64_t n) { return (n + SCAN_TILE - 1) / SCAN_TILE + 2; }

// One pass (decoupled look-back): a CTA takes the next tile number from a ticket
// counter (so every tile it waits for belongs to a CTA that is already running), posts its
// tile sum, and warp 0 walks back over the predecessors' posts -- a tile sum (state 1) or
// the inclusive prefix (state 2) -- until an inclusive prefix ends the walk.  Integer sums,
// so the result does not depend on which posts a tile happens to see.  The last CTA to
// finish (done counter) clears the posts and both counters, so `tmp` is all zero between
// scans: no memset launch, and a captured graph replays the same kernels.
//   tmp[0] = ticket counter, tmp[1] = done counter, tmp[2 + t] = post of tile t
//   post = state << 62 | value (sums are < 2^62).
constexpr unsigned long long POST_AGG = 1ull << 62, POST_INC = 2ull << 62, POST_VAL = (1ull << 62) - 1;

__device__ __forceinline__ unsigned long long load_post(const unsigned long long* p) {
  return *reinterpret_cast<const volatile unsigned long long*>(p);
}
__device__ __forceinline__ void store_post(unsigned long long* p, unsigned long long v) {
  *reinterpret_cast<volatile unsigned long long*>(p) = v;
}

template <typename In, typename Out>
__global__ void __launch_bounds__(THREADS) k_scan(const In* __restrict__ in, Out* __restrict__ out, int64_t n,
                                                  int64_t ntiles, int64_t* __restrict__ total_dev,
                                                  unsigned long long* __restrict__ tmp, bool write_total) {
  __shared__ int64_t scratch[THREADS / 32 + 1];
  __shared__ int64_t s_tile, s_excl;
  __shared__ int s_last;
  if (threadIdx.x == 0) s_tile = (int64_t)atomicAdd(&tmp[0], 1ull);
  __syncthreads();
  const int64_t tile = s_tile;
  unsigned long long* post = tmp + 2;
  const int64_t base = tile * SCAN_TILE + (int64_t)threadIdx.x * SCAN_ITEMS;
  int64_t v[SCAN_ITEMS];
  int64_t s = 0;
#pragma unroll
  for (int i = 0; i < SCAN_ITEMS; ++i) {
    const int64_t idx = base + i;
    v[i] = idx < n ? (int64_t)in[idx] : 0;
    s += v[i];
  }
  int64_t total;
  const int64_t ex = block_exclusive_sum<int64_t>(s, scratch, &total);
  if (threadIdx.x < 32) {
    const int lane = threadIdx.x;
    int64_t excl = 0;
    if (tile == 0) {
      if (lane == 0) store_post(&post[0], POST_INC | (unsigned long long)total);
    } else {
      if (lane == 0) store_post(&post[tile], POST_AGG | (unsigned long long)total);
      int64_t j = tile - 1 - lane;           // this lane's predecessor in the current window
      while (true) {
        unsigned long long w = j >= 0 ? load_post(&post[j]) : POST_INC;
        // wait until every predecessor of the window has posted something
        while (__any_sync(0xffffffffu, (w >> 62) == 0)) {
          if ((w >> 62) == 0) w = load_post(&post[j]);
        }
        const unsigned inc = __ballot_sync(0xffffffffu, (w >> 62) == 2);
        // lanes up to (and including) the nearest inclusive prefix contribute
        const int stop = inc ? __ffs(inc) - 1 : 31;
        int64_t add = lane <= stop && j >= 0 ? (int64_t)(w & POST_VAL) : 0;
#pragma unroll
        for (int d = 16; d > 0; d >>= 1) add += __shfl_xor_sync(0xffffffffu, add, d);
        excl += add;
        if (inc) break;
        j -= 32;
      }
      if (lane == 0) store_post(&post[tile], POST_INC | (unsigned long long)(excl + total));
    }
    if (lane == 0) s_excl = excl;
  }
  __syncthreads();
  int64_t run = s_excl + ex;
#pragma unroll
  for (int i = 0; i < SCAN_ITEMS; ++i) {
    const int64_t idx = base + i;
    if (idx < n) out[idx] = (Out)run;
    run += v[i];
  }
  if (tile == ntiles - 1 && threadIdx.x == 0) {
    *total_dev = s_excl + total;
    if (write_total) out[n] = (Out)(s_excl + total);
  }
  // the last CTA to finish clears the posts: every other CTA has finished its walk
  if (threadIdx.x == 0) {
    __threadfence();
    s_last = atomicAdd(&tmp[1], 1ull) == (unsigned long long)(ntiles - 1);
  }
  __syncthreads();
  if (s_last) {
    __threadfence();
    for (int64_t t = threadIdx.x; t < ntiles; t += THREADS) post[t] = 0;
    if (threadIdx.x == 0) { tmp[0] = 0; tmp[1] = 0; }
  }
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
  k_scan<In, Out><<<(unsigned)ntiles, THREADS, 0, st>>>(in, out, n, ntiles, total_dev,
                                                        reinterpret_cast<unsigned long long*>(tmp), write_total);
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
