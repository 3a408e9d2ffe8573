// Stage 4 — output matrix and chunk copy (§3.5): "in parallel, we
// iterate over all chunks and copy their data to the newly allocated C.  Each chunk
// uses a complete block of threads to copy data in a coalesced fashion."
//
// A chunk's rows are contiguous in its data and, apart from a shared first / last
// row (supplied by the merged copy, L428), contiguous in C as well, so every chunk is
// a single contiguous copy.  Shared rows copy their merged data from the merge pool.
#include "kernels.cuh"

namespace acs {

template <typename T>
__device__ __forceinline__ void block_copy(const int32_t* __restrict__ scol, const T* __restrict__ sval,
                                           int32_t* __restrict__ dcol, T* __restrict__ dval, int n) {
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    dcol[i] = scol[i];
    dval[i] = sval[i];
  }
}

template <typename T>
__global__ void __launch_bounds__(256) k_copy(CopyArgs a) {
  const int64_t x = blockIdx.x;
  if (x < a.max_chunks) {
    if (x >= *a.total_chunks_dev) return;
    const ChunkDesc d = a.dense[x];
    const int s = (d.flags & 1) ? d.first_count : 0;
    const int e = (d.flags & 2) ? d.count - d.last_count : d.count;
    if (s >= e) return;
    const int dst_row = (d.flags & 1) ? d.first_row + 1 : d.first_row;
    const int64_t dst = a.row_ptr[dst_row];
    block_copy<T>(a.pool_col + d.data_off + s, reinterpret_cast<const T*>(a.pool_val) + d.data_off + s,
                  a.c_col + dst, reinterpret_cast<T*>(a.c_val) + dst, e - s);
  } else {
    const int64_t i = x - a.max_chunks;
    if (i >= a.nshared) return;
    const SharedRow sh = a.shared[i];
    const int64_t dst = a.row_ptr[sh.row];
    block_copy<T>(a.merge_col + sh.merge_off, reinterpret_cast<const T*>(a.merge_val) + sh.merge_off,
                  a.c_col + dst, reinterpret_cast<T*>(a.c_val) + dst, sh.merged);
  }
}

void launch_copy(const CopyArgs& a, bool f64, cudaStream_t st) {
  const int64_t grid = a.max_chunks + a.nshared;
  if (grid <= 0) return;
  if (f64) k_copy<double><<<(unsigned)grid, 256, 0, st>>>(a);
  else k_copy<float><<<(unsigned)grid, 256, 0, st>>>(a);
}

}  // namespace acs
