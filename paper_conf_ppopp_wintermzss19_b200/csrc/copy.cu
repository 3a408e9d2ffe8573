// Stage 4 — output matrix and chunk copy (§3.5): "in parallel, we
// iterate over all chunks and copy their data to the newly allocated C.  Each chunk
// uses a complete block of threads to copy data in a coalesced fashion."
//
// A chunk's rows are contiguous in its data and, apart from a shared first / last
// row (supplied by the merged copy, L428), contiguous in C as well, so every chunk is
// a single contiguous copy.  Shared rows copy their merged data from the merge pool.
// B200: one warp per chunk (chunks average a few hundred elements), streaming
// (evict-first) loads and stores since neither side is re-read.
#include <algorithm>
#include <climits>
#include "kernels.cuh"

namespace acs {

// One warp per chunk (or shared row): 8 independent element loads per lane in flight
// (the copy is bound by DRAM latency x bytes in flight, not by instructions).
template <typename T>
__device__ __forceinline__ void warp_copy(const int32_t* __restrict__ scol, const T* __restrict__ sval,
                                          int32_t* __restrict__ dcol, T* __restrict__ dval, int n, int lane) {
#ifndef ACS_COPY_U
#define ACS_COPY_U 8
#endif
  constexpr int U = ACS_COPY_U;
  int i = lane;
  for (; i + 32 * (U - 1) < n; i += 32 * U) {
    int32_t c[U];
    T v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) { c[u] = __ldcs(scol + i + 32 * u); v[u] = __ldcs(sval + i + 32 * u); }
#pragma unroll
    for (int u = 0; u < U; ++u) { __stcs(dcol + i + 32 * u, c[u]); __stcs(dval + i + 32 * u, v[u]); }
  }
  int32_t c[U];
  T v[U];
#pragma unroll
  for (int u = 0; u < U; ++u) {
    if (i + 32 * u < n) { c[u] = __ldcs(scol + i + 32 * u); v[u] = __ldcs(sval + i + 32 * u); }
  }
#pragma unroll
  for (int u = 0; u < U; ++u) {
    if (i + 32 * u < n) { __stcs(dcol + i + 32 * u, c[u]); __stcs(dval + i + 32 * u, v[u]); }
  }
}

#ifndef ACS_COPY_WARPS
#define ACS_COPY_WARPS 8
#endif
constexpr int COPY_WARPS = ACS_COPY_WARPS;

template <typename T>
__global__ void __launch_bounds__(32 * COPY_WARPS, 5) k_copy(CopyArgs a) {   // 5 CTAs per SM: <= 48 registers
  const int64_t x = (int64_t)blockIdx.x * COPY_WARPS + (threadIdx.x >> 5);
  const int lane = threadIdx.x & 31;
  if (x < a.max_chunks) {
    if (x >= *a.total_chunks_dev) return;
    const ChunkDesc d = a.dense[x];
    const int s = (d.flags & 1) ? d.first_count : 0;
    const int e = (d.flags & 2) ? d.count - d.last_count : d.count;
    if (s >= e) return;
    const int dst_row = (d.flags & 1) ? d.first_row + 1 : d.first_row;
    const int64_t dst = a.row_ptr[dst_row];
    warp_copy<T>(a.pool_col + d.data_off + s, reinterpret_cast<const T*>(a.pool_val) + d.data_off + s,
                 a.c_col + dst, reinterpret_cast<T*>(a.c_val) + dst, e - s, lane);
  } else {
    const int64_t i = x - a.max_chunks;
    if (i >= a.nshared) return;
    const SharedRow sh = a.shared[i];
    const int64_t dst = a.row_ptr[sh.row];
    if (sh.merge_off >= 0)
      warp_copy<T>(a.merge_col + sh.merge_off, reinterpret_cast<const T*>(a.merge_val) + sh.merge_off,
                   a.c_col + dst, reinterpret_cast<T*>(a.c_val) + dst, sh.merged, lane);
    else {                               // merged in place in the chunk pool (merge.cu): the first
      const ChunkDesc d0 = a.dense[sh.first_chunk];              // piece's room, then the second's
      const int64_t b0 = d0.data_off + d0.count - d0.last_count;
      const int64_t b1 = a.dense[sh.first_chunk + 1].data_off;
      const int n0 = min(sh.merged, d0.last_count);
      const T* pv = reinterpret_cast<const T*>(a.pool_val);
      T* cv = reinterpret_cast<T*>(a.c_val);
      warp_copy<T>(a.pool_col + b0, pv + b0, a.c_col + dst, cv + dst, n0, lane);
      warp_copy<T>(a.pool_col + b1, pv + b1, a.c_col + dst + n0, cv + dst + n0, sh.merged - n0, lane);
    }
  }
}

void launch_copy(const CopyArgs& a, bool f64, cudaStream_t st) {
  const int64_t items = a.max_chunks + a.nshared;
  if (items <= 0) return;
  const unsigned grid = (unsigned)((items + COPY_WARPS - 1) / COPY_WARPS);
  if (f64) k_copy<double><<<grid, 32 * COPY_WARPS, 0, st>>>(a);
  else k_copy<float><<<grid, 32 * COPY_WARPS, 0, st>>>(a);
}

// min / max of col[0, n) into out[0] / out[1] (set to INT_MAX-ish / 0 first): the B rows a
// row piece of A reaches (acspgemm_multiply_host's input pipeline).
__global__ void k_col_range(const int32_t* __restrict__ col, int64_t n, int32_t* __restrict__ out) {
  int mn = INT_MAX, mx = INT_MIN;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int c = col[i];
    mn = min(mn, c);
    mx = max(mx, c);
  }
  mn = __reduce_min_sync(0xffffffffu, mn);
  mx = __reduce_max_sync(0xffffffffu, mx);
  if ((threadIdx.x & 31) == 0) {
    atomicMin(&out[0], mn);
    atomicMax(&out[1], mx);
  }
}

void launch_col_range(const int32_t* col, int64_t n, int32_t* out, cudaStream_t st) {
  cudaMemsetAsync(out, 0x7F, sizeof(int32_t), st);
  cudaMemsetAsync(out + 1, 0, sizeof(int32_t), st);
  if (n <= 0) return;
  const unsigned grid = (unsigned)std::min<int64_t>((n + 255) / 256, 148 * 4);
  k_col_range<<<grid, 256, 0, st>>>(col, n, out);
}

// Small read-backs go to mapped host memory through the SM (a copy-engine transfer would
// queue behind a large device->host copy running on another stream).
__global__ void k_read_back(const uint32_t* __restrict__ src, volatile uint32_t* dst, int nwords) {
  const int i = threadIdx.x;
  if (i < nwords) dst[i] = src[i];
}

void launch_read_back(const void* src, void* mapped_dst, int nbytes, cudaStream_t st) {
  const int nw = (nbytes + 3) / 4;
  k_read_back<<<1, 32 * ((nw + 31) / 32), 0, st>>>(static_cast<const uint32_t*>(src),
                                                   static_cast<uint32_t*>(mapped_dst), nw);
}

__global__ void k_read_back2(const uint32_t* __restrict__ src1, volatile uint32_t* dst1, int n1,
                             const uint32_t* __restrict__ src2, volatile uint32_t* dst2, int n2) {
  const int i = threadIdx.x;
  if (i < n1) dst1[i] = src1[i];
  if (i < n2) dst2[i] = src2[i];
}

void launch_read_back2(const void* src1, void* dst1, int nbytes1, const void* src2, void* dst2, int nbytes2,
                       cudaStream_t st) {
  const int n1 = (nbytes1 + 3) / 4, n2 = (nbytes2 + 3) / 4, nw = n1 > n2 ? n1 : n2;
  k_read_back2<<<1, 32 * ((nw + 31) / 32), 0, st>>>(static_cast<const uint32_t*>(src1), static_cast<uint32_t*>(dst1),
                                                    n1, static_cast<const uint32_t*>(src2),
                                                    static_cast<uint32_t*>(dst2), n2);
}

__global__ void k_copy_offset(int32_t* __restrict__ dst, const int32_t* __restrict__ src, int64_t n, int32_t off) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    dst[i] = src[i] + off;
}

void launch_copy_offset(int32_t* dst, const int32_t* src, int64_t n, int32_t off, cudaStream_t st) {
  if (n <= 0) return;
  const unsigned grid = (unsigned)std::min<int64_t>((n + 255) / 256, 148 * 8);
  k_copy_offset<<<grid, 256, 0, st>>>(dst, src, n, off);
}

// src == nullptr: dst[i] = off (the row pointers of an empty product)
template <typename I>
__global__ void k_rowptr_out(I* __restrict__ dst, const int64_t* __restrict__ src, int64_t n, I off) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    dst[i] = (src ? (I)src[i] : (I)0) + off;
}

void launch_rowptr_out(int32_t* dst, const int64_t* src, int64_t n, int32_t off, cudaStream_t st) {
  if (n <= 0) return;
  const unsigned grid = (unsigned)std::min<int64_t>((n + 255) / 256, 148 * 8);
  k_rowptr_out<int32_t><<<grid, 256, 0, st>>>(dst, src, n, off);
}

void launch_rowptr_out(int64_t* dst, const int64_t* src, int64_t n, int64_t off, cudaStream_t st) {
  if (n <= 0) return;
  const unsigned grid = (unsigned)std::min<int64_t>((n + 255) / 256, 148 * 8);
  k_rowptr_out<int64_t><<<grid, 256, 0, st>>>(dst, src, n, off);
}

__global__ void k_add_offset(int32_t* __restrict__ p, int64_t n, int32_t off) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    p[i] += off;
}

void launch_add_offset(int32_t* p, int64_t n, int32_t off, cudaStream_t st) {
  if (n <= 0 || off == 0) return;
  const unsigned grid = (unsigned)std::min<int64_t>((n + 255) / 256, 148 * 8);
  k_add_offset<<<grid, 256, 0, st>>>(p, n, off);
}

}  // namespace acs
