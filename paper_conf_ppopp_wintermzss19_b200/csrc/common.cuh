// Shared constants, data structures and block/warp primitives of the AC-SpGEMM
// CUDA path (sm_100a).  Nothing here is shared with oracle/ (the test oracle).
//
// Tile constants (§4: "sorts 8 elements per thread and keeps up
// to 4 elements per thread"; "256/512 non-zeros" per block for global load
// balancing).  They are fixed per build: they decide the summation tree and hence
// the bits of every result (reading R7 in DESIGN.md).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace acs {

#ifndef ACS_THREADS
#define ACS_THREADS 128
#endif
#ifndef ACS_ITEMS
#define ACS_ITEMS 16
#endif
#ifndef ESC_MIN_BLOCKS
#define ESC_MIN_BLOCKS (ACS_THREADS == 256 ? 3 : 4)
#endif
constexpr int THREADS = ACS_THREADS;         // threads per CTA (paper: 256, L344)
constexpr int ITEMS = ACS_ITEMS;             // sorted elements per thread (paper: 8, L556)
constexpr int CAP = THREADS * ITEMS;         // products per local ESC iteration (2048)
constexpr int IDXBITS = 31 - __builtin_clz(CAP); // log2(CAP): position bits in a sort word
constexpr int NPB = 512;                     // NNZ_PER_BLOCK (Alg. 1, Alg. 2; L556 "256/512")
constexpr int NNZ_PER_THREAD = NPB / THREADS;// A entries per thread
#ifndef ACS_KEEP_PER_THREAD
#define ACS_KEEP_PER_THREAD 4
#endif
constexpr int KEEP_PER_THREAD = ACS_KEEP_PER_THREAD; // "keeps up to 4 elements per thread" (L556)
constexpr int CAP_SMALL = 512;               // small-tile AC-ESC (esc_small.cu, reading R32)
constexpr int KEEP = KEEP_PER_THREAD * THREADS; // max kept elements of the last row
#ifndef ACS_RADIX_BITS
#define ACS_RADIX_BITS 5
#endif
constexpr int RADIX_BITS = ACS_RADIX_BITS;   // digit width of one radix-sort pass
constexpr int DEFAULT_SEGMENTS = 8;          // canonical segments
constexpr int MAX_SEGMENTS = 64;
constexpr int PATH_MAX_CHUNKS = 32;          // Path Merge limit (reading R12)
// long rows (§3.4): an entry whose B row has more than PTR_LEN entries becomes
// its own chunk (a·B_k, no sort); at most PTR_MAX such entries per block
#ifndef ACS_PTR_LEN
#define ACS_PTR_LEN (ACS_THREADS * ACS_ITEMS)
#endif
constexpr int PTR_LEN = ACS_PTR_LEN;
constexpr int PTR_MAX = 160;
constexpr int SEARCH_MAXP = 1024;            // Search Merge limit; longer chunk lists: dense slices (R30)
#ifndef ACS_GIANT_SLICE
#define ACS_GIANT_SLICE 8192
#endif
constexpr int GIANT_SLICE = ACS_GIANT_SLICE;  // columns of a dense slice (one accumulator)
#ifndef ACS_DENSE_SPAN_RATIO
#define ACS_DENSE_SPAN_RATIO 16
#endif
constexpr int DENSE_SPAN_RATIO = ACS_DENSE_SPAN_RATIO;  // dense slices when span <= 16 x pre-merge elements
#ifndef ACS_PAIR_MAX
#define ACS_PAIR_MAX 512
#endif
constexpr int PAIR_MAX = ACS_PAIR_MAX;     // two-chunk rows up to this many elements: one warp each (k_pair_merge)
// hash accumulator (hash.cu, reading R31)
#ifndef ACS_HASH_WARPS
#define ACS_HASH_WARPS 4
#endif
constexpr int HASH_WARPS = ACS_HASH_WARPS;   // warps per CTA; each emits one chunk per block
constexpr int ACC_MAX_WARPS = 8;             // most warps (= chunks) an accumulator uses per block (k_dict)
static_assert(HASH_WARPS <= ACC_MAX_WARPS, "chunk slots per block (k_block_bounds)");
constexpr int HASH_THREADS = 32 * HASH_WARPS;
#ifndef ACS_HASH_T
#define ACS_HASH_T 512
#endif
constexpr int HASH_T = ACS_HASH_T;           // table slots per warp (a multiple of 32)
constexpr int HASH_UMAX = HASH_T / 2;        // max distinct columns of a row (load <= 1/2)
#ifndef ACS_HASH_UBOUND
#define ACS_HASH_UBOUND 192
#endif
// POOL_BOUND (reading R40): an accumulator row's output cap, so a candidate block's region
// is sum min(row products, HASH_UBOUND); a row with more distinct columns sends its block
// to AC-ESC (deferred, exact region) in that mode only
constexpr int HASH_UBOUND = ACS_HASH_UBOUND;
static_assert(HASH_UBOUND <= HASH_UMAX, "the bound cap cannot exceed the table's row limit");
#ifndef ACS_HASH_PROWMAX
#define ACS_HASH_PROWMAX 2048
#endif
constexpr int HASH_PROWMAX = ACS_HASH_PROWMAX; // blocks with a longer row (in products) go to AC-ESC
#ifndef HASH_MIN_BLOCKS
#define HASH_MIN_BLOCKS 5
#endif                // two-chunk rows up to this size: warp merge
static_assert((1 << IDXBITS) == CAP, "IDXBITS must be log2(CAP)");
static_assert(KEEP <= CAP / 2, "kept row must leave room for new products");
static_assert(NPB % THREADS == 0, "NPB must be a multiple of THREADS");

// A chunk of C (§3.2.4: "each chunk holds its starting row, element
// count and number of elements in the first and last row"; the chunk id (block,
// running number) gives the global order, L430).  Column indices and values live in
// the pool arrays at [data_off, data_off + count).
struct ChunkDesc {
  int64_t data_off;
  int32_t first_row, last_row;
  int32_t count, first_count, last_count;
  int32_t flags;          // bit0: first row shared, bit1: last row shared (set by MCC)
};
static_assert(sizeof(ChunkDesc) == 32, "ChunkDesc layout");

// A row of C that spans >= 2 chunks (the "shared rows" array, L432).
struct SharedRow {
  int32_t row;
  int32_t first_chunk;    // dense global chunk index of the first chunk holding the row
  int32_t nchunks;
  int32_t total;          // sum of the row's element counts over its chunks (pre-merge)
  int64_t merge_off;      // where the merged row goes in the merge pool; < 0: a two-chunk row
                          // merged in place over its pieces (first piece's room, then the second's)
  int32_t merged;         // merged element count (written by the merge kernels)
  int32_t kind;           // 0 multi (block), 1 path, 2 search, 3 multi (warp pair), 4 dense slices
};

// ---------------------------------------------------------------- helpers --

// Per-block trace for the multiprocessor-load report (Table 3's mpL, L760; acspgemm_sm_load):
// tr[3b] = SM id, tr[3b+1] = start, tr[3b+2] = end (%globaltimer, ns).
__device__ __forceinline__ uint64_t global_timer() {
  uint64_t t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__device__ __forceinline__ uint32_t sm_id() {
  uint32_t s;
  asm volatile("mov.u32 %0, %%smid;" : "=r"(s));
  return s;
}
__device__ __forceinline__ void trace_block(uint64_t* tr, int64_t b, uint64_t t0) {
  if (tr) {
    tr[3 * b] = sm_id();
    tr[3 * b + 1] = t0;
    tr[3 * b + 2] = global_timer();
  }
}

__device__ __forceinline__ int bit_width_u64(uint64_t x) { return x ? 64 - __clzll((long long)x) : 0; }

template <typename T> struct ValueTraits;
template <> struct ValueTraits<float> { static constexpr int bytes = 4; };
template <> struct ValueTraits<double> { static constexpr int bytes = 8; };

__device__ __forceinline__ int warp_id() { return threadIdx.x >> 5; }
__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }

// Block-wide exclusive prefix sum of one value per thread (fixed shuffle tree).
// `scratch` needs THREADS/32 + 1 elements.  Returns the exclusive prefix; *total
// receives the block sum.  Contains two __syncthreads().
template <typename V>
__device__ __forceinline__ V block_exclusive_sum(V x, V* scratch, V* total) {
  constexpr int NW = THREADS / 32;
  const int lane = lane_id(), w = warp_id();
  V inc = x;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    V y = __shfl_up_sync(0xffffffffu, inc, d);
    if (lane >= d) inc += y;
  }
  if (lane == 31) scratch[w] = inc;
  __syncthreads();
  // every warp scans the NW warp totals in its low lanes (no serial loop)
  V t = lane < NW ? scratch[lane] : (V)0;
  V ti = t;
#pragma unroll
  for (int d = 1; d < NW; d <<= 1) {
    V y = __shfl_up_sync(0xffffffffu, ti, d);
    if (lane >= d) ti += y;
  }
  const V wpre = __shfl_sync(0xffffffffu, ti - t, w);
  *total = __shfl_sync(0xffffffffu, ti, NW - 1);
  __syncthreads();          // scratch may be reused by the caller right away
  return wpre + inc - x;
}

// Block-wide inclusive max scan (one value per thread).  Two __syncthreads().
__device__ __forceinline__ int block_inclusive_max(int x, int* scratch) {
  const int lane = lane_id(), w = warp_id();
  int inc = x;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    int y = __shfl_up_sync(0xffffffffu, inc, d);
    if (lane >= d) inc = max(inc, y);
  }
  if (lane == 31) scratch[w] = inc;
  __syncthreads();
  if (threadIdx.x == 0) {
    int run = 0;
    for (int i = 0; i < THREADS / 32; ++i) { int t = scratch[i]; scratch[i] = run; run = max(run, t); }
  }
  __syncthreads();
  int res = max(scratch[w], inc);
  __syncthreads();
  return res;
}

// Block-wide exclusive max scan (identity 0, the "clear(Offsets)" value of Alg. 2).
__device__ __forceinline__ int block_exclusive_max(int x, int* scratch) {
  constexpr int NW = THREADS / 32;
  const int lane = lane_id(), w = warp_id();
  int inc = x;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    int y = __shfl_up_sync(0xffffffffu, inc, d);
    if (lane >= d) inc = max(inc, y);
  }
  int ex = __shfl_up_sync(0xffffffffu, inc, 1);
  if (lane == 0) ex = 0;
  if (lane == 31) scratch[w] = inc;
  __syncthreads();
  int t = lane < NW ? scratch[lane] : 0;
#pragma unroll
  for (int d = 1; d < NW; d <<= 1) {
    int y = __shfl_up_sync(0xffffffffu, t, d);
    if (lane >= d) t = max(t, y);
  }
  int wpre = __shfl_up_sync(0xffffffffu, t, 1);
  wpre = __shfl_sync(0xffffffffu, lane == 0 ? 0 : wpre, w);
  __syncthreads();
  return max(wpre, ex);
}

// Block-wide min/max reduction of four ints (rmin, rmax, cmin, cmax).
__device__ __forceinline__ void block_minmax4(int& a_min, int& a_max, int& b_min, int& b_max, int* scratch) {
  constexpr int NW = THREADS / 32;
  a_min = __reduce_min_sync(0xffffffffu, a_min);
  a_max = __reduce_max_sync(0xffffffffu, a_max);
  b_min = __reduce_min_sync(0xffffffffu, b_min);
  b_max = __reduce_max_sync(0xffffffffu, b_max);
  const int w = warp_id(), lane = lane_id();
  if (lane == 0) {
    scratch[4 * w + 0] = a_min; scratch[4 * w + 1] = a_max;
    scratch[4 * w + 2] = b_min; scratch[4 * w + 3] = b_max;
  }
  __syncthreads();
  const int q = lane < NW ? lane : 0;
  a_min = __reduce_min_sync(0xffffffffu, scratch[4 * q + 0]);
  a_max = __reduce_max_sync(0xffffffffu, scratch[4 * q + 1]);
  b_min = __reduce_min_sync(0xffffffffu, scratch[4 * q + 2]);
  b_max = __reduce_max_sync(0xffffffffu, scratch[4 * q + 3]);
  __syncthreads();
}

}  // namespace acs
