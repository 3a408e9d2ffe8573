// Internal host-side launchers of the AC-SpGEMM stage kernels (not part of the C ABI).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>
#include "common.cuh"

namespace acs {

struct CsrView {              // device CSR view; row_ptr values index col/val directly
  int64_t rows, cols;
  const int32_t* row_ptr;
  const int32_t* col;
  const void* val;
};

// ---- stage 1: global load balancing (glb.cu) ----------------------------------
// Explicit segment row boundaries, passed BY VALUE as a kernel argument (so a captured
// graph and an asynchronous launch keep their own copy); n == 0: canonical segments.
struct SegRows {
  int32_t n;
  int64_t r[MAX_SEGMENTS + 1];
};
// Device words the first kernel of a multiply zeroes (counters of the later stages), so
// that no memset launch is needed: ZeroList::p[i][0 .. n[i]) = 0.
struct ZeroList {
  int64_t* p[4];
  int32_t n[4];
};
// Writes seg tables to `seg` (device, int64[4*(MAX_SEGMENTS+1)]): rows | nz | block base;
// also zeroes `zero`.
void launch_segments(const CsrView& A, int nseg, const SegRows& explicit_rows,
                     int64_t* seg, int32_t* nblocks_dev, cudaStream_t st, const ZeroList& zero = ZeroList{});
// row_count (nullable): zeroed, one word per row of A
void launch_glb(const CsrView& A, int nseg, const int64_t* seg, int32_t* block_row_starts,
                int64_t max_blocks, cudaStream_t st, int32_t* row_count = nullptr);
void launch_block_bounds(const CsrView& A, const CsrView& B, int nseg, const int64_t* seg,
                         const int32_t* nblocks_dev, int64_t max_blocks, int32_t* blk_nz_begin,
                         int32_t* blk_nz_end, int64_t* blk_products, int64_t* blk_slots,
                         int32_t* blk_hash_ok /* nullable: hash-accumulator candidates (R31) */,
                         int64_t* ncand /* nullable: their count (zeroed by the caller) */,
                         int64_t* max_products /* atomicMax of block products > INT_MAX (zeroed) */,
                         int64_t* nblocks_out /* nullable: the block count as int64 */,
                         const int32_t* block_row_starts, int64_t rows_a,
                         int64_t* est /* nullable: POOL_BOUND region per block (reading R40) */, cudaStream_t st);

// ---- device-wide exclusive scan (scan.cu) --------------------------------------
// out[i] = sum_{j<i} in[j] for i < n, total -> *total_dev.  tmp needs scan_tmp_elems(n)
// words, all zero before the first scan; every scan leaves them zero again.
int64_t scan_tmp_elems(int64_t n);
void launch_scan_i64(const int64_t* in, int64_t* out, int64_t n, int64_t* total_dev, int64_t* tmp, cudaStream_t st);
void launch_scan_i32(const int32_t* in, int64_t* out, int64_t n, int64_t* total_dev, int64_t* tmp, cudaStream_t st);
// row_ptr: exclusive scan of int32 counts into int64 row_ptr[n+1] (+ the total).
void launch_scan_rowptr(const int32_t* in, int64_t* row_ptr, int64_t n, int64_t* total_dev, int64_t* tmp,
                        cudaStream_t st);

// ---- stage 2: AC-ESC (esc.cu) ---------------------------------------------------
struct EscArgs {
  CsrView A, B;
  int32_t nblocks;
  const int32_t* blk_nz_begin;
  const int32_t* blk_nz_end;
  const int32_t* block_row_starts;
  const int64_t* pool_off;      // per block, elements
  const int64_t* desc_off;      // per block, descriptor slots
  int32_t* pool_col;
  void* pool_val;
  ChunkDesc* descs;
  int32_t* nchunks;             // per block
  int32_t* used;                // per block: chunk elements written
  int32_t* row_count;           // per row of C
  int32_t* hash_done;           // per block: in: 1 = hash candidate (k_block_bounds); out: 2 = finished
                                // by k_dict, 1 = by k_hash, 3 = by k_rows, 0 = AC-ESC (nullptr: none)
  int64_t* hash_count;          // blocks finished by k_dict or k_hash (atomic counter, info only)
  int64_t* dict_count;          // blocks finished by k_dict (atomic counter, info only)
  int64_t* rows_count;          // blocks finished by k_rows (atomic counter, info only)
  int32_t* esc_list;            // adaptive: blocks left to AC-ESC [nblocks]
  int64_t* esc_count;           // adaptive: their number (zeroed before launch_hash)
  int64_t* esc_next;            // adaptive: grab counter of the persistent k_esc (zeroed)
  const int64_t* blk_products;  // per block product count
  uint64_t* trace;              // nullable: per-block (SM, start, end) of this launch's kernel (mpL)
  int32_t* esc_list_small;      // adaptive: left blocks of <= CAP_SMALL products [nblocks]
  int64_t* esc_count_small;     // (zeroed) -- the small-tile AC-ESC's list, counter
  int64_t* esc_next_small;      // (zeroed)
  int64_t* rows_next;           // adaptive: batch counter of the persistent k_rows (zeroed)
  int64_t* hash_next;           // adaptive: block counter of the persistent k_hash (zeroed)
  int32_t* rows_list;           // adaptive: blocks k_hash saw and did not finish, for k_rows
  int64_t* rows_list_count;     // (zeroed) their number; nullptr: k_rows scans hash_done
  int32_t rows_batch;           // blocks per k_rows batch, 0: one CTA per block (set by launch_rows)
  int32_t bound;                // POOL_BOUND (reading R40): warp runs packed by min(row products,
                                // HASH_UMAX); a block left to AC-ESC whose region is below its
                                // products is deferred (hash_done = 4) instead of listed
  const int64_t* region;        // POOL_BOUND: each block's pool region (elements)
  int64_t* defer;               // POOL_BOUND: [0] deferred blocks, [1] their products (zeroed)
};
void launch_esc(const EscArgs& a, bool f64, cudaStream_t st);
// adaptive alternative (hash.cu, reading R31): must run before launch_esc on the same stream
void launch_hash(const EscArgs& a, bool f64, cudaStream_t st);
// column-dictionary accumulator (dict.cu, reading R33): runs before launch_hash on the
// same stream; blocks it finishes get hash_done = 2, the rest stay hash candidates
void launch_dict(const EscArgs& a, bool f64, cudaStream_t st);
// per-row accumulator for blocks of short rows (rows.cu, reading R34): after launch_hash,
// on the blocks no accumulator finished; the ones it finishes get hash_done = 3, the
// others go onto the AC-ESC lists (esc_list / esc_list_small) for launch_esc
// hash_ran: an accumulator ran before (persistent batches), else one CTA per block
void launch_rows(const EscArgs& a, bool f64, bool hash_ran, cudaStream_t st);
// POOL_BOUND second pass (rows.cu, reading R40): flag[b] = products of deferred blocks;
// after its scan, their regions off[b] = base + scan[b] and the AC-ESC lists
void launch_defer_flags(const EscArgs& a, int64_t* flag, cudaStream_t st);
void launch_defer_place(const EscArgs& a, const int64_t* scan, int64_t base, int64_t* off, cudaStream_t st);

// ---- stage 3: chunk ordering, shared rows, merges (merge.cu) --------------------
struct MergeState {
  int32_t nblocks;
  const int64_t* desc_off;
  const int32_t* nchunks;
  const int64_t* chunk_base;     // exclusive scan of nchunks
  const ChunkDesc* descs;
  ChunkDesc* dense;              // dense global chunk array [total_chunks]
  int64_t max_chunks;            // host upper bound (total slots)
  const int64_t* total_chunks_dev;
  int32_t* shared_flag;          // [max_chunks] 1 where a shared row starts
  int64_t* shared_pos;           // [max_chunks] exclusive scan of shared_flag
  SharedRow* shared;             // [max_chunks]
  const int32_t* pool_col;       // chunk columns (row spans for the merge classification)
  int64_t* scan_tmp;
};
void launch_gather_chunks(const MergeState& m, cudaStream_t st);

struct MergeLists {
  int64_t nshared;
  SharedRow* shared;
  int32_t* kind_flag;            // [nshared] scratch
  int64_t* kind_pos;             // [nshared] scratch
  int32_t* multi_idx;            // [nshared]
  int32_t* path_idx;
  int32_t* search_idx;
  int32_t* pair_idx;             // two-chunk rows of <= PAIR_MAX elements (warp merge)
  int32_t* giant_idx;            // rows of > SEARCH_MAXP chunks (dense slices)
  int64_t* counts_dev;           // [8]: nmulti, npath, nsearch, npair, merge_total, ngiant, multi_total
  int64_t* merge_total_scan;     // [nshared] exclusive scan of totals -> merge offsets
  int64_t* multi_scan;           // [nshared]
  int32_t* group_of;             // [nshared]
  int32_t* group_start;          // [max groups + 1]
  int64_t* scan_tmp;
};
// shared rows, their kinds and merge offsets in one pass (lists sized by m.max_chunks)
// L.counts_dev[0 .. 6) must be zero on entry.
void launch_find_shared(const MergeState& m, const MergeLists& L, int64_t* total_shared_dev, cudaStream_t st);
void launch_multi_groups(const MergeLists& L, int64_t nmulti, int64_t ngroups, cudaStream_t st);

struct MergeArgs {
  const ChunkDesc* dense;
  SharedRow* shared;
  const int32_t* list;           // indices into shared for this kind
  int64_t nlist;
  const int32_t* group_start;    // multi merge only: [ngroups+1] starts then [ngroups+1] ends
  const int64_t* multi_scan;     // multi merge only: exclusive scan of totals over the list
  int64_t ngroups;
  const int32_t* pool_col;
  const void* pool_val;
  int32_t* merge_col;
  void* merge_val;
  int32_t* cur_first;            // per dense chunk cursors (path/search)
  int32_t* cur_last;
  int32_t* row_count;
  int32_t* error_flag;
};
void launch_multi_merge(const MergeArgs& a, bool f64, cudaStream_t st);
void launch_pair_merge(const MergeArgs& a, bool f64, cudaStream_t st);
void launch_path_merge(const MergeArgs& a, bool f64, cudaStream_t st);
void launch_search_merge(const MergeArgs& a, bool f64, cudaStream_t st);
struct GiantArgs {                // dense-slice merge of rows with > SEARCH_MAXP chunks
  const int32_t* list;            // [n] indices into shared
  int64_t n;
  int32_t* glo;                   // [n] first column of the row's span
  int32_t* ghi;                   // [n] last column of the row's span
  int64_t* gnsl;                  // [n] slices of the row
  int64_t* gbase;                 // [n] exclusive scan of gnsl
  int64_t* gmn;                   // [n] slices x pieces of the row
  int64_t* gmbase;                // [n] exclusive scan of gmn
  int32_t* pos;                   // [sum gmn] start of each piece's entries in each slice
  int32_t* gent;                  // [nslices] pre-merge entries per slice
  int64_t* gpos;                  // [nslices] exclusive scan of gent
  int32_t* tcnt;                  // [nslices] merged entries per slice
};
void launch_giant_span(const MergeArgs& a, const GiantArgs& g, cudaStream_t st);
void launch_giant_count(const MergeArgs& a, const GiantArgs& g, int64_t nslices, cudaStream_t st);
void launch_giant_merge(const MergeArgs& a, const GiantArgs& g, int64_t nslices, bool f64, cudaStream_t st);

// ---- stage 4: chunk copy (copy.cu) ----------------------------------------------
struct CopyArgs {
  const ChunkDesc* dense;
  const int64_t* total_chunks_dev;
  int64_t max_chunks;
  const SharedRow* shared;
  int64_t nshared;
  const int32_t* pool_col;
  const void* pool_val;
  const int32_t* merge_col;
  const void* merge_val;
  const int64_t* row_ptr;        // C's row pointers (plan memory, int64)
  int32_t* c_col;
  void* c_val;
};
void launch_copy(const CopyArgs& a, bool f64, cudaStream_t st);
// C.row_ptr from the plan's int64 row pointers: dst[i] = src[i] + off (int32 or int64 dst;
// src nullptr: dst[i] = off)
void launch_rowptr_out(int32_t* dst, const int64_t* src, int64_t n, int32_t off, cudaStream_t st);
void launch_rowptr_out(int64_t* dst, const int64_t* src, int64_t n, int64_t off, cudaStream_t st);
// dst[i] = src[i] + off (row pointers of a row piece placed after earlier pieces)
void launch_copy_offset(int32_t* dst, const int32_t* src, int64_t n, int32_t off, cudaStream_t st);
// out[0] = min, out[1] = max of col[0, n) (n = 0: out = {0x7F7F7F7F, 0})
void launch_col_range(const int32_t* col, int64_t n, int32_t* out, cudaStream_t st);
// nbytes (multiple of 4, <= 4096) from device memory to mapped host memory, by a kernel
void launch_read_back(const void* src, void* mapped_dst, int nbytes, cudaStream_t st);
// two read-backs in one launch
void launch_read_back2(const void* src1, void* mapped_dst1, int nbytes1, const void* src2, void* mapped_dst2,
                       int nbytes2, cudaStream_t st);
// p[i] += off for i < n (row pointers of a row piece placed after earlier pieces)
void launch_add_offset(int32_t* p, int64_t n, int32_t off, cudaStream_t st);

// Resident CTAs of `kern` on the current device (SMs x CTAs per SM at `threads` threads and
// `smem` dynamic shared memory), worked out once per device per kernel (the host calls
// sit between a read-back and the next launch: on the critical path of small
// multiplies); raises the kernel's dynamic shared-memory limit to `smem` the same once.
struct ResidentCache {
  int grid[16] = {0};
};
template <typename K>
inline int resident_ctas(ResidentCache& c, K kern, int threads, size_t smem) {
  int dev = 0;
  cudaGetDevice(&dev);
  int* slot = (dev >= 0 && dev < 16) ? &c.grid[dev] : nullptr;
  if (slot && *slot > 0) return *slot;
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  int sms = 148, per = 1;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per, kern, threads, smem);
  const int g = sms * (per > 0 ? per : 1);
  if (slot) *slot = g;
  return g;
}

// ---- validation ----------------------------------------------------------------
void launch_validate(const CsrView& M, int32_t* bad_flag, cudaStream_t st);

}  // namespace acs

// small-tile AC-ESC over esc_list_small (esc_small.cu, reading R32); args: acs::EscArgs
void acs_launch_esc_small(const void* args, bool f64, cudaStream_t st);
