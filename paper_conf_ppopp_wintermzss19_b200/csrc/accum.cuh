// Shared pieces of the per-block accumulators of the adaptive strategy (hash.cu,
// reading R31; dict.cu, reading R33): exact IEEE product/sum and Fetch A.
#pragma once
#include <climits>
#include <type_traits>
#include "kernels.cuh"

namespace acs {

__device__ __forceinline__ float vmul(float x, float y) { return __fmul_rn(x, y); }
__device__ __forceinline__ double vmul(double x, double y) { return __dmul_rn(x, y); }
__device__ __forceinline__ float vadd(float x, float y) { return __fadd_rn(x, y); }
__device__ __forceinline__ double vadd(double x, double y) { return __dadd_rn(x, y); }

// A compacted entry and its A value in one 16-byte record (k_hash reads a wave's entry
// with one shared-memory load); fetch_block fills it when E is EntA<T> (a_val unused).
template <typename T>
struct alignas(16) EntA {
  int x, y;   // B row start, B row length
  T a;        // the A value
};

// Block-wide exclusive prefix sum for a CTA of NT threads (the fixed shuffle tree of
// common.cuh's block_exclusive_sum).  `scratch` needs NT/32 + 1 elements.  Two
// __syncthreads().
template <int NT, typename V>
__device__ __forceinline__ V block_exclusive_sum_nt(V x, V* scratch, V* total) {
  constexpr int NW = NT / 32;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  V inc = x;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    V y = __shfl_up_sync(0xffffffffu, inc, d);
    if (lane >= d) inc += y;
  }
  if (lane == 31) scratch[w] = inc;
  __syncthreads();
  V t = lane < NW ? scratch[lane] : (V)0;
  V ti = t;
#pragma unroll
  for (int d = 1; d < NW; d <<= 1) {
    V y = __shfl_up_sync(0xffffffffu, ti, d);
    if (lane >= d) ti += y;
  }
  const V wpre = __shfl_sync(0xffffffffu, ti - t, w);
  *total = __shfl_sync(0xffffffffu, ti, NW - 1);
  __syncthreads();
  return wpre + inc - x;
}

// Fetch A (§3.2.1) for one block of NPB nonzeros, as in AC-ESC, by NT
// threads (default THREADS):
//   * entries whose B row is empty add no products and are dropped; the others are
//     compacted in storage order: ent[ci].x = B row start, ent[ci].y = its length,
//     a_val[ci] = A value, wd[ci] = exclusive product prefix (the WDState of Alg. 2),
//     wd[nent] = the block's products;
//   * the block's rows are numbered by rank: row_first[lr] = first compacted entry of
//     local row lr (row_first[nrows] = nent), row_of[lr] = the row of A (and C).
// rp_cache needs NPB + 1 ints and may alias other storage after the call; scratch needs
// 2 (NT/32 + 1) ints, 8-byte aligned.  Ends with a __syncthreads().  Returns whether this thread saw a B row
// longer than 32 entries.
template <typename T, typename E, int NT = THREADS>
__device__ __forceinline__ bool fetch_block(const EscArgs& a, int b, int* rp_cache, int* row_of, int* row_first,
                                            E* ent, T* a_val, int* wd, int* scratch, int& nrows, int& nent,
                                            int& total) {
  const int tid = threadIdx.x;
  const int32_t* __restrict__ arp = a.A.row_ptr;
  const int32_t* __restrict__ acol = a.A.col;
  const T* __restrict__ aval = reinterpret_cast<const T*>(a.A.val);
  const int32_t* __restrict__ brp = a.B.row_ptr;
  const int nzb = a.blk_nz_begin[b];
  const int n_a = a.blk_nz_end[b] - nzb;
  const int r0 = a.block_row_starts[b];
  const int64_t rowsA = a.A.rows;
  constexpr int NPT = NPB / NT;          // A entries per thread (blocked)
  static_assert(NPB % NT == 0, "NPB must be a multiple of NT");
  // the entries' loads and their B row gathers are issued before the row pointers'
  // barrier, so the two chains of global loads overlap
  int len[NPT], row[NPT], bst[NPT];
  T av[NPT];
#pragma unroll
  for (int j = 0; j < NPT; ++j) {
    const int e = tid * NPT + j;
    len[j] = 0;
    bst[j] = 0;
    av[j] = (T)0;
    if (e < n_a) {
      const int k = acol[nzb + e];
      av[j] = aval[nzb + e];
      bst[j] = brp[k];
      len[j] = brp[k + 1] - bst[j];
    }
  }
  for (int t = tid; t <= NPB; t += NT) {
    const int64_t r = (int64_t)r0 + t;
    rp_cache[t] = r <= rowsA ? arp[r] : INT_MAX;
  }
  __syncthreads();
  int prev = 0;                          // local row of this thread's previous entry
#pragma unroll
  for (int j = 0; j < NPT; ++j) {
    const int e = tid * NPT + j;
    row[j] = INT_MAX;
    if (e < n_a) {
      const int nz = nzb + e;
      int r;
      if (nz < rp_cache[NPB]) {
        // consecutive entries: a few steps on from the previous entry's row, else a
        // binary search over the rest (rp_cache[lo] <= nz < rp_cache[lo + 1])
        int lo = prev;
#pragma unroll
        for (int step = 0; step < 2; ++step)
          if (rp_cache[lo + 1] <= nz) ++lo;
        if (rp_cache[lo + 1] <= nz) {
          int hi = NPB - 1;
          while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (rp_cache[mid] <= nz) lo = mid; else hi = mid - 1;
          }
        }
        prev = lo;
        r = r0 + lo;
      } else {
        int64_t lo = (int64_t)r0 + NPB, hi = rowsA - 1;
        while (lo < hi) {
          const int64_t mid = (lo + hi + 1) >> 1;
          if (arp[mid] <= nz) lo = mid; else hi = mid - 1;
        }
        r = (int)lo;
      }
      row[j] = r;
    }
    row_of[e] = row[j];        // temporarily: row per entry
  }
  __syncthreads();
  // one packed scan numbers the rows (low 16 bits) and the nonempty entries (high 16)
  int f[NPT], packed = 0, psum = 0;
  bool longb = false;
#pragma unroll
  for (int j = 0; j < NPT; ++j) {
    const int e = tid * NPT + j;
    f[j] = (e < n_a) && (e == 0 || row_of[e - 1] != row[j]);
    packed += f[j] + ((len[j] > 0) << 16);
    psum += len[j];
    longb |= len[j] > 32;
  }
  // one scan for both: (rows, entries) in the high word, products in the low word
  long long tot2;
  // (a block's products are < 2^31: the symbolic pass refuses larger blocks, k_block_bounds)
  const long long ex2 = block_exclusive_sum_nt<NT, long long>(((long long)packed << 32) | (long long)(uint32_t)psum,
                                                              reinterpret_cast<long long*>(scratch), &tot2);
  int ex = (int)(ex2 >> 32), pex = (int)(ex2 & 0xFFFFFFFFll);
  const int tot_packed = (int)(tot2 >> 32);
  total = (int)(tot2 & 0xFFFFFFFFll);
  nrows = tot_packed & 0xFFFF;
  nent = tot_packed >> 16;
#pragma unroll
  for (int j = 0; j < NPT; ++j) {
    const int lr = ex & 0xFFFF, ci = ex >> 16;
    if (f[j]) {
      row_first[lr] = ci;
      row_of[lr] = row[j];
    }
    if (len[j] > 0) {
      if constexpr (std::is_same<E, EntA<T>>::value) {
        ent[ci] = EntA<T>{bst[j], len[j], av[j]};
      } else {
        ent[ci].x = bst[j];
        ent[ci].y = len[j];
        a_val[ci] = av[j];
      }
      wd[ci] = pex;
    }
    ex += f[j] + ((len[j] > 0) << 16);
    pex += len[j];
  }
  if (tid == 0) {
    row_first[nrows] = nent;
    wd[nent] = total;
  }
  __syncthreads();
  return longb;
}

// Rows -> warps by product count: warp w of NW owns the rows whose first product lies in
// [w·P/NW, (w+1)·P/NW).  Lane 0 of each warp writes wrow[w] (wrow[NW] = nrows); the
// caller synchronises.
template <int NW>
__device__ __forceinline__ void split_rows(const int* wd, const int* row_first, int nrows, int total, int* wrow) {
  const int w = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (lane == 0) {
    const int L = (int)((int64_t)w * total / NW);
    int lo = 0, hi = nrows;              // first r with start(r) >= L
    while (lo < hi) {
      const int mid = (lo + hi) >> 1;
      if (wd[row_first[mid]] < L) lo = mid + 1; else hi = mid;
    }
    wrow[w] = w == 0 ? 0 : lo;
    if (w == NW - 1) wrow[NW] = nrows;
  }
}

// One chunk descriptor per warp that emitted rows (L424-L428), in warp order = row
// order; wout[q] = {count, first_row, last_row, first_count, last_count}; counts the
// block in *counter (info only).  Thread 0.
// Where (relative to the block's pool region) the warp owning rows [rlo, ..) writes: exact
// pools: after the products of the rows before it; POOL_BOUND (reading R40): after
// sum min(products, HASH_UBOUND) over them -- the accumulators' output bound, so the runs
// pack into min(products, rows x HASH_UMAX).  All lanes of the warp call it.
__device__ __forceinline__ int warp_out_base(const EscArgs& a, const int* wd, const int* row_first, int rlo,
                                             int nrows, int lane) {
  if (rlo >= nrows) return 0;
  if (!a.bound) return wd[row_first[rlo]];
  int s = 0;
  for (int r = lane; r < rlo; r += 32) s += min(wd[row_first[r + 1]] - wd[row_first[r]], HASH_UBOUND);
  return __reduce_add_sync(0xffffffffu, s);
}

// wout[w]: count, first_row, last_row, first_count, last_count, warp_out_base
__device__ __forceinline__ void emit_warp_chunks(const EscArgs& a, int b, int nw, const int* wrow, const int (*wout)[6],
                                                 const int* wd, const int* row_first, int64_t* counter) {
  const int64_t pool_base = a.pool_off[b];
  const int64_t desc_base = a.desc_off[b];
  int seq = 0, used = 0;
  (void)wrow; (void)wd; (void)row_first;
  for (int q = 0; q < nw; ++q) {
    if (wout[q][0] == 0) continue;
    ChunkDesc d;
    d.data_off = pool_base + wout[q][5];
    d.first_row = wout[q][1];
    d.last_row = wout[q][2];
    d.count = wout[q][0];
    d.first_count = wout[q][3];
    d.last_count = wout[q][4];
    d.flags = 0;
    a.descs[desc_base + seq] = d;
    ++seq;
    used += wout[q][0];
  }
  a.nchunks[b] = seq;
  a.used[b] = used;
  atomicAdd(reinterpret_cast<unsigned long long*>(counter), 1ull);
}

}  // namespace acs
