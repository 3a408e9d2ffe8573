// Stage 2, adaptive alternative — per-row accumulation for blocks of short rows
// (reading R34).
//
// PAPER.md L850 (§5): "choose between alternative approaches (ESC, hashing, merging)
// depending on the load currently seen by the work distribution".  Blocks whose rows
// each hold only a few products and columns (AMG prolongation A·P: 7 products, <= 4
// columns per row; the Galerkin product R·(A·P): <= 32 products, 7 columns) sort a tile
// of 512 products in AC-ESC (R32) to find them.  Here one LANE owns one row:
//   * it walks the row's products in expansion order (A entries in storage order, each
//     B row in order) and accumulates a_ik * b_kj into a private list of <= ROWS_LMAX
//     (column, value) slots in shared memory (column-major over the CTA's lanes, so the
//     lanes of a warp touch consecutive banks): a column seen before is added to its
//     slot, a new column takes the next slot with the product itself (= -0.0 + product,
//     the identity start of the other accumulators).  Every output is therefore the left
//     fold of its products in A-entry order -- Gustavson's order, the same bits as the
//     hash and dictionary accumulators (R31, R33);
//   * the list is insertion-sorted by column and written to the warp's chunk; a warp
//     owns a contiguous run of the block's rows and takes them 32 at a time, lane order
//     = row order, so the chunk holds its rows in order (L424-L428).
// Blocks with a row of more than ROWS_PMAX products are not taken; a row reaching more
// than ROWS_LMAX distinct columns abandons the block (both tests depend only on the
// data: the choice is deterministic).  Such blocks stay with AC-ESC.  hash_done[b] = 3
// marks a block finished here.
#include "accum.cuh"

namespace acs {

constexpr int ROWS_WARPS = THREADS / 32;
#ifndef ACS_ROWS_LMAX
#define ACS_ROWS_LMAX 8
#endif
constexpr int ROWS_LMAX = ACS_ROWS_LMAX;  // distinct columns of one row (per-lane list; 8 keeps
                                          // shared memory at 26 KB: 8 CTAs per SM, cfg4a A·P
                                          // 5.4 -> 4.2 ms against 16 slots)
constexpr int ROWS_PMAX = 256;           // products of one row
constexpr int ROWS_U = 8;                // products per lane with their B loads in flight

template <typename T>
struct RowsSmem {
  T a_val[NPB];
  int2 ent[NPB];                 // (B row start, length) per nonempty entry (fetch_block)
  int wd[NPB + 1];
  int row_first[NPB + 1];
  int row_of[NPB];
  union {
    int rp_cache[NPB + 1];
    struct {
      int col[ROWS_LMAX][THREADS];   // lane tid's slot j at [j][tid]
      T val[ROWS_LMAX][THREADS];
    } l;
  } u;
  int wrow[ROWS_WARPS + 1];
  int wout[ROWS_WARPS][6];
  alignas(8) int scratch[40];
  int flag;
  int batch[32];                 // the current batch's blocks no accumulator finished
  int nbatch, bbase;
};

// A block left to AC-ESC: onto the big- or small-tile list (reading R32).
__device__ __forceinline__ void rows_give_up(const EscArgs& a, int b) {
  if (a.bound && a.region[b] < a.blk_products[b]) {
    // POOL_BOUND: AC-ESC needs the block's exact bound; deferred to a second pass (R40)
    a.hash_done[b] = 4;
    atomicAdd(reinterpret_cast<unsigned long long*>(a.defer), 1ull);
    atomicAdd(reinterpret_cast<unsigned long long*>(a.defer + 1), (unsigned long long)a.blk_products[b]);
    return;
  }
  const bool small = a.esc_list_small && a.blk_products[b] <= CAP_SMALL;
  int64_t* cnt = small ? a.esc_count_small : a.esc_count;
  int32_t* list = small ? a.esc_list_small : a.esc_list;
  list[atomicAdd(reinterpret_cast<unsigned long long*>(cnt), 1ull)] = b;
}

// One block: finished here (hash_done[b] = 3) or left to AC-ESC (listed).
template <typename T>
__device__ __forceinline__ void rows_block(RowsSmem<T>& S, const EscArgs& a, const int b) {
  const unsigned FULL = 0xffffffffu;
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const uint64_t t_start = a.trace ? global_timer() : 0;
  const int32_t* __restrict__ bcol = a.B.col;
  const T* __restrict__ bval = reinterpret_cast<const T*>(a.B.val);
  if (tid == 0) S.flag = 0;
  int nrows, nent, total;
  fetch_block<T, int2, THREADS>(a, b, S.u.rp_cache, S.row_of, S.row_first, S.ent, S.a_val, S.wd, S.scratch, nrows,
                                nent, total);
  bool big = false;
  for (int r = tid; r < nrows; r += THREADS) big |= S.wd[S.row_first[r + 1]] - S.wd[S.row_first[r]] > ROWS_PMAX;
  if (__syncthreads_or(big)) {           // a long row: AC-ESC
    if (tid == 0) rows_give_up(a, b);
    return;
  }
  split_rows<ROWS_WARPS>(S.wd, S.row_first, nrows, total, S.wrow);
  __syncthreads();
  const int rlo = S.wrow[w], rhi = S.wrow[w + 1];
  const int wrel = warp_out_base(a, S.wd, S.row_first, rlo, nrows, lane);
  const int64_t wbase = a.pool_off[b] + wrel;
  T* pval = reinterpret_cast<T*>(a.pool_val);
  int32_t* pcol = a.pool_col;
  int(*lc)[THREADS] = S.u.l.col;
  T(*lv)[THREADS] = S.u.l.val;
  int out = 0, first_row = -1, last_row = -1, first_count = 0, last_count = 0;
  for (int r0 = rlo; r0 < rhi; r0 += 32) {
    // another warp abandoned the block: one lane reads the flag, the warp follows it
    // (per-lane atomics could disagree and split the warp)
    if (__shfl_sync(0xffffffffu, lane == 0 ? atomicOr(&S.flag, 0) : 0, 0)) break;
    const int r = r0 + lane;
    int cnt = 0;
    bool over = false;
    if (r < rhi) {
      // products in expansion order, ROWS_U at a time: their B loads are all in flight
      // before the first one is accumulated
      int c = S.row_first[r];
      const int c1 = S.row_first[r + 1];
      int q = 0, qe = 0;
      T av = (T)0;
      if (c < c1) { const int2 e = S.ent[c]; q = e.x; qe = e.x + e.y; av = S.a_val[c]; }
      while (c < c1) {
        int col[ROWS_U];
        T v[ROWS_U];
        int n = 0;
#pragma unroll
        for (int u = 0; u < ROWS_U; ++u) {
          if (c < c1) {
            col[u] = __ldg(bcol + q);
            v[u] = vmul(av, __ldg(bval + q));
            n = u + 1;
            if (++q == qe && ++c < c1) { const int2 e = S.ent[c]; q = e.x; qe = e.x + e.y; av = S.a_val[c]; }
          }
        }
#pragma unroll
        for (int u = 0; u < ROWS_U; ++u) {
          if (u < n) {
            int j = 0;
            while (j < cnt && lc[j][tid] != col[u]) ++j;
            if (j < cnt) {
              lv[j][tid] = vadd(lv[j][tid], v[u]);
            } else if (cnt < ROWS_LMAX) {
              lc[cnt][tid] = col[u];
              lv[cnt][tid] = v[u];
              ++cnt;
            } else {
              over = true;
            }
          }
        }
      }
      // insertion sort of the row's columns (equal columns do not occur)
      for (int i = 1; i < cnt; ++i) {
        const int kc = lc[i][tid];
        const T kv = lv[i][tid];
        int j = i - 1;
        while (j >= 0 && lc[j][tid] > kc) {
          lc[j + 1][tid] = lc[j][tid];
          lv[j + 1][tid] = lv[j][tid];
          --j;
        }
        lc[j + 1][tid] = kc;
        lv[j + 1][tid] = kv;
      }
    }
    if (__any_sync(FULL, over)) {        // uniform per warp; the block goes to AC-ESC
      if (lane == 0) atomicExch(&S.flag, 1);
      break;
    }
    int inc = cnt;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int y = __shfl_up_sync(FULL, inc, d);
      if (lane >= d) inc += y;
    }
    const int tot = __shfl_sync(FULL, inc, 31);
    const int64_t dst = wbase + out + (inc - cnt);
    for (int i = 0; i < cnt; ++i) {
      pcol[dst + i] = lc[i][tid];
      pval[dst + i] = lv[i][tid];
    }
    const int grow = r < rhi ? S.row_of[r] : -1;
    if (cnt > 0) a.row_count[grow] = cnt;          // per-row counter (L362)
    const unsigned m = __ballot_sync(FULL, cnt > 0);
    if (m) {
      const int fl = __ffs(m) - 1, ll = 31 - __clz(m);
      const int frow = __shfl_sync(FULL, grow, fl), fcnt = __shfl_sync(FULL, cnt, fl);
      const int lrow = __shfl_sync(FULL, grow, ll), lcnt = __shfl_sync(FULL, cnt, ll);
      if (first_row < 0) { first_row = frow; first_count = fcnt; }
      last_row = lrow;
      last_count = lcnt;
    }
    out += tot;
  }
  if (lane == 0) {
    S.wout[w][0] = out;
    S.wout[w][1] = first_row;
    S.wout[w][2] = last_row;
    S.wout[w][3] = first_count;
    S.wout[w][4] = last_count;
    S.wout[w][5] = wrel;
  }
  __syncthreads();
  if (tid == 0) trace_block(a.trace, b, t_start);
  if (tid == 0) {
    if (!S.flag) {
      emit_warp_chunks(a, b, ROWS_WARPS, S.wrow, S.wout, S.wd, S.row_first, a.rows_count);
      a.hash_done[b] = 3;
    } else {
      rows_give_up(a, b);
    }
  }
}

// The blocks it gives up go onto the AC-ESC lists (no list pass).  Without a hash
// candidate it runs one CTA per block; after k_hash / k_dict (most blocks done) it is
// persistent: a CTA takes rows_batch (<= ROWS_BATCH) consecutive block numbers at a time
// (rows_next) and runs those no accumulator finished (hash_done == 0, in order) -- no
// grid of nblocks CTAs that mostly exit at once (cfg2: all 108,880 blocks are k_hash's).
constexpr int ROWS_BATCH = 32;

template <typename T>
__global__ void __launch_bounds__(THREADS, 8) k_rows(EscArgs a) {   // 8 CTAs per SM (26 KB shared memory each)
  extern __shared__ __align__(16) unsigned char smem_raw[];
  RowsSmem<T>& S = *reinterpret_cast<RowsSmem<T>*>(smem_raw);
  const int tid = threadIdx.x;
  if (a.rows_batch == 0) {               // one CTA per block (most blocks are k_rows' own)
    if (a.hash_done[blockIdx.x] == 0) rows_block<T>(S, a, blockIdx.x);
    return;
  }
  for (;;) {
    if (tid < 32) {
      int base = 0;
      if (tid == 0)
        base = (int)atomicAdd(reinterpret_cast<unsigned long long*>(a.rows_next), (unsigned long long)a.rows_batch);
      base = __shfl_sync(0xffffffffu, base, 0);
      // after k_hash: its list of the blocks it left; otherwise every block, by flag
      const int limit = a.rows_list ? (int)*a.rows_list_count : a.nblocks;
      const int i = base + tid;
      const int b = a.rows_list ? (i < limit ? a.rows_list[i] : 0) : i;
      const bool need = tid < a.rows_batch && i < limit && a.hash_done[b] == 0;
      const unsigned m = __ballot_sync(0xffffffffu, need);
      if (need) S.batch[__popc(m & ((1u << tid) - 1u))] = b;
      if (tid == 0) { S.nbatch = __popc(m); S.bbase = base < limit ? 0 : 1; }
    }
    __syncthreads();
    const int bbase = S.bbase, n = S.nbatch;
    __syncthreads();                     // read before warp 0 overwrites them (n == 0)
    if (bbase) break;                    // past the last block
    for (int k = 0; k < n; ++k) {
      rows_block<T>(S, a, S.batch[k]);
      __syncthreads();                   // shared memory is reused by the next block
    }
  }
}

// POOL_BOUND second pass (reading R40): the deferred blocks (hash_done == 4) get regions of
// their exact product bound appended to the pool, in block order (a scan), and go onto
// the AC-ESC lists (big / small tile).
__global__ void k_defer_flags(const int32_t* __restrict__ hash_done, const int64_t* __restrict__ prod, int n,
                              int64_t* __restrict__ flag) {
  const int b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b < n) flag[b] = hash_done[b] == 4 ? prod[b] : 0;
}

__global__ void k_defer_place(EscArgs a, const int64_t* __restrict__ scan, int64_t base, int64_t* __restrict__ off) {
  const int b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= a.nblocks || a.hash_done[b] != 4) return;
  off[b] = base + scan[b];
  const bool small = a.esc_list_small && a.blk_products[b] <= CAP_SMALL;
  int64_t* cnt = small ? a.esc_count_small : a.esc_count;
  int32_t* list = small ? a.esc_list_small : a.esc_list;
  list[atomicAdd(reinterpret_cast<unsigned long long*>(cnt), 1ull)] = b;
}

void launch_defer_flags(const EscArgs& a, int64_t* flag, cudaStream_t st) {
  if (a.nblocks > 0) k_defer_flags<<<(a.nblocks + 255) / 256, 256, 0, st>>>(a.hash_done, a.blk_products, a.nblocks, flag);
}

void launch_defer_place(const EscArgs& a, const int64_t* scan, int64_t base, int64_t* off, cudaStream_t st) {
  if (a.nblocks > 0) k_defer_place<<<(a.nblocks + 255) / 256, 256, 0, st>>>(a, scan, base, off);
}

template <typename T>
static void launch_rows_t(const EscArgs& a, bool hash_ran, cudaStream_t st) {
  const size_t smem = sizeof(RowsSmem<T>);
  static ResidentCache rc;
  // batches of up to ROWS_BATCH blocks, at least ~16 per CTA (a short tail), one block
  // per batch when there are fewer blocks than CTAs
  const int64_t slots = resident_ctas(rc, k_rows<T>, THREADS, smem);   // also sets the smem limit
  EscArgs b = a;
  if (!hash_ran) {                       // no accumulator ran: one CTA per block
    b.rows_batch = 0;
    k_rows<T><<<a.nblocks, THREADS, smem, st>>>(b);
    return;
  }
  b.rows_batch = (int)std::max<int64_t>(1, std::min<int64_t>(ROWS_BATCH, a.nblocks / (slots * 16)));
  const int64_t batches = (a.nblocks + b.rows_batch - 1) / b.rows_batch;
  const int grid = (int)std::min<int64_t>(batches, slots);
  k_rows<T><<<grid, THREADS, smem, st>>>(b);
}

void launch_rows(const EscArgs& a, bool f64, bool hash_ran, cudaStream_t st) {
  if (a.nblocks <= 0) return;
  if (f64) launch_rows_t<double>(a, hash_ran, st); else launch_rows_t<float>(a, hash_ran, st);
}

}  // namespace acs
