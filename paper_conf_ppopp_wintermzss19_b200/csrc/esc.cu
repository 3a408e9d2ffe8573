// Stage 2 — Adaptive chunk-based ESC (§3.2).
//
// One CTA per block of NPB nonzeros of A.  Per CTA:
//   Fetch A (§3.2.1): coalesced load of the block's A entries, B row starts and
//     lengths, and a dense local row dictionary (local id = rank of the row among the
//     block's rows; its bit width is bounded by log2(NPB) like the paper's dictionary).
//   placework (Alg. 2), then iterate:
//     receivework(CAP - kept) -> expand (§3.2.3) -> radix sort of
//     (row, col) keys with the bit range reduced to the rows and columns present
//     (L342-L344) -> compaction scan (Alg. 3) -> completed rows go to a chunk, the
//     last row is kept in shared memory when it is not yet complete and has at most
//     KEEP elements (L364-L366) -> per-row counts (L362).
// Long rows (§3.4): an entry of A whose B row has more than PTR_LEN = CAP
// entries would be loaded and sorted without change; instead it is removed from the
// work distribution and becomes its own chunk, a·B_k written by a coalesced streaming
// copy (no sort), placed in the chunk order where its products belong: the iteration
// before it stops at its position ("we break up chunks at the position of the long
// row", L548), and the row is merged with the rest of its chunks in the merge stage.
// Chunk allocation is deterministic (reading R8): block b writes its chunks to a
// slot range sized from its exact product count (stage 1), so no atomics, no
// restarts, and the chunk id (block, running number) is the global order (L430).
#include <algorithm>
#include <climits>
#include "esc_core.cuh"
#include "kernels.cuh"

namespace acs {

template <typename T>
struct EscSmem {
  SortSmem<T> s;
  T a_val[NPB];
  int a_bstart[NPB];
  int a_lrow[NPB];
  int row_of[NPB];
  int wd[NPB + 1];
  int rp_cache[NPB + 1];
};

struct EscState {
  int kept, kofs, kept_lrow, kept_cmin, kept_cmax;  // kept row lives in the staging area
  int seq;
  int64_t wofs;
  int stop_row;     // local row of the next long-row chunk: the current iteration ends at its
                    // position, a complete last row below it is not kept (INT_MIN: none)
  bool keep_ok;     // the block's rows average at most CAP/2 products (reading R38): keeping
                    // the last row (L366) can spare a merge; longer rows span iterations anyway
};

// Staging slot of compacted element p.  Each thread emits ITEMS consecutive elements, so
// the lanes of one store are ~ITEMS slots apart; a rotation inside every 32 (4-byte
// columns) / 16 (8-byte values) slots by the row number spreads them over the banks,
// and consecutive p (the coalesced read-out) stay conflict-free.  A permutation inside
// each aligned group, so slots stay below CAP.
__device__ __forceinline__ int stage_slot32(int p) { return (p & ~31) | ((p + (p >> 5)) & 31); }
template <typename T>
__device__ __forceinline__ int stage_slot(int p) {
  return sizeof(T) == 8 ? ((p & ~15) | ((p + (p >> 4)) & 15)) : stage_slot32(p);
}

// Sort + compaction (Alg. 3) + emission of one local ESC iteration whose sort words are
// already in s.words: completed rows become a chunk, the last row is kept.  Only the
// key bits [IDXBITS, IDXBITS + sortbits) are sorted (0: words already sorted).
// colof(key, pos) yields an element's output column.
template <typename Word, typename T, typename ColOf>
__device__ __forceinline__ void esc_tail(EscSmem<T>& S, const EscArgs& a, EscState& st, int n, int size_after,
                                         int rmin, int sortbits, int colbits, int64_t pool_base, int64_t desc_base,
                                         ColOf colof) {
  const int tid = threadIdx.x;
  Word k[ITEMS];
  T ev[ITEMS];
  load_and_sort<Word, T>(S.s, sortbits, k);
  const ScanCtx<Word, T> ctx = compaction_prepare<Word, T>(S.s, k, n, colbits, ev);
  int* stage_col = reinterpret_cast<int*>(S.s.words);
  T* stage_val = S.s.vals;
  int* misc = S.s.misc;
  // element n-1 (the last valid one) ends the last run and row: its state gives the
  // compacted total and the last row's count; publish it first
  const int owner = (n - 1) / ITEMS;
  if (threadIdx.x == owner) {
    compaction_emit<Word, T>(k, ev, n, colbits, ctx, [&](int idx, Word key, T, uint32_t state, bool) {
      if (idx == n - 1) {
        misc[0] = st_count(state);
        misc[1] = st_row_count(state);
        misc[2] = (int)(key >> colbits);
      }
    });
  }
  __syncthreads();   // also: every read of the sort buffers is done, staging may start
  const int total = misc[0], rc_last = misc[1], lastrel = misc[2];
  // keep the last row for the next iteration (L366) unless the block is done or the
  // row no longer fits the kept budget (reading R13: then it is written as a partial
  // chunk and merged later)
  const bool keep = st.keep_ok && size_after > 0 && rc_last <= KEEP && rmin + lastrel >= st.stop_row;
  const int nchunk = total - (keep ? rc_last : 0);
  // compacted element p goes to staging slot stage_slot(p): [0, nchunk) is the chunk,
  // the kept row stays at [nchunk, total) for the next iteration
  compaction_emit<Word, T>(k, ev, n, colbits, ctx, [&](int, Word key, T val, uint32_t state, bool row_end) {
    const int p = st_count(state) - 1;
    stage_col[stage_slot32(p)] = colof(key, 0);
    stage_val[stage_slot<T>(p)] = val;
    if (row_end && p < nchunk) {
      const int rc = st_row_count(state);
      const int rel = (int)(key >> colbits);
      a.row_count[S.row_of[rmin + rel]] = rc;        // per-row counter (L362)
      if (rel == 0) misc[3] = rc;
      if (p == nchunk - 1) { misc[4] = rel; misc[5] = rc; }
    }
  });
  __syncthreads();
  if (nchunk > 0) {
    // chunk write through shared memory for coalescing (L424-L426)
    const int64_t dst = pool_base + st.wofs;
    T* pv = reinterpret_cast<T*>(a.pool_val);
    for (int p = tid; p < nchunk; p += THREADS) {
      a.pool_col[dst + p] = stage_col[stage_slot32(p)];
      pv[dst + p] = stage_val[stage_slot<T>(p)];
    }
    if (tid == 0) {
      ChunkDesc d;
      d.data_off = dst;
      d.first_row = S.row_of[rmin];
      d.last_row = S.row_of[rmin + misc[4]];
      d.count = nchunk;
      d.first_count = misc[3];
      d.last_count = misc[5];
      d.flags = 0;
      a.descs[desc_base + st.seq] = d;
    }
    st.seq += 1;
    st.wofs += nchunk;
  }
  st.kept = keep ? rc_last : 0;
  st.kofs = nchunk;
  if (keep) {
    st.kept_lrow = rmin + lastrel;
    st.kept_cmin = stage_col[stage_slot32(nchunk)];
    st.kept_cmax = stage_col[stage_slot32(total - 1)];
  }
  __syncthreads();
}


// Radix path: key = (local row - rmin, column - cmin), all key bits sorted.
// One local ESC iteration after expansion (values already at s.vals[pos]): build the
// sort words, sort, compact (Alg. 3), emit completed rows as a chunk, keep the last row.
template <typename Word, typename T>
__device__ __forceinline__ void esc_iteration(EscSmem<T>& S, const EscArgs& a, EscState& st, int consume,
                                              int size_after, const int (&ares)[ITEMS], const int (&col)[ITEMS],
                                              const int (&kc)[KEEP_PER_THREAD], int rmin, int cmin, int rowbits,
                                              int colbits, int64_t pool_base, int64_t desc_base) {
  const int tid = threadIdx.x;
  const int kept = st.kept;
  const int n = kept + consume;
  Word* sw = reinterpret_cast<Word*>(S.s.words);
  // positions: kept elements first (they sort before equal keys, L366), then product c
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    if (ares[i] >= 0) {
      const int pos = kept + i * THREADS + tid;
      const Word key = ((Word)(S.a_lrow[ares[i]] - rmin) << colbits) | (Word)(col[i] - cmin);
      sw[pad32(pos)] = (key << IDXBITS) | (Word)pos;
    }
  }
#pragma unroll
  for (int j = 0; j < KEEP_PER_THREAD; ++j) {
    const int p = j * THREADS + tid;
    if (p < kept) {
      const Word key = ((Word)(st.kept_lrow - rmin) << colbits) | (Word)(kc[j] - cmin);
      sw[pad32(p)] = (key << IDXBITS) | (Word)p;
    }
  }
  for (int p = n + tid; p < CAP; p += THREADS) sw[pad32(p)] = ~(Word)0;
  __syncthreads();
  const Word colmask = colbits ? (((Word)1 << colbits) - (Word)1) : (Word)0;
  esc_tail<Word, T>(S, a, st, n, size_after, rmin, rowbits + colbits, colbits, pool_base, desc_base,
                    [&](Word key, int) { return cmin + (int)(key & colmask); });
}


// Split-word path for keys of 21..31 bits (R-MAT, LP: 20-bit columns plus row bits):
// instead of 64-bit sort words, sort 32-bit words (low 20 key bits | position) over
// their key bits, then the remaining high key bits, read by position from a 16-bit side
// array, in further stable passes.  Halves the shared-memory traffic of every pass.
// The sorted words are then widened to 64-bit (key | position) for the compaction.
template <typename T>
__device__ __forceinline__ void esc_iteration_split(EscSmem<T>& S, const EscArgs& a, EscState& st, int consume,
                                                    int size_after, const int (&ares)[ITEMS], const int (&col)[ITEMS],
                                                    const int (&kc)[KEEP_PER_THREAD], int rmin, int cmin, int rowbits,
                                                    int colbits, int64_t pool_base, int64_t desc_base) {
  constexpr int LOBITS = 31 - IDXBITS;                      // 20: pads (all ones) stay last
  const int tid = threadIdx.x;
  const int kept = st.kept;
  const int n = kept + consume;
  const int keybits = rowbits + colbits;
  uint32_t* sw = reinterpret_cast<uint32_t*>(S.s.words);
  uint16_t* hi16 = reinterpret_cast<uint16_t*>(S.s.words + CAP_PAD / 2);   // upper half of the buffer
  const uint64_t lomask = (1ull << LOBITS) - 1ull;
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    if (ares[i] >= 0) {
      const int pos = kept + i * THREADS + tid;
      const uint64_t key = ((uint64_t)(S.a_lrow[ares[i]] - rmin) << colbits) | (uint64_t)(col[i] - cmin);
      sw[pad32(pos)] = ((uint32_t)(key & lomask) << IDXBITS) | (uint32_t)pos;
      hi16[pos] = (uint16_t)(key >> LOBITS);
    }
  }
#pragma unroll
  for (int j = 0; j < KEEP_PER_THREAD; ++j) {
    const int p = j * THREADS + tid;
    if (p < kept) {
      const uint64_t key = ((uint64_t)(st.kept_lrow - rmin) << colbits) | (uint64_t)(kc[j] - cmin);
      sw[pad32(p)] = ((uint32_t)(key & lomask) << IDXBITS) | (uint32_t)p;
      hi16[p] = (uint16_t)(key >> LOBITS);
    }
  }
  for (int p = n + tid; p < CAP; p += THREADS) { sw[pad32(p)] = ~0u; hi16[p] = 0xFFFFu; }
  __syncthreads();
  uint32_t k[ITEMS];
  const int bb = pad32(tid * ITEMS);
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) k[i] = sw[bb + i];
  block_radix_sort<uint32_t>(k, sw, S.s.u.cnt, S.s.swarp, IDXBITS, IDXBITS + LOBITS);
  __syncthreads();
  block_radix_sort<uint32_t>(k, sw, S.s.u.cnt, S.s.swarp, 0, keybits - LOBITS,
                             [&](uint32_t w, int bit) { return (uint32_t)hi16[w & (uint32_t)(CAP - 1)] >> bit; });
  uint64_t k64[ITEMS];
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    const uint32_t pos = k[i] & (uint32_t)(CAP - 1);
    const uint64_t key = ((uint64_t)hi16[pos] << LOBITS) | (uint64_t)(k[i] >> IDXBITS);
    k64[i] = tid * ITEMS + i < n ? ((key << IDXBITS) | pos) : ~0ull;
  }
  __syncthreads();
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) S.s.words[bb + i] = k64[i];
  __syncthreads();
  const uint64_t colmask = colbits ? ((1ull << colbits) - 1ull) : 0ull;
  esc_tail<uint64_t, T>(S, a, st, n, size_after, rmin, 0, colbits, pool_base, desc_base,
                        [&](uint64_t key, int) { return cmin + (int)(key & colmask); });
}

// AC-ESC of one block b.
template <typename T>
__device__ __forceinline__ void esc_block(EscSmem<T>& S, const EscArgs& a, const int b) {
  const int tid = threadIdx.x;
  const int32_t* __restrict__ arp = a.A.row_ptr;
  const int32_t* __restrict__ acol = a.A.col;
  const T* __restrict__ aval = reinterpret_cast<const T*>(a.A.val);
  const int32_t* __restrict__ brp = a.B.row_ptr;
  const int32_t* __restrict__ bcol = a.B.col;
  const T* __restrict__ bval = reinterpret_cast<const T*>(a.B.val);
  const int nzb = a.blk_nz_begin[b];
  const int n_a = a.blk_nz_end[b] - nzb;
  const int r0 = a.block_row_starts[b];
  const int64_t rowsA = a.A.rows;

  // ---------------- Fetch A (§3.2.1) ----------------
  // row_ptr[r0 .. r0+NPB] covers every row of the block unless it has empty rows
  for (int t = tid; t <= NPB; t += THREADS) {
    const int64_t r = (int64_t)r0 + t;
    S.rp_cache[t] = r <= rowsA ? arp[r] : INT_MAX;
  }
  __syncthreads();
  int len[NNZ_PER_THREAD], row[NNZ_PER_THREAD];
#pragma unroll
  for (int j = 0; j < NNZ_PER_THREAD; ++j) {
    const int e = tid * NNZ_PER_THREAD + j;
    if (e < n_a) {
      const int nz = nzb + e;
      const int k = acol[nz];
      S.a_val[e] = aval[nz];
      const int bs = brp[k];
      S.a_bstart[e] = bs;
      len[j] = brp[k + 1] - bs;
      int r;
      if (nz < S.rp_cache[NPB]) {                 // row within the cached window
        int lo = 0, hi = NPB - 1;
        while (lo < hi) {
          const int mid = (lo + hi + 1) >> 1;
          if (S.rp_cache[mid] <= nz) lo = mid; else hi = mid - 1;
        }
        r = r0 + lo;
      } else {                                    // many (empty) rows: search globally
        int64_t lo = (int64_t)r0 + NPB, hi = rowsA - 1;
        while (lo < hi) {
          const int64_t mid = (lo + hi + 1) >> 1;
          if (arp[mid] <= nz) lo = mid; else hi = mid - 1;
        }
        r = (int)lo;
      }
      row[j] = r;
    } else {
      len[j] = 0;
      row[j] = INT_MAX;
    }
    if (e < NPB) S.a_lrow[e] = row[j];
  }
  __syncthreads();
  // dense local row ids: rank of the row among the block's rows
  int f[NNZ_PER_THREAD], cnt = 0;
#pragma unroll
  for (int j = 0; j < NNZ_PER_THREAD; ++j) {
    const int e = tid * NNZ_PER_THREAD + j;
    f[j] = (e < n_a) && (e == 0 || S.a_lrow[e - 1] != row[j]);
    cnt += f[j];
  }
  int tot;
  int run = block_exclusive_sum<int>(cnt, S.s.scratch, &tot);
#pragma unroll
  for (int j = 0; j < NNZ_PER_THREAD; ++j) {
    const int e = tid * NNZ_PER_THREAD + j;
    run += f[j];
    if (e < n_a) {
      S.a_lrow[e] = run - 1;
      if (f[j]) S.row_of[run - 1] = row[j];
    }
  }
  // long rows (§3.4): entries with B rows of more than PTR_LEN entries (at most PTR_MAX
  // per block, in entry order) leave the work distribution; their list (entry, products
  // before it) lives in rp_cache's storage, dead after Fetch A
  static_assert(3 * PTR_MAX <= NPB + 1, "long-row list fits rp_cache");
  int* ptr_e = S.rp_cache;                      // entry
  int* ptr_p = S.rp_cache + PTR_MAX;            // products of the entries before it
  int* ptr_n = S.rp_cache + 2 * PTR_MAX;        // its B row length
  int np_loc = 0;
#pragma unroll
  for (int j = 0; j < NNZ_PER_THREAD; ++j) np_loc += len[j] > PTR_LEN;
  int np_tot;
  const int prank0 = block_exclusive_sum<int>(np_loc, S.s.scratch, &np_tot);
  int prank[NNZ_PER_THREAD], plen[NNZ_PER_THREAD];
  {
    int r = prank0;
#pragma unroll
    for (int j = 0; j < NNZ_PER_THREAD; ++j) {
      const bool lng = len[j] > PTR_LEN;
      prank[j] = lng && r < PTR_MAX ? r : -1;   // beyond PTR_MAX: AC-ESC as any entry
      r += lng;
      plen[j] = len[j];
      if (prank[j] >= 0) len[j] = 0;
    }
  }
  wd_placework(len, S.wd, S.s.scratch);          // ends with a barrier: rp_cache is free
#pragma unroll
  for (int j = 0; j < NNZ_PER_THREAD; ++j) {
    if (prank[j] >= 0) {
      const int e = tid * NNZ_PER_THREAD + j;
      ptr_e[prank[j]] = e;
      ptr_p[prank[j]] = S.wd[e];
      ptr_n[prank[j]] = plen[j];
    }
  }
  const int np = min(np_tot, PTR_MAX);
  __syncthreads();

  EscState st{0, 0, 0, 0, 0, 0, 0, INT_MIN, true};
  const int64_t pool_base = a.pool_off[b];
  const int64_t desc_base = a.desc_off[b];
  const int total_products = S.wd[NPB];
  st.keep_ok = (int64_t)total_products <= (int64_t)(CAP / 2) * tot;
  int size = total_products;
  int pc = 0;                                   // next long-row entry
  // the long-row chunks whose position has been reached: a·B_k streamed into the pool
  auto emit_long = [&](int upto_products) {
    while (pc < np && ptr_p[pc] <= upto_products) {
      const int e = ptr_e[pc];
      const int n = ptr_n[pc];
      const int bs = S.a_bstart[e];
      const T av = S.a_val[e];
      const int64_t dst = pool_base + st.wofs;
      T* pv = reinterpret_cast<T*>(a.pool_val);
      for (int i = tid; i < n; i += THREADS) {
        a.pool_col[dst + i] = __ldg(bcol + bs + i);
        pv[dst + i] = av * __ldg(bval + bs + i);
      }
      if (tid == 0) {
        const int grow = S.row_of[S.a_lrow[e]];
        ChunkDesc d;
        d.data_off = dst;
        d.first_row = grow;
        d.last_row = grow;
        d.count = n;
        d.first_count = n;
        d.last_count = n;
        d.flags = 0;
        a.descs[desc_base + st.seq] = d;
        a.row_count[grow] = n;                  // a row with other chunks is merged (count rewritten)
      }
      st.seq += 1;
      st.wofs += n;
      ++pc;
    }
  };
  while (size > 0 || pc < np) {
    const int consumed = total_products - size;
    emit_long(consumed);
    if (size == 0) break;
    // stop at the next long-row chunk's position (L548); keep no complete row below it
    int consume = min(CAP - st.kept, size);
    st.stop_row = INT_MIN;
    if (pc < np && ptr_p[pc] - consumed <= consume) {
      consume = ptr_p[pc] - consumed;           // this iteration ends at the long row(s)
      // the last row may stay (be kept) only if it is the row of the last long-row chunk
      // emitted at this position: every chunk of a row must stay adjacent (L430)
      int last = pc;
      while (last + 1 < np && ptr_p[last + 1] == ptr_p[pc]) ++last;
      st.stop_row = S.a_lrow[ptr_e[last]];
    }
    // the kept row sits in the staging area, which the new values overwrite: pull it
    // into registers first (receivework's barriers order this before the writes)
    int kc[KEEP_PER_THREAD];
    T kv[KEEP_PER_THREAD];
#pragma unroll
    for (int j = 0; j < KEEP_PER_THREAD; ++j) {
      const int p = j * THREADS + tid;
      if (p < st.kept) {
        kc[j] = reinterpret_cast<int*>(S.s.words)[stage_slot32(st.kofs + p)];
        kv[j] = S.s.vals[stage_slot<T>(st.kofs + p)];
      } else {
        kc[j] = 0;
        kv[j] = (T)0;
      }
    }
    int ares[ITEMS], bres[ITEMS];
    wd_receivework(consume, S.wd, S.s.u.offsets, S.s.scratch, ares, bres);
    const int size_after = S.wd[NPB];
    // ---------------- expand (L340) ----------------
    int col[ITEMS];
    int rmin = INT_MAX, rmax = INT_MIN, cmin = INT_MAX, cmax = INT_MIN;
    // B addresses first, then all B loads of a half in flight, then the products
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) bres[i] = ares[i] >= 0 ? S.a_bstart[ares[i]] + bres[i] : 0;
    constexpr int HALF = ITEMS / 2;
#pragma unroll
    for (int h = 0; h < ITEMS; h += HALF) {
      T bv[HALF];
#pragma unroll
      for (int u = 0; u < HALF; ++u) {
        const int i = h + u;
        if (ares[i] >= 0) { col[i] = __ldg(bcol + bres[i]); bv[u] = __ldg(bval + bres[i]); }
        else { col[i] = 0; bv[u] = (T)0; }
      }
#pragma unroll
      for (int u = 0; u < HALF; ++u) {
        const int i = h + u;
        if (ares[i] >= 0) {
          const int e = ares[i];
          S.s.vals[st.kept + i * THREADS + tid] = S.a_val[e] * bv[u];
          const int lr = S.a_lrow[e];
          rmin = min(rmin, lr); rmax = max(rmax, lr);
          cmin = min(cmin, col[i]); cmax = max(cmax, col[i]);
        }
      }
    }
#pragma unroll
    for (int j = 0; j < KEEP_PER_THREAD; ++j) {
      const int p = j * THREADS + tid;
      if (p < st.kept) S.s.vals[p] = kv[j];
    }
    if (st.kept > 0) {
      rmin = min(rmin, st.kept_lrow); rmax = max(rmax, st.kept_lrow);
      cmin = min(cmin, st.kept_cmin); cmax = max(cmax, st.kept_cmax);
    }
    block_minmax4(rmin, rmax, cmin, cmax, S.s.scratch);
    // dynamic bit reduction (L342-L344): only the row and column ranges present
    const int rowbits = bit_width_u64((uint64_t)(rmax - rmin));
    const int colbits = bit_width_u64((uint64_t)((int64_t)cmax - (int64_t)cmin));
    if (rowbits + colbits + IDXBITS < 32)
      esc_iteration<uint32_t, T>(S, a, st, consume, size_after, ares, col, kc, rmin, cmin, rowbits, colbits,
                                 pool_base, desc_base);
    else if (rowbits + colbits <= 31 - IDXBITS + 16)
      esc_iteration_split<T>(S, a, st, consume, size_after, ares, col, kc, rmin, cmin, rowbits, colbits,
                             pool_base, desc_base);
    else
      esc_iteration<uint64_t, T>(S, a, st, consume, size_after, ares, col, kc, rmin, cmin, rowbits, colbits,
                                 pool_base, desc_base);
    size = size_after;
  }
  emit_long(INT_MAX);
  if (tid == 0) {
    a.nchunks[b] = st.seq;
    a.used[b] = (int32_t)st.wofs;
  }
}

// One CTA per block; with the adaptive strategy (hash_done set) a persistent grid takes
// the blocks the hash accumulator did not finish (reading R31) from a list, one at a time
// through an atomic counter, instead of launching a CTA per finished block.  Blocks are
// independent and write only their own chunk range: the order does not change any result.
template <typename T>
__global__ void __launch_bounds__(THREADS, ESC_MIN_BLOCKS) k_esc(EscArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  EscSmem<T>& S = *reinterpret_cast<EscSmem<T>*>(smem_raw);
  if (!a.hash_done) {
    const uint64_t t0 = a.trace ? global_timer() : 0;
    esc_block<T>(S, a, blockIdx.x);
    if (threadIdx.x == 0) trace_block(a.trace, blockIdx.x, t0);
    return;
  }
  const int64_t n = *a.esc_count;
  for (;;) {
    if (threadIdx.x == 0)
      S.s.misc[15] = (int)atomicAdd(reinterpret_cast<unsigned long long*>(a.esc_next), 1ull);
    __syncthreads();
    const int i = S.s.misc[15];
    __syncthreads();
    if (i >= n) break;
    const uint64_t t0 = a.trace ? global_timer() : 0;
    esc_block<T>(S, a, a.esc_list[i]);
    if (threadIdx.x == 0) trace_block(a.trace, a.esc_list[i], t0);
    __syncthreads();                                  // shared memory is reused by the next block
  }
}

template <typename T>
static void launch_esc_t(const EscArgs& a, cudaStream_t st) {
  const size_t smem = sizeof(EscSmem<T>);
  static ResidentCache rc;
  const int resident = resident_ctas(rc, k_esc<T>, THREADS, smem);   // also sets the smem limit
  int grid = a.nblocks;
  if (a.hash_done) grid = std::min<int>(a.nblocks, std::max(1, resident));
  k_esc<T><<<grid, THREADS, smem, st>>>(a);
}

void launch_esc(const EscArgs& a, bool f64, cudaStream_t st) {
  if (a.nblocks <= 0) return;
  if (f64) launch_esc_t<double>(a, st); else launch_esc_t<float>(a, st);
}

}  // namespace acs
