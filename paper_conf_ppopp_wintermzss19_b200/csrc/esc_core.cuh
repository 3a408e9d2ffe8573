// Block-level building blocks of local ESC, shared by the AC-ESC kernel, the three
// merge kernels and the debug entry points:
//   * the local work distribution (Alg. 2, §3.2.2),
//   * a stable block radix sort over packed (key | position) words with dynamic bit
//     range (§3.2.3),
//   * the compaction scan with the CombineScanOperator (Alg. 3).
#pragma once
#include "common.cuh"

namespace acs {

// =====================================================================
// Alg. 2 — local work distribution.  WDState[NPB+1] lives in shared memory.
// =====================================================================

// placework (lines 2-7): inclusive prefix sum of the products owed per A entry.
// Entries are in blocked layout: thread t owns entries t*NNZ_PER_THREAD + j (reading
// R5: line 5's index is tid*NNZ_PER_THREAD + i + 1).
__device__ __forceinline__ void wd_placework(const int (&len)[NNZ_PER_THREAD], int* wd, int* scratch) {
  int s = 0;
#pragma unroll
  for (int j = 0; j < NNZ_PER_THREAD; ++j) s += len[j];
  int total;
  int run = block_exclusive_sum<int>(s, scratch, &total);
#pragma unroll
  for (int j = 0; j < NNZ_PER_THREAD; ++j) {
    run += len[j];
    wd[threadIdx.x * NNZ_PER_THREAD + j + 1] = run;
  }
  if (threadIdx.x == 0) wd[0] = 0;
  __syncthreads();
}

// receivework (lines 10-38) for `consume` (<= size()) products.  On return thread t
// holds products c = i*THREADS + t (striped, line 25) as (ares[i], bres[i]); ares = -1
// marks c >= consume.  Bres is the offset inside the A entry's B row counted down from
// the row's remaining end (line 29).  `offsets` needs CAP ints.
__device__ __forceinline__ void wd_receivework(int consume, int* wd, int* offsets, int* scratch,
                                               int (&ares)[ITEMS], int (&bres)[ITEMS]) {
  const int tid = threadIdx.x;
  // line 14: clear(Offsets) — 0 is the identity of the max scan (reading R5)
  for (int c = tid; c < consume; c += THREADS) offsets[c] = 0;
  __syncthreads();
  // lines 16-20: mark the first product of every entry that starts inside the draw
#pragma unroll
  for (int i = 0; i < NNZ_PER_THREAD; ++i) {
    const int e = i * THREADS + tid;
    const int a = wd[e], an = wd[e + 1];
    if (a < consume && a != an) offsets[a] = e;
  }
  __syncthreads();
  // line 24: block max scan, blocked layout
  int loc[ITEMS];
  int m = 0;
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    const int c = tid * ITEMS + i;
    m = max(m, c < consume ? offsets[c] : 0);
    loc[i] = m;
  }
  const int ex = block_exclusive_max(m, scratch);
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    const int c = tid * ITEMS + i;
    if (c < consume) offsets[c] = max(ex, loc[i]);
  }
  __syncthreads();
  // line 25: blocked -> striped; lines 26-32
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    const int c = i * THREADS + tid;
    if (c < consume) {
      const int e = offsets[c];
      ares[i] = e;
      bres[i] = wd[e + 1] - c - 1;
    } else {
      ares[i] = -1;
      bres[i] = -1;
    }
  }
  __syncthreads();
  // lines 34-36
#pragma unroll
  for (int i = 0; i < NNZ_PER_THREAD; ++i) {
    const int j = tid + i * THREADS + 1;
    wd[j] = max(0, wd[j] - consume);
  }
  __syncthreads();
}

// =====================================================================
// Stable block radix sort of packed words, blocked layout.
// A word is  key << IDXBITS | position.  Sorting only the key bits with a stable LSD
// radix sort keeps equal keys in position order, i.e. the expansion order (kept
// elements first, then products by A entry) that the paper's stable sort preserves
// for bit-stable sums (L198).  Ranking uses per-thread 16-bit digit counters packed
// two per word (RADIX_BITS = 5 -> 32 digits = 16 counter lanes x 2 halves), a raking
// exclusive scan over (lane, thread) order, and a scatter through shared memory.
// =====================================================================

constexpr int CNT_LANES = 16;
constexpr int CNT_WORDS = CNT_LANES * THREADS;
constexpr int CNT_PADDED = CNT_WORDS + CNT_WORDS / 32;
constexpr int RAKE = CNT_WORDS / THREADS;
static_assert(RADIX_BITS <= 5, "two 16-bit halves x 16 lanes");

__device__ __forceinline__ int cpad(int w) { return w + (w >> 5); }

template <typename Word>
__device__ __forceinline__ void block_radix_sort(Word (&k)[ITEMS], Word* s_words, uint32_t* s_cnt,
                                                 uint32_t* s_scan, int begin_bit, int end_bit) {
  const int tid = threadIdx.x;
  uint16_t* c16 = reinterpret_cast<uint16_t*>(s_cnt);
  for (int bit = begin_bit; bit < end_bit; bit += RADIX_BITS) {
    const int nb = min(RADIX_BITS, end_bit - bit);
    const uint32_t mask = (1u << nb) - 1u;
#pragma unroll
    for (int j = 0; j < RAKE; ++j) s_cnt[cpad(tid * RAKE + j)] = 0u;
    __syncthreads();
    int cidx[ITEMS];
    uint32_t pre[ITEMS];
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) {
      const uint32_t d = (uint32_t)(k[i] >> bit) & mask;
      const int W = (int)(d & 15u) * THREADS + tid;
      cidx[i] = cpad(W) * 2 + (int)(d >> 4);
      pre[i] = c16[cidx[i]];
      c16[cidx[i]] = (uint16_t)(pre[i] + 1u);
    }
    __syncthreads();
    uint32_t seg[RAKE];
    uint32_t sum = 0;
#pragma unroll
    for (int j = 0; j < RAKE; ++j) { seg[j] = s_cnt[cpad(tid * RAKE + j)]; sum += seg[j]; }
    uint32_t total;
    const uint32_t excl = block_exclusive_sum<uint32_t>(sum, s_scan, &total);
    uint32_t run = excl + ((total & 0xFFFFu) << 16);   // digits 16..31 follow all of 0..15
#pragma unroll
    for (int j = 0; j < RAKE; ++j) { const uint32_t v = seg[j]; s_cnt[cpad(tid * RAKE + j)] = run; run += v; }
    __syncthreads();
    int rank[ITEMS];
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) rank[i] = (int)c16[cidx[i]] + (int)pre[i];
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) s_words[rank[i]] = k[i];
    __syncthreads();
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) k[i] = s_words[tid * ITEMS + i];
  }
}

// =====================================================================
// Alg. 3 — compaction scan.
// Element: key (row bits above `colbits`, column bits below), value, 32-bit state:
//   bit 0 run end (end of a combine sequence), bits 1-15 compacted-element counter,
//   bit 16 row end, bits 17-31 per-row counter (L348, L354).
// =====================================================================

constexpr uint32_t ST_END_ROW = 0x00030003u;   // L354 "end row"
constexpr uint32_t ST_END_COMP = 0x00020003u;  // L354 "end comp"

template <typename Key, typename T>
struct CElem {
  Key key;
  T val;
  uint32_t state;
};

// CombineScanOperator (L352-L360) with reading R6: equal rows keep both counters and
// clear the flag bits (& 0xFFFEFFFE); a new row also clears the row counter
// (& 0x0000FFFE).  Keys are sorted, so a.key == b.key means all of b continues a's run.
template <typename Key, typename T>
__device__ __forceinline__ CElem<Key, T> combine_op(const CElem<Key, T>& a, const CElem<Key, T>& b, int colbits) {
  CElem<Key, T> r;
  const bool eq_row = (a.key >> colbits) == (b.key >> colbits);
  const uint32_t st = eq_row ? (a.state & 0xFFFEFFFEu) : (a.state & 0x0000FFFEu);
  r.key = b.key;
  r.val = (a.key == b.key) ? a.val + b.val : b.val;
  r.state = st + b.state;
  return r;
}

template <typename Key, typename T>
__device__ __forceinline__ CElem<Key, T> shfl_up_elem(const CElem<Key, T>& x, int d) {
  CElem<Key, T> y;
  y.key = __shfl_up_sync(0xffffffffu, x.key, d);
  y.val = __shfl_up_sync(0xffffffffu, x.val, d);
  y.state = __shfl_up_sync(0xffffffffu, x.state, d);
  return y;
}

// Inclusive block scan of ITEMS elements per thread (blocked layout) with the fixed
// tree: thread-sequential, warp Kogge-Stone, then the warps in order.  The tree is
// fixed by (THREADS, ITEMS), so results are bit-stable run to run.
template <typename Key, typename T>
__device__ __forceinline__ void block_compaction_scan(CElem<Key, T> (&x)[ITEMS], int colbits,
                                                      CElem<Key, T>* s_warp) {
  const int lane = lane_id(), w = warp_id();
#pragma unroll
  for (int i = 1; i < ITEMS; ++i) x[i] = combine_op(x[i - 1], x[i], colbits);
  CElem<Key, T> inc = x[ITEMS - 1];
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    CElem<Key, T> y = shfl_up_elem(inc, d);
    if (lane >= d) inc = combine_op(y, inc, colbits);
  }
  CElem<Key, T> ex = shfl_up_elem(inc, 1);
  if (lane == 31) s_warp[w] = inc;
  __syncthreads();
  bool has = false;
  CElem<Key, T> pre;
  if (w > 0) {
    pre = s_warp[0];
    for (int j = 1; j < w; ++j) pre = combine_op(pre, s_warp[j], colbits);
    has = true;
  }
  if (lane > 0) {
    pre = has ? combine_op(pre, ex, colbits) : ex;
    has = true;
  }
  if (has) {
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) x[i] = combine_op(pre, x[i], colbits);
  }
  __syncthreads();
}

__device__ __forceinline__ int st_count(uint32_t s) { return (int)((s >> 1) & 0x7FFFu); }
__device__ __forceinline__ int st_row_count(uint32_t s) { return (int)((s >> 17) & 0x7FFFu); }
__device__ __forceinline__ bool st_run_end(uint32_t s) { return s & 1u; }
__device__ __forceinline__ bool st_row_end(uint32_t s) { return (s >> 16) & 1u; }

// Shared-memory workspace for sort + compaction (one per CTA).
template <typename T>
struct SortSmem {
  union {
    int offsets[CAP];                 // Alg. 2 Offsets
    uint32_t cnt[CNT_PADDED];         // radix counters
    int wprefix[CAP + 1];             // merge window prefix
  } u;
  uint64_t words[CAP];                // sort buffer (uint32 words use the first half);
                                      // reused as int32 staging of output columns
  T vals[CAP];                        // values by position; reused as output staging
  CElem<uint64_t, T> warp_agg[THREADS / 32];
  uint32_t scan32[THREADS / 32 + 1];
  int scratch[40];
  int misc[16];
};

// Load the sorted words (blocked), run the compaction scan and leave per element
// (key, run sum, state).  Words in s.words[0..CAP) hold key<<IDXBITS|pos, positions
// >= n are padding (all ones) and sort last.
template <typename Word, typename T>
__device__ __forceinline__ void sort_and_scan(SortSmem<T>& s, int n, int keybits, int colbits,
                                              CElem<Word, T> (&x)[ITEMS]) {
  Word* sw = reinterpret_cast<Word*>(s.words);
  Word k[ITEMS];
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) k[i] = sw[threadIdx.x * ITEMS + i];
  block_radix_sort<Word>(k, sw, s.u.cnt, s.scan32, IDXBITS, IDXBITS + keybits);
  // after the last pass the sorted words are also in sw (blocked order); with zero
  // passes sw already is the input order
  const Word posmask = (Word)(CAP - 1);
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    const int idx = threadIdx.x * ITEMS + i;
    const Word key = k[i] >> IDXBITS;
    Word nkey;
    if (i + 1 < ITEMS) nkey = k[i + 1] >> IDXBITS;
    else nkey = (idx + 1 < CAP) ? (sw[idx + 1] >> IDXBITS) : key;
    const bool valid = idx < n;
    const bool last = idx == n - 1;
    x[i].key = valid ? key : ~(Word)0;
    x[i].val = valid ? s.vals[(int)(k[i] & posmask)] : (T)0;
    uint32_t st = 0;
    if (valid) {
      const bool run_end = last || nkey != key;
      const bool row_end = last || (nkey >> colbits) != (key >> colbits);
      st = row_end ? ST_END_ROW : (run_end ? ST_END_COMP : 0u);
    }
    x[i].state = st;
  }
  __syncthreads();   // all reads of words / vals done
  block_compaction_scan<Word, T>(x, colbits, reinterpret_cast<CElem<Word, T>*>(s.warp_agg));
}

}  // namespace acs
