// Block-level building blocks of local ESC, shared by the AC-ESC kernel, the three
// merge kernels and the debug entry points:
//   * the local work distribution (Alg. 2, §3.2.2),
//   * a stable block radix sort over packed (key | position) words with dynamic bit
//     range (§3.2.3),
//   * the compaction scan with the CombineScanOperator (Alg. 3).
// Shared-memory arrays that are read in blocked order (thread t reads t*ITEMS + i) use
// one padding word per 32 (`pad32`) so those reads are bank-conflict free.
#pragma once
#include "common.cuh"

namespace acs {

__device__ __forceinline__ int pad32(int i) { return i + (i >> 5); }
constexpr int CAP_PAD = CAP + CAP / 32;

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
// the row's remaining end (line 29).  `offsets` needs CAP_PAD ints.
__device__ __forceinline__ void wd_receivework(int consume, int* wd, int* offsets, int* scratch,
                                               int (&ares)[ITEMS], int (&bres)[ITEMS]) {
  const int tid = threadIdx.x;
  // line 14: clear(Offsets) — 0 is the identity of the max scan (reading R5)
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    const int c = i * THREADS + tid;
    if (c < consume) offsets[pad32(c)] = 0;
  }
  __syncthreads();
  // lines 16-20: mark the first product of every entry that starts inside the draw
#pragma unroll
  for (int i = 0; i < NNZ_PER_THREAD; ++i) {
    const int e = i * THREADS + tid;
    const int a = wd[e], an = wd[e + 1];
    if (a < consume && a != an) offsets[pad32(a)] = e;
  }
  __syncthreads();
  // line 24: block max scan, blocked layout
  int loc[ITEMS];
  int m = 0;
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    const int c = tid * ITEMS + i;
    m = max(m, c < consume ? offsets[pad32(c)] : 0);
    loc[i] = m;
  }
  const int ex = block_exclusive_max(m, scratch);
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    const int c = tid * ITEMS + i;
    if (c < consume) offsets[pad32(c)] = max(ex, loc[i]);
  }
  __syncthreads();
  // line 25: blocked -> striped; lines 26-32
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    const int c = i * THREADS + tid;
    if (c < consume) {
      const int e = offsets[pad32(c)];
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
// for bit-stable sums (L198).  Ranking: per-thread 16-bit digit counters packed two per
// word (RADIX_BITS = b -> 2^b digits = 2^(b-1) counter lanes x 2 halves), a raking exclusive
// scan over (lane, virtual thread) order, a scatter through shared memory.  Five
// barriers per pass.  Words live at pad32(index).
// =====================================================================

constexpr int CNT_LANES = 1 << (RADIX_BITS - 1);               // two 16-bit digits per word
// Each thread counts its ITEMS keys as VT "virtual threads" of ITEMS/VT consecutive keys
// with separate counter columns: the VT read-increment-write chains are independent, so
// their shared-memory latencies overlap; the (lane, virtual thread) scan order keeps the
// ranking stable because virtual thread tid*VT + v holds keys tid*ITEMS + v*ITEMS/VT ...
#ifndef ACS_VT
#define ACS_VT 1
#endif
constexpr int VT = ACS_VT;
constexpr int VTHREADS = THREADS * VT;
// ACS_ROT_RAKE: counter lanes without padding (LANE_STRIDE = VTHREADS, a multiple of 32)
// make the counting accesses bank-conflict free for any digits; the raking scan then
// reads its 16-word segment in a per-thread rotated order (conflict free as well) and
// undoes the rotation arithmetically.
#ifndef ACS_ROT_RAKE
#define ACS_ROT_RAKE 0
#endif
#ifndef ACS_LANE_STRIDE
#if ACS_ROT_RAKE
#define ACS_LANE_STRIDE (ACS_THREADS * ACS_VT)
#else
#define ACS_LANE_STRIDE (ACS_THREADS * ACS_VT + ACS_THREADS * ACS_VT / 32)
#endif
#endif
constexpr int LANE_STRIDE = ACS_LANE_STRIDE;                // padded words per counter lane
constexpr int CNT_PADDED = CNT_LANES * LANE_STRIDE;
constexpr int RAKE = CNT_LANES * VT;                        // words per thread in the raking scan
static_assert(RADIX_BITS >= 2 && RADIX_BITS <= 6, "two 16-bit halves x CNT_LANES lanes");
static_assert(VTHREADS % 32 == 0 && RAKE <= 32 && 32 % RAKE == 0, "raking layout");
static_assert(ITEMS <= 32 && 32 % ITEMS == 0, "blocked items must not straddle padding");
static_assert(ITEMS % VT == 0, "virtual threads split the items evenly");

struct ShiftDigit {
  template <typename Word>
  __device__ __forceinline__ uint32_t operator()(Word w, int bit) const { return (uint32_t)(w >> bit); }
};

// digit(word, bit) >> 0 & mask is the digit of a pass (default: the word's own bits)
template <typename Word, typename Digit = ShiftDigit>
__device__ __forceinline__ void block_radix_sort(Word (&k)[ITEMS], Word* s_words, uint32_t* s_cnt,
                                                 uint32_t* s_warp, int begin_bit, int end_bit,
                                                 Digit digit = Digit()) {
  constexpr int IPV = ITEMS / VT;                           // items per virtual thread
  const int tid = threadIdx.x, lane = lane_id(), w = warp_id();
  uint16_t* c16 = reinterpret_cast<uint16_t*>(s_cnt);
  // my raking segment: logical counter words [tid*RAKE, (tid+1)*RAKE) = lane L, virtual
  // threads v0 .. v0+RAKE-1 (contiguous: RAKE divides 32)
  const int v0 = (tid * RAKE) % VTHREADS;
#if ACS_ROT_RAKE
  static_assert(RAKE == 16 && VT == 1, "rotated raking layout");
  const int seg0 = ((tid * RAKE) / VTHREADS) * LANE_STRIDE + v0;
  const int rot = 4 * ((tid >> 3) & 3) + ((tid & 7) >> 1);  // distinct banks across a warp
#define ACS_CIDX(vt) (2 * (vt))
#define ACS_RK(j) (seg0 + (((j) + rot) & (RAKE - 1)))
#else
  const int seg0 = ((tid * RAKE) / VTHREADS) * LANE_STRIDE + v0 + (v0 >> 5);
#define ACS_CIDX(vt) (2 * ((vt) + ((vt) >> 5)))
#define ACS_RK(j) (seg0 + (j))
#endif
  const int bb = pad32(tid * ITEMS);                        // my blocked items (contiguous)
  if (begin_bit >= end_bit) return;
#pragma unroll
  for (int j = 0; j < RAKE; ++j) s_cnt[ACS_RK(j)] = 0u;
  __syncthreads();
  for (int bit = begin_bit; bit < end_bit; bit += RADIX_BITS) {
    const int nb = min(RADIX_BITS, end_bit - bit);
    const uint32_t mask = (1u << nb) - 1u;
    int cidx[ITEMS];
    uint32_t pre[ITEMS];
#pragma unroll
    for (int q = 0; q < IPV; ++q) {
#pragma unroll
      for (int v = 0; v < VT; ++v) {
        const int i = v * IPV + q;
        const int vt = tid * VT + v;
        const uint32_t d = digit(k[i], bit) & mask;
        cidx[i] = (int)(d & (CNT_LANES - 1)) * (2 * LANE_STRIDE) + (int)(d >> (RADIX_BITS - 1)) + ACS_CIDX(vt);
        pre[i] = c16[cidx[i]];
        c16[cidx[i]] = (uint16_t)(pre[i] + 1u);
      }
    }
    __syncthreads();
    uint32_t seg[RAKE];
    uint32_t sum = 0;
#pragma unroll
    for (int j = 0; j < RAKE; ++j) { seg[j] = s_cnt[ACS_RK(j)]; sum += seg[j]; }
    uint32_t inc = sum;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, inc, d);
      if (lane >= d) inc += y;
    }
    if (lane == 31) s_warp[w] = inc;
    __syncthreads();
    uint32_t wt = lane < THREADS / 32 ? s_warp[lane] : 0u;
#pragma unroll
    for (int d = 1; d < THREADS / 32; d <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, wt, d);
      if (lane >= d) wt += y;
    }
    const uint32_t grand = __shfl_sync(0xffffffffu, wt, THREADS / 32 - 1);
    uint32_t wpre = __shfl_up_sync(0xffffffffu, wt, 1);
    wpre = __shfl_sync(0xffffffffu, lane == 0 ? 0u : wpre, w);
    // digits in the high halves follow all digits in the low halves
    uint32_t run = wpre + inc - sum + ((grand & 0xFFFFu) << 16);
#if ACS_ROT_RAKE
    {
      // seg[m] holds counter (m + rot) mod 16 of the segment; its natural exclusive
      // prefix is R(m) - H + (m < 16 - rot ? sum : 0), R the rotated running sum and
      // H the sum of the first 16 - rot rotated words
      uint32_t H = 0, R = 0;
#pragma unroll
      for (int j = 0; j < RAKE; ++j) H += j < RAKE - rot ? seg[j] : 0u;
#pragma unroll
      for (int j = 0; j < RAKE; ++j) {
        // every packed half stays non-negative: no borrow between the two digits
        s_cnt[ACS_RK(j)] = run + (j < RAKE - rot ? (sum - H) + R : R - H);
        R += seg[j];
      }
    }
#else
#pragma unroll
    for (int j = 0; j < RAKE; ++j) { const uint32_t v = seg[j]; s_cnt[seg0 + j] = run; run += v; }
#endif
    __syncthreads();
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) {
      const int rank = (int)c16[cidx[i]] + (int)pre[i];
      s_words[pad32(rank)] = k[i];
    }
    __syncthreads();
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) k[i] = s_words[bb + i];
    if (bit + RADIX_BITS < end_bit) {
#pragma unroll
      for (int j = 0; j < RAKE; ++j) s_cnt[ACS_RK(j)] = 0u;
      __syncthreads();
    }
  }
#undef ACS_CIDX
#undef ACS_RK
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

__device__ __forceinline__ int st_count(uint32_t s) { return (int)((s >> 1) & 0x7FFFu); }
__device__ __forceinline__ int st_row_count(uint32_t s) { return (int)((s >> 17) & 0x7FFFu); }
__device__ __forceinline__ bool st_run_end(uint32_t s) { return s & 1u; }
__device__ __forceinline__ bool st_row_end(uint32_t s) { return (s >> 16) & 1u; }

// Shared-memory workspace for sort + compaction (one per CTA).
template <typename T>
struct SortSmem {
  union {
    int offsets[CAP_PAD];             // Alg. 2 Offsets (padded)
    uint32_t cnt[CNT_PADDED];         // radix counters
    int wprefix[CAP + 1];             // merge window prefix / path samples
  } u;
  uint64_t words[CAP_PAD];            // sort buffer at pad32(i) (uint32 words use the first
                                      // half); after the sort: int32 staging of output
                                      // columns at plain index p
  T vals[CAP];                        // values by position; after the sort: output staging
  CElem<uint64_t, T> warp_agg[2 * (THREADS / 32) + 1];
  uint8_t warp_has[2 * (THREADS / 32) + 1];
  uint32_t swarp[THREADS / 32];
  int scratch[40];
  int misc[16];
};

// The compaction scan (Alg. 3) over the sorted words of a thread (blocked layout).
// Within a thread the scan is a left fold; because the input is sorted, applying the
// CombineScanOperator to the running element and the next item only needs to know
// whether the previous item ended a run / a row (a.key == b.key  <=>  no run end
// between them; equalRow  <=>  no row end).  Across threads the operator itself
// combines the per-thread aggregates (warp Kogge-Stone, then the warps in order).
// Padding words (all ones) sort after the n valid elements and carry a key larger than
// every valid key (callers guarantee keybits + IDXBITS < word width), so they only form
// trailing runs of their own and never change a valid element's scan result; no
// per-item validity predicates are needed.
//   prepare: values into registers, the thread aggregate, the block scan of the
//            aggregates; returns the carry-in and publishes element n-1's scan result.
//   emit:    re-folds the thread's items from the carry and calls
//            f(idx, key, value, state, row_end) at every run end with idx < n.
// The tree is fixed by (THREADS, ITEMS): results are bit-stable run to run.
template <typename Word, typename T>
struct ScanCtx {
  CElem<Word, T> carry;
  bool has_carry;
  Word next_last;        // key following this thread's last item
};

template <typename Word, typename T>
__device__ __forceinline__ ScanCtx<Word, T> compaction_prepare(SortSmem<T>& s, const Word (&k)[ITEMS], int n,
                                                                int colbits, T (&ev)[ITEMS]) {
  const int lane = lane_id(), w = warp_id();
  const Word* sw = reinterpret_cast<const Word*>(s.words);
  const Word posmask = (Word)(CAP - 1);
  const int base = threadIdx.x * ITEMS;
  ScanCtx<Word, T> ctx;
  ctx.next_last = (base + ITEMS < CAP) ? (sw[pad32(base + ITEMS)] >> IDXBITS) : ~(Word)0;
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) ev[i] = s.vals[(int)(k[i] & posmask)];
  // thread-local fold (state bits: see Alg. 3)
  T val = ev[0];
  uint32_t state = 0;
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    const Word key = k[i] >> IDXBITS;
    const Word nkey = (i + 1 < ITEMS) ? (k[i + 1] >> IDXBITS) : ctx.next_last;
    const bool run_end = nkey != key;
    const bool row_end = (nkey >> colbits) != (key >> colbits);
    const uint32_t st0 = row_end ? ST_END_ROW : (run_end ? ST_END_COMP : 0u);
    if (i > 0) {
      const Word pkey = k[i - 1] >> IDXBITS;
      val = pkey != key ? ev[i] : val + ev[i];
      state = ((pkey >> colbits) != (key >> colbits) ? (state & 0x0000FFFEu) : (state & 0xFFFEFFFEu)) + st0;
    } else {
      state = st0;
    }
  }
  CElem<Word, T> inc;
  inc.key = k[ITEMS - 1] >> IDXBITS;
  inc.val = val;
  inc.state = state;
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    const CElem<Word, T> y = shfl_up_elem(inc, d);
    if (lane >= d) inc = combine_op(y, inc, colbits);
  }
  const CElem<Word, T> ex = shfl_up_elem(inc, 1);
  CElem<Word, T>* wagg = reinterpret_cast<CElem<Word, T>*>(s.warp_agg);
  if (lane == 31) wagg[w] = inc;
  __syncthreads();
  // one thread turns the warp aggregates into inclusive warp prefixes (fixed order)
  if (threadIdx.x == 0) {
    CElem<Word, T> run = wagg[0];
    for (int q = 1; q < THREADS / 32; ++q) {
      run = combine_op(run, wagg[q], colbits);
      wagg[q] = run;
    }
  }
  __syncthreads();
  if (w > 0) {
    const CElem<Word, T> wp = wagg[w - 1];
    ctx.carry = lane > 0 ? combine_op(wp, ex, colbits) : wp;
    ctx.has_carry = true;
  } else {
    ctx.carry = ex;
    ctx.has_carry = lane > 0;
  }
  return ctx;
}

template <typename Word, typename T, bool ALL = false, typename F>
__device__ __forceinline__ void compaction_emit(const Word (&k)[ITEMS], const T (&ev)[ITEMS], int n, int colbits,
                                                const ScanCtx<Word, T>& ctx, F&& f) {
  const int base = threadIdx.x * ITEMS;
  T val;
  uint32_t state;
  Word pkey;
  if (ctx.has_carry) {
    val = ctx.carry.val;
    state = ctx.carry.state;
    pkey = ctx.carry.key;
  }
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) {
    const Word key = k[i] >> IDXBITS;
    const Word nkey = (i + 1 < ITEMS) ? (k[i + 1] >> IDXBITS) : ctx.next_last;
    const bool run_end = nkey != key;
    const bool row_end = (nkey >> colbits) != (key >> colbits);
    const uint32_t st0 = row_end ? ST_END_ROW : (run_end ? ST_END_COMP : 0u);
    if (i > 0 || ctx.has_carry) {
      val = pkey != key ? ev[i] : val + ev[i];
      state = ((pkey >> colbits) != (key >> colbits) ? (state & 0x0000FFFEu) : (state & 0xFFFEFFFEu)) + st0;
    } else {
      val = ev[0];
      state = st0;
    }
    pkey = key;
    const int idx = base + i;
    if ((ALL || run_end) && idx < n) f(idx, key, val, state, row_end);
  }
}

// Load the n input words (written at pad32(pos), padding = all ones beyond n), sort the
// key bits.  On return k holds the sorted words of this thread (blocked) and s.words the
// whole sorted array at pad32(index).
template <typename Word, typename T>
__device__ __forceinline__ void load_and_sort(SortSmem<T>& s, int keybits, Word (&k)[ITEMS]) {
  Word* sw = reinterpret_cast<Word*>(s.words);
  const int bb = pad32(threadIdx.x * ITEMS);      // ITEMS divides 32: no padding inside
#pragma unroll
  for (int i = 0; i < ITEMS; ++i) k[i] = sw[bb + i];
  block_radix_sort<Word>(k, sw, s.u.cnt, s.swarp, IDXBITS, IDXBITS + keybits);
}

}  // namespace acs
