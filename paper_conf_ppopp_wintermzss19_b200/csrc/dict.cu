// Stage 2, adaptive alternative — column-dictionary accumulation (reading R33).
//
// PAPER.md L850 (§5) names the direction: "choose between alternative approaches (ESC,
// hashing, merging) depending on the load currently seen by the work distribution";
// L654: ESC's sort is "simply too high" a cost where rows compact strongly.  The hash
// accumulator (hash.cu, R31) removed the sort of the products but still pays a table
// probe per product and a sort per row.  In a block whose rows reuse the same B rows
// (stencils, meshes: the blocks k_block_bounds marks as candidates) both can be paid
// once per block instead of once per product and per row:
//   * Distinct B rows.  The block's NPB entries reference far fewer distinct B rows
//     (27-point stencil: ~190 for 512 entries); they are found with a small hash on the
//     B row start and staged back to back (offsets by a block scan).
//   * Dictionary.  Every column of the staged B rows sets a bit in a bitmap over the
//     block's column span [cmin, cmax]; a prefix of the word popcounts ranks them: the
//     dictionary index of column c is the number of distinct block columns below c.  So
//     the dictionary is sorted by column, without a sort.  Each staged B entry stores its
//     index (16 bits).
//   * Accumulation.  A warp owns a contiguous run of the block's rows (one chunk, as in
//     hash.cu) and a dense accumulator over the dictionary.  Per row it walks the
//     products in expansion order -- one entry of A times <= 32 entries of its B row per
//     wave -- and adds a_ik * b_kj to acc[index]; a B row has unique columns, so the lanes
//     of a wave touch distinct slots, and waves run in order: every output is the left
//     fold of its products in A-entry order from -0.0, exactly what the hash accumulator
//     computes (bit-identical results; fp64 rows inside a block equal the oracle's
//     Gustavson order bit for bit).  A 16-bit row stamp per slot marks the row's columns.
//   * Emission.  The stamps are scanned in dictionary order (= column order) with warp
//     ballots; the row's entries are written to the chunk coalesced, already sorted.
// A block whose distinct B rows hold more than DICT_NSMAX entries, whose span exceeds
// DICT_SPAN columns or whose dictionary exceeds DICT_DMAX columns is left to k_hash
// (hash_done stays 1; the test depends only on the data, so the choice is
// deterministic, and both kernels give the same bits).  hash_done[b] = 2 marks a block
// finished here: k_hash and AC-ESC skip it.
#include <cstdint>
#include "accum.cuh"

namespace acs {

constexpr int DICT_WARPS = 4;
constexpr int DICT_THREADS = 32 * DICT_WARPS;
static_assert(DICT_THREADS == THREADS, "fetch_block and the block scans assume THREADS");
constexpr int DICT_DMAX = 768;           // distinct columns of a block (dense accumulator slots)
constexpr int DICT_NSMAX = 6144;         // staged B entries (distinct B rows) of a block
constexpr int DICT_WORDS = 4096;         // bitmap words: column span <= 131,072
constexpr int64_t DICT_SPAN = 32LL * DICT_WORDS;
constexpr int DICT_RH = 1024;            // distinct-row hash slots (>= 2 NPB: never full)
constexpr int DICT_W = 4;                // waves per batch (loads of the next batch in flight)
static_assert(DICT_DMAX <= 32 * 32, "one ballot word per lane covers the dictionary");
static_assert(DICT_NSMAX < 65536 && DICT_DMAX < 65536, "16-bit indices");
static_assert(NPB < 65535, "16-bit row stamps");

template <typename T>
struct DictSmem {
  T a_val[NPB];                  // nonempty entries of the block, compacted (fetch_block)
  int4 ent[NPB];                 // (B row start, B row length, staged offset, distinct row id)
  int wd[NPB + 1];               // exclusive product prefix over compacted entries
  int row_first[NPB + 1];
  int row_of[NPB];
  int drow[NPB];                 // distinct B row -> one compacted entry referencing it
  int dsoff[NPB + 1];            // distinct B row -> staged offset
  uint16_t sidx[DICT_NSMAX];     // dictionary index of every staged B entry
  int dcol[DICT_DMAX];           // dictionary index -> column
  union {
    int rp_cache[NPB + 1];
    struct { int key[DICT_RH]; int id[DICT_RH]; } rh;                     // distinct B rows
    struct { uint32_t bits[DICT_WORDS]; uint16_t pre[DICT_WORDS]; } bm;    // column bitmap + ranks
    struct { T acc[DICT_WARPS][DICT_DMAX + 1]; uint16_t mark[DICT_WARPS][DICT_DMAX + 2]; } w;  // [DMAX]: dummy
  } u;
  int wrow[DICT_WARPS + 1];
  int wout[DICT_WARPS][5];
  int scratch[40];
  int nd, cmin, cmax, bad;
};

// position of the n-th (0-based) set bit of x (x has more than n set bits)
__device__ __forceinline__ int nth_set_bit(uint32_t x, int n) {
  int pos = 0;
#pragma unroll
  for (int s = 16; s > 0; s >>= 1) {
    const int c = __popc(x & ((1u << s) - 1u));
    if (n >= c) { n -= c; x >>= s; pos += s; }
  }
  return pos;
}

// Waves of one row: wave (entry c, offset o) = B entries [o, o+32) of entry c's row.
template <typename T>
struct DictCursor {
  int c, o, c1;
  int4 e;
  T ea;
  __device__ __forceinline__ void init(const DictSmem<T>& S, int c0, int c1_) {
    c = c0; o = 0; c1 = c1_;
    e = S.ent[c0];
    ea = S.a_val[c0];
  }
  __device__ __forceinline__ bool more() const { return c < c1; }
  // this lane's staged position, B position and A value of the current wave; advance
  __device__ __forceinline__ bool take(const DictSmem<T>& S, int lane, int& s, unsigned& q, T& a) {
    const bool live = c < c1;
    const bool v = live && o + lane < e.y;
    s = e.z + o + lane;
    q = (unsigned)(e.x + o + lane);
    a = ea;
    if (live) {
      if (o + 32 < e.y) {
        o += 32;
      } else {
        o = 0;
        ++c;
        if (c < c1) { e = S.ent[c]; ea = S.a_val[c]; }
      }
    }
    return v;
  }
};

// All products of one row, DICT_W waves at a time; the next batch's loads are issued
// before the current batch is accumulated.  Lanes without a product use the dummy slot
// DICT_DMAX, so every wave's read-modify-write runs converged and in wave order.
template <typename T>
__device__ __forceinline__ void dict_row(const DictSmem<T>& S, int c0, int c1, const T* __restrict__ bval, T* acc,
                                         uint16_t* mark, uint16_t stamp, int lane) {
  constexpr int W = DICT_W;
  DictCursor<T> cur;
  cur.init(S, c0, c1);
  int idx[W];
  T av[W], bv[W];
#pragma unroll
  for (int w = 0; w < W; ++w) {
    int s;
    unsigned q;
    const bool v = cur.take(S, lane, s, q, av[w]);
    idx[w] = v ? (int)S.sidx[s] : DICT_DMAX;
    bv[w] = v ? __ldg(bval + q) : (T)0;
  }
  for (;;) {
    const bool more = cur.more();
    int nidx[W];
    T nav[W], nbv[W];
#pragma unroll
    for (int w = 0; w < W; ++w) {
      int s;
      unsigned q;
      const bool v = cur.take(S, lane, s, q, nav[w]);
      nidx[w] = v ? (int)S.sidx[s] : DICT_DMAX;
      nbv[w] = v ? __ldg(bval + q) : (T)0;
    }
#pragma unroll
    for (int w = 0; w < W; ++w) {
      const T p = vmul(av[w], bv[w]);
      acc[idx[w]] = vadd(acc[idx[w]], p);
      mark[idx[w]] = stamp;
    }
    if (!more) break;
#pragma unroll
    for (int w = 0; w < W; ++w) { idx[w] = nidx[w]; av[w] = nav[w]; bv[w] = nbv[w]; }
  }
  __syncwarp();
}

template <typename T>
__global__ void __launch_bounds__(DICT_THREADS, 3) k_dict(EscArgs a) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  DictSmem<T>& S = *reinterpret_cast<DictSmem<T>*>(smem_raw);
  const unsigned FULL = 0xffffffffu;
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const int b = blockIdx.x;
  if (a.hash_done[b] != 1) return;       // not a candidate (k_block_bounds)
  const int32_t* __restrict__ bcol = a.B.col;
  const T* __restrict__ bval = reinterpret_cast<const T*>(a.B.val);

  // ---------------- Fetch A (§3.2.1) ----------------
  int nrows, nent, total;
  fetch_block<T>(a, b, S.u.rp_cache, S.row_of, S.row_first, S.ent, S.a_val, S.wd, S.scratch, nrows, nent, total);

  // ---------------- distinct B rows ----------------
  for (int i = tid; i < DICT_RH; i += DICT_THREADS) S.u.rh.key[i] = -1;
  if (tid == 0) { S.nd = 0; S.cmin = INT_MAX; S.cmax = INT_MIN; S.bad = 0; }
  __syncthreads();
  int myslot[NNZ_PER_THREAD];
#pragma unroll
  for (int j = 0; j < NNZ_PER_THREAD; ++j) {
    const int ci = tid + j * DICT_THREADS;
    myslot[j] = -1;
    if (ci < nent) {
      const int key = S.ent[ci].x;       // B row start: unique among nonempty B rows
      int h = (int)(((uint32_t)key * 2654435761u) >> 22);
      for (;;) {
        int k = S.u.rh.key[h];
        if (k == -1) {
          k = atomicCAS(&S.u.rh.key[h], -1, key);
          if (k == -1) {
            const int id = atomicAdd(&S.nd, 1);
            S.u.rh.id[h] = id;
            S.drow[id] = ci;
            break;
          }
        }
        if (k == key) break;
        h = (h + 1) & (DICT_RH - 1);
      }
      myslot[j] = h;
    }
  }
  __syncthreads();
  const int nd = S.nd;
#pragma unroll
  for (int j = 0; j < NNZ_PER_THREAD; ++j)
    if (myslot[j] >= 0) S.ent[tid + j * DICT_THREADS].w = S.u.rh.id[myslot[j]];
  // staged offsets of the distinct rows (blocked), and the block's column range
  int dl[NNZ_PER_THREAD], ssum = 0, cmn = INT_MAX, cmx = INT_MIN;
#pragma unroll
  for (int j = 0; j < NNZ_PER_THREAD; ++j) {
    const int d = tid * NNZ_PER_THREAD + j;
    dl[j] = 0;
    if (d < nd) {
      const int4 e = S.ent[S.drow[d]];
      dl[j] = e.y;
      cmn = min(cmn, bcol[e.x]);           // canonical B: columns ascending (R3)
      cmx = max(cmx, bcol[e.x + e.y - 1]);
    }
    ssum += dl[j];
  }
  cmn = __reduce_min_sync(FULL, cmn);
  cmx = __reduce_max_sync(FULL, cmx);
  if (lane == 0) { atomicMin(&S.cmin, cmn); atomicMax(&S.cmax, cmx); }
  int NS;
  int sex = block_exclusive_sum<int>(ssum, S.scratch, &NS);   // barriers: the id reads are done
#pragma unroll
  for (int j = 0; j < NNZ_PER_THREAD; ++j) {
    const int d = tid * NNZ_PER_THREAD + j;
    if (d < nd) S.dsoff[d] = sex;
    sex += dl[j];
  }
  const int cmin = S.cmin;
  const int64_t span = (int64_t)S.cmax - cmin + 1;
  if (NS > DICT_NSMAX || span > DICT_SPAN) return;     // uniform: k_hash takes the block
  const int nwords = (int)((span + 31) >> 5);
  for (int i = tid; i < nwords; i += DICT_THREADS) S.u.bm.bits[i] = 0;
  __syncthreads();                                     // dsoff, bitmap
#pragma unroll
  for (int j = 0; j < NNZ_PER_THREAD; ++j) {
    const int ci = tid + j * DICT_THREADS;
    if (ci < nent) S.ent[ci].z = S.dsoff[S.ent[ci].w];
  }

  // ---------------- dictionary: column bitmap over [cmin, cmax] ----------------
  for (int d = w; d < nd; d += DICT_WARPS) {
    const int4 e = S.ent[S.drow[d]];
    for (int j = lane; j < e.y; j += 32) {
      const int c = bcol[e.x + j] - cmin;
      if ((unsigned)c < (unsigned)span) atomicOr(&S.u.bm.bits[c >> 5], 1u << (c & 31));
      else S.bad = 1;                                  // non-canonical B row
    }
  }
  __syncthreads();
  if (S.bad) return;
  // ranks: warp w scans words [w·wpw, (w+1)·wpw)
  const int wpw = ((nwords + DICT_THREADS - 1) / DICT_THREADS) * 32;
  {
    int run = 0;
    const int i1 = min((w + 1) * wpw, nwords);
    for (int i0 = w * wpw; i0 < i1; i0 += 32) {
      const int i = i0 + lane;
      const int c = i < i1 ? __popc(S.u.bm.bits[i]) : 0;
      int inc = c;
#pragma unroll
      for (int d = 1; d < 32; d <<= 1) {
        const int y = __shfl_up_sync(FULL, inc, d);
        if (lane >= d) inc += y;
      }
      if (i < i1) S.u.bm.pre[i] = (uint16_t)(run + inc - c);
      run += __shfl_sync(FULL, inc, 31);
    }
    if (lane == 0) S.scratch[w] = run;
  }
  split_rows<DICT_WARPS>(S.wd, S.row_first, nrows, total, S.wrow);
  __syncthreads();
  int wbase = 0, D = 0;
#pragma unroll
  for (int q = 0; q < DICT_WARPS; ++q) {
    const int t = S.scratch[q];
    wbase += q < w ? t : 0;
    D += t;
  }
  if (D > DICT_DMAX) return;                           // uniform: k_hash takes the block
  if (wbase) {
    const int i1 = min((w + 1) * wpw, nwords);
    for (int i = w * wpw + lane; i < i1; i += 32) S.u.bm.pre[i] += (uint16_t)wbase;
  }
  __syncthreads();
  // dictionary index of every staged B entry; dcol inverts it
  for (int d = w; d < nd; d += DICT_WARPS) {
    const int4 e = S.ent[S.drow[d]];
    const int so = S.dsoff[d];
    for (int j = lane; j < e.y; j += 32) {
      const int col = bcol[e.x + j];
      const int c = col - cmin;
      const int idx = S.u.bm.pre[c >> 5] + __popc(S.u.bm.bits[c >> 5] & ((1u << (c & 31)) - 1u));
      S.sidx[so + j] = (uint16_t)idx;
      S.dcol[idx] = col;
    }
  }
  __syncthreads();                                     // the bitmap is dead: accumulators

  // ---------------- rows: accumulate, emit in dictionary (= column) order ----------------
  T* acc = S.u.w.acc[w];
  uint16_t* mark = S.u.w.mark[w];
  for (int i = lane; i <= DICT_DMAX; i += 32) { acc[i] = (T)(-0.0); mark[i] = 0; }
  __syncwarp();
  const int rlo = S.wrow[w], rhi = S.wrow[w + 1];
  const int64_t wbase_pool = a.pool_off[b] + (rlo < nrows ? S.wd[S.row_first[rlo]] : 0);
  T* pval = reinterpret_cast<T*>(a.pool_val);
  int32_t* pcol = a.pool_col;
  const int nwin = (D + 31) >> 5;
  int out = 0, first_row = -1, last_row = -1, first_count = 0, last_count = 0;
  for (int r = rlo; r < rhi; ++r) {
    const int c0 = S.row_first[r], c1 = S.row_first[r + 1];
    if (c0 == c1) continue;              // no products
    const uint16_t stamp = (uint16_t)(r + 1);
    dict_row<T>(S, c0, c1, bval, acc, mark, stamp, lane);
    // lane k holds the ballot of dictionary window k (columns 32k .. 32k+31)
    uint32_t myword = 0;
    for (int k = 0; k < nwin; ++k) {
      const int i = k * 32 + lane;
      const uint32_t bal = __ballot_sync(FULL, i < D && mark[i] == stamp);
      if (lane == k) myword = bal;
    }
    const int cnt = __popc(myword);
    int inc = cnt;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int y = __shfl_up_sync(FULL, inc, d);
      if (lane >= d) inc += y;
    }
    const int wpre = inc - cnt;
    const int U = __shfl_sync(FULL, inc, 31);
    const int64_t dst = wbase_pool + out;
    for (int j0 = 0; j0 < U; j0 += 32) {
      const int j = j0 + lane;
      int pos = 0;                       // last window whose prefix is <= j
#pragma unroll
      for (int step = 16; step > 0; step >>= 1) {
        const int x = __shfl_sync(FULL, wpre, pos + step);
        if (x <= j) pos += step;
      }
      const uint32_t word = __shfl_sync(FULL, myword, pos);
      const int rank = j - __shfl_sync(FULL, wpre, pos);
      if (j < U) {
        const int idx = pos * 32 + nth_set_bit(word, rank);
        pcol[dst + j] = S.dcol[idx];
        pval[dst + j] = acc[idx];
        acc[idx] = (T)(-0.0);
      }
    }
    __syncwarp();
    const int grow = S.row_of[r];
    if (lane == 0) a.row_count[grow] = U;     // per-row counter (L362)
    if (first_row < 0) { first_row = grow; first_count = U; }
    last_row = grow;
    last_count = U;
    out += U;
  }
  if (lane == 0) {
    S.wout[w][0] = out;
    S.wout[w][1] = first_row;
    S.wout[w][2] = last_row;
    S.wout[w][3] = first_count;
    S.wout[w][4] = last_count;
  }
  __syncthreads();
  if (tid == 0) {
    emit_warp_chunks(a, b, DICT_WARPS, S.wrow, S.wout, S.wd, S.row_first);
    a.hash_done[b] = 2;
    atomicAdd(reinterpret_cast<unsigned long long*>(a.dict_count), 1ull);
  }
}

template <typename T>
static void launch_dict_t(const EscArgs& a, cudaStream_t st) {
  const size_t smem = sizeof(DictSmem<T>);
  cudaFuncSetAttribute(k_dict<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  k_dict<T><<<a.nblocks, DICT_THREADS, smem, st>>>(a);
}

void launch_dict(const EscArgs& a, bool f64, cudaStream_t st) {
  if (a.nblocks <= 0) return;
  if (f64) launch_dict_t<double>(a, st); else launch_dict_t<float>(a, st);
}

}  // namespace acs
