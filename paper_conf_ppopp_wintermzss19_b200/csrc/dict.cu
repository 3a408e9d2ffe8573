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
//     B row start and staged back to back, each padded to whole waves of 32 (offsets by
//     a block scan; pads hold a per-lane dummy index).
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
//     Gustavson order bit for bit).  A byte per dictionary slot marks the row's columns.
//   * Emission.  Lane k turns the marks of dictionary window k (32 slots) into a word; a
//     warp scan of the popcounts orders the row's indices into a list, and the row's
//     entries are written to the chunk coalesced in dictionary order = column order:
//     already sorted.
// A block whose distinct B rows hold more than DICT_NSMAX entries, whose span exceeds
// DICT_SPAN columns or whose dictionary exceeds DICT_DMAX columns is left to k_hash
// (hash_done stays 1; the test depends only on the data, so the choice is
// deterministic, and both kernels give the same bits).  hash_done[b] = 2 marks a block
// finished here: k_hash and AC-ESC skip it.
#include <cstdint>
#include "accum.cuh"

namespace acs {

#ifndef ACS_DICT_WARPS
#define ACS_DICT_WARPS ACC_MAX_WARPS
#endif
constexpr int DICT_WARPS = ACS_DICT_WARPS;  // 8: a block's rows over 8 warps, one chunk each
static_assert(DICT_WARPS <= ACC_MAX_WARPS, "chunk slots per block (k_block_bounds)");
constexpr int DICT_THREADS = 32 * DICT_WARPS;
constexpr int DICT_NPT = NPB / DICT_THREADS;   // A entries per thread in the block phases
#ifndef ACS_DICT_DMAX
#define ACS_DICT_DMAX 768
#endif
constexpr int DICT_DMAX = ACS_DICT_DMAX;  // distinct columns of a block (dense accumulator slots)
constexpr int DICT_NSMAX = 7168;         // staged B entries of a block (distinct B rows, padded to waves)
constexpr int DICT_WORDS = 4096;         // bitmap words: column span <= 131,072
constexpr int64_t DICT_SPAN = 32LL * DICT_WORDS;
constexpr int DICT_RH = 1024;            // distinct-row hash slots (>= 2 NPB: never full)
constexpr int DICT_W = 4;                // waves per batch (loads of the next batch in flight)
static_assert(DICT_DMAX <= 32 * 32, "one ballot word per lane covers the dictionary");
static_assert(DICT_NSMAX < 65536 && DICT_DMAX < 65536, "16-bit indices");

constexpr int DICT_EPAD = 2 * DICT_W;   // entries past the last one a prefetching row loop may read

// One warp's accumulator over the dictionary: acc[i] sums the current row's products of
// dictionary column i, mark[i] = 1 when the row has column i, list = the row's indices
// in column order while it is emitted.  Slots DICT_DMAX + lane are the idle lanes'
// dummies (one per lane: no two lanes of a wave ever touch one slot).
template <typename T>
struct DictWarp {
  T acc[DICT_DMAX + 32];
  union {                        // the marks are read into registers before the list is built
    alignas(16) uint8_t mark[DICT_DMAX + 32];
    uint16_t list[DICT_DMAX];
  };
};

template <typename T>
struct DictSmem {
  T a_val[NPB + DICT_EPAD];      // nonempty entries of the block, compacted (fetch_block)
  int4 ent[NPB + DICT_EPAD];     // (B row start, B row length, staged offset, last B position)
  int wd[NPB + 1];               // exclusive product prefix over compacted entries
  int row_first[NPB + 1];
  int row_of[NPB];
  uint16_t sidx[DICT_NSMAX + 32];  // dictionary index of every staged B entry; pads: DICT_DMAX + lane
  int dcol[DICT_DMAX];           // dictionary index -> column
  union {
    int rp_cache[NPB + 1];
    struct {                     // distinct B rows
      int key[DICT_RH];
      int id[DICT_RH];
      int drow[NPB];             // distinct B row -> a compacted entry referencing it
    } rh;
    struct {                     // staging: column bitmap + ranks, distinct rows' staged waves
      uint32_t bits[DICT_WORDS];
      uint16_t pre[DICT_WORDS];
      int dsoff[NPB];            // distinct B row -> staged offset (a multiple of 32)
      int2 dinfo[NPB];           // distinct B row -> (B row start, length)
      uint16_t wtab[DICT_NSMAX / 32];  // staged wave -> distinct B row
    } bm;
    DictWarp<T> w[DICT_WARPS];
  } u;
  int wrow[DICT_WARPS + 1];
  int wout[DICT_WARPS][6];
  alignas(8) int scratch[40];
  int nd, cmin, cmax, bad;
};
static_assert(DICT_DMAX % 32 == 0, "the dummy slots lie outside the emitted windows");

// Waves of one row: wave (entry c, offset o) = B entries [o, o+32) of entry c's row.
// Staged B rows are padded to whole waves with the dummy index, so a lane past the B row
// needs no test; past the row's last entry the wave reads the pad at DICT_NSMAX.  Global
// B positions are clamped to the B row's last entry (ent.w).
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
  __device__ __forceinline__ void take(const DictSmem<T>& S, int lane, int& s, unsigned& q, T& a) {
    const bool live = c < c1;
    s = live ? e.z + o + lane : DICT_NSMAX + lane;
    q = (unsigned)min(e.x + o + lane, e.w);
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
  }
};

// Accumulate one batch of waves and mark their dictionary indices.  Lanes without a
// product use their own dummy slot DICT_DMAX + lane (the staged pads hold it), so every
// wave's read-modify-write runs converged; __syncwarp orders the waves (left fold).
template <int W, typename T>
__device__ __forceinline__ void dict_accumulate(DictWarp<T>& Wp, const int (&idx)[W], const T (&av)[W],
                                                const T (&bv)[W]) {
#pragma unroll
  for (int w = 0; w < W; ++w) {
    const T p = vmul(av[w], bv[w]);
    Wp.acc[idx[w]] = vadd(Wp.acc[idx[w]], p);
    Wp.mark[idx[w]] = 1;
    __syncwarp();                        // wave w's writes are visible to wave w+1's lanes
  }
}

// Loads of W short waves, one per entry c .. c+W-1 (every lane: staged rows are padded,
// B positions clamped; the entries past the block are zero-filled pads).
template <int W, typename T>
__device__ __forceinline__ void dict_short_load(const DictSmem<T>& S, int c, const T* __restrict__ bval, int lane,
                                                int (&idx)[W], T (&av)[W], T (&bv)[W]) {
#pragma unroll
  for (int w = 0; w < W; ++w) {
    const int4 e = S.ent[c + w];
    av[w] = S.a_val[c + w];
    idx[w] = S.sidx[e.z + lane];
    bv[w] = __ldg(bval + (unsigned)min(e.x + lane, e.w));
  }
}

// Rows whose B rows all fit a wave (<= 32 entries): one wave per entry.  Full batches of
// DICT_W entries, the next batch's loads in flight while the current one accumulates;
// the remaining < DICT_W entries one wave at a time.
template <typename T>
__device__ __forceinline__ void dict_row_short(const DictSmem<T>& S, int c0, int c1, const T* __restrict__ bval,
                                               DictWarp<T>& Wp, int lane) {
  constexpr int W = DICT_W;
  const int nfull = (c1 - c0) / W;
  int c = c0;
  if (nfull > 0) {
    int ia[W], ib[W];
    T aa[W], ba[W], ab[W], bb[W];
    dict_short_load<W, T>(S, c, bval, lane, ia, aa, ba);
    for (int k = 0;;) {
      dict_short_load<W, T>(S, c + W, bval, lane, ib, ab, bb);
      dict_accumulate<W, T>(Wp, ia, aa, ba);
      c += W;
      if (++k == nfull) break;
      dict_short_load<W, T>(S, c + W, bval, lane, ia, aa, ba);
      dict_accumulate<W, T>(Wp, ib, ab, bb);
      c += W;
      if (++k == nfull) break;
    }
  }
  for (; c < c1; ++c) {
    int i1[1];
    T a1[1], b1[1];
    dict_short_load<1, T>(S, c, bval, lane, i1, a1, b1);
    dict_accumulate<1, T>(Wp, i1, a1, b1);
  }
  __syncwarp();
}

// Any row (B rows of any length): waves from DictCursor, DICT_W at a time; the next
// batch's loads are issued before the current batch is accumulated.
template <typename T>
__device__ __forceinline__ void dict_row(const DictSmem<T>& S, int c0, int c1, const T* __restrict__ bval,
                                         DictWarp<T>& Wp, int lane) {
  constexpr int W = DICT_W;
  DictCursor<T> cur;
  cur.init(S, c0, c1);
  int idx[W];
  T av[W], bv[W];
#pragma unroll
  for (int w = 0; w < W; ++w) {
    int s;
    unsigned q;
    cur.take(S, lane, s, q, av[w]);
    idx[w] = S.sidx[s];
    bv[w] = __ldg(bval + q);
  }
  for (;;) {
    const bool more = cur.more();
    int nidx[W];
    T nav[W], nbv[W];
#pragma unroll
    for (int w = 0; w < W; ++w) {
      int s;
      unsigned q;
      cur.take(S, lane, s, q, nav[w]);
      nidx[w] = S.sidx[s];
      nbv[w] = __ldg(bval + q);
    }
    dict_accumulate<W, T>(Wp, idx, av, bv);
    if (!more) break;
#pragma unroll
    for (int w = 0; w < W; ++w) { idx[w] = nidx[w]; av[w] = nav[w]; bv[w] = nbv[w]; }
  }
  __syncwarp();
}

template <typename T>
__global__ void __launch_bounds__(DICT_THREADS, DICT_WARPS == 8 ? 2 : 3) k_dict(EscArgs a) {
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
  const bool longb = fetch_block<T, int4, DICT_THREADS>(a, b, S.u.rp_cache, S.row_of, S.row_first, S.ent, S.a_val,
                                                        S.wd, S.scratch, nrows, nent, total);
  const bool short_rows = !__syncthreads_or(longb);

  // ---------------- distinct B rows ----------------
  if (tid < DICT_EPAD) {                 // entries a prefetching row loop reads past the last one
    S.ent[nent + tid] = make_int4(0, 0, 0, 0);
    S.a_val[nent + tid] = (T)0;
  }
  if (tid < 32) S.sidx[DICT_NSMAX + tid] = DICT_DMAX + tid;   // the pad wave of finished rows
  for (int i = tid; i < DICT_RH; i += DICT_THREADS) S.u.rh.key[i] = -1;
  if (tid == 0) { S.nd = 0; S.cmin = INT_MAX; S.cmax = INT_MIN; S.bad = 0; }
  __syncthreads();
  int myslot[DICT_NPT];
#pragma unroll
  for (int j = 0; j < DICT_NPT; ++j) {
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
            S.u.rh.drow[id] = ci;
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
  for (int j = 0; j < DICT_NPT; ++j)
    if (myslot[j] >= 0) S.ent[tid + j * DICT_THREADS].w = S.u.rh.id[myslot[j]];
  // staged offsets of the distinct rows (blocked; each padded to whole waves of 32), and
  // the block's column range
  int dl[DICT_NPT], dbst[DICT_NPT], ssum = 0, cmn = INT_MAX, cmx = INT_MIN;
#pragma unroll
  for (int j = 0; j < DICT_NPT; ++j) {
    const int d = tid * DICT_NPT + j;
    dl[j] = 0;
    dbst[j] = 0;
    if (d < nd) {
      const int4 e = S.ent[S.u.rh.drow[d]];
      dl[j] = e.y;
      dbst[j] = e.x;
      cmn = min(cmn, bcol[e.x]);           // canonical B: columns ascending (R3)
      cmx = max(cmx, bcol[e.x + e.y - 1]);
    }
    ssum += (dl[j] + 31) & ~31;
  }
  cmn = __reduce_min_sync(FULL, cmn);
  cmx = __reduce_max_sync(FULL, cmx);
  if (lane == 0) { atomicMin(&S.cmin, cmn); atomicMax(&S.cmax, cmx); }
  int NS;
  int sex = block_exclusive_sum_nt<DICT_THREADS, int>(ssum, S.scratch, &NS);   // barriers: rh is dead
  const int cmin = S.cmin;
  const int64_t span = (int64_t)S.cmax - cmin + 1;
  if (NS > DICT_NSMAX || span > DICT_SPAN) return;     // uniform: k_hash takes the block
#pragma unroll
  for (int j = 0; j < DICT_NPT; ++j) {
    const int d = tid * DICT_NPT + j;
    if (d < nd) {
      S.u.bm.dsoff[d] = sex;
      S.u.bm.dinfo[d] = make_int2(dbst[j], dl[j]);
      for (int g = sex >> 5; g < (sex + dl[j] + 31) >> 5; ++g) S.u.bm.wtab[g] = (uint16_t)d;
    }
    sex += (dl[j] + 31) & ~31;
  }
  const int nwords = (int)((span + 31) >> 5);
  for (int i = tid; i < nwords; i += DICT_THREADS) S.u.bm.bits[i] = 0;
  __syncthreads();                                     // dsoff, dinfo, wtab, bitmap
#pragma unroll
  for (int j = 0; j < DICT_NPT; ++j) {
    const int ci = tid + j * DICT_THREADS;
    if (ci < nent) {
      int4& e = S.ent[ci];
      e.z = S.u.bm.dsoff[e.w];
      e.w = e.x + e.y - 1;
    }
  }

  // ---------------- dictionary: column bitmap over [cmin, cmax] ----------------
  // warp-uniform over the staged waves (wave g = 32 staged positions of row wtab[g]),
  // SU waves per warp in flight
  constexpr int SU = 4;
  const int nwaves = NS >> 5;
  for (int g0 = w; g0 < nwaves; g0 += SU * DICT_WARPS) {
    int col[SU];
    bool v[SU];
#pragma unroll
    for (int u = 0; u < SU; ++u) {
      const int g = g0 + u * DICT_WARPS;
      const int d = g < nwaves ? S.u.bm.wtab[g] : 0;
      const int2 di = S.u.bm.dinfo[d];
      const int o = 32 * g + lane - S.u.bm.dsoff[d];
      v[u] = g < nwaves && o < di.y;
      col[u] = v[u] ? bcol[di.x + o] : cmin;
    }
#pragma unroll
    for (int u = 0; u < SU; ++u) {
      const int c = col[u] - cmin;
      if ((unsigned)c < (unsigned)span) {
        if (v[u]) atomicOr(&S.u.bm.bits[c >> 5], 1u << (c & 31));
      } else {
        S.bad = 1;                                     // non-canonical B row
      }
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
  // dictionary index of every staged B entry (pads: the dummy); dcol inverts it
  for (int g0 = w; g0 < nwaves; g0 += SU * DICT_WARPS) {
    int col[SU];
    bool v[SU];
#pragma unroll
    for (int u = 0; u < SU; ++u) {
      const int g = g0 + u * DICT_WARPS;
      const int d = g < nwaves ? S.u.bm.wtab[g] : 0;
      const int2 di = S.u.bm.dinfo[d];
      const int o = 32 * g + lane - S.u.bm.dsoff[d];
      v[u] = g < nwaves && o < di.y;
      col[u] = v[u] ? bcol[di.x + o] : cmin;
    }
#pragma unroll
    for (int u = 0; u < SU; ++u) {
      const int g = g0 + u * DICT_WARPS;
      if (g < nwaves) {
        const int c = col[u] - cmin;
        int idx = DICT_DMAX + lane;      // pad: this lane's dummy
        if (v[u]) {
          idx = S.u.bm.pre[c >> 5] + __popc(S.u.bm.bits[c >> 5] & ((1u << (c & 31)) - 1u));
          S.dcol[idx] = col[u];
        }
        S.sidx[32 * g + lane] = (uint16_t)idx;
      }
    }
  }
  __syncthreads();                                     // the bitmap is dead: accumulators

  // ---------------- rows: accumulate, emit in dictionary (= column) order ----------------
  DictWarp<T>& Wp = S.u.w[w];
  for (int i = lane; i < DICT_DMAX + 32; i += 32) Wp.acc[i] = (T)(-0.0);
  for (int i = lane; i < DICT_DMAX + 32; i += 32) Wp.mark[i] = 0;
  __syncwarp();
  const int rlo = S.wrow[w], rhi = S.wrow[w + 1];
  const int wrel = warp_out_base(a, S.wd, S.row_first, rlo, nrows, lane);
  const int64_t wbase_pool = a.pool_off[b] + wrel;
  T* pval = reinterpret_cast<T*>(a.pool_val);
  int32_t* pcol = a.pool_col;
  const int nwin = (D + 31) >> 5;
  int out = 0, first_row = -1, last_row = -1, first_count = 0, last_count = 0;
  for (int r = rlo; r < rhi; ++r) {
    const int c0 = S.row_first[r], c1 = S.row_first[r + 1];
    if (c0 == c1) continue;              // no products
    if (short_rows) dict_row_short<T>(S, c0, c1, bval, Wp, lane);
    else dict_row<T>(S, c0, c1, bval, Wp, lane);
    // lane k turns the marks of dictionary window k (indices 32k .. 32k+31) into a word
    uint32_t myword = 0;
    if (lane < nwin) {
      const uint4* mw = reinterpret_cast<const uint4*>(Wp.mark + 32 * lane);
      const uint4 m0 = mw[0], m1 = mw[1];
      const uint32_t q[8] = {m0.x, m0.y, m0.z, m0.w, m1.x, m1.y, m1.z, m1.w};
#pragma unroll
      for (int i = 0; i < 8; ++i) myword |= ((q[i] * 0x01020408u) >> 24) << (4 * i);   // bytes 0/1 -> 4 bits
    }
    __syncwarp();                        // marks read: the list may overwrite them
    const int cnt = __popc(myword);
    int inc = cnt;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int y = __shfl_up_sync(FULL, inc, d);
      if (lane >= d) inc += y;
    }
    const int U = __shfl_sync(FULL, inc, 31);
    // the row's dictionary indices in order (each lane lists its window's), then coalesced out
    for (int pos = inc - cnt; myword; myword &= myword - 1u, ++pos)
      Wp.list[pos] = (uint16_t)(32 * lane + __ffs(myword) - 1);
    __syncwarp();
    const int64_t dst = wbase_pool + out;
    for (int j = lane; j < U; j += 32) {
      const int idx = Wp.list[j];
      pcol[dst + j] = S.dcol[idx];
      pval[dst + j] = Wp.acc[idx];
      Wp.acc[idx] = (T)(-0.0);
    }
    __syncwarp();                        // list read: clear the marks for the next row
    if (lane < nwin) {
      uint4* mw = reinterpret_cast<uint4*>(Wp.mark + 32 * lane);
      mw[0] = make_uint4(0, 0, 0, 0);
      mw[1] = make_uint4(0, 0, 0, 0);
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
    S.wout[w][5] = wrel;
  }
  __syncthreads();
  if (tid == 0) {
    emit_warp_chunks(a, b, DICT_WARPS, S.wrow, S.wout, S.wd, S.row_first, a.hash_count);
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
