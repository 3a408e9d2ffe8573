// Stage 1 — Global Load Balancing (§3.1, Alg. 1) plus the
// per-block product bound used by the deterministic chunk allocator.
//
// A is split into canonical segments (nnz-balanced row ranges, reading
// R21) and each segment into blocks of NPB consecutive nonzeros counted from the
// segment's first nonzero ("splits the non-zeros of A uniformly, assigning the same
// number to each thread block", L194).  Rows never straddle segments, so the block
// decomposition -- and therefore every summation tree -- is the same whether the
// segments run on one GPU or on several.
#include <climits>
#include "kernels.cuh"

namespace acs {

// seg layout: [0, MAX_SEGMENTS] rows | [MAX_SEGMENTS+1, ...] first nonzero | block base
constexpr int SEG_STRIDE = MAX_SEGMENTS + 1;

__global__ void k_segments(const int32_t* __restrict__ rp, int64_t rows, int nseg, SegRows explicit_rows,
                           int64_t* __restrict__ seg, int32_t* __restrict__ nblocks, ZeroList zero) {
  __shared__ int64_t s_rows[SEG_STRIDE], s_nz[SEG_STRIDE];
  const int s = threadIdx.x;
#pragma unroll
  for (int i = 0; i < 4; ++i)
    for (int j = s; j < zero.n[i]; j += blockDim.x) zero.p[i][j] = 0;
  const int64_t base = rp[0];
  const int64_t nnz = (int64_t)rp[rows] - base;
  if (s <= nseg) {
    int64_t r;
    if (explicit_rows.n > 0) {
      r = explicit_rows.r[s];
    } else if (s == 0) {
      r = 0;
    } else if (s == nseg) {
      r = rows;
    } else {
      // first row r with rp[r] - base >= ceil(s * nnz / nseg)
      const int64_t target = (s * nnz + nseg - 1) / nseg;
      int64_t lo = 0, hi = rows;
      while (lo < hi) {
        const int64_t mid = (lo + hi) >> 1;
        if ((int64_t)rp[mid] - base < target) lo = mid + 1; else hi = mid;
      }
      r = lo;
    }
    s_rows[s] = r;
    s_nz[s] = rp[r];
  }
  __syncthreads();
  if (s == 0) {
    int64_t acc = 0;
    for (int i = 0; i <= nseg; ++i) {
      seg[i] = s_rows[i];
      seg[SEG_STRIDE + i] = s_nz[i];
      seg[2 * SEG_STRIDE + i] = acc;
      if (i < nseg) acc += (s_nz[i + 1] - s_nz[i] + NPB - 1) / NPB;
    }
    *nblocks = (int32_t)acc;
  }
}

void launch_segments(const CsrView& A, int nseg, const SegRows& explicit_rows, int64_t* seg,
                     int32_t* nblocks_dev, cudaStream_t st, const ZeroList& zero) {
  k_segments<<<1, 128, 0, st>>>(A.row_ptr, A.rows, nseg, explicit_rows, seg, nblocks_dev, zero);
}

// Alg. 1: one thread per row of A.  Reading R4: rows with a == b are skipped.
__global__ void k_glb(const int32_t* __restrict__ rp, int64_t rows, int nseg, const int64_t* __restrict__ seg,
                      int32_t* __restrict__ block_row_starts, int32_t* __restrict__ row_count) {
  __shared__ int64_t s_rows[SEG_STRIDE], s_nz[SEG_STRIDE], s_base[SEG_STRIDE];
  for (int i = threadIdx.x; i <= nseg; i += blockDim.x) {
    s_rows[i] = seg[i];
    s_nz[i] = seg[SEG_STRIDE + i];
    s_base[i] = seg[2 * SEG_STRIDE + i];
  }
  __syncthreads();
  const int64_t tid = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (tid >= rows) return;
  if (row_count) row_count[tid] = 0;
  const int64_t a0 = rp[tid], b0 = rp[tid + 1];
  if (a0 == b0) return;
  int s = 0;                                   // segment holding row tid
  while (s + 1 < nseg && s_rows[s + 1] <= tid) ++s;
  const int64_t a = a0 - s_nz[s], b = b0 - s_nz[s];
  int64_t blocka = (a + NPB - 1) / NPB;        // divup(a, NNZ_PER_BLOCK)
  const int64_t blockb = (b - 1) / NPB;        // (b - 1) / NNZ_PER_BLOCK
  while (blocka <= blockb) {
    block_row_starts[s_base[s] + blocka] = (int32_t)tid;
    ++blocka;
  }
}

void launch_glb(const CsrView& A, int nseg, const int64_t* seg, int32_t* brs, int64_t max_blocks, cudaStream_t st,
                int32_t* row_count) {
  (void)max_blocks;
  if (A.rows == 0) return;
  const int T = 256;
  k_glb<<<(unsigned)((A.rows + T - 1) / T), T, 0, st>>>(A.row_ptr, A.rows, nseg, seg, brs, row_count);
}

// Per block: nonzero range and the exact product count sum_p len(B_row(A.col[p])),
// "inspecting B now comes with little additional cost" (L206).  One warp per block.
// slots = ceil(products / (CAP - KEEP)) bounds the number of chunks the block emits
// (every local ESC iteration consumes at least CAP - KEEP products and emits at most
// one chunk), and products bounds its chunk elements (compaction never grows data).
//
// Hash accumulator candidate (reading R31), two deterministic tests on the block's own
// entries: (1) its waves (one entry x <= 32 entries of the entry's B row) keep at least
// half of the lanes busy -- short B rows stay in AC-ESC, whose draws pack them densely;
// (2) the rows are likely to compact: the B rows of adjacent entries share at least a
// quarter of their columns (8 sampled pairs, first <= 32 columns of each) -- random-
// column rows barely compact, and AC-ESC's sort is cheaper than hashing and then
// sorting them.  The candidates are counted (ncand) so that no k_hash is launched when
// there is none.
__global__ void k_block_bounds(const int32_t* __restrict__ arp, const int32_t* __restrict__ acol,
                               const int32_t* __restrict__ brp, const int32_t* __restrict__ bcol, int nseg,
                               const int64_t* __restrict__ seg, const int32_t* __restrict__ nblocks_dev,
                               int64_t max_blocks, int32_t* __restrict__ nz_begin, int32_t* __restrict__ nz_end,
                               int64_t* __restrict__ products, int64_t* __restrict__ slots,
                               int32_t* __restrict__ hash_ok, int64_t* __restrict__ ncand,
                               int64_t* __restrict__ max_products, int64_t* __restrict__ nblocks_out,
                               const int32_t* __restrict__ brs, int64_t rows_a, int64_t* __restrict__ est) {
  __shared__ int64_t s_nz[SEG_STRIDE], s_base[SEG_STRIDE];
  __shared__ int s_cand;
  for (int i = threadIdx.x; i <= nseg; i += blockDim.x) {
    s_nz[i] = seg[SEG_STRIDE + i];
    s_base[i] = seg[2 * SEG_STRIDE + i];
  }
  if (threadIdx.x == 0) s_cand = 0;
  __syncthreads();
  const int64_t b = ((int64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int nblocks = *nblocks_dev;
  if (nblocks_out && blockIdx.x == 0 && threadIdx.x == 0) *nblocks_out = nblocks;
  if (b < max_blocks && b >= nblocks && lane == 0) {
    products[b] = 0; slots[b] = 0; nz_begin[b] = 0; nz_end[b] = 0;
    if (est) est[b] = 0;
    if (hash_ok) hash_ok[b] = 0;
  }
  if (b < nblocks) {
    int s = 0;
    while (s + 1 < nseg && s_base[s + 1] <= b) ++s;
    const int64_t nzb = s_nz[s] + (b - s_base[s]) * NPB;
    const int64_t nze = min(nzb + (int64_t)NPB, s_nz[s + 1]);
    int64_t sum = 0, waves = 0;
    int nlong = 0;                            // long-row chunks (§3.4): one chunk + one split each
    // all of the block's column loads first (NPB / 32 per lane), then the B row gathers
    constexpr int PER_LANE = NPB / 32;
    int k[PER_LANE];
#pragma unroll
    for (int j = 0; j < PER_LANE; ++j) {
      const int64_t p = nzb + lane + 32 * j;
      k[j] = p < nze ? acol[p] : -1;
    }
#pragma unroll
    for (int j = 0; j < PER_LANE; ++j) {
      if (k[j] >= 0) {
        const int len = brp[k[j] + 1] - brp[k[j]];
        sum += len;
        waves += (len + 31) >> 5;
        nlong += len > PTR_LEN;
      }
    }
#pragma unroll
    for (int d = 16; d > 0; d >>= 1) {
      sum += __shfl_xor_sync(0xffffffffu, sum, d);
      waves += __shfl_xor_sync(0xffffffffu, waves, d);
      nlong += __shfl_xor_sync(0xffffffffu, nlong, d);
    }
    int hok = 0;
    if (hash_ok && sum > 0 && 2 * sum >= 32 * waves) {
      constexpr int NS = 8;                   // sampled adjacent pairs
      const int64_t n = nze - nzb;
      int ov = 0, mn = 0;
      if (n >= 2) {
        int v1[NS], v2[NS], l1[NS], l2[NS];
#pragma unroll
        for (int q = 0; q < NS; ++q) {
          const int64_t p = nzb + ((int64_t)q * (n - 1)) / NS;
          const int k1 = acol[p], k2 = acol[p + 1];
          const int a0 = brp[k1], b0 = brp[k2];
          l1[q] = min(brp[k1 + 1] - a0, 32);
          l2[q] = min(brp[k2 + 1] - b0, 32);
          v1[q] = lane < l1[q] ? bcol[a0 + lane] : INT_MAX;
          v2[q] = lane < l2[q] ? bcol[b0 + lane] : INT_MAX;
        }
#pragma unroll
        for (int q = 0; q < NS; ++q) {
          // position of v1 among the sorted v2 (held across the lanes): count of v2 < v1
          int pos = 0;
#pragma unroll
          for (int step = 16; step > 0; step >>= 1) {
            const int x = __shfl_sync(0xffffffffu, v2[q], pos + step - 1);
            if (x < v1[q]) pos += step;
          }
          const int at = __shfl_sync(0xffffffffu, v2[q], pos & 31);
          ov += lane < l1[q] && pos < 32 && at == v1[q];
          mn += min(l1[q], l2[q]);
        }
      }
      ov = __reduce_add_sync(0xffffffffu, ov);
      hok = mn > 0 && 4 * ov >= mn;
    }
    if (lane == 0) {
      // the block kernels count a block's products in 32 bits (fetch_block): a block of
      // >= 2^31 products is refused by the symbolic pass (read back with the totals)
      if (sum > (int64_t)INT_MAX) atomicMax(reinterpret_cast<unsigned long long*>(max_products), (unsigned long long)sum);
      if (hash_ok) hash_ok[b] = hok;
      if (hok) atomicAdd(&s_cand, 1);
      products[b] = sum;
      if (est) {
        // POOL_BOUND (reading R40): a candidate's accumulator output is at most HASH_UBOUND
        // columns per row (k_hash) or fewer (k_rows); its rows lie in [brs[b], brs[b+1]]
        const int64_t last = b + 1 < nblocks ? (int64_t)brs[b + 1] : rows_a - 1;
        const int64_t nr = last - brs[b] + 1;
        est[b] = hok ? min(sum, nr * (int64_t)HASH_UBOUND) : sum;
      }
      // the accumulators (R31, R33) emit up to one chunk per warp
      slots[b] = sum > 0 ? max((sum + (CAP - KEEP) - 1) / (CAP - KEEP), (int64_t)ACC_MAX_WARPS) +
                               2 * (int64_t)min(nlong, PTR_MAX) : 0;
      nz_begin[b] = (int32_t)nzb;
      nz_end[b] = (int32_t)nze;
    }
  }
  __syncthreads();
  if (threadIdx.x == 0 && ncand && s_cand)
    atomicAdd(reinterpret_cast<unsigned long long*>(ncand), (unsigned long long)s_cand);
}

void launch_block_bounds(const CsrView& A, const CsrView& B, int nseg, const int64_t* seg,
                         const int32_t* nblocks_dev, int64_t max_blocks, int32_t* nzb, int32_t* nze,
                         int64_t* products, int64_t* slots, int32_t* hash_ok, int64_t* ncand,
                         int64_t* max_products, int64_t* nblocks_out, const int32_t* brs, int64_t rows_a,
                         int64_t* est, cudaStream_t st) {
  if (max_blocks == 0) return;
  const int T = 256, WPB = T / 32;
  k_block_bounds<<<(unsigned)((max_blocks + WPB - 1) / WPB), T, 0, st>>>(
      A.row_ptr, A.col, B.row_ptr, B.col, nseg, seg, nblocks_dev, max_blocks, nzb, nze, products, slots, hash_ok,
      ncand, max_products, nblocks_out, brs, rows_a, est);
}

// Canonical-CSR check (reading R3): row_ptr monotone, columns strictly increasing and
// in range.  Only run when acspgemm_options.validate_inputs is set.
__global__ void k_validate(const int32_t* __restrict__ rp, const int32_t* __restrict__ col, int64_t rows,
                           int64_t cols, int32_t* bad) {
  const int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (r >= rows) return;
  const int64_t a = rp[r], b = rp[r + 1];
  if (b < a) { *bad = 1; return; }
  for (int64_t p = a; p < b; ++p) {
    const int c = col[p];
    if (c < 0 || c >= cols || (p > a && col[p - 1] >= c)) { *bad = 1; return; }
  }
}

void launch_validate(const CsrView& M, int32_t* bad, cudaStream_t st) {
  if (M.rows == 0) return;
  k_validate<<<(unsigned)((M.rows + 255) / 256), 256, 0, st>>>(M.row_ptr, M.col, M.rows, M.cols, bad);
}

}  // namespace acs
