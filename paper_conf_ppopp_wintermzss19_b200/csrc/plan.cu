// Host orchestration of AC-SpGEMM (Fig. 2; §3.5) behind
// the C ABI declared in include/acspgemm.h.
//
// Stage sequence on one caller stream:
//   GLB      segments -> Alg. 1 -> per-block nonzero range and exact product count ->
//            scans giving every block a deterministic chunk-pool range and descriptor
//            slot range                                     [read-back 1: totals]
//   ESC      one CTA per block                               (esc.cu)
//   MCC      dense chunk order, shared rows                  [read-back 2: counts]
//            classification, merge offsets, Multi-Merge packing [read-back 3]
//   MM/PM/SM the three merges                                (merge.cu)
//   SCAN     row_ptr of C                                    [read-back 4: nnz(C)]
//   CC       (numeric) chunk copy into C                     (copy.cu)
#include <cmath>
#include <cstdio>
#include <cstring>
#include <new>
#include <string>
#include <vector>
#include <array>

#include <algorithm>

#include "../../include/acspgemm.h"
#include "esc_core.cuh"
#include "kernels.cuh"

namespace acs {
thread_local long long tl_launches = 0;
}

namespace {

using namespace acs;

thread_local std::string tl_err;

acspgemm_status set_err(acspgemm_status s, const std::string& msg) {
  tl_err = msg;
  return s;
}

#define ACS_CUDA(call)                                                                        \
  do {                                                                                        \
    cudaError_t e_ = (call);                                                                  \
    if (e_ != cudaSuccess) {                                                                  \
      if (e_ == cudaErrorMemoryAllocation) {                                                  \
        cudaGetLastError();                                                                   \
        return set_err(ACSPGEMM_ERR_OUT_OF_MEMORY, std::string(#call) + ": " + cudaGetErrorString(e_)); \
      }                                                                                       \
      return set_err(ACSPGEMM_ERR_CUDA, std::string(#call) + ": " + cudaGetErrorString(e_)); \
    }                                                                                         \
  } while (0)

struct DevBuf {
  void* p = nullptr;
  size_t bytes = 0;
};

// mapped host buffer h_scal: [0, 32) read-backs, [32, 97) unused, [97, 162) segment
// boundaries read back for acspgemm_info
constexpr int H_SEG_ROWS = 32;
constexpr int H_SEG_INFO = H_SEG_ROWS + MAX_SEGMENTS + 1;
constexpr int H_SCAL_WORDS = H_SEG_INFO + MAX_SEGMENTS + 1;
// S_HASHEND: end of the accumulator part of the ESC stage (stage 8 "HASH": k_dict + k_hash);
// S_DICTEND: end of its column-dictionary part (stage 9 "DICT": k_dict)
enum Stage { S_GLB = 0, S_ESC, S_MCC, S_MM, S_PM, S_SM, S_SCAN, S_CC, S_END, S_HASHEND, S_DICTEND, NSTAGE_EV };

}  // namespace

struct acspgemm_plan_s {
  acspgemm_options opt;
  int nseg_explicit = 0;
  int64_t seg_rows_explicit[MAX_SEGMENTS + 1];
  // buffers
  DevBuf seg, scal, brs, nzb, nze, bprod, bslot, pool_off, desc_off, nchunks, chunk_base, rows_list;
  DevBuf pool_col, pool_val, descs, dense, sflag, spos, shared, row_count, row_ptr, scan_tmp;
  DevBuf kflag, kpos, lmulti, lpath, lsearch, lpair, mscan, mtscan, group_of, gstart, merge_col, merge_val;
  DevBuf cur_first, cur_last, err, bused, bused_scan, hdone, esc_list, esc_list_small;
  DevBuf lgiant, g_lo, g_nsl, g_base, g_pos, g_tcol, g_tval, g_tcnt;
  DevBuf best, boff, bdef, bdef_scan;   // POOL_BOUND (R40): regions, their scan, deferred flags + scan   // dense-slice merge (R30): lists, spans, slices
  DevBuf trace;                  // acspgemm_set_trace: per block (SM, start, end) x 4 kernels (mpL)
  bool trace_on = false;
  int64_t trace_blocks = 0;
  // acspgemm_multiply_host: device copies of A and B, two C piece buffers, copy stream
  DevBuf hp_a[3], hp_b[3], hp_c[2][3];
  cudaStream_t hp_cs = nullptr;
  cudaEvent_t hp_ready = nullptr, hp_copied[2] = {nullptr, nullptr};
  cudaStream_t hp_in = nullptr;             // input copies (multiply_host), piece by piece
  cudaEvent_t hp_start = nullptr, hp_inev[MAX_SEGMENTS + 1] = {};   // [S]: B when it is not A
  DevBuf hp_rng;                            // a piece's column range
  int64_t* h_scal = nullptr;     // pinned read-back buffer
  cudaEvent_t ev[NSTAGE_EV];
  bool ev_ok = false;
  // last problem
  bool ready = false;
  bool empty = true;
  bool f64 = true;
  int64_t rows = 0, cols = 0, nnz = 0;
  int64_t max_chunks = 0, total_chunks = 0, nshared = 0;
  acspgemm_info info;
  long long launches_sym = 0;
  int dev = 0;
  // pattern replay (acspgemm_numeric_update): the host values of every read-back of the
  // last symbolic, in order, and the problem they describe; replaying them makes the
  // launch sequence sync-free, so it is captured once into a CUDA graph
  std::vector<std::vector<int64_t>> rec;
  size_t rec_pos = 0;
  bool replay = false;
  int64_t rec_dims[6] = {-1, -1, -1, -1, -1, -1};   // A rows, cols, nnz; B rows, cols, nnz
  int rec_dtype = -1;
  cudaGraphExec_t gexec = nullptr;
  const void* gkey[9] = {};
  // acspgemm_multiply_budget: the pieces' C buffers (row_ptr, col, val), kept for reuse
  std::vector<std::array<DevBuf, 3>> bp;
};

namespace {

acspgemm_status ensure(DevBuf& b, size_t bytes) {
  if (bytes == 0) bytes = 16;
  if (b.bytes >= bytes) return ACSPGEMM_OK;
  if (b.p) {
    cudaError_t e = cudaFree(b.p);
    if (e != cudaSuccess) return set_err(ACSPGEMM_ERR_CUDA, std::string("cudaFree: ") + cudaGetErrorString(e));
    b.p = nullptr;
    b.bytes = 0;
  }
  size_t want = bytes + bytes / 8;          // headroom so repeated calls do not re-allocate
  cudaError_t e = cudaMalloc(&b.p, want);
  if (e != cudaSuccess) {
    cudaGetLastError();
    b.p = nullptr;
    return set_err(ACSPGEMM_ERR_OUT_OF_MEMORY,
                   "cudaMalloc(" + std::to_string(want) + " bytes): " + cudaGetErrorString(e));
  }
  b.bytes = want;
  return ACSPGEMM_OK;
}

#define ACS_ENSURE(buf, bytes)                          \
  do {                                                  \
    acspgemm_status s_ = ensure((buf), (size_t)(bytes)); \
    if (s_ != ACSPGEMM_OK) return s_;                   \
  } while (0)

// Grow a buffer to `bytes`, keeping its first `keep` bytes (POOL_BOUND's deferred regions).
acspgemm_status grow_keep(DevBuf& b, size_t bytes, size_t keep, cudaStream_t st) {
  if (b.bytes >= bytes) return ACSPGEMM_OK;
  void* np = nullptr;
  const size_t want = bytes + bytes / 8;
  cudaError_t e = cudaMalloc(&np, want);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return set_err(ACSPGEMM_ERR_OUT_OF_MEMORY, "cudaMalloc(" + std::to_string(want) + " bytes): " + cudaGetErrorString(e));
  }
  if (keep && b.p) {
    e = cudaMemcpyAsync(np, b.p, keep, cudaMemcpyDeviceToDevice, st);
    if (e != cudaSuccess) return set_err(ACSPGEMM_ERR_CUDA, std::string("cudaMemcpyAsync: ") + cudaGetErrorString(e));
  }
  if (b.p) cudaFree(b.p);                  // synchronises: the copy is done
  b.p = np;
  b.bytes = want;
  return ACSPGEMM_OK;
}

// scan_tmp: zero when (re)allocated; the scans leave it zero (scan.cu)
acspgemm_status ensure_scan_tmp(DevBuf& b, int64_t elems, cudaStream_t st) {
  void* old = b.p;
  acspgemm_status s = ensure(b, sizeof(int64_t) * elems);
  if (s == ACSPGEMM_OK && b.p != old) {
    cudaError_t e = cudaMemsetAsync(b.p, 0, b.bytes, st);
    if (e != cudaSuccess) return set_err(ACSPGEMM_ERR_CUDA, std::string("cudaMemsetAsync: ") + cudaGetErrorString(e));
  }
  return s;
}

#define ACS_ENSURE_SCAN_TMP(buf, elems, st)                  \
  do {                                                       \
    acspgemm_status s_ = ensure_scan_tmp((buf), (elems), (st)); \
    if (s_ != ACSPGEMM_OK) return s_;                        \
  } while (0)

template <typename P>
P* ptr(DevBuf& b) { return reinterpret_cast<P*>(b.p); }

void free_buf(DevBuf& b) {
  if (b.p) cudaFree(b.p);
  b.p = nullptr;
  b.bytes = 0;
}

void record(acspgemm_plan p, int stage, cudaStream_t st) {
  if (p->opt.collect_stage_times && p->ev_ok && !p->replay) cudaEventRecord(p->ev[stage], st);
}

acspgemm_status check_in(const acspgemm_csr_in* M, const char* name) {
  if (!M) return set_err(ACSPGEMM_ERR_INVALID_ARG, std::string(name) + " is NULL");
  if (M->rows < 0 || M->cols < 0 || M->nnz < 0)
    return set_err(ACSPGEMM_ERR_INVALID_ARG, std::string(name) + ": negative size");
  if (M->rows >= (int64_t(1) << 31) - 1 || M->cols >= (int64_t(1) << 31) - 1 || M->nnz >= (int64_t(1) << 31))
    return set_err(ACSPGEMM_ERR_INVALID_ARG, std::string(name) + ": size exceeds int32 indexing");
  if (M->rows > 0 && !M->row_ptr) return set_err(ACSPGEMM_ERR_INVALID_ARG, std::string(name) + ".row_ptr is NULL");
  if (M->nnz > 0 && (!M->col_idx || !M->val))
    return set_err(ACSPGEMM_ERR_INVALID_ARG, std::string(name) + ": NULL col_idx/val with nnz > 0");
  return ACSPGEMM_OK;
}

int64_t helper_bytes(acspgemm_plan p) {
  DevBuf* bs[] = {&p->seg, &p->scal, &p->brs, &p->nzb, &p->nze, &p->bprod, &p->bslot,
                  &p->pool_off, &p->desc_off, &p->nchunks, &p->chunk_base, &p->descs, &p->dense, &p->sflag,
                  &p->spos, &p->shared, &p->row_count, &p->row_ptr, &p->scan_tmp, &p->kflag, &p->kpos,
                  &p->lmulti, &p->lpath, &p->lsearch, &p->lpair, &p->mscan, &p->mtscan, &p->group_of, &p->gstart,
                  &p->merge_col, &p->merge_val, &p->cur_first, &p->cur_last, &p->err, &p->bused, &p->bused_scan, &p->hdone, &p->esc_list, &p->esc_list_small, &p->rows_list, &p->best, &p->boff, &p->bdef, &p->bdef_scan};
  int64_t t = 0;
  for (DevBuf* b : bs) t += (int64_t)b->bytes;
  return t;
}

// Read n device words into h_scal (a host round trip), recorded for pattern replay; in
// replay the recorded values are used instead (no launch, no synchronisation).
// extra_*: a second read-back in the same launch (not recorded; skipped in replay).
acspgemm_status sync_read(acspgemm_plan p, const int64_t* dev, int n, cudaStream_t st, const void* extra_src = nullptr,
                          void* extra_dst = nullptr, int extra_bytes = 0) {
  if (p->replay) {
    if (p->rec_pos >= p->rec.size() || (int)p->rec[p->rec_pos].size() != n)
      return set_err(ACSPGEMM_ERR_INTERNAL, "pattern replay out of step");
    std::memcpy(p->h_scal, p->rec[p->rec_pos].data(), sizeof(int64_t) * n);
    ++p->rec_pos;
    return ACSPGEMM_OK;
  }
  if (extra_src)
    launch_read_back2(dev, p->h_scal, (int)sizeof(int64_t) * n, extra_src, extra_dst, extra_bytes, st);
  else
    launch_read_back(dev, p->h_scal, (int)sizeof(int64_t) * n, st);
  tl_launches += 1;
  ACS_CUDA(cudaStreamSynchronize(st));
  p->rec.emplace_back(p->h_scal, p->h_scal + n);
  return ACSPGEMM_OK;
}

acspgemm_status symbolic_impl(acspgemm_plan p, const acspgemm_csr_in* A, const acspgemm_csr_in* B,
                              acspgemm_dtype dtype, cudaStream_t st, int64_t* nnz_c) {
  acspgemm_status s;
  if ((s = check_in(A, "A")) != ACSPGEMM_OK) return s;
  if ((s = check_in(B, "B")) != ACSPGEMM_OK) return s;
  if (!nnz_c) return set_err(ACSPGEMM_ERR_INVALID_ARG, "nnz_c is NULL");
  if (dtype != ACSPGEMM_F32 && dtype != ACSPGEMM_F64) return set_err(ACSPGEMM_ERR_INVALID_ARG, "bad dtype");
  if (A->cols != B->rows) return set_err(ACSPGEMM_ERR_DIM_MISMATCH, "A.cols != B.rows");
  ACS_CUDA(cudaGetDevice(&p->dev));
  const long long l0 = tl_launches;
  if (p->replay) {
    p->rec_pos = 0;
  } else {
    p->rec.clear();
    if (p->gexec) { cudaGraphExecDestroy(p->gexec); p->gexec = nullptr; }
    const int64_t dims[6] = {A->rows, A->cols, A->nnz, B->rows, B->cols, B->nnz};
    std::memcpy(p->rec_dims, dims, sizeof(dims));
    p->rec_dtype = (int)dtype;
  }
  p->ready = false;
  p->f64 = dtype == ACSPGEMM_F64;
  p->rows = A->rows;
  p->cols = B->cols;
  std::memset(&p->info, 0, sizeof(p->info));
  const int vbytes = p->f64 ? 8 : 4;
  p->info.pool_estimate_bytes =
      acspgemm_pool_estimate_bytes(A->rows, A->nnz, B->rows, B->cols, B->nnz, vbytes);
  const CsrView Av{A->rows, A->cols, A->row_ptr, A->col_idx, A->val};
  const CsrView Bv{B->rows, B->cols, B->row_ptr, B->col_idx, B->val};

  // empty inputs are legal (reading R18): C has no entries, no kernels run
  if (A->rows == 0 || A->nnz == 0 || B->nnz == 0) {
    p->empty = true;
    p->nnz = 0;
    p->ready = true;
    *nnz_c = 0;
    p->info.nsegments = 0;
    p->launches_sym = 0;
    return ACSPGEMM_OK;
  }
  p->empty = false;
  ACS_ENSURE(p->scal, sizeof(int64_t) * 32);
  ACS_ENSURE(p->err, sizeof(int32_t) * 4);
  int64_t* scal = ptr<int64_t>(p->scal);

  if (p->opt.validate_inputs && !p->replay) {
    ACS_CUDA(cudaMemsetAsync(p->err.p, 0, sizeof(int32_t) * 4, st));
    launch_validate(Av, ptr<int32_t>(p->err), st);
    launch_validate(Bv, ptr<int32_t>(p->err), st);
    tl_launches += 2;
    launch_read_back(p->err.p, p->h_scal, sizeof(int32_t), st);
    tl_launches += 1;
    ACS_CUDA(cudaStreamSynchronize(st));
    if (*reinterpret_cast<volatile int32_t*>(p->h_scal) != 0)
      return set_err(ACSPGEMM_ERR_INVALID_ARG, "input is not canonical CSR (row_ptr/col order/range)");
  }

  // ------------------------------------------------------------ GLB -----------
  record(p, S_GLB, st);
  int nseg = p->nseg_explicit > 0 ? p->nseg_explicit : p->opt.num_segments;
  if (nseg < 1) nseg = DEFAULT_SEGMENTS;
  if (nseg > MAX_SEGMENTS) nseg = MAX_SEGMENTS;
  const int64_t max_blocks = (A->nnz + NPB - 1) / NPB + nseg;
  ACS_ENSURE(p->seg, sizeof(int64_t) * 3 * (MAX_SEGMENTS + 1));
  SegRows explicit_rows;
  explicit_rows.n = 0;
  if (p->nseg_explicit > 0) {
    if (p->seg_rows_explicit[p->nseg_explicit] != A->rows)
      return set_err(ACSPGEMM_ERR_INVALID_ARG, "explicit segments do not end at A.rows");
    // by value in the kernel arguments: a captured graph (numeric_update) keeps this
    // copy, whatever later calls do to the plan's segments
    explicit_rows.n = nseg + 1;
    for (int i = 0; i <= nseg; ++i) explicit_rows.r[i] = p->seg_rows_explicit[i];
  }
  ACS_ENSURE(p->brs, sizeof(int32_t) * max_blocks);
  ACS_ENSURE(p->nzb, sizeof(int32_t) * max_blocks);
  ACS_ENSURE(p->nze, sizeof(int32_t) * max_blocks);
  ACS_ENSURE(p->bprod, sizeof(int64_t) * max_blocks);
  ACS_ENSURE(p->bslot, sizeof(int64_t) * max_blocks);
  ACS_ENSURE(p->pool_off, sizeof(int64_t) * max_blocks);
  ACS_ENSURE(p->desc_off, sizeof(int64_t) * max_blocks);
  ACS_ENSURE(p->nchunks, sizeof(int32_t) * max_blocks);
  ACS_ENSURE(p->chunk_base, sizeof(int64_t) * max_blocks);
  ACS_ENSURE(p->bused, sizeof(int32_t) * max_blocks);
  ACS_ENSURE(p->bused_scan, sizeof(int64_t) * max_blocks);
  ACS_ENSURE(p->hdone, sizeof(int32_t) * max_blocks);
  ACS_ENSURE(p->esc_list, sizeof(int32_t) * max_blocks);
  ACS_ENSURE(p->esc_list_small, sizeof(int32_t) * max_blocks);
  ACS_ENSURE(p->rows_list, sizeof(int32_t) * max_blocks);
  // POOL_BOUND / AUTO (reading R40): per-block regions bounded by the accumulators' output
  const bool want_bound = p->opt.pool_mode != ACSPGEMM_POOL_EXACT && p->opt.strategy != ACSPGEMM_STRATEGY_ESC &&
                          p->opt.strategy != ACSPGEMM_STRATEGY_DICT;
  if (want_bound) {
    ACS_ENSURE(p->best, sizeof(int64_t) * max_blocks);
    ACS_ENSURE(p->boff, sizeof(int64_t) * max_blocks);
  }
  const int64_t tmp_n = scan_tmp_elems(std::max<int64_t>(max_blocks, A->rows) * 2 + 1024);
  ACS_ENSURE_SCAN_TMP(p->scan_tmp, tmp_n, st);
  ACS_ENSURE(p->row_count, sizeof(int32_t) * A->rows);
  int32_t* nblocks_dev = reinterpret_cast<int32_t*>(scal + 20);
  // scal words: 0 products, 1 slots, 2 nblocks, 3 ncand / total chunks, 4 max block
  // products / shared rows, 5 bounded pool / chunk elements, 6 hash blocks, 7 dict
  // blocks, 8..14 merge class counts, 15 k_rows blocks, 16 nnz(C), 17-18 deferred blocks
  // and their products, 20 nblocks (int32), 21 k_rows list, 22 in-place merged elements,
  // 23-25 dense slices, 26 k_rows
  // batches, 27 k_hash blocks, 28-31
  // AC-ESC lists.  The counters are zeroed by k_segments, the
  // first kernel (with err), and k_glb zeroes the per-row counters: no memset launches.
  ZeroList zero{};
  zero.p[0] = scal + 3; zero.n[0] = 2;
  zero.p[1] = scal + 6; zero.n[1] = 13;
  zero.p[2] = scal + 21; zero.n[2] = 11;
  zero.p[3] = reinterpret_cast<int64_t*>(p->err.p); zero.n[3] = 2;
  launch_segments(Av, nseg, explicit_rows, ptr<int64_t>(p->seg), nblocks_dev, st, zero);
  tl_launches += 1;
  launch_glb(Av, nseg, ptr<int64_t>(p->seg), ptr<int32_t>(p->brs), max_blocks, st, ptr<int32_t>(p->row_count));
  tl_launches += 1;
  launch_block_bounds(Av, Bv, nseg, ptr<int64_t>(p->seg), nblocks_dev, max_blocks, ptr<int32_t>(p->nzb),
                      ptr<int32_t>(p->nze), ptr<int64_t>(p->bprod), ptr<int64_t>(p->bslot),
                      p->opt.strategy != ACSPGEMM_STRATEGY_ESC ? ptr<int32_t>(p->hdone) : nullptr, scal + 3, scal + 4,
                      scal + 2, ptr<int32_t>(p->brs), A->rows, want_bound ? ptr<int64_t>(p->best) : nullptr, st);
  tl_launches += 1;
  launch_scan_i64(ptr<int64_t>(p->bprod), ptr<int64_t>(p->pool_off), max_blocks, scal + 0, ptr<int64_t>(p->scan_tmp), st);
  launch_scan_i64(ptr<int64_t>(p->bslot), ptr<int64_t>(p->desc_off), max_blocks, scal + 1, ptr<int64_t>(p->scan_tmp), st);
  tl_launches += 2;
  if (want_bound) {
    launch_scan_i64(ptr<int64_t>(p->best), ptr<int64_t>(p->boff), max_blocks, scal + 5, ptr<int64_t>(p->scan_tmp), st);
    tl_launches += 1;
  }
  ACS_CUDA(cudaGetLastError());
  // segment boundaries (for info) ride along with the first read-back (replay: unchanged)
  if ((s = sync_read(p, scal, want_bound ? 6 : 5, st, p->seg.p, p->h_scal + H_SEG_INFO,
                     (int)sizeof(int64_t) * (nseg + 1))) != ACSPGEMM_OK)
    return s;
  const int64_t products = p->h_scal[0], slots = p->h_scal[1], nblocks = p->h_scal[2], ncand = p->h_scal[3];
  if (p->h_scal[4] > 0)
    return set_err(ACSPGEMM_ERR_INDEX_OVERFLOW, "a block of NPB nonzeros of A has " + std::to_string(p->h_scal[4]) +
                                                    " >= 2^31 products (32-bit block counters)");
  p->info.products = products;
  p->info.nblocks = nblocks;
  p->info.nsegments = nseg;
  for (int i = 0; i <= nseg; ++i) p->info.segment_rows[i] = p->h_scal[H_SEG_INFO + i];
  const int64_t bound_elems = want_bound ? p->h_scal[5] : products;
  const bool over_limit = p->opt.pool_limit_bytes && (size_t)(products * (4 + vbytes)) > p->opt.pool_limit_bytes;
  const bool use_bound = want_bound && (p->opt.pool_mode == ACSPGEMM_POOL_BOUND || over_limit);
  const int64_t pool_elems = use_bound ? bound_elems : products;
  const int64_t pool_bytes = pool_elems * (4 + vbytes);
  if (p->opt.pool_limit_bytes && (size_t)pool_bytes > p->opt.pool_limit_bytes)
    return set_err(ACSPGEMM_ERR_OUT_OF_MEMORY, std::string(use_bound ? "bounded" : "exact") + " chunk-pool size " +
                                                   std::to_string(pool_bytes) + " B exceeds pool_limit_bytes");
  p->info.pool_mode = use_bound ? ACSPGEMM_POOL_BOUND : ACSPGEMM_POOL_EXACT;
  p->info.ndeferred_blocks = 0;
  ACS_ENSURE(p->pool_col, sizeof(int32_t) * pool_elems);
  ACS_ENSURE(p->pool_val, (size_t)vbytes * pool_elems);
  ACS_ENSURE(p->descs, sizeof(ChunkDesc) * slots);
  // scans later run over up to `slots` chunks / shared rows
  ACS_ENSURE_SCAN_TMP(p->scan_tmp, scan_tmp_elems(std::max<int64_t>(std::max(max_blocks, A->rows), slots) + 1), st);
  p->info.pool_bytes = (int64_t)(p->pool_col.bytes + p->pool_val.bytes);

  // ------------------------------------------------------------ ESC -----------
  record(p, S_ESC, st);
  EscArgs ea;
  ea.A = Av;
  ea.B = Bv;
  ea.nblocks = (int32_t)nblocks;
  ea.blk_nz_begin = ptr<int32_t>(p->nzb);
  ea.blk_nz_end = ptr<int32_t>(p->nze);
  ea.block_row_starts = ptr<int32_t>(p->brs);
  ea.pool_off = use_bound ? ptr<int64_t>(p->boff) : ptr<int64_t>(p->pool_off);
  ea.bound = use_bound ? 1 : 0;
  ea.region = use_bound ? ptr<int64_t>(p->best) : nullptr;
  ea.defer = scal + 17;
  ea.desc_off = ptr<int64_t>(p->desc_off);
  ea.pool_col = ptr<int32_t>(p->pool_col);
  ea.pool_val = p->pool_val.p;
  ea.descs = ptr<ChunkDesc>(p->descs);
  ea.nchunks = ptr<int32_t>(p->nchunks);
  ea.used = ptr<int32_t>(p->bused);
  ea.row_count = ptr<int32_t>(p->row_count);
  ea.hash_done = nullptr;
  ea.hash_count = scal + 6;
  ea.dict_count = scal + 7;
  ea.rows_count = scal + 15;
  ea.esc_list = ptr<int32_t>(p->esc_list);
  ea.esc_count = scal + 28;
  ea.esc_next = scal + 29;
  ea.rows_next = scal + 26;
  ea.hash_next = scal + 27;
  ea.rows_list = nullptr;
  ea.rows_list_count = nullptr;
  ea.blk_products = ptr<int64_t>(p->bprod);
  ea.esc_list_small = nullptr;
  ea.trace = nullptr;
  uint64_t* trace_base = nullptr;        // kernel k's records at trace_base + k * 3 * nblocks
  if (p->trace_on && !p->replay) {
    ACS_ENSURE(p->trace, sizeof(uint64_t) * 3 * 4 * nblocks);
    ACS_CUDA(cudaMemsetAsync(p->trace.p, 0, sizeof(uint64_t) * 3 * 4 * nblocks, st));
    trace_base = ptr<uint64_t>(p->trace);
    p->trace_blocks = nblocks;
  }
  auto trace_of = [&](int k) { return trace_base ? trace_base + (int64_t)k * 3 * nblocks : nullptr; };
  ea.esc_count_small = scal + 30;
  ea.esc_next_small = scal + 31;
  if (p->opt.strategy != ACSPGEMM_STRATEGY_ESC) {
    // hash accumulator first (reading R31); blocks it does not finish go to AC-ESC,
    // small ones (<= 512 products) to the small-tile AC-ESC (reading R32)
    ea.hash_done = ptr<int32_t>(p->hdone);
    ea.esc_list_small = ptr<int32_t>(p->esc_list_small);
  }
  // column dictionary first (reading R33): by default for fp32 only -- with fp64 values its
  // per-warp accumulators allow 2 CTAs (16 warps) per SM and it measured slower than the
  // hash table (cfg2: 10.5 vs 10.1 ms; fp32: 7.8 vs 9.5 ms); both give the same bits
  const bool use_dict = p->opt.strategy == ACSPGEMM_STRATEGY_DICT;
  if (ea.hash_done && ncand > 0 && use_dict) {
    launch_dict(ea, p->f64, st);
    tl_launches += nblocks > 0 ? 1 : 0;
  }
  record(p, S_DICTEND, st);
  if (ea.hash_done && ncand > 0) {
    ea.trace = trace_of(0);
    ea.rows_list = ptr<int32_t>(p->rows_list);   // k_hash lists the blocks it leaves for k_rows
    ea.rows_list_count = scal + 21;
    launch_hash(ea, p->f64, st);         // blocks k_dict left (reading R31)
    tl_launches += nblocks > 0 ? 1 : 0;
  }
  record(p, S_HASHEND, st);
  if (ea.hash_done) {
    ea.trace = trace_of(1);
    launch_rows(ea, p->f64, ncand > 0, st);   // blocks of short rows (reading R34)
    tl_launches += nblocks > 0 ? 1 : 0;
  }
  if (ea.hash_done) {
    ea.trace = trace_of(3);
    acs_launch_esc_small(&ea, p->f64, st);   // k_rows listed the blocks left to AC-ESC
    tl_launches += nblocks > 0 ? 1 : 0;
  }
  ea.trace = trace_of(2);
  launch_esc(ea, p->f64, st);
  tl_launches += nblocks > 0 ? 1 : 0;
  ea.trace = nullptr;
  ACS_CUDA(cudaGetLastError());
  if (use_bound) {
    // POOL_BOUND (reading R40): candidates that ended in AC-ESC were deferred; their
    // exact regions are appended to the pool (grown by a copy) and AC-ESC runs on them
    if ((s = sync_read(p, scal + 17, 2, st)) != ACSPGEMM_OK) return s;
    const int64_t ndef = p->h_scal[0], def_products = p->h_scal[1];
    p->info.ndeferred_blocks = ndef;
    if (ndef > 0) {
      const int64_t total = bound_elems + def_products;
      if (p->opt.pool_limit_bytes && (size_t)(total * (4 + vbytes)) > p->opt.pool_limit_bytes)
        return set_err(ACSPGEMM_ERR_OUT_OF_MEMORY, "bounded chunk pool plus the deferred blocks' exact bounds (" +
                                                       std::to_string(total * (4 + vbytes)) + " B) exceeds pool_limit_bytes");
      if ((s = grow_keep(p->pool_col, sizeof(int32_t) * total, sizeof(int32_t) * bound_elems, st)) != ACSPGEMM_OK)
        return s;
      if ((s = grow_keep(p->pool_val, (size_t)vbytes * total, (size_t)vbytes * bound_elems, st)) != ACSPGEMM_OK)
        return s;
      ea.pool_col = ptr<int32_t>(p->pool_col);
      ea.pool_val = p->pool_val.p;
      ACS_ENSURE(p->bdef, sizeof(int64_t) * max_blocks);
      ACS_ENSURE(p->bdef_scan, sizeof(int64_t) * max_blocks);
      ACS_CUDA(cudaMemsetAsync(scal + 28, 0, 4 * sizeof(int64_t), st));
      launch_defer_flags(ea, ptr<int64_t>(p->bdef), st);
      launch_scan_i64(ptr<int64_t>(p->bdef), ptr<int64_t>(p->bdef_scan), nblocks, scal + 19, ptr<int64_t>(p->scan_tmp),
                      st);
      launch_defer_place(ea, ptr<int64_t>(p->bdef_scan), bound_elems, ptr<int64_t>(p->boff), st);
      acs_launch_esc_small(&ea, p->f64, st);
      launch_esc(ea, p->f64, st);
      tl_launches += 5;
      ACS_CUDA(cudaGetLastError());
      p->info.pool_bytes = (int64_t)(p->pool_col.bytes + p->pool_val.bytes);
    }
  }

  // ------------------------------------------------------------ MCC -----------
  record(p, S_MCC, st);
  ACS_ENSURE(p->dense, sizeof(ChunkDesc) * slots);
  ACS_ENSURE(p->sflag, sizeof(int32_t) * slots);
  ACS_ENSURE(p->spos, sizeof(int64_t) * slots);
  ACS_ENSURE(p->shared, sizeof(SharedRow) * slots);
  launch_scan_i32(ptr<int32_t>(p->nchunks), ptr<int64_t>(p->chunk_base), nblocks, scal + 3, ptr<int64_t>(p->scan_tmp), st);
  launch_scan_i32(ptr<int32_t>(p->bused), ptr<int64_t>(p->bused_scan), nblocks, scal + 5, ptr<int64_t>(p->scan_tmp), st);
  tl_launches += 2;
  MergeState ms;
  ms.nblocks = (int32_t)nblocks;
  ms.desc_off = ptr<int64_t>(p->desc_off);
  ms.nchunks = ptr<int32_t>(p->nchunks);
  ms.chunk_base = ptr<int64_t>(p->chunk_base);
  ms.descs = ptr<ChunkDesc>(p->descs);
  ms.dense = ptr<ChunkDesc>(p->dense);
  ms.max_chunks = slots;
  ms.total_chunks_dev = scal + 3;
  ms.shared_flag = ptr<int32_t>(p->sflag);
  ms.shared_pos = ptr<int64_t>(p->spos);
  ms.shared = ptr<SharedRow>(p->shared);
  ms.pool_col = ptr<int32_t>(p->pool_col);
  ms.scan_tmp = ptr<int64_t>(p->scan_tmp);
  // merge lists sized by the chunk bound: shared rows, their kinds and merge offsets
  // are found in one pass, and one read-back serves MCC
  ACS_ENSURE(p->kflag, sizeof(int32_t) * std::max<int64_t>(slots, 1));
  ACS_ENSURE(p->lmulti, sizeof(int32_t) * std::max<int64_t>(slots, 1));
  ACS_ENSURE(p->lpath, sizeof(int32_t) * std::max<int64_t>(slots, 1));
  ACS_ENSURE(p->lsearch, sizeof(int32_t) * std::max<int64_t>(slots, 1));
  ACS_ENSURE(p->lpair, sizeof(int32_t) * std::max<int64_t>(slots, 1));
  ACS_ENSURE(p->lgiant, sizeof(int32_t) * std::max<int64_t>(slots, 1));
  ACS_ENSURE(p->mtscan, sizeof(int64_t) * std::max<int64_t>(slots, 1));
  MergeLists L;
  L.nshared = 0;
  L.shared = ptr<SharedRow>(p->shared);
  L.kind_flag = ptr<int32_t>(p->kflag);
  L.kind_pos = nullptr;
  L.multi_idx = ptr<int32_t>(p->lmulti);
  L.path_idx = ptr<int32_t>(p->lpath);
  L.search_idx = ptr<int32_t>(p->lsearch);
  L.pair_idx = ptr<int32_t>(p->lpair);
  L.giant_idx = ptr<int32_t>(p->lgiant);
  L.counts_dev = scal + 8;
  L.merge_total_scan = ptr<int64_t>(p->mtscan);
  L.multi_scan = nullptr;
  L.group_of = nullptr;
  L.group_start = nullptr;
  L.scan_tmp = ptr<int64_t>(p->scan_tmp);
  launch_gather_chunks(ms, st);
  launch_find_shared(ms, L, scal + 4, st);
  tl_launches += 1 + (slots > 0 ? 7 : 0);
  ACS_CUDA(cudaGetLastError());
  if ((s = sync_read(p, scal + 2, 21, st)) != ACSPGEMM_OK) return s;
  const int64_t inplace_total = p->h_scal[20];   // scal + 22: elements of rows merged in place
  p->info.nrow_blocks = p->h_scal[13];
  p->info.nhash_blocks = p->h_scal[4];
  p->info.ndict_blocks = p->h_scal[5];
  p->total_chunks = p->h_scal[1];
  p->nshared = p->h_scal[2];
  p->max_chunks = slots;
  p->info.nchunks = p->total_chunks;
  p->info.nshared = p->nshared;
  p->info.chunk_elems = p->h_scal[3];
  const int64_t nsh = p->nshared;
  int64_t nmulti = 0, npath = 0, nsearch = 0, npair = 0, merge_total = 0, ngroups = 0, ngiant = 0;
  if (nsh > 0) {
    ACS_ENSURE(p->mscan, sizeof(int64_t) * nsh);
    ACS_ENSURE(p->group_of, sizeof(int32_t) * nsh);
    L.nshared = nsh;
    L.multi_scan = ptr<int64_t>(p->mscan);
    L.group_of = ptr<int32_t>(p->group_of);
    for (int i = 0; i < 6; ++i) p->h_scal[i] = p->h_scal[6 + i];   // the class counts (scal + 8 ..)
    nmulti = p->h_scal[0];
    npath = p->h_scal[1];
    nsearch = p->h_scal[2];
    npair = p->h_scal[3];
    merge_total = p->h_scal[4];
    ngiant = p->h_scal[5];
    // Multi-Merge packing needs the multi totals: scan them over the multi list
    if (nmulti > 0) {
      // upper bound of groups from merge_total (multi totals <= merge_total)
      int64_t gmax = 2 * ((merge_total + inplace_total + CAP - 1) / CAP) + 2;
      ACS_ENSURE(p->gstart, sizeof(int32_t) * 2 * (gmax + 1));
      L.group_start = ptr<int32_t>(p->gstart);
      launch_multi_groups(L, nmulti, gmax, st);
      tl_launches += 1 + 1 + 1 + 1;
      ngroups = gmax;
    }
    ACS_ENSURE(p->merge_col, sizeof(int32_t) * merge_total);
    ACS_ENSURE(p->merge_val, (size_t)vbytes * merge_total);
    ACS_ENSURE(p->cur_first, sizeof(int32_t) * p->total_chunks);
    ACS_ENSURE(p->cur_last, sizeof(int32_t) * p->total_chunks);
    MergeArgs ma;
    ma.dense = ptr<ChunkDesc>(p->dense);
    ma.shared = ptr<SharedRow>(p->shared);
    ma.group_start = ptr<int32_t>(p->gstart);
    ma.multi_scan = ptr<int64_t>(p->mscan);
    ma.ngroups = ngroups;
    ma.pool_col = ptr<int32_t>(p->pool_col);
    ma.pool_val = p->pool_val.p;
    ma.merge_col = ptr<int32_t>(p->merge_col);
    ma.merge_val = p->merge_val.p;
    ma.cur_first = ptr<int32_t>(p->cur_first);
    ma.cur_last = ptr<int32_t>(p->cur_last);
    ma.row_count = ptr<int32_t>(p->row_count);
    ma.error_flag = ptr<int32_t>(p->err);
    record(p, S_MM, st);
    ma.list = ptr<int32_t>(p->lmulti);
    ma.nlist = nmulti;
    if (nmulti > 0) { launch_multi_merge(ma, p->f64, st); tl_launches += 1; }
    ma.list = ptr<int32_t>(p->lpair);
    ma.nlist = npair;
    if (npair > 0) { launch_pair_merge(ma, p->f64, st); tl_launches += 1; }
    record(p, S_PM, st);
    ma.list = ptr<int32_t>(p->lpath);
    ma.nlist = npath;
    if (npath > 0) { launch_path_merge(ma, p->f64, st); tl_launches += 1; }
    record(p, S_SM, st);
    ma.list = ptr<int32_t>(p->lsearch);
    ma.nlist = nsearch;
    if (nsearch > 0) { launch_search_merge(ma, p->f64, st); tl_launches += 1; }
    if (ngiant > 0) {
      // rows of > SEARCH_MAXP chunks: dense column slices (reading R30)
      ACS_ENSURE(p->g_lo, sizeof(int32_t) * 2 * ngiant);          // first | last column
      ACS_ENSURE(p->g_nsl, sizeof(int64_t) * 2 * ngiant);         // slices | slices x pieces
      ACS_ENSURE(p->g_base, sizeof(int64_t) * 2 * ngiant);        // their scans
      GiantArgs g;
      g.list = ptr<int32_t>(p->lgiant);
      g.n = ngiant;
      g.glo = ptr<int32_t>(p->g_lo);
      g.ghi = g.glo + ngiant;
      g.gnsl = ptr<int64_t>(p->g_nsl);
      g.gmn = g.gnsl + ngiant;
      g.gbase = ptr<int64_t>(p->g_base);
      g.gmbase = g.gbase + ngiant;
      launch_giant_span(ma, g, st);
      launch_scan_i64(g.gmn, g.gmbase, ngiant, scal + 23, ptr<int64_t>(p->scan_tmp), st);
      launch_scan_i64(g.gnsl, g.gbase, ngiant, scal + 24, ptr<int64_t>(p->scan_tmp), st);
      tl_launches += 1 + 2;
      ACS_CUDA(cudaGetLastError());
      if ((s = sync_read(p, scal + 23, 2, st)) != ACSPGEMM_OK) return s;
      const int64_t npos = p->h_scal[0], nslices = p->h_scal[1];
      ACS_ENSURE(p->g_pos, sizeof(int32_t) * npos);
      ACS_ENSURE(p->g_tcol, sizeof(int32_t) * nslices);            // entries per slice
      ACS_ENSURE(p->g_tval, sizeof(int64_t) * nslices);            // their scan
      ACS_ENSURE(p->g_tcnt, sizeof(int32_t) * nslices);
      ACS_ENSURE_SCAN_TMP(p->scan_tmp, scan_tmp_elems(nslices + 1), st);
      g.pos = ptr<int32_t>(p->g_pos);
      g.gent = ptr<int32_t>(p->g_tcol);
      g.gpos = ptr<int64_t>(p->g_tval);
      g.tcnt = ptr<int32_t>(p->g_tcnt);
      launch_giant_count(ma, g, nslices, st);
      launch_scan_i32(g.gent, g.gpos, nslices, scal + 25, ptr<int64_t>(p->scan_tmp), st);
      launch_giant_merge(ma, g, nslices, p->f64, st);
      tl_launches += 2 + 1 + 2;
    }
    ACS_CUDA(cudaGetLastError());
  } else {
    record(p, S_MM, st);
    record(p, S_PM, st);
    record(p, S_SM, st);
  }
  p->info.nmulti = nmulti + npair;
  p->info.npath = npath;
  p->info.nsearch = nsearch + ngiant;
  p->info.nmulti_groups = ngroups;
  p->info.merge_elems = merge_total;

  // ------------------------------------------------------------ SCAN ----------
  record(p, S_SCAN, st);
  // int64 row pointers in plan memory (any nnz(C)); C gets int32 or int64 copies
  ACS_ENSURE(p->row_ptr, sizeof(int64_t) * (A->rows + 1));
  launch_scan_rowptr(ptr<int32_t>(p->row_count), ptr<int64_t>(p->row_ptr), A->rows, scal + 16,
                     ptr<int64_t>(p->scan_tmp), st);
  tl_launches += 1;
  ACS_CUDA(cudaGetLastError());
  record(p, S_CC, st);
  int64_t nnz;
  int32_t errflag;
  if (p->replay) {
    if (p->rec_pos >= p->rec.size() || p->rec[p->rec_pos].size() != 2)
      return set_err(ACSPGEMM_ERR_INTERNAL, "pattern replay out of step");
    nnz = p->rec[p->rec_pos][0];
    errflag = (int32_t)p->rec[p->rec_pos][1];
    ++p->rec_pos;
  } else {
    launch_read_back2(scal + 16, p->h_scal, sizeof(int64_t), p->err.p, p->h_scal + 1, sizeof(int32_t), st);
    tl_launches += 1;
    ACS_CUDA(cudaStreamSynchronize(st));
    nnz = p->h_scal[0];
    errflag = *reinterpret_cast<int32_t*>(p->h_scal + 1);
    p->rec.push_back({nnz, (int64_t)errflag});
  }
  if (errflag) return set_err(ACSPGEMM_ERR_INTERNAL, "a shared row spans more chunks than one merge block handles");
  p->nnz = nnz;
  p->info.nnz_c = nnz;
  p->info.helper_bytes = helper_bytes(p);
  p->launches_sym = tl_launches - l0;
  p->ready = true;
  *nnz_c = nnz;
  return ACSPGEMM_OK;
}

// Numeric pass into C with row pointers of type I (int32: acspgemm_csr_out, int64:
// acspgemm_csr_out64), shifted by row_off (row pieces placed after earlier pieces).
template <typename Out, typename I>
acspgemm_status numeric_impl_t(acspgemm_plan p, Out* C, cudaStream_t st, I row_off) {
  if (!p->ready) return set_err(ACSPGEMM_ERR_NOT_READY, "numeric called without a successful symbolic");
  if (!C) return set_err(ACSPGEMM_ERR_INVALID_ARG, "C is NULL");
  if (p->rows > 0 && !C->row_ptr) return set_err(ACSPGEMM_ERR_INVALID_ARG, "C.row_ptr is NULL");
  if (p->nnz > 0 && (!C->col_idx || !C->val)) return set_err(ACSPGEMM_ERR_INVALID_ARG, "C.col_idx/val is NULL");
  if (sizeof(I) == 4 && (int64_t)row_off + p->nnz >= (int64_t(1) << 31))
    return set_err(ACSPGEMM_ERR_INDEX_OVERFLOW, "nnz(C) >= 2^31: int32 row_ptr (use acspgemm_numeric64)");
  const long long l0 = tl_launches;
  C->rows = p->rows;
  C->cols = p->cols;
  C->nnz = p->nnz;
  if (p->empty) {
    if (p->rows >= 0 && C->row_ptr) launch_rowptr_out(C->row_ptr, nullptr, p->rows + 1, row_off, st);
    p->info.kernel_launches = p->launches_sym;
    return ACSPGEMM_OK;
  }
  launch_rowptr_out(C->row_ptr, ptr<int64_t>(p->row_ptr), p->rows + 1, row_off, st);
  tl_launches += 1;
  record(p, S_CC, st);
  CopyArgs ca;
  ca.dense = ptr<ChunkDesc>(p->dense);
  ca.total_chunks_dev = ptr<int64_t>(p->scal) + 3;
  ca.max_chunks = p->total_chunks;
  ca.shared = ptr<SharedRow>(p->shared);
  ca.nshared = p->nshared;
  ca.pool_col = ptr<int32_t>(p->pool_col);
  ca.pool_val = p->pool_val.p;
  ca.merge_col = ptr<int32_t>(p->merge_col);
  ca.merge_val = p->merge_val.p;
  ca.row_ptr = ptr<int64_t>(p->row_ptr);
  ca.c_col = C->col_idx;
  ca.c_val = C->val;
  launch_copy(ca, p->f64, st);
  if (p->total_chunks + p->nshared > 0) tl_launches += 1;
  record(p, S_END, st);
  ACS_CUDA(cudaGetLastError());
  p->info.kernel_launches = p->launches_sym + (tl_launches - l0);
  return ACSPGEMM_OK;
}

acspgemm_status numeric_impl(acspgemm_plan p, acspgemm_csr_out* C, cudaStream_t st, int32_t row_off = 0) {
  return numeric_impl_t<acspgemm_csr_out, int32_t>(p, C, st, row_off);
}

// ------------------------------------------------------------ debug kernels ------

__global__ void k_debug_wd(const int32_t* lengths, int nentries, const int32_t* draws, int ndraws, int32_t* ares_out,
                           int32_t* bres_out, int32_t* rem_out) {
  __shared__ int wd[NPB + 1];
  __shared__ int offsets[CAP_PAD];
  __shared__ int scratch[40];
  int len[NNZ_PER_THREAD];
#pragma unroll
  for (int j = 0; j < NNZ_PER_THREAD; ++j) {
    const int e = threadIdx.x * NNZ_PER_THREAD + j;
    len[j] = e < nentries ? lengths[e] : 0;
  }
  wd_placework(len, wd, scratch);
  int off = 0;
  for (int d = 0; d < ndraws; ++d) {
    const int consume = draws[d];
    int ares[ITEMS], bres[ITEMS];
    wd_receivework(consume, wd, offsets, scratch, ares, bres);
#pragma unroll
    for (int i = 0; i < ITEMS; ++i) {
      const int c = i * THREADS + threadIdx.x;
      if (c < consume) { ares_out[off + c] = ares[i]; bres_out[off + c] = bres[i]; }
    }
    for (int e = threadIdx.x; e < nentries; e += THREADS) rem_out[d * nentries + e] = wd[e + 1] - wd[e];
    off += consume;
    __syncthreads();
  }
}

__global__ void k_debug_sort_compact(const int32_t* rows, const int32_t* cols, const double* vals, int n,
                                     int32_t* orow, int32_t* ocol, double* oval, uint32_t* ostate) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  SortSmem<double>& S = *reinterpret_cast<SortSmem<double>*>(smem_raw);
  const int tid = threadIdx.x;
  int rmin = INT_MAX, rmax = INT_MIN, cmin = INT_MAX, cmax = INT_MIN;
  for (int p = tid; p < n; p += THREADS) {
    rmin = min(rmin, rows[p]); rmax = max(rmax, rows[p]);
    cmin = min(cmin, cols[p]); cmax = max(cmax, cols[p]);
  }
  block_minmax4(rmin, rmax, cmin, cmax, S.scratch);
  if (n == 0) return;
  const int rowbits = bit_width_u64((uint64_t)(rmax - rmin));
  const int colbits = bit_width_u64((uint64_t)((int64_t)cmax - cmin));
  for (int p = tid; p < CAP; p += THREADS) {
    if (p < n) {
      const uint64_t key = ((uint64_t)(rows[p] - rmin) << colbits) | (uint64_t)(cols[p] - cmin);
      S.words[pad32(p)] = (key << IDXBITS) | (uint64_t)p;
      S.vals[p] = vals[p];
    } else {
      S.words[pad32(p)] = ~0ull;
    }
  }
  __syncthreads();
  uint64_t k[ITEMS];
  double ev[ITEMS];
  load_and_sort<uint64_t, double>(S, rowbits + colbits, k);
  const ScanCtx<uint64_t, double> ctx = compaction_prepare<uint64_t, double>(S, k, n, colbits, ev);
  const uint64_t colmask = colbits ? ((1ull << colbits) - 1) : 0;
  compaction_emit<uint64_t, double, true>(k, ev, n, colbits, ctx,
                                          [&](int idx, uint64_t key, double val, uint32_t state, bool) {
    orow[idx] = rmin + (int)(key >> colbits);
    ocol[idx] = cmin + (int)(key & colmask);
    oval[idx] = val;
    ostate[idx] = state;
  });
}

// Restores a plan's explicit segments when acspgemm_multiply_host returns (any path)
// and leaves both of its streams idle.
struct HostPipeGuard {
  acspgemm_plan plan;
  cudaStream_t st;
  int saved_nseg;
  int64_t saved_rows[MAX_SEGMENTS + 1];
  explicit HostPipeGuard(acspgemm_plan p, cudaStream_t s) : plan(p), st(s), saved_nseg(p->nseg_explicit) {
    for (int i = 0; i <= MAX_SEGMENTS; ++i) saved_rows[i] = p->seg_rows_explicit[i];
  }
  ~HostPipeGuard() {
    if (plan->hp_cs) cudaStreamSynchronize(plan->hp_cs);
    if (plan->hp_in) cudaStreamSynchronize(plan->hp_in);
    cudaStreamSynchronize(st);
    plan->nseg_explicit = saved_nseg;
    for (int i = 0; i <= MAX_SEGMENTS; ++i) plan->seg_rows_explicit[i] = saved_rows[i];
  }
};

template <typename P>
struct Scratch {
  P* d = nullptr;
  ~Scratch() { if (d) cudaFree(d); }
};

}  // namespace

// ======================================================================= C ABI ====

extern "C" {

void acspgemm_options_default(acspgemm_options* opt) {
  if (!opt) return;
  opt->pool_limit_bytes = 0;
  opt->validate_inputs = 0;
  opt->collect_stage_times = 0;
  opt->num_segments = DEFAULT_SEGMENTS;
  opt->strategy = ACSPGEMM_STRATEGY_ADAPTIVE;
  opt->pool_mode = ACSPGEMM_POOL_BOUND;
}

acspgemm_status acspgemm_plan_create(acspgemm_plan* plan, const acspgemm_options* opt) {
  if (!plan) return set_err(ACSPGEMM_ERR_INVALID_ARG, "plan is NULL");
  acspgemm_plan p = new (std::nothrow) acspgemm_plan_s();
  if (!p) return set_err(ACSPGEMM_ERR_OUT_OF_MEMORY, "host allocation");
  acspgemm_options_default(&p->opt);
  if (opt) p->opt = *opt;
  if (p->opt.num_segments <= 0) p->opt.num_segments = DEFAULT_SEGMENTS;
  if (p->opt.num_segments > MAX_SEGMENTS) {
    delete p;
    return set_err(ACSPGEMM_ERR_INVALID_ARG, "num_segments > 64");
  }
  if (p->opt.strategy < ACSPGEMM_STRATEGY_ADAPTIVE || p->opt.strategy > ACSPGEMM_STRATEGY_DICT) {
    delete p;
    return set_err(ACSPGEMM_ERR_INVALID_ARG, "unknown strategy");
  }
  std::memset(&p->info, 0, sizeof(p->info));
  // mapped: read-backs are written by a kernel (launch_read_back), not a copy engine
  cudaError_t e = cudaHostAlloc(&p->h_scal, sizeof(int64_t) * H_SCAL_WORDS, cudaHostAllocMapped);
  if (e != cudaSuccess) {
    delete p;
    return set_err(ACSPGEMM_ERR_CUDA, std::string("cudaHostAlloc: ") + cudaGetErrorString(e));
  }
  p->ev_ok = true;
  for (int i = 0; i < NSTAGE_EV; ++i)
    if (cudaEventCreate(&p->ev[i]) != cudaSuccess) p->ev_ok = false;
  *plan = p;
  return ACSPGEMM_OK;
}

void acspgemm_plan_destroy(acspgemm_plan p) {
  if (!p) return;
  cudaDeviceSynchronize();
  DevBuf* bs[] = {&p->seg, &p->scal, &p->brs, &p->nzb, &p->nze, &p->bprod, &p->bslot,
                  &p->pool_off, &p->desc_off, &p->nchunks, &p->chunk_base, &p->pool_col, &p->pool_val,
                  &p->descs, &p->dense, &p->sflag, &p->spos, &p->shared, &p->row_count, &p->row_ptr,
                  &p->scan_tmp, &p->kflag, &p->kpos, &p->lmulti, &p->lpath, &p->lsearch, &p->lpair, &p->mscan,
                  &p->mtscan, &p->group_of, &p->gstart, &p->merge_col, &p->merge_val, &p->cur_first,
                  &p->cur_last, &p->err, &p->bused, &p->bused_scan, &p->lgiant, &p->g_lo, &p->g_nsl,
                  &p->g_base, &p->g_pos, &p->g_tcol, &p->g_tval, &p->g_tcnt, &p->hdone, &p->esc_list,
                  &p->esc_list_small, &p->trace, &p->best, &p->boff, &p->bdef, &p->bdef_scan};
  for (DevBuf* b : bs) free_buf(*b);
  for (auto& pb : p->bp) for (DevBuf& b : pb) free_buf(b);
  if (p->gexec) cudaGraphExecDestroy(p->gexec);
  for (int i = 0; i < 3; ++i) {
    free_buf(p->hp_a[i]);
    free_buf(p->hp_b[i]);
    free_buf(p->hp_c[0][i]);
    free_buf(p->hp_c[1][i]);
  }
  if (p->hp_cs) cudaStreamDestroy(p->hp_cs);
  if (p->hp_in) cudaStreamDestroy(p->hp_in);
  if (p->hp_start) cudaEventDestroy(p->hp_start);
  for (cudaEvent_t e : p->hp_inev) if (e) cudaEventDestroy(e);
  free_buf(p->hp_rng);
  if (p->hp_ready) cudaEventDestroy(p->hp_ready);
  for (cudaEvent_t e : p->hp_copied) if (e) cudaEventDestroy(e);
  if (p->h_scal) cudaFreeHost(p->h_scal);
  if (p->ev_ok)
    for (int i = 0; i < NSTAGE_EV; ++i) cudaEventDestroy(p->ev[i]);
  delete p;
}

acspgemm_status acspgemm_set_segments(acspgemm_plan p, int nseg, const int64_t* rows_host) {
  if (!p) return set_err(ACSPGEMM_ERR_INVALID_ARG, "plan is NULL");
  if (nseg == 0) { p->nseg_explicit = 0; return ACSPGEMM_OK; }
  if (nseg < 0 || nseg > MAX_SEGMENTS || !rows_host) return set_err(ACSPGEMM_ERR_INVALID_ARG, "bad segments");
  if (rows_host[0] != 0) return set_err(ACSPGEMM_ERR_INVALID_ARG, "segments must start at row 0");
  for (int i = 0; i < nseg; ++i)
    if (rows_host[i + 1] < rows_host[i]) return set_err(ACSPGEMM_ERR_INVALID_ARG, "segments must be non-decreasing");
  for (int i = 0; i <= nseg; ++i) p->seg_rows_explicit[i] = rows_host[i];
  p->nseg_explicit = nseg;
  return ACSPGEMM_OK;
}

acspgemm_status acspgemm_canonical_segments(const acspgemm_csr_in* A, int nseg, int64_t* rows_host, void* stream) {
  acspgemm_status s = check_in(A, "A");
  if (s != ACSPGEMM_OK) return s;
  if (nseg < 1 || nseg > MAX_SEGMENTS || !rows_host) return set_err(ACSPGEMM_ERR_INVALID_ARG, "bad nseg");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  if (A->rows == 0) {
    for (int i = 0; i <= nseg; ++i) rows_host[i] = 0;
    return ACSPGEMM_OK;
  }
  Scratch<int64_t> seg;
  ACS_CUDA(cudaMalloc(&seg.d, sizeof(int64_t) * (3 * (MAX_SEGMENTS + 1) + 2)));
  const CsrView Av{A->rows, A->cols, A->row_ptr, A->col_idx, A->val};
  launch_segments(Av, nseg, SegRows{}, seg.d, reinterpret_cast<int32_t*>(seg.d + 3 * (MAX_SEGMENTS + 1)), st);
  ACS_CUDA(cudaGetLastError());
  ACS_CUDA(cudaMemcpyAsync(rows_host, seg.d, sizeof(int64_t) * (nseg + 1), cudaMemcpyDeviceToHost, st));
  ACS_CUDA(cudaStreamSynchronize(st));
  return ACSPGEMM_OK;
}

acspgemm_status acspgemm_symbolic(acspgemm_plan p, const acspgemm_csr_in* A, const acspgemm_csr_in* B,
                                  acspgemm_dtype dtype, void* stream, int64_t* nnz_c) {
  if (!p) return set_err(ACSPGEMM_ERR_INVALID_ARG, "plan is NULL");
  return symbolic_impl(p, A, B, dtype, reinterpret_cast<cudaStream_t>(stream), nnz_c);
}

acspgemm_status acspgemm_numeric(acspgemm_plan p, acspgemm_csr_out* C, void* stream) {
  if (!p) return set_err(ACSPGEMM_ERR_INVALID_ARG, "plan is NULL");
  return numeric_impl(p, C, reinterpret_cast<cudaStream_t>(stream));
}

acspgemm_status acspgemm_numeric_update(acspgemm_plan p, const acspgemm_csr_in* A, const acspgemm_csr_in* B,
                                        acspgemm_csr_out* C, void* stream) {
  if (!p || !A || !B || !C) return set_err(ACSPGEMM_ERR_INVALID_ARG, "NULL argument");
  if (!p->ready || p->rec_dtype < 0)
    return set_err(ACSPGEMM_ERR_NOT_READY, "numeric_update needs a successful symbolic of the same pattern");
  const int64_t dims[6] = {A->rows, A->cols, A->nnz, B->rows, B->cols, B->nnz};
  if (std::memcmp(dims, p->rec_dims, sizeof(dims)) != 0)
    return set_err(ACSPGEMM_ERR_INVALID_ARG, "numeric_update: A/B dimensions differ from the last symbolic");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  const acspgemm_dtype dtype = (acspgemm_dtype)p->rec_dtype;
  if (p->empty) {                        // no entries: only the row pointers
    int64_t nnz = 0;
    acspgemm_status s = symbolic_impl(p, A, B, dtype, st, &nnz);
    return s == ACSPGEMM_OK ? numeric_impl(p, C, st) : s;
  }
  const void* key[9] = {A->row_ptr, A->col_idx, A->val, B->row_ptr, B->col_idx, B->val,
                        C->row_ptr, C->col_idx, C->val};
  if (p->gexec && std::memcmp(key, p->gkey, sizeof(key)) == 0) {
    ACS_CUDA(cudaGraphLaunch(p->gexec, st));
    return ACSPGEMM_OK;
  }
  if (p->gexec) { cudaGraphExecDestroy(p->gexec); p->gexec = nullptr; }
  // the legacy default stream cannot be captured: replay without a graph (still sync-free)
  const bool capture = st != nullptr && st != cudaStreamLegacy && st != cudaStreamPerThread;
  cudaGraph_t g = nullptr;
  if (capture) ACS_CUDA(cudaStreamBeginCapture(st, cudaStreamCaptureModeRelaxed));
  p->replay = true;
  int64_t nnz = 0;
  acspgemm_status s = symbolic_impl(p, A, B, dtype, st, &nnz);
  if (s == ACSPGEMM_OK) s = numeric_impl(p, C, st);
  p->replay = false;
  if (capture) {
    const cudaError_t e = cudaStreamEndCapture(st, &g);
    if (s == ACSPGEMM_OK && e != cudaSuccess) s = set_err(ACSPGEMM_ERR_CUDA, cudaGetErrorString(e));
    if (s == ACSPGEMM_OK) {
      const cudaError_t ei = cudaGraphInstantiate(&p->gexec, g, 0);
      if (ei != cudaSuccess) { p->gexec = nullptr; s = set_err(ACSPGEMM_ERR_CUDA, cudaGetErrorString(ei)); }
    }
    if (g) cudaGraphDestroy(g);
    if (s == ACSPGEMM_OK) {
      std::memcpy(p->gkey, key, sizeof(key));
      const cudaError_t el = cudaGraphLaunch(p->gexec, st);
      if (el != cudaSuccess) s = set_err(ACSPGEMM_ERR_CUDA, cudaGetErrorString(el));
    }
  }
  return s;
}

acspgemm_status acspgemm_numeric64(acspgemm_plan p, acspgemm_csr_out64* C, void* stream) {
  if (!p) return set_err(ACSPGEMM_ERR_INVALID_ARG, "plan is NULL");
  return numeric_impl_t<acspgemm_csr_out64, int64_t>(p, C, static_cast<cudaStream_t>(stream), 0);
}

acspgemm_status acspgemm_multiply(const acspgemm_csr_in* A, const acspgemm_csr_in* B, acspgemm_csr_out* C,
                                  void* stream, acspgemm_dtype dtype) {
  if (!C) return set_err(ACSPGEMM_ERR_INVALID_ARG, "C is NULL");
  acspgemm_plan p = nullptr;
  acspgemm_status s = acspgemm_plan_create(&p, nullptr);
  if (s != ACSPGEMM_OK) return s;
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  int64_t nnz = 0;
  s = acspgemm_symbolic(p, A, B, dtype, stream, &nnz);
  if (s == ACSPGEMM_OK && nnz >= (int64_t(1) << 31))
    s = set_err(ACSPGEMM_ERR_INDEX_OVERFLOW, "nnz(C) >= 2^31: int32 row_ptr (use acspgemm_numeric64)");
  if (s == ACSPGEMM_OK) {
    const size_t vb = dtype == ACSPGEMM_F64 ? 8 : 4;
    C->row_ptr = nullptr; C->col_idx = nullptr; C->val = nullptr;
    cudaError_t e = cudaMallocAsync((void**)&C->row_ptr, sizeof(int32_t) * (A->rows + 1), st);
    if (e == cudaSuccess) e = cudaMallocAsync((void**)&C->col_idx, sizeof(int32_t) * (nnz > 0 ? nnz : 1), st);
    if (e == cudaSuccess) e = cudaMallocAsync(&C->val, vb * (nnz > 0 ? nnz : 1), st);
    if (e != cudaSuccess) {
      cudaGetLastError();
      acspgemm_free_csr(C, stream);
      s = set_err(ACSPGEMM_ERR_OUT_OF_MEMORY, std::string("cudaMallocAsync: ") + cudaGetErrorString(e));
    } else {
      s = acspgemm_numeric(p, C, stream);
    }
  }
  if (s == ACSPGEMM_OK) cudaStreamSynchronize(st);
  acspgemm_plan_destroy(p);
  return s;
}

acspgemm_status acspgemm_rap(const acspgemm_csr_in* R, const acspgemm_csr_in* A, const acspgemm_csr_in* P,
                             acspgemm_csr_out* C, void* stream, acspgemm_dtype dtype) {
  if (!R || !A || !P || !C) return set_err(ACSPGEMM_ERR_INVALID_ARG, "NULL argument");
  if (R->cols != A->rows) return set_err(ACSPGEMM_ERR_DIM_MISMATCH, "R.cols != A.rows");
  acspgemm_csr_out AP{};
  acspgemm_status s = acspgemm_multiply(A, P, &AP, stream, dtype);
  if (s != ACSPGEMM_OK) return s;
  const acspgemm_csr_in APin{AP.rows, AP.cols, AP.nnz, AP.row_ptr, AP.col_idx, AP.val};
  s = acspgemm_multiply(R, &APin, C, stream, dtype);
  acspgemm_free_csr(&AP, stream);
  if (s == ACSPGEMM_OK) ACS_CUDA(cudaStreamSynchronize(reinterpret_cast<cudaStream_t>(stream)));
  return s;
}

acspgemm_status acspgemm_multiply_budget(acspgemm_plan p, const acspgemm_csr_in* A, const acspgemm_csr_in* B,
                                         acspgemm_dtype dtype, void* stream, acspgemm_csr_out* C, int* npieces,
                                         int* nrestarts) {
  if (!p || !C) return set_err(ACSPGEMM_ERR_INVALID_ARG, "NULL argument");
  acspgemm_status s;
  if ((s = check_in(A, "A")) != ACSPGEMM_OK) return s;
  if ((s = check_in(B, "B")) != ACSPGEMM_OK) return s;
  if (dtype != ACSPGEMM_F32 && dtype != ACSPGEMM_F64) return set_err(ACSPGEMM_ERR_INVALID_ARG, "bad dtype");
  if (A->cols != B->rows) return set_err(ACSPGEMM_ERR_DIM_MISMATCH, "A.cols != B.rows");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  const size_t vb = dtype == ACSPGEMM_F64 ? 8 : 4;
  const int S = p->opt.num_segments;
  int pieces = 0, restarts = 0;
  C->rows = A->rows;
  C->cols = B->cols;
  C->nnz = 0;
  C->row_ptr = nullptr; C->col_idx = nullptr; C->val = nullptr;
  if (A->rows == 0 || A->nnz == 0 || B->nnz == 0) {         // no entries: one empty piece
    int64_t nnz = 0;
    if ((s = symbolic_impl(p, A, B, dtype, st, &nnz)) != ACSPGEMM_OK) return s;
    ACS_CUDA(cudaMallocAsync((void**)&C->row_ptr, sizeof(int32_t) * (A->rows + 1), st));
    if ((s = numeric_impl(p, C, st)) != ACSPGEMM_OK) return s;
    if (npieces) *npieces = 1;
    if (nrestarts) *nrestarts = 0;
    ACS_CUDA(cudaStreamSynchronize(st));
    return ACSPGEMM_OK;
  }
  HostPipeGuard guard(p, st);
  // canonical segments of A: row and nonzero boundaries (one read-back)
  int64_t seg[2 * (MAX_SEGMENTS + 1)];
  {
    ACS_ENSURE(p->seg, sizeof(int64_t) * (4 * (MAX_SEGMENTS + 1) + 2));
    int64_t* sd = ptr<int64_t>(p->seg);
    const CsrView Av{A->rows, A->cols, A->row_ptr, A->col_idx, A->val};
    launch_segments(Av, S, SegRows{}, sd, reinterpret_cast<int32_t*>(sd + 4 * (MAX_SEGMENTS + 1)), st);
    ACS_CUDA(cudaGetLastError());
    ACS_CUDA(cudaMemcpyAsync(seg, sd, sizeof(int64_t) * 2 * (MAX_SEGMENTS + 1), cudaMemcpyDeviceToHost, st));
    ACS_CUDA(cudaStreamSynchronize(st));
  }
  const int64_t* seg_nz = seg + (MAX_SEGMENTS + 1);
  struct Piece { int64_t r0, rows, nnz; };
  std::vector<Piece> out;
  int64_t off = 0;
  for (int s0 = 0; s0 < S;) {
    int s1 = S;
    int64_t nnz_g = 0;
    for (;;) {                               // the largest run of whole segments within budget
      const int64_t r0 = seg[s0], r1 = seg[s1];
      p->nseg_explicit = s1 - s0;
      for (int i = 0; i <= s1 - s0; ++i) p->seg_rows_explicit[i] = seg[s0 + i] - r0;
      const acspgemm_csr_in V{r1 - r0, A->cols, seg_nz[s1] - seg_nz[s0], A->row_ptr + r0, A->col_idx, A->val};
      s = symbolic_impl(p, &V, B, dtype, st, &nnz_g);
      if (s == ACSPGEMM_OK) break;
      if (s != ACSPGEMM_ERR_OUT_OF_MEMORY || s1 - s0 == 1) return s;
      ++restarts;                            // pool over budget: retry on fewer segments
      s1 = s0 + (s1 - s0) / 2;
    }
    if (off + nnz_g >= (int64_t(1) << 31)) return set_err(ACSPGEMM_ERR_INDEX_OVERFLOW, "nnz(C) >= 2^31");
    Piece q{seg[s0], seg[s1] - seg[s0], nnz_g};
    if (p->bp.size() <= out.size()) p->bp.emplace_back();
    std::array<DevBuf, 3>& pb = p->bp[out.size()];
    if ((s = ensure(pb[0], sizeof(int32_t) * (q.rows + 1))) != ACSPGEMM_OK ||
        (s = ensure(pb[1], sizeof(int32_t) * nnz_g)) != ACSPGEMM_OK || (s = ensure(pb[2], vb * nnz_g)) != ACSPGEMM_OK)
      return s;
    acspgemm_csr_out Cg{q.rows, B->cols, nnz_g, ptr<int32_t>(pb[0]), ptr<int32_t>(pb[1]), pb[2].p};
    out.push_back(q);
    if ((s = numeric_impl(p, &Cg, st, (int32_t)off)) != ACSPGEMM_OK) return s;
    off += nnz_g;
    ++pieces;
    s0 = s1;
  }
  // concatenate the pieces into C (allocated like acspgemm_multiply)
  cudaError_t e = cudaMallocAsync((void**)&C->row_ptr, sizeof(int32_t) * (A->rows + 1), st);
  if (e == cudaSuccess) e = cudaMallocAsync((void**)&C->col_idx, sizeof(int32_t) * (off > 0 ? off : 1), st);
  if (e == cudaSuccess) e = cudaMallocAsync(&C->val, vb * (off > 0 ? off : 1), st);
  if (e != cudaSuccess) {
    cudaGetLastError();
    acspgemm_free_csr(C, stream);
    return set_err(ACSPGEMM_ERR_OUT_OF_MEMORY, std::string("cudaMallocAsync: ") + cudaGetErrorString(e));
  }
  int64_t o = 0;
  for (size_t g = 0; g < out.size(); ++g) {
    const Piece& q = out[g];
    std::array<DevBuf, 3>& pb = p->bp[g];
    ACS_CUDA(cudaMemcpyAsync(C->row_ptr + q.r0, pb[0].p, sizeof(int32_t) * (q.rows + 1), cudaMemcpyDeviceToDevice, st));
    if (q.nnz > 0) {
      ACS_CUDA(cudaMemcpyAsync(C->col_idx + o, pb[1].p, sizeof(int32_t) * q.nnz, cudaMemcpyDeviceToDevice, st));
      ACS_CUDA(cudaMemcpyAsync(static_cast<char*>(C->val) + vb * o, pb[2].p, vb * q.nnz, cudaMemcpyDeviceToDevice, st));
    }
    o += q.nnz;
  }
  ACS_CUDA(cudaStreamSynchronize(st));
  C->nnz = off;
  if (npieces) *npieces = pieces;
  if (nrestarts) *nrestarts = restarts;
  return ACSPGEMM_OK;
}

acspgemm_status acspgemm_multiply_host(acspgemm_plan p, const acspgemm_csr_in* A, const acspgemm_csr_in* B,
                                       acspgemm_dtype dtype, void* stream, int npieces, acspgemm_csr_out* C,
                                       int64_t capacity) {
  if (!p) return set_err(ACSPGEMM_ERR_INVALID_ARG, "plan is NULL");
  acspgemm_status s;
  if ((s = check_in(A, "A")) != ACSPGEMM_OK) return s;
  if ((s = check_in(B, "B")) != ACSPGEMM_OK) return s;
  if (!C) return set_err(ACSPGEMM_ERR_INVALID_ARG, "C is NULL");
  if (dtype != ACSPGEMM_F32 && dtype != ACSPGEMM_F64) return set_err(ACSPGEMM_ERR_INVALID_ARG, "bad dtype");
  if (A->cols != B->rows) return set_err(ACSPGEMM_ERR_DIM_MISMATCH, "A.cols != B.rows");
  const int S = p->opt.num_segments;
  if (npieces < 1 || npieces > S) return set_err(ACSPGEMM_ERR_INVALID_ARG, "npieces must be in [1, num_segments]");
  if (capacity < 0 || (capacity > 0 && (!C->col_idx || !C->val)))
    return set_err(ACSPGEMM_ERR_INVALID_ARG, "bad C capacity / buffers");
  if (!C->row_ptr) return set_err(ACSPGEMM_ERR_INVALID_ARG, "C.row_ptr is NULL");
  const size_t vb = dtype == ACSPGEMM_F64 ? 8 : 4;
  C->rows = A->rows;
  C->cols = B->cols;
  C->nnz = 0;
  if (A->rows == 0) { C->row_ptr[0] = 0; return ACSPGEMM_OK; }
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  HostPipeGuard guard(p, st);
  if (!p->hp_cs) ACS_CUDA(cudaStreamCreateWithFlags(&p->hp_cs, cudaStreamNonBlocking));
  if (!p->hp_ready) ACS_CUDA(cudaEventCreateWithFlags(&p->hp_ready, cudaEventDisableTiming));
  for (cudaEvent_t& e : p->hp_copied)
    if (!e) ACS_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  // inputs host -> device into plan memory (B once when it is A): the row pointers first
  // (the segments need them), then the columns and values on an input stream, B whole
  // (when it is not A) and A piece by piece, so piece g's multiply overlaps the copies of
  // the pieces after it
  if (!p->hp_in) ACS_CUDA(cudaStreamCreateWithFlags(&p->hp_in, cudaStreamNonBlocking));
  if (!p->hp_start) ACS_CUDA(cudaEventCreateWithFlags(&p->hp_start, cudaEventDisableTiming));
  for (cudaEvent_t& e : p->hp_inev)
    if (!e) ACS_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  const bool same = B->row_ptr == A->row_ptr && B->col_idx == A->col_idx && B->val == A->val &&
                    B->rows == A->rows && B->nnz == A->nnz;
  const acspgemm_csr_in* M[2] = {A, B};
  DevBuf* Dm[2] = {p->hp_a, p->hp_b};
  acspgemm_csr_in D[2];
  int64_t hbase[2] = {0, 0};
  for (int m = 0; m < (same ? 1 : 2); ++m) {
    const acspgemm_csr_in* H = M[m];
    DevBuf* d = Dm[m];
    const int64_t base = H->rows > 0 ? H->row_ptr[0] : 0;
    hbase[m] = base;
    ACS_ENSURE(d[0], sizeof(int32_t) * (H->rows + 1));
    ACS_ENSURE(d[1], sizeof(int32_t) * H->nnz);
    ACS_ENSURE(d[2], vb * H->nnz);
    ACS_CUDA(cudaMemcpyAsync(d[0].p, H->row_ptr, sizeof(int32_t) * (H->rows + 1), cudaMemcpyHostToDevice, st));
    // device view: row_ptr values index col / val directly (base shifted away)
    D[m] = acspgemm_csr_in{H->rows, H->cols, H->nnz, ptr<const int32_t>(d[0]), ptr<const int32_t>(d[1]) - base,
                           static_cast<const char*>(d[2].p) - vb * base};
  }
  if (same) D[1] = D[0];
  hbase[1] = same ? hbase[0] : hbase[1];
  // canonical segments of the whole A (plan memory, one read-back), grouped into pieces
  int64_t seg[MAX_SEGMENTS + 1];
  {
    ACS_ENSURE(p->seg, sizeof(int64_t) * (4 * (MAX_SEGMENTS + 1) + 2));
    int64_t* sd = ptr<int64_t>(p->seg);
    const CsrView Av{D[0].rows, D[0].cols, D[0].row_ptr, D[0].col_idx, D[0].val};
    launch_segments(Av, S, SegRows{}, sd, reinterpret_cast<int32_t*>(sd + 4 * (MAX_SEGMENTS + 1)), st);
    tl_launches += 1;
    ACS_CUDA(cudaGetLastError());
    ACS_CUDA(cudaMemcpyAsync(seg, sd, sizeof(int64_t) * (S + 1), cudaMemcpyDeviceToHost, st));
    ACS_CUDA(cudaStreamSynchronize(st));
  }
  auto piece_rows = [&](int g, int64_t& r0, int64_t& r1) {
    r0 = seg[(int)((int64_t)g * S / npieces)];
    r1 = seg[(int)((int64_t)(g + 1) * S / npieces)];
  };
  ACS_CUDA(cudaEventRecord(p->hp_start, st));            // the input buffers are free from here
  ACS_CUDA(cudaStreamWaitEvent(p->hp_in, p->hp_start, 0));
  auto copy_nz = [&](int m, int64_t z0, int64_t z1) -> acspgemm_status {   // entries [z0, z1) of M[m]
    if (z1 <= z0) return ACSPGEMM_OK;
    const acspgemm_csr_in* H = M[m];
    const int64_t o = z0 - hbase[m];
    ACS_CUDA(cudaMemcpyAsync(ptr<int32_t>(Dm[m][1]) + o, H->col_idx + z0, sizeof(int32_t) * (z1 - z0),
                             cudaMemcpyHostToDevice, p->hp_in));
    ACS_CUDA(cudaMemcpyAsync(static_cast<char*>(Dm[m][2].p) + vb * o, static_cast<const char*>(H->val) + vb * z0,
                             vb * (z1 - z0), cudaMemcpyHostToDevice, p->hp_in));
    return ACSPGEMM_OK;
  };
  if (!same) {
    if ((s = copy_nz(1, hbase[1], hbase[1] + B->nnz)) != ACSPGEMM_OK) return s;
    ACS_CUDA(cudaEventRecord(p->hp_inev[S], p->hp_in));
  }
  for (int g = 0; g < npieces; ++g) {
    int64_t r0, r1;
    piece_rows(g, r0, r1);
    if ((s = copy_nz(0, A->row_ptr[r0], A->row_ptr[r1])) != ACSPGEMM_OK) return s;
    ACS_CUDA(cudaEventRecord(p->hp_inev[g], p->hp_in));
  }
  ACS_ENSURE(p->hp_rng, 2 * sizeof(int32_t));
  int64_t off = 0;
  bool overflow = false;
  for (int g = 0; g < npieces; ++g) {
    const int s0 = (int)((int64_t)g * S / npieces), s1 = (int)((int64_t)(g + 1) * S / npieces);
    const int64_t r0 = seg[s0], r1 = seg[s1];
    ACS_CUDA(cudaStreamWaitEvent(st, p->hp_inev[g], 0));     // the piece's own rows of A
    if (!same) {
      ACS_CUDA(cudaStreamWaitEvent(st, p->hp_inev[S], 0));
    } else if (A->row_ptr[r1] > A->row_ptr[r0]) {
      // B is A: the rows of A this piece reaches, from its entries' column range (one
      // read-back); the pieces holding them must have arrived
      launch_col_range(D[0].col_idx + A->row_ptr[r0], (int64_t)A->row_ptr[r1] - A->row_ptr[r0], ptr<int32_t>(p->hp_rng), st);
      launch_read_back(p->hp_rng.p, p->h_scal, 2 * sizeof(int32_t), st);
      tl_launches += 2;
      ACS_CUDA(cudaStreamSynchronize(st));
      const int32_t* rng = reinterpret_cast<const int32_t*>(p->h_scal);
      const int64_t z0 = A->row_ptr[rng[0]], z1 = A->row_ptr[(int64_t)rng[1] + 1];
      for (int c = 0; c < npieces; ++c) {
        int64_t q0, q1;
        piece_rows(c, q0, q1);
        if (c != g && A->row_ptr[q0] < z1 && A->row_ptr[q1] > z0) ACS_CUDA(cudaStreamWaitEvent(st, p->hp_inev[c], 0));
      }
    }
    p->nseg_explicit = s1 - s0;
    for (int i = 0; i <= s1 - s0; ++i) p->seg_rows_explicit[i] = seg[s0 + i] - r0;
    const acspgemm_csr_in V{r1 - r0, A->cols, (int64_t)A->row_ptr[r1] - A->row_ptr[r0], D[0].row_ptr + r0,
                            D[0].col_idx, D[0].val};
    int64_t nnz_g = 0;
    if ((s = symbolic_impl(p, &V, &D[1], dtype, st, &nnz_g)) != ACSPGEMM_OK) return s;
    if (off + nnz_g >= (int64_t(1) << 31)) return set_err(ACSPGEMM_ERR_INDEX_OVERFLOW, "nnz(C) >= 2^31");
    if (off + nnz_g > capacity) overflow = true;
    if (!overflow) {
      // piece buffer k alternates; its previous copy-out (piece g - 2) must be done
      DevBuf* cb = p->hp_c[g & 1];
      ACS_CUDA(cudaStreamWaitEvent(st, p->hp_copied[g & 1], 0));
      if (cb[0].bytes < sizeof(int32_t) * (V.rows + 1) || cb[1].bytes < sizeof(int32_t) * nnz_g ||
          cb[2].bytes < vb * nnz_g)
        ACS_CUDA(cudaEventSynchronize(p->hp_copied[g & 1]));   // about to re-allocate it
      ACS_ENSURE(cb[0], sizeof(int32_t) * (V.rows + 1));
      ACS_ENSURE(cb[1], sizeof(int32_t) * nnz_g);
      ACS_ENSURE(cb[2], vb * nnz_g);
      acspgemm_csr_out Cg{V.rows, B->cols, nnz_g, ptr<int32_t>(cb[0]), ptr<int32_t>(cb[1]), cb[2].p};
      if ((s = numeric_impl(p, &Cg, st, (int32_t)off)) != ACSPGEMM_OK) return s;
      ACS_CUDA(cudaGetLastError());
      // copy piece g out on the copy stream while piece g + 1 is multiplied
      ACS_CUDA(cudaEventRecord(p->hp_ready, st));
      ACS_CUDA(cudaStreamWaitEvent(p->hp_cs, p->hp_ready, 0));
      // (the size queries of later pieces read back through mapped memory, never through
      // a copy engine, so they do not queue behind these copies)
      ACS_CUDA(cudaMemcpyAsync(C->row_ptr + r0, Cg.row_ptr, sizeof(int32_t) * (V.rows + 1), cudaMemcpyDeviceToHost,
                               p->hp_cs));
      if (nnz_g > 0) {
        ACS_CUDA(cudaMemcpyAsync(C->col_idx + off, Cg.col_idx, sizeof(int32_t) * nnz_g, cudaMemcpyDeviceToHost,
                                 p->hp_cs));
        ACS_CUDA(cudaMemcpyAsync(static_cast<char*>(C->val) + vb * off, Cg.val, vb * nnz_g, cudaMemcpyDeviceToHost,
                                 p->hp_cs));
      }
      ACS_CUDA(cudaEventRecord(p->hp_copied[g & 1], p->hp_cs));
    }
    off += nnz_g;
  }
  ACS_CUDA(cudaStreamSynchronize(p->hp_cs));
  C->nnz = off;
  if (overflow) return set_err(ACSPGEMM_ERR_INVALID_ARG, "C capacity " + std::to_string(capacity) +
                                                         " < nnz(C) = " + std::to_string(off));
  return ACSPGEMM_OK;
}

acspgemm_status acspgemm_free_csr(acspgemm_csr_out* C, void* stream) {
  if (!C) return set_err(ACSPGEMM_ERR_INVALID_ARG, "C is NULL");
  cudaStream_t st = reinterpret_cast<cudaStream_t>(stream);
  if (C->row_ptr) cudaFreeAsync(C->row_ptr, st);
  if (C->col_idx) cudaFreeAsync(C->col_idx, st);
  if (C->val) cudaFreeAsync(C->val, st);
  C->row_ptr = nullptr; C->col_idx = nullptr; C->val = nullptr;
  ACS_CUDA(cudaGetLastError());
  return ACSPGEMM_OK;
}

acspgemm_status acspgemm_stage_times(acspgemm_plan p, float* ms_out, int n) {
  if (!p || !ms_out) return set_err(ACSPGEMM_ERR_INVALID_ARG, "NULL argument");
  if (!p->opt.collect_stage_times || !p->ev_ok) return set_err(ACSPGEMM_ERR_NOT_READY, "stage times not collected");
  if (p->empty) {
    for (int i = 0; i < n && i < 10; ++i) ms_out[i] = 0.f;
    return ACSPGEMM_OK;
  }
  ACS_CUDA(cudaEventSynchronize(p->ev[S_END]));
  for (int i = 0; i < n && i < 10; ++i) {
    float ms = 0.f;
    // stages 8 (HASH: k_dict + k_hash) and 9 (DICT: k_dict) are parts of stage 1 (ESC)
    const int a = i < 8 ? i : (int)S_ESC, b = i < 8 ? i + 1 : (i == 8 ? (int)S_HASHEND : (int)S_DICTEND);
    if (cudaEventElapsedTime(&ms, p->ev[a], p->ev[b]) != cudaSuccess) { cudaGetLastError(); ms = -1.f; }
    ms_out[i] = ms;
  }
  return ACSPGEMM_OK;
}

acspgemm_status acspgemm_set_trace(acspgemm_plan p, int enable) {
  if (!p) return set_err(ACSPGEMM_ERR_INVALID_ARG, "NULL plan");
  p->trace_on = enable != 0;
  p->trace_blocks = 0;
  return ACSPGEMM_OK;
}

acspgemm_status acspgemm_sm_load(acspgemm_plan p, int kernel, double* per_sm_ms, int nsm, double* mpl,
                                 int64_t* nblocks_traced) {
  if (!p || !mpl) return set_err(ACSPGEMM_ERR_INVALID_ARG, "NULL argument");
  if (kernel < 0 || kernel > 3) return set_err(ACSPGEMM_ERR_INVALID_ARG, "kernel must be 0..3");
  if (!p->trace_on || p->trace_blocks <= 0 || !p->trace.p)
    return set_err(ACSPGEMM_ERR_NOT_READY, "no traced multiply (acspgemm_set_trace before the symbolic pass)");
  int dev = p->dev, sms = 0;
  ACS_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  const int64_t n = p->trace_blocks;
  std::vector<uint64_t> h((size_t)(3 * n));
  ACS_CUDA(cudaMemcpy(h.data(), ptr<uint64_t>(p->trace) + (int64_t)kernel * 3 * n, sizeof(uint64_t) * 3 * n,
                      cudaMemcpyDeviceToHost));
  std::vector<double> busy((size_t)sms, 0.0);
  int64_t traced = 0;
  for (int64_t b = 0; b < n; ++b) {
    const uint64_t sm = h[3 * b], t0 = h[3 * b + 1], t1 = h[3 * b + 2];
    if (t1 == 0 || t1 < t0 || sm >= (uint64_t)sms) continue;
    busy[(size_t)sm] += (double)(t1 - t0) * 1e-6;
    ++traced;
  }
  double mx = 0.0, mn = 0.0;
  if (traced > 0) {
    mx = *std::max_element(busy.begin(), busy.end());
    mn = *std::min_element(busy.begin(), busy.end());
  }
  *mpl = mx > 0.0 ? mn / mx : 0.0;
  if (nblocks_traced) *nblocks_traced = traced;
  if (per_sm_ms)
    for (int i = 0; i < nsm && i < sms; ++i) per_sm_ms[i] = busy[(size_t)i];
  return ACSPGEMM_OK;
}

acspgemm_status acspgemm_plan_info(acspgemm_plan p, acspgemm_info* info) {
  if (!p || !info) return set_err(ACSPGEMM_ERR_INVALID_ARG, "NULL argument");
  *info = p->info;
  return ACSPGEMM_OK;
}

acspgemm_status acspgemm_block_row_starts(acspgemm_plan p, int32_t* host_out, int64_t n) {
  if (!p || (!host_out && n > 0)) return set_err(ACSPGEMM_ERR_INVALID_ARG, "NULL argument");
  if (!p->ready) return set_err(ACSPGEMM_ERR_NOT_READY, "no symbolic pass");
  if (n > p->info.nblocks) n = p->info.nblocks;
  if (n <= 0) return ACSPGEMM_OK;
  ACS_CUDA(cudaMemcpy(host_out, p->brs.p, sizeof(int32_t) * n, cudaMemcpyDeviceToHost));
  return ACSPGEMM_OK;
}

double acspgemm_pool_estimate_bytes(int64_t nA, int64_t nnzA, int64_t nB, int64_t mB, int64_t nnzB,
                                    int value_bytes) {
  double S = 0.0;
  if (nA > 0 && nB > 0 && mB > 0 && nnzA > 0 && nnzB > 0) {
    const double a = (double)nnzA / (double)nA;
    const double b = (double)nnzB / (double)nB;
    const double pb = b / (double)mB;
    S = pb < 1.0 ? (double)nA * b * (-std::expm1(a * std::log1p(-pb))) / pb : (double)nA * b;
  }
  const double bytes = S * (4.0 + value_bytes) * 1.2;
  return bytes > 100e6 ? bytes : 100e6;
}

acspgemm_status acspgemm_debug_work_distribution(const int32_t* lengths, int nentries, const int32_t* draws,
                                                 int ndraws, int32_t* ares, int32_t* bres, int32_t* remaining) {
  if (nentries < 0 || nentries > NPB || ndraws < 0 || (!lengths && nentries) || (!draws && ndraws))
    return set_err(ACSPGEMM_ERR_INVALID_ARG, "bad arguments");
  int64_t total_len = 0, total_draw = 0;
  for (int i = 0; i < nentries; ++i) total_len += lengths[i];
  for (int d = 0; d < ndraws; ++d) {
    if (draws[d] < 0 || draws[d] > CAP) return set_err(ACSPGEMM_ERR_INVALID_ARG, "draw > CAP");
    total_draw += draws[d];
  }
  if (total_draw > total_len) return set_err(ACSPGEMM_ERR_INVALID_ARG, "draws exceed the work");
  Scratch<int32_t> dl, dd, da, db, dr;
  ACS_CUDA(cudaMalloc(&dl.d, sizeof(int32_t) * (nentries + 1)));
  ACS_CUDA(cudaMalloc(&dd.d, sizeof(int32_t) * (ndraws + 1)));
  ACS_CUDA(cudaMalloc(&da.d, sizeof(int32_t) * (total_draw + 1)));
  ACS_CUDA(cudaMalloc(&db.d, sizeof(int32_t) * (total_draw + 1)));
  ACS_CUDA(cudaMalloc(&dr.d, sizeof(int32_t) * ((int64_t)ndraws * nentries + 1)));
  if (nentries) ACS_CUDA(cudaMemcpy(dl.d, lengths, sizeof(int32_t) * nentries, cudaMemcpyHostToDevice));
  if (ndraws) ACS_CUDA(cudaMemcpy(dd.d, draws, sizeof(int32_t) * ndraws, cudaMemcpyHostToDevice));
  k_debug_wd<<<1, THREADS>>>(dl.d, nentries, dd.d, ndraws, da.d, db.d, dr.d);
  ACS_CUDA(cudaGetLastError());
  ACS_CUDA(cudaDeviceSynchronize());
  if (total_draw) {
    ACS_CUDA(cudaMemcpy(ares, da.d, sizeof(int32_t) * total_draw, cudaMemcpyDeviceToHost));
    ACS_CUDA(cudaMemcpy(bres, db.d, sizeof(int32_t) * total_draw, cudaMemcpyDeviceToHost));
  }
  if ((int64_t)ndraws * nentries)
    ACS_CUDA(cudaMemcpy(remaining, dr.d, sizeof(int32_t) * ndraws * nentries, cudaMemcpyDeviceToHost));
  return ACSPGEMM_OK;
}

acspgemm_status acspgemm_debug_sort_compact(const int32_t* rows, const int32_t* cols, const double* vals, int n,
                                            int32_t* out_rows, int32_t* out_cols, double* out_vals,
                                            uint32_t* out_state) {
  if (n < 0 || n > CAP) return set_err(ACSPGEMM_ERR_INVALID_ARG, "n must be in [0, CAP]");
  if (n == 0) return ACSPGEMM_OK;
  Scratch<int32_t> dr, dc, orow, ocol;
  Scratch<double> dv, oval;
  Scratch<uint32_t> ost;
  ACS_CUDA(cudaMalloc(&dr.d, sizeof(int32_t) * n));
  ACS_CUDA(cudaMalloc(&dc.d, sizeof(int32_t) * n));
  ACS_CUDA(cudaMalloc(&dv.d, sizeof(double) * n));
  ACS_CUDA(cudaMalloc(&orow.d, sizeof(int32_t) * n));
  ACS_CUDA(cudaMalloc(&ocol.d, sizeof(int32_t) * n));
  ACS_CUDA(cudaMalloc(&oval.d, sizeof(double) * n));
  ACS_CUDA(cudaMalloc(&ost.d, sizeof(uint32_t) * n));
  ACS_CUDA(cudaMemcpy(dr.d, rows, sizeof(int32_t) * n, cudaMemcpyHostToDevice));
  ACS_CUDA(cudaMemcpy(dc.d, cols, sizeof(int32_t) * n, cudaMemcpyHostToDevice));
  ACS_CUDA(cudaMemcpy(dv.d, vals, sizeof(double) * n, cudaMemcpyHostToDevice));
  const size_t smem = sizeof(SortSmem<double>);
  ACS_CUDA(cudaFuncSetAttribute(k_debug_sort_compact, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  k_debug_sort_compact<<<1, THREADS, smem>>>(dr.d, dc.d, dv.d, n, orow.d, ocol.d, oval.d, ost.d);
  ACS_CUDA(cudaGetLastError());
  ACS_CUDA(cudaDeviceSynchronize());
  ACS_CUDA(cudaMemcpy(out_rows, orow.d, sizeof(int32_t) * n, cudaMemcpyDeviceToHost));
  ACS_CUDA(cudaMemcpy(out_cols, ocol.d, sizeof(int32_t) * n, cudaMemcpyDeviceToHost));
  ACS_CUDA(cudaMemcpy(out_vals, oval.d, sizeof(double) * n, cudaMemcpyDeviceToHost));
  ACS_CUDA(cudaMemcpy(out_state, ost.d, sizeof(uint32_t) * n, cudaMemcpyDeviceToHost));
  return ACSPGEMM_OK;
}

int acspgemm_const(int id) {
  switch (id) {
    case 0: return NPB;
    case 1: return THREADS;
    case 2: return ITEMS;
    case 3: return CAP;
    case 4: return KEEP;
    case 5: return RADIX_BITS;
    case 6: return DEFAULT_SEGMENTS;
    case 7: return PATH_MAX_CHUNKS;
    default: return -1;
  }
}

const char* acspgemm_status_string(acspgemm_status s) {
  switch (s) {
    case ACSPGEMM_OK: return "ok";
    case ACSPGEMM_ERR_INVALID_ARG: return "invalid argument";
    case ACSPGEMM_ERR_DIM_MISMATCH: return "dimension mismatch";
    case ACSPGEMM_ERR_INDEX_OVERFLOW: return "index overflow";
    case ACSPGEMM_ERR_OUT_OF_MEMORY: return "out of memory";
    case ACSPGEMM_ERR_CUDA: return "cuda error";
    case ACSPGEMM_ERR_NOT_READY: return "not ready";
    case ACSPGEMM_ERR_INTERNAL: return "internal limit";
  }
  return "unknown";
}

const char* acspgemm_last_error(void) { return tl_err.c_str(); }

int acspgemm_abi_version(void) { return ACSPGEMM_ABI_VERSION; }

}  // extern "C"
