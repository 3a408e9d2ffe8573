/*
 * acspgemm.h — C ABI of the B200 (sm_100a) AC-SpGEMM library: C = A·B on CSR with the
 * adaptive chunk-based ESC method of Winter, Mlakar, Zayer, Seidel, Steinberger,
 * "Adaptive Sparse Matrix-Matrix Multiplication on the GPU", PPoPP'19.  Citations
 * "L<n>" are PAPER.md line numbers (the paper transcript).
 *
 * Operation (Eq. (1)):  C_ij = sum_k A_ik · B_kj  with pattern
 *   {(i,j) : exists k, A_ik and B_kj stored}.  Structural zeros (exact cancellations)
 *   are kept; columns of every row of C are ascending and unique.
 * Method (L100-L104, Fig. 2): global load balancing (Alg. 1) -> AC-ESC with the local
 *   work distribution (Alg. 2), block radix sort and compaction scan (Alg. 3) writing
 *   chunks of C -> chunk ordering and Multi / Path / Search Merge of rows shared by
 *   several chunks -> row-pointer prefix sum -> chunk copy into C (§3.5).
 * Determinism: the block decomposition is fixed by A's nonzeros and the canonical
 *   segments; chunk slots are allocated per block (no atomics decide any placement or
 *   order); every sum follows a fixed order (AC-ESC: the compaction scan tree of Alg. 3;
 *   the adaptive accumulators: the left fold of a row's products in A-entry order).
 *   Results are bit-identical run to run and
 *   for any split of the segments over GPUs ("bit-stable", L34, L198, L430).
 *
 * Conventions for every entry point:
 *   - All matrix pointers are DEVICE pointers (cudaMalloc / torch CUDA memory) unless a
 *     parameter says "host".  `stream` is a cudaStream_t passed as void* (NULL = legacy
 *     default stream).  All device work is enqueued on that stream.
 *   - Index arrays are int32; values are float (ACSPGEMM_F32) or double (ACSPGEMM_F64),
 *     and A, B, C all use the same value type.  fp32 products and sums are computed in
 *     fp32, fp64 in fp64; no fast-math, IEEE NaN/Inf propagate.
 *   - Input CSR must be canonical: row_ptr non-decreasing, columns strictly increasing
 *     within a row and in [0, cols) (L52, L546).  row_ptr[0] may be non-zero: the
 *     matrix is then a row-range view whose row_ptr values index col_idx / val directly
 *     (used to hand one GPU its canonical segments of a larger A).
 *   - Ownership: the caller owns A and B (read only; keep them alive until the stream
 *     work completes) and, in the two-phase API, C.  A plan owns all intermediate memory
 *     (chunk pool, helpers) until acspgemm_plan_destroy.  No global state: distinct plans
 *     may be used concurrently from different threads / devices.
 *   - Errors are returned as acspgemm_status; the library never aborts.  The text of the
 *     last error of the calling thread is available from acspgemm_last_error().
 */
#ifndef ACSPGEMM_H_
#define ACSPGEMM_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define ACSPGEMM_ABI_VERSION 2   /* 2: acspgemm_options.pool_mode, acspgemm_info.pool_mode / ndeferred_blocks */

typedef enum { ACSPGEMM_F32 = 0, ACSPGEMM_F64 = 1 } acspgemm_dtype;

typedef enum {
  ACSPGEMM_OK = 0,
  ACSPGEMM_ERR_INVALID_ARG = 1,     /* null pointer with nnz > 0, negative size, non-canonical input */
  ACSPGEMM_ERR_DIM_MISMATCH = 2,    /* A.cols != B.rows */
  ACSPGEMM_ERR_INDEX_OVERFLOW = 3,  /* nnz(C) >= 2^31 with int32 C.row_ptr (acspgemm_numeric64 has none) */
  ACSPGEMM_ERR_OUT_OF_MEMORY = 4,   /* device allocation failed or pool_limit_bytes exceeded */
  ACSPGEMM_ERR_CUDA = 5,            /* a CUDA runtime error; see acspgemm_last_error() */
  ACSPGEMM_ERR_NOT_READY = 6,       /* acspgemm_numeric without a successful acspgemm_symbolic */
  ACSPGEMM_ERR_INTERNAL = 7         /* an internal limit was hit (e.g. > 2048 chunks in one row) */
} acspgemm_status;

/* Input CSR (device pointers).  rows+1 row_ptr entries; nnz = row_ptr[rows]-row_ptr[0]. */
typedef struct {
  int64_t rows, cols, nnz;
  const int32_t* row_ptr;
  const int32_t* col_idx;
  const void* val;
} acspgemm_csr_in;

/* Output CSR (device pointers).  row_ptr[rows+1] with row_ptr[0] = 0. */
typedef struct {
  int64_t rows, cols, nnz;
  int32_t* row_ptr;
  int32_t* col_idx;
  void* val;
} acspgemm_csr_out;

/* Output CSR with 64-bit row pointers (for nnz(C) >= 2^31; column indices stay int32). */
typedef struct {
  int64_t rows, cols, nnz;
  int64_t* row_ptr;
  int32_t* col_idx;
  void* val;
} acspgemm_csr_out64;

typedef struct acspgemm_plan_s* acspgemm_plan;

typedef struct {
  size_t pool_limit_bytes;   /* 0 = no limit; else symbolic fails with OUT_OF_MEMORY when the
                                chunk pool the pool_mode sizes exceeds it */
  int validate_inputs;       /* 1: check that A and B are canonical CSR (one extra sync) */
  int collect_stage_times;   /* 1: record CUDA events between stages (acspgemm_stage_times) */
  int num_segments;          /* canonical segments S (default 8, max 64) */
  int strategy;              /* ACSPGEMM_STRATEGY_ADAPTIVE (default): each candidate block is tried
                                by the hash accumulator (R31) and falls back to AC-ESC; blocks of
                                short rows go to the per-row accumulator (R34);
                                ACSPGEMM_STRATEGY_ESC: every block through AC-ESC;
                                ACSPGEMM_STRATEGY_HASH: hash accumulator, then AC-ESC;
                                ACSPGEMM_STRATEGY_DICT: block dictionary (R33), hash, AC-ESC.
                                ADAPTIVE, HASH and DICT give the same results bit for bit. */
  int pool_mode;             /* chunk-pool sizing (L556, L580; reading R40):
                                ACSPGEMM_POOL_BOUND (default): a hash-accumulator candidate block
                                owns min(products, rows x HASH_UBOUND = 192) (the accumulators'
                                output bound; in this mode a row of more distinct columns sends
                                its block to AC-ESC); a candidate that ends in AC-ESC is deferred
                                and run after the first pass in a region of its exact bound
                                appended to the pool (one more read-back; the pool grows by a
                                copy); other blocks own their exact product bound.  Same bytes of C;
                                ACSPGEMM_POOL_EXACT: every block owns its exact product bound,
                                products x (4 + value size) in all -- no overflow path;
                                ACSPGEMM_POOL_AUTO: EXACT when the exact bound fits
                                pool_limit_bytes (or there is no limit), else BOUND.
                                The DICT strategy always uses EXACT. */
} acspgemm_options;

#define ACSPGEMM_POOL_EXACT 0
#define ACSPGEMM_POOL_BOUND 1
#define ACSPGEMM_POOL_AUTO 2

#define ACSPGEMM_STRATEGY_ADAPTIVE 0
#define ACSPGEMM_STRATEGY_ESC 1
#define ACSPGEMM_STRATEGY_HASH 2
#define ACSPGEMM_STRATEGY_DICT 3

/* Counters of the last multiply of a plan (host values). */
typedef struct {
  int64_t products;          /* intermediate products sum_k nnz(A_:,k) nnz(B_k,:) ("temp", Table 2) */
  int64_t nnz_c;
  int64_t nblocks;           /* AC-ESC blocks (Alg. 1) */
  int64_t nchunks;           /* chunks written by AC-ESC */
  int64_t chunk_elems;       /* elements written to chunks (Table 3 "used") */
  int64_t nshared;           /* rows held by >= 2 chunks (the shared-rows array, L432) */
  int64_t nmulti, npath, nsearch, nmulti_groups;
  int64_t merge_elems;       /* pre-merge elements of shared rows */
  int64_t pool_bytes;        /* chunk pool reserved (exact bound, reading R8) */
  int64_t helper_bytes;      /* all other plan memory */
  double pool_estimate_bytes;/* the paper's estimate (L556, L580), for comparison */
  int64_t kernel_launches;   /* kernels launched by the last symbolic + numeric */
  int32_t nsegments;
  int64_t segment_rows[65];
  int64_t nhash_blocks;      /* blocks completed by an accumulator (dictionary or hash; R33, R31) */
  int64_t ndict_blocks;      /* of them, blocks completed by the column-dictionary accumulator (R33) */
  int64_t nrow_blocks;       /* blocks completed by the per-row accumulator for short rows (R34) */
  int64_t ndeferred_blocks;  /* POOL_BOUND: candidate blocks that ended in AC-ESC (second pass) */
  int32_t pool_mode;         /* the sizing the last symbolic used (EXACT or BOUND) */
} acspgemm_info;

/* Defaults: no pool limit, no validation, no stage times, 8 segments, adaptive strategy,
   exact pool. */
void acspgemm_options_default(acspgemm_options* opt);

/* Create a plan.  opt may be NULL (defaults).  *plan receives the handle. */
acspgemm_status acspgemm_plan_create(acspgemm_plan* plan, const acspgemm_options* opt);

/* Release a plan and all device memory it owns (synchronises the device). */
void acspgemm_plan_destroy(acspgemm_plan plan);

/* Explicit segment row boundaries for A (host array of nseg+1 row indices relative to A,
 * rows_host[0] = 0, rows_host[nseg] = A.rows, non-decreasing).  nseg = 0 restores the
 * canonical segmentation (boundary s = first row r with row_ptr[r]-row_ptr[0] >=
 * ceil(s·nnz/S)).  Used by the multi-GPU driver so that a GPU holding segments
 * [g0, g1) of the full A decomposes them exactly as a single GPU would. */
acspgemm_status acspgemm_set_segments(acspgemm_plan plan, int nseg, const int64_t* rows_host);

/* Canonical segment boundaries of A (nseg+1 host int64 values written to rows_host).
 * Runs one kernel on `stream` and synchronises it. */
acspgemm_status acspgemm_canonical_segments(const acspgemm_csr_in* A, int nseg, int64_t* rows_host, void* stream);

/* Symbolic + merge pass.  Runs global load balancing, AC-ESC, chunk ordering, the
 * merges and the row-pointer scan on `stream`; chunk data and C's row_ptr stay in plan
 * memory.  *nnz_c (host) receives nnz(C).  Synchronises `stream` (the size query is
 * the one mandatory host round trip; three more small counter read-backs size the
 * chunk pool and the merge launches). */
acspgemm_status acspgemm_symbolic(acspgemm_plan plan, const acspgemm_csr_in* A, const acspgemm_csr_in* B,
                                  acspgemm_dtype dtype, void* stream, int64_t* nnz_c);

/* Numeric pass: copy row_ptr and the chunk data into caller-allocated C
 * (row_ptr[rows+1], col_idx[nnz_c], val[nnz_c] of the dtype given to symbolic).
 * C->rows/cols/nnz are filled in.  Asynchronous on `stream`.  Returns
 * ACSPGEMM_ERR_INDEX_OVERFLOW when nnz(C) >= 2^31 (int32 row_ptr): use acspgemm_numeric64. */
acspgemm_status acspgemm_numeric(acspgemm_plan plan, acspgemm_csr_out* C, void* stream);

/* Re-multiply with new VALUES on the pattern of the plan's last acspgemm_symbolic (SURVEY
 * §8(f)-2, e.g. an AMG hierarchy re-setup): A and B must have exactly the structure
 * (row_ptr, col_idx contents, dimensions, dtype) of that call -- the caller guarantees it,
 * the library checks only the dimensions -- and C is caller-allocated with the nnz that
 * call returned.  Produces the same bits as a fresh symbolic + numeric on the new values.
 * No host synchronisation: the sizes the symbolic read back are replayed, and the whole
 * launch sequence is captured once into a CUDA graph (re-captured when any pointer
 * changes; on the legacy default stream it runs uncaptured).  Asynchronous on `stream`.
 * Any later acspgemm_symbolic on the plan starts a new pattern.  Stage times are not
 * collected by this call. */
acspgemm_status acspgemm_numeric_update(acspgemm_plan plan, const acspgemm_csr_in* A, const acspgemm_csr_in* B,
                                        acspgemm_csr_out* C, void* stream);

/* Numeric pass into a C with int64 row_ptr[rows+1] (any nnz(C); outputs
 * beyond 2^31 entries, e.g. skewed graph products).  Otherwise as acspgemm_numeric. */
acspgemm_status acspgemm_numeric64(acspgemm_plan plan, acspgemm_csr_out64* C, void* stream);

/* One-shot C = A·B.  The library allocates C->row_ptr/col_idx/val with cudaMallocAsync
 * on `stream`; release them with acspgemm_free_csr.  Uses a temporary plan. */
acspgemm_status acspgemm_multiply(const acspgemm_csr_in* A, const acspgemm_csr_in* B, acspgemm_csr_out* C,
                                  void* stream, acspgemm_dtype dtype);

/* End-to-end C = A·B with A, B and C in HOST memory: inputs host -> device on `stream`,
 * the multiply, the result device -> host.  A_host / B_host carry host pointers (page-
 * locked memory gives asynchronous full-speed copies; pageable memory works, slower);
 * B_host may alias A_host (copied once).  The multiply runs in `npieces` row pieces of
 * whole canonical segments (1 <= npieces <= the plan's num_segments), so
 * the device -> host copy of piece g (on an internal stream) overlaps the multiply of
 * piece g + 1; C is bit-identical to a one-piece multiply.  C->row_ptr (rows+1 entries),
 * C->col_idx and C->val (`capacity` entries) are caller-allocated HOST buffers.  If
 * nnz(C) > capacity the call returns ACSPGEMM_ERR_INVALID_ARG with C->nnz = nnz(C), which
 * makes capacity = 0 a size query.  The device copies of A and B and two alternating
 * piece buffers of C are plan memory (kept for reuse until acspgemm_plan_destroy); the
 * plan's segment setting is restored.  The plan's counters and stage times describe the
 * last piece.  Synchronises `stream`. */
acspgemm_status acspgemm_multiply_host(acspgemm_plan plan, const acspgemm_csr_in* A_host,
                                       const acspgemm_csr_in* B_host, acspgemm_dtype dtype, void* stream,
                                       int npieces, acspgemm_csr_out* C_host, int64_t capacity);

/* C = A·B within the plan's pool_limit_bytes (the paper restarts a
 * kernel when its chunk pool runs out, L254, L844).  A and B are device CSR.  Instead of
 * failing with OUT_OF_MEMORY when the exact pool bound exceeds the budget, the multiply
 * runs in pieces of whole canonical segments: each piece is the longest run of
 * segments whose bound fits (a piece over budget is retried on half as many segments --
 * a "restart", which costs only the global load balancing of the refused piece).  Every
 * block, chunk and merge is that of the one-piece multiply, so C is bit-identical to
 * it.  C is allocated like acspgemm_multiply (cudaMallocAsync on `stream`, free with
 * acspgemm_free_csr); the pieces are concatenated into it (their buffers are plan
 * memory, kept for the next call).  *npieces / *nrestarts
 * (nullable) receive the piece and restart counts.  A single segment over budget
 * returns OUT_OF_MEMORY.  Synchronises `stream`; the plan's segment setting is restored. */
acspgemm_status acspgemm_multiply_budget(acspgemm_plan plan, const acspgemm_csr_in* A, const acspgemm_csr_in* B,
                                         acspgemm_dtype dtype, void* stream, acspgemm_csr_out* C, int* npieces,
                                         int* nrestarts);

/* Galerkin triple product C = R·(A·P) as two ordered AC-SpGEMMs (SURVEY §8(f)-2,
 * reading R24: the association R·(A·P)).  A·P lives in temporary device memory that is
 * released before return; C is allocated like acspgemm_multiply (cudaMallocAsync on
 * `stream`, free with acspgemm_free_csr).  Requires R.cols == A.rows, A.cols == P.rows.
 * Synchronises `stream`. */
acspgemm_status acspgemm_rap(const acspgemm_csr_in* R, const acspgemm_csr_in* A, const acspgemm_csr_in* P,
                             acspgemm_csr_out* C, void* stream, acspgemm_dtype dtype);

/* Free C allocated by acspgemm_multiply or acspgemm_rap (cudaFreeAsync on `stream`). */
acspgemm_status acspgemm_free_csr(acspgemm_csr_out* C, void* stream);

/* Per-stage device times (ms) of the last symbolic + numeric when collect_stage_times
 * was set, in the order of Fig. 7 (L740): GLB, ESC, MCC, MM, PM, SM, SCAN, CC, then HASH:
 * the part of ESC spent in the accumulators (column dictionary + hash table, readings
 * R33, R31), then DICT: the part spent in the column-dictionary accumulator.
 * Writes min(n, 10) values.  Synchronises the plan's events. */
acspgemm_status acspgemm_stage_times(acspgemm_plan plan, float* ms_out, int n);

/* Counters of the last multiply. */
acspgemm_status acspgemm_plan_info(acspgemm_plan plan, acspgemm_info* info);

/* Multiprocessor load (Table 3's "lowest multiprocessor load", mpL, L746-L760, L832).
 * acspgemm_set_trace(plan, 1) makes the following symbolic passes record, for every block
 * a stage-2 kernel processes, the SM it ran on (%smid) and its start / end time
 * (%globaltimer); 0 turns it off (the default; recording costs two timer reads and three
 * stores per block).  acspgemm_sm_load then reports, for kernel 0 = hash accumulator
 * (k_hash), 1 = per-row accumulator (k_rows), 2 = AC-ESC (k_esc), 3 = small-tile AC-ESC:
 * per SM the summed block time in ms (per_sm_ms, host, nsm entries; nullable) and
 * *mpl = min over SMs / max over SMs of that busy time (1 = perfectly balanced; reading
 * R36), and *nblocks_traced (nullable) = blocks the kernel processed.  Synchronous (reads
 * the records back).  NOT_READY if the last symbolic was not traced. */
acspgemm_status acspgemm_set_trace(acspgemm_plan plan, int enable);
acspgemm_status acspgemm_sm_load(acspgemm_plan plan, int kernel, double* per_sm_ms, int nsm, double* mpl,
                                 int64_t* nblocks_traced);

/* Copy the last blockRowStarts array (Alg. 1 output, one int32 per block) to host. */
acspgemm_status acspgemm_block_row_starts(acspgemm_plan plan, int32_t* host_out, int64_t n);

/* The paper's chunk-pool estimate in bytes (L556, L580): S = nA·b·(1-(1-p_b)^a)/p_b
 * with a = nnzA/nA, b = nnzB/nB, p_b = b/mB, times (4 + value_bytes) times 1.2, at
 * least 100 MB.  Host-only arithmetic. */
double acspgemm_pool_estimate_bytes(int64_t nA, int64_t nnzA, int64_t nB, int64_t mB, int64_t nnzB,
                                    int value_bytes);

/* ---- unit entry points for parity tests of single steps (host buffers; one CTA) ----
 * Work distribution (Alg. 2): placework(lengths[0..nentries)), then receivework for each
 * draws[d] (each <= CAP and <= the remaining size).  ares/bres receive sum(draws)
 * values in draw order (product c of draw d at offset sum(draws[<d]) + c);
 * remaining receives ndraws*nentries values: products still owed per entry after each
 * draw.  nentries <= acspgemm_const(0) (NNZ_PER_BLOCK). */
acspgemm_status acspgemm_debug_work_distribution(const int32_t* lengths, int nentries, const int32_t* draws,
                                                 int ndraws, int32_t* ares, int32_t* bres, int32_t* remaining);

/* Block radix sort + compaction scan (Alg. 3) of n <= CAP (row, col, value) triples in
 * input order (fp64 values).  Outputs, per sorted position: row, col, scanned value and
 * the 32-bit Alg. 3 state word. */
acspgemm_status acspgemm_debug_sort_compact(const int32_t* rows, const int32_t* cols, const double* vals, int n,
                                            int32_t* out_rows, int32_t* out_cols, double* out_vals,
                                            uint32_t* out_state);

/* Build constants: 0 NNZ_PER_BLOCK, 1 THREADS, 2 ITEMS, 3 CAP, 4 KEEP, 5 RADIX_BITS,
 * 6 default segments, 7 PATH_MAX_CHUNKS.  Returns -1 for an unknown id. */
int acspgemm_const(int id);

const char* acspgemm_status_string(acspgemm_status s);
const char* acspgemm_last_error(void);
int acspgemm_abi_version(void);

#ifdef __cplusplus
}
#endif
#endif /* ACSPGEMM_H_ */
