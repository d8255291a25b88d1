/* =============================================================================
 * sr.h — C ABI of the B200 row-reordered, adaptively tiled SpMM / SDDMM library
 * ("sr" = sparse reorder).  Jiang, Hong & Agrawal, PPoPP'20.
 * P:N = /root/reference/PAPER.md line N; R<n> = reading listed in DESIGN.md §3.
 *
 * Conventions
 *  - Every function returns int status: SR_OK (0) or a negative SR_E* code; the
 *    message of the last error on the calling thread is sr_last_error().  No C++
 *    exception crosses the ABI.
 *  - Handles are not thread-safe: one handle per stream, or serialise calls.
 *  - Dense operands (B, X, Y, C, out) are caller-owned DEVICE memory on the
 *    handle's device, fp32, row-major with a leading dimension in elements.
 *    The library owns only its CSR copy, its plan and its scratch.
 *  - sr_spmm / sr_sddmm are asynchronous on `stream` and never synchronise the
 *    host.  sr_reorder synchronises (the clustering runs on the host).
 *  - `stream` is a cudaStream_t (NULL = legacy default stream).
 * ============================================================================= */
#ifndef SR_H_
#define SR_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SR_OK 0
#define SR_EINVAL (-1)       /* bad argument, malformed CSR, duplicate entry, ld < K ... */
#define SR_ENOMEM (-2)       /* host or device allocation failed                         */
#define SR_ECUDA (-3)        /* a CUDA runtime call failed (see sr_last_error)           */
#define SR_ESTATE (-4)       /* call out of order (e.g. sr_reorder twice)                */
#define SR_EUNSUPPORTED (-5) /* valid but unsupported (nnz >= 2^31, bsize > 2, ...)      */

#define SR_REORDER_AUTO 0  /* P:265, P:332 decision rules                              */
#define SR_REORDER_FORCE 1 /* both reordering rounds always                            */
#define SR_REORDER_OFF 2   /* original order, ASpT tiles only ("ASpT-NR")       */

typedef struct CUstream_st* sr_stream; /* == cudaStream_t */
typedef struct sr_csr_s* sr_csr;       /* opaque handle owned by the library */

/* -----------------------------------------------------------------------------
 * sr_csr_create — ingest a CSR matrix (Fig 1): rowptr[i] is the first
 * nnz of row i, colidx / vals hold the nnz row by row.
 *   nrows, ncols : M, N >= 0, both < 2^31;   nnz < 2^31.
 *   rowptr       : HOST int64[nrows+1], rowptr[0] = 0, non-decreasing, rowptr[M] = nnz
 *   colidx       : HOST int32[nnz], 0 <= colidx < ncols, no duplicate (row, col)
 *   vals         : HOST fp32[nnz]
 *   device       : CUDA device ordinal that will hold the matrix
 * Deep-copies (the caller keeps its arrays).  Rows need not be column-sorted:
 * they are sorted internally and SDDMM results still come back in the caller's
 * nnz order (R22).  The handle starts with the identity plan (no tiles): spmm /
 * sddmm work right away as the plain row-wise kernels of P:101 (its device arrays are built on
 * the first spmm / sddmm / set_values call, synchronously, unless a plan is installed first).
 * Errors: SR_EINVAL (malformed / duplicates), SR_EUNSUPPORTED, SR_ENOMEM, SR_ECUDA.
 * ---------------------------------------------------------------------------*/
int sr_csr_create(int64_t nrows, int64_t ncols, int64_t nnz, const int64_t* rowptr,
                  const int32_t* colidx, const float* vals, int device, sr_csr* out);

/* -----------------------------------------------------------------------------
 * Reorder / tiling parameters (Alg 3 inputs S, siglen, bsize, threshold_size,
 * P:160-162; values used by the paper P:366; ASpT parameters R17).
 * ---------------------------------------------------------------------------*/
typedef struct {
  int32_t siglen;          /* minhash signature length, 128                       */
  int32_t bsize;           /* LSH band size, 2; siglen % bsize == 0; 1 or 2 here   */
  int32_t threshold_size;  /* cluster size that freezes a cluster, 256, >= 2       */
  int32_t max_bucket;      /* LSH bucket chunk cap (R14); 0 = unlimited (paper-exact)      */
  uint64_t seed;           /* hash-family seed (O3); the plan is bit-exact per seed        */
  int32_t panel_rows;      /* ASpT row-panel height (P:111 example: 3), 1..128             */
  int32_t dense_min;       /* dense column = >= dense_min nnz in the panel (2), >= 1 */
  int32_t tile_cols;       /* dense columns per shared-memory tile, 1..1024                */
  int32_t mode;            /* SR_REORDER_AUTO | SR_REORDER_FORCE | SR_REORDER_OFF          */
  int32_t skip_dense_num, skip_dense_den; /* skip round 1 iff DenseRatio0 > num/den (1/10) */
  int32_t skip_sim_num, skip_sim_den;     /* skip round 2 iff AvgSim > num/den (1/10)      */
  int32_t world, rank;     /* row-panel shard owned by this handle; 1, 0 = whole matrix    */
  int32_t auto_dense_min;  /* dense criterion of the AUTO DenseRatio0 decision (R28);
                              0 = dense_min.  Lets the decision ask "does the original order
                              already share columns?" while the kernels run with a higher
                              execution threshold                           */
  int32_t reserved0;       /* must be 0                                                    */
} sr_reorder_params;

/* Fill *p with the defaults above (siglen 128, bsize 2, threshold 256, max_bucket 32,
 * seed 4, panel_rows 64, dense_min 2, tile_cols 64, AUTO, 1/10, 1/10, world 1, rank 0,
 * auto_dense_min 0). */
void sr_default_params(sr_reorder_params* p);

/* The parameters of h's plan (after sr_reorder or sr_plan_load; the defaults before).
 * Errors: SR_EINVAL (NULL). */
int sr_get_params(sr_csr h, sr_reorder_params* out);

/* -----------------------------------------------------------------------------
 * sr_reorder — build the plan (Fig 5 workflow):
 *   round 1: LSH candidate pairs of A's rows (minhash + banding on the GPU,
 *            P:151-153) -> exact Jaccard (GPU) -> Alg 3 clustering (host,
 *            P:155-222) -> perm1;  skipped under AUTO if DenseRatio0 > 1/10
 *            (DenseRatio0 with the dense criterion auto_dense_min, R28).
 *   ASpT tiling of perm1's row panels: dense columns + remainder.
 *   round 2: the same on the remainder rows -> perm2; skipped under AUTO if the
 *            remainder's consecutive-row AvgSim > 1/10.
 *   world > 1: keep only panels [cut_rank, cut_rank+1) of the nnz-balanced
 *            contiguous partition.
 * Synchronous.  Callable once per handle.  Errors: SR_EINVAL, SR_EUNSUPPORTED,
 * SR_ESTATE (second call), SR_ENOMEM, SR_ECUDA.
 * ---------------------------------------------------------------------------*/
int sr_reorder(sr_csr h, const sr_reorder_params* p, sr_stream stream);

/* -----------------------------------------------------------------------------
 * sr_spmm — C := A·B (Alg 1, overwrite semantics R1).
 *   B : device fp32 [ncols × K], leading dimension ldb >= K
 *   C : device fp32, leading dimension ldc >= K;
 *       world == 1: [nrows × K], original row order;
 *       world  > 1: [sr_shard_nrows × K], this shard's rows packed in plan order
 *                   (original ids from sr_shard_rows).
 *   K >= 1.  The 16-byte vector path needs K % 4 == 0, ldb % 4 == 0, ldc % 4 == 0 and
 *   16-byte aligned B / C; anything else takes the scalar path.
 * Asynchronous on `stream`.  Errors: SR_EINVAL, SR_ECUDA (launch).
 * ---------------------------------------------------------------------------*/
int sr_spmm(sr_csr h, const float* B, int64_t K, int64_t ldb, float* C, int64_t ldc,
            sr_stream stream);

/* -----------------------------------------------------------------------------
 * sr_sddmm — out[p] := vals[p] · <X[row(p), :], Y[colidx[p], :]> (Alg 2, P:78-92,
 *   readings R2, R22: X is the row-side M×K operand, Y the column-side N×K one).
 *   out : device fp32;  world == 1: [nnz] in the caller's original nnz order;
 *         world > 1: [sr_shard_nnz] packed in plan order (ids from sr_shard_nnz_ids).
 * Asynchronous on `stream`.  Errors: SR_EINVAL, SR_ECUDA.
 * ---------------------------------------------------------------------------*/
int sr_sddmm(sr_csr h, const float* X, int64_t ldx, const float* Y, int64_t ldy, int64_t K,
             float* out, sr_stream stream);

/* -----------------------------------------------------------------------------
 * sr_set_values — replace the nonzero values the kernels use; pattern and plan unchanged.
 *   For iterative applications that reuse one plan with changing values, e.g. the
 *   collaborative-filtering gradient loop: E := SDDMM(U, V) − R on the
 *   pattern, then E·V with the same plan.
 *   vals : DEVICE fp32 in the handle's OUTPUT order (the order sr_sddmm writes):
 *          world == 1: [nnz], the caller's original nnz order; world > 1: [sr_shard_nnz],
 *          this shard's packed order.
 *   The device plan keeps the new values until the next sr_set_values; a later sr_reorder /
 *   sr_plan_load rebuilds the plan from the values given to sr_csr_create.
 * Asynchronous on `stream` (the caller keeps `vals` alive until it completes).
 * Errors: SR_EINVAL, SR_ECUDA.
 * ---------------------------------------------------------------------------*/
int sr_set_values(sr_csr h, const float* vals, sr_stream stream);

/* Free all host and device state.  NULL-safe.  Synchronises the device. */
int sr_destroy(sr_csr h);

/* -----------------------------------------------------------------------------
 * Offline reordering ("data reordering can be performed offline", the
 * preprocessing "amortized across iterations"): a plan is fully determined by the matrix,
 * the parameters and the two row orders, so it can be saved once and loaded later without
 * LSH or clustering (the tiling and the execution plan are rebuilt from perm1 / perm2).
 *
 * sr_plan_save — canonical byte image of h's plan into the HOST buffer buf[cap]:
 *   "SRPLAN01" | u32 version 1 | u32 reserved | i64 M, N, nnz | u64 matrix fingerprint
 *   (64-bit hash of the canonical rowptr / colidx) | sr_reorder_params | sr_plan_stats |
 *   i64 len1, i32 perm1[len1] | i64 len2, i32 perm2[len2] | u64 checksum of all preceding
 *   bytes.  *len gets the image size; buf may be NULL (size query).  The image does not
 *   depend on world / rank (perm2 is global; a shard filters it).
 *   Errors: SR_ESTATE (no plan: sr_reorder / sr_plan_load not called), SR_EINVAL (cap).
 * sr_plan_load — install a saved plan on a handle of the SAME matrix (fingerprint checked)
 *   that has no plan yet; world / rank select the shard (1, 0 = single GPU).  Synchronous.
 *   Errors: SR_EINVAL (bad / corrupted image, other matrix, bad permutation, bad world /
 *   rank), SR_ESTATE (the handle already has a plan), SR_ENOMEM, SR_ECUDA.
 * ---------------------------------------------------------------------------*/
int sr_plan_save(sr_csr h, void* buf, int64_t cap, int64_t* len);
int sr_plan_load(sr_csr h, const void* buf, int64_t len, int32_t world, int32_t rank, sr_stream stream);

/* -----------------------------------------------------------------------------
 * sr_trial — trial-and-error plan selection ("perform row-reordering in the first
 *   iteration and do SpMM or SDDMM on both the reordered matrix and the original matrix. If
 *   the reordered matrix is faster, keep the row-reordering").  Times op (SR_OP_SPMM:
 *   C := A·B with U = B, V unused, out = C; SR_OP_SDDMM: out := A ⊙ (U·Vᵀ) with U = X, V = Y)
 *   `reps` times on each of the n candidate handles (plans of the same matrix: equal
 *   nrows / ncols / nnz and shard output sizes, e.g. a reordered handle and a fresh one in the
 *   original order) after one warm-up call each, on `stream` with CUDA events.  ms[i] gets the
 *   median device time of candidate i (HOST array of n floats, may be NULL); *best the index
 *   of the fastest.  Operands are DEVICE memory as in sr_spmm / sr_sddmm; `out` holds the last
 *   candidate's result on return.  Synchronous.  Errors: SR_EINVAL (n < 1, NULL, candidates
 *   of different shapes, reps < 1, bad op), SR_ECUDA.
 * ---------------------------------------------------------------------------*/
#define SR_OP_SPMM 0
#define SR_OP_SDDMM 1
int sr_trial(const sr_csr* cands, int32_t n, int32_t op, const float* U, int64_t ldu, const float* V,
             int64_t ldv, int64_t K, float* out, int64_t ldo, int32_t reps, sr_stream stream, int32_t* best,
             float* ms);

/* ---------------------------------------------------------------------------
 * Plan metadata (bit-exact parity with the oracle; the gather/scatter step).
 * All output pointers are HOST memory of capacity `cap` elements; *len gets the
 * full length even when cap is too small (then SR_EINVAL and nothing written).
 * -------------------------------------------------------------------------*/
/* which = 1: perm1[M] (perm1[position] = original row);
 * which = 2: perm2 (positions of the non-empty remainder rows, processing order). */
int sr_get_perm(sr_csr h, int which, int32_t* out, int64_t cap, int64_t* len);

typedef struct {
  int64_t nnz;
  int64_t dense0;        /* dense-tile nnz of the original order under the AUTO decision's
                            criterion (auto_dense_min, else dense_min): DenseRatio0 = dense0/nnz */
  int64_t dense1;        /* dense-tile nnz of the plan:           DenseRatio  = dense1/nnz */
  uint64_t avgsim_num;   /* AvgSim of the remainder = num/den (R27 fixed point)          */
  uint64_t avgsim_den;
  int32_t round1, round2;/* rounds performed                                             */
  int64_t E1, E2;        /* LSH candidate pairs of round 1 / round 2                     */
  int64_t npanels;
  int64_t ndense_cols;   /* Σ_p |D_p|                                                    */
  int64_t ntiles;        /* Σ_p ceil(|D_p| / tile_cols)                                   */
  int64_t n_perm2;       /* non-empty remainder rows                                     */
  int64_t shard_panel_begin, shard_panel_end; /* panels owned by this handle             */
  int64_t shard_nrows, shard_nnz;
  double t_lsh1_s, t_cluster1_s, t_tile_s, t_lsh2_s, t_cluster2_s, t_total_s; /* wall time */
  double t_plan_s;       /* wall time of the device execution plan build (tasks, uploads)  */
} sr_plan_stats;

int sr_get_plan_stats(sr_csr h, sr_plan_stats* out);

/* Tiling arrays of the WHOLE plan (positions q = index into perm1), as the oracle's
 * O10 emits them.  Any pointer may be NULL to skip it; lengths:
 *   dense_ptr[npanels+1], dense_cols[ndense_cols],
 *   drow_ptr[M+1], d_slot[dense1], d_pos[dense1]        (dense nnz per position, slot asc)
 *   rrow_ptr[M+1], r_col[nnz-dense1], r_pos[nnz-dense1]  (remainder per position, CSR order)
 * d_pos / r_pos are the caller's ORIGINAL nnz indices. */
int sr_export_tiles(sr_csr h, int64_t* dense_ptr, int32_t* dense_cols, int64_t* drow_ptr,
                    int32_t* d_slot, int64_t* d_pos, int64_t* rrow_ptr, int32_t* r_col,
                    int64_t* r_pos);

/* Original row ids of this handle's shard, in the packed order sr_spmm writes. */
int sr_shard_rows(sr_csr h, int32_t* rows_out, int64_t cap, int64_t* len);
/* Original nnz ids of this handle's shard, in the packed order sr_sddmm writes. */
int sr_shard_nnz_ids(sr_csr h, int64_t* ids_out, int64_t cap, int64_t* len);

/* Gather helpers for sharded plans: after an all-gather of the packed shard
 * outputs, scatter them back to original positions.  All pointers are DEVICE memory.
 *   sr_scatter_rows  : dst[rows[r], 0:K] = src[r, 0:K] for r < n (rows[r] < 0 skipped)
 *   sr_scatter_values: dst[ids[i]] = src[i] for i < n (ids[i] < 0 skipped)
 * Asynchronous on `stream`.  Errors: SR_EINVAL, SR_ECUDA. */
int sr_scatter_rows(const float* src, int64_t lds, const int32_t* rows, int64_t n, int64_t K, float* dst,
                    int64_t ldd, sr_stream stream);
int sr_scatter_values(const float* src, const int64_t* ids, int64_t n, float* dst, sr_stream stream);

/* Kernel launches the last sr_spmm / sr_sddmm call issued on this handle. */
int sr_last_launch_count(sr_csr h, int32_t* n);

/* ---------------------------------------------------------------------------
 * Measurement hooks (bench.py): the bytes model of the current plan and per-launch
 * device times of the last sr_spmm / sr_sddmm call.
 * -------------------------------------------------------------------------*/
typedef struct {
  int64_t dense_nnz, sparse_nnz;        /* nnz served by phase D (tiles) / phase S (remainder) */
  int64_t dense_panels, sparse_items;   /* CTAs of phase D; warps (work items) of phase S      */
  int64_t dense_rows;                   /* rows written by phase D                             */
  int64_t sparse_rows;                  /* remainder rows (phase S writes or read-modify-writes) */
  int64_t zero_rows;                    /* rows with no nnz (phase S zero-fills them)          */
  int64_t rmw_rows;                     /* rows with both dense-tile and remainder nnz         */
  int64_t dense_col_loads;              /* Σ_p |D_p|: B/Y rows staged into shared memory */
  int64_t dense_distinct_cols;          /* distinct columns over all D_p                       */
  int64_t sparse_group_loads;           /* access model O14 of phase S (8 warps per CTA) */
  int64_t sparse_distinct_cols;         /* distinct columns of the remainder                   */
} sr_traffic_model;

int sr_get_traffic_model(sr_csr h, sr_traffic_model* out);

/* enable != 0: every later sr_spmm / sr_sddmm records a CUDA event pair around each of its
 * kernel launches on the call's stream. */
int sr_set_profiling(sr_csr h, int enable);

/* Device time of each launch of the last sr_spmm / sr_sddmm call (waits for its events).
 * kinds: 1 = spmm phase D (TMA shared-memory tiles), 2 = spmm phase S, 3 = sddmm phase D (TMA),
 *        4 = sddmm phase S, 5 = spmm phase D on register tiles, 6 = sddmm phase D on register tiles. */
int sr_last_kernel_times(sr_csr h, int32_t* kinds, float* ms, int32_t cap, int32_t* n);

const char* sr_last_error(void);

/* ---------------------------------------------------------------------------
 * Host-only entry points (no GPU needed; the host half of the pipeline).
 * -------------------------------------------------------------------------*/
/* Alg 3 (readings R3-R12) over a column-sorted CSR given as HOST
 * arrays, with candidate pairs packed (i<<32|j), i<j, sorted ascending and
 * unique, and their exact (inter, uni) (NULL: computed here).  Output perm[M]
 * in rule-B order.  Returns SR_OK / SR_EINVAL. */
int sr_host_cluster(int64_t M, const int64_t* rowptr, const int32_t* colidx, int64_t npairs,
                    const uint64_t* pairs, const uint32_t* inter, const uint32_t* uni,
                    int32_t threshold_size, int32_t* perm);

/* nnz-balanced contiguous partition of `npanels` weights into G shards
 * (cuts[0] = 0, cuts[G] = npanels; cuts[g] = smallest p with prefix(p)·G >= g·total). */
int sr_host_partition(int64_t npanels, const int64_t* weights, int32_t G, int64_t* cuts);

/* Library version string. */
const char* sr_version(void);

#ifdef __cplusplus
}
#endif
#endif /* SR_H_ */
