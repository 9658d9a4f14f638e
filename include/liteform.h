/*
 * liteform.h -- C ABI of liblf.so, the B200 (sm_100a) implementation of the
 * data-parallel hot path of LiteForm (Peng, Thomadakis, Pienaar, Kestor,
 * HPDC'25): CSR -> CELL conversion and the CELL SpMM  C = A . B.
 *
 * Citations: P:L<a>-<b> = lines of the paper text.  Readings of
 * passages the paper leaves silent or that the extraction garbled are listed
 * in DESIGN.md "Readings" (R1..R17, = SURVEY.md 8(c) C1..C17).
 *
 * Conventions for every call:
 *   - Pointers marked (device) are CUDA device pointers on the current device;
 *     (host) pointers are ordinary host memory.  No call takes ownership of a
 *     caller pointer.
 *   - lf_stream_t is a cudaStream_t (NULL = the legacy default stream).  All
 *     device work is enqueued on that stream; a call returns before the work
 *     completes unless documented as synchronising.
 *   - Errors are reported only through lf_status; no exception or abort
 *     crosses the ABI.  Argument checks are done on the host before any
 *     device work.  On LF_ERR_CUDA, lf_last_error_detail() holds the CUDA
 *     error string (thread-local, valid until the next call on the thread).
 *     A call that launches work first clears a non-sticky CUDA error left
 *     pending by earlier runtime calls of the thread, so its status reflects
 *     its own launches (a sticky error still fails its first launch).
 *   - Matrices: A is I x K sparse (CSR on input, CELL after build); B is a
 *     dense K x J fp32 row-major matrix with leading dimension ldb >= J
 *     (elements); C is dense I x J fp32 row-major with ldc >= J.
 *   - Precision (reading R14): fp32 values, fp32 products and fp32
 *     accumulation; partial results of one C row coming from several CELL
 *     rows are combined with fp32 atomic adds (order-dependent rounding).
 */
#ifndef LITEFORM_H
#define LITEFORM_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define LF_ABI_VERSION 1
#define LF_MAX_PARTS 64   /* maximum number of column partitions P */
#define LF_MAX_LOG2 30    /* maximum log2 of a bucket width or block size */

#if defined(__GNUC__)
#define LF_API __attribute__((visibility("default")))
#else
#define LF_API
#endif

typedef void *lf_stream_t; /* cudaStream_t */

typedef enum lf_status {
    LF_OK = 0,
    LF_ERR_INVALID_ARG = 1,    /* a size, pointer or parameter is out of range        */
    LF_ERR_UNSORTED_CSR = 2,   /* LF_VALIDATE=1 found unsorted / out-of-range columns  */
    LF_ERR_INDEX_OVERFLOW = 3, /* a CELL array would exceed int32 row or column range */
    LF_ERR_NO_MEMORY = 4,      /* the allocator returned NULL                          */
    LF_ERR_CUDA = 5,           /* a CUDA runtime call failed (see lf_last_error_detail) */
    LF_ERR_UNSUPPORTED = 6     /* a valid request this build does not implement        */
} lf_status;

/* Sparse A in CSR (Alg. 1 inputs rowPtr, colInd, val: P:L132-137).
 * All three arrays are (device), caller-owned, and must stay alive and
 * unmodified while a call that reads them runs (and, for a handle built with
 * use_cell = 0, for the handle's lifetime).
 *   row_ptr[n_rows+1]  int64, non-decreasing.  row_ptr[0] may be non-zero: a
 *                      row-shard view into a larger CSR; positions are
 *                      absolute indexes into col_ind / val.
 *   col_ind[...]       int32 in [0, n_cols), non-decreasing within each row
 *                      (duplicates allowed; they are kept and summed).
 *   val[...]           fp32 (explicit zeros allowed and kept).
 *   nnz                row_ptr[n_rows] - row_ptr[0]  (passed by the caller
 *                      so the host never reads device memory to size work). */
typedef struct lf_csr {
    int64_t n_rows;
    int64_t n_cols;
    int64_t nnz;
    const int64_t *row_ptr;
    const int32_t *col_ind;
    const float *val;
} lf_csr;

/* Device-memory provider for the handle's arrays (e.g. PyTorch's caching
 * allocator).  alloc must return a 256-byte-aligned device pointer usable on
 * stream s, or NULL; free releases it (stream-ordered on s).  Passing a NULL
 * lf_allocator* uses cudaMallocFromPoolAsync / cudaFreeAsync on the call's
 * stream with the library's private per-device memory pool (release
 * threshold 512 MiB; the device's default pool is left untouched). */
typedef struct lf_allocator {
    void *ctx;
    void *(*alloc)(void *ctx, size_t bytes, lf_stream_t s);
    void (*free)(void *ctx, void *ptr, size_t bytes, lf_stream_t s);
} lf_allocator;

/* CELL composition parameters (section 4, section 5).
 *   use_cell            1: CELL (section 4); 0: keep CSR and run Alg. 1
 *                       (the "fixed format" of section 5.1).
 *   n_parts             P >= 1 column partitions; partition p holds columns
 *                       [p*S, min(p*S+S, n_cols)), S = ceil(n_cols/P)
 *                       ("evenly divides the columns", R3).
 *   max_width_log2[p]   e_p: partition p's maximum bucket width W_p = 2^e_p
 *                       (P:L840-846); rows longer than W_p are folded into
 *                       ceil(l/W_p) rows of the max bucket (R4).
 *   block_nnz_log2[p]   k_p >= e_p: every block holds 2^k_p slots, i.e.
 *                       2^(k_p - t) rows of bucket t (R2).
 * Entries beyond n_parts are ignored. */
typedef struct lf_cell_params {
    int32_t use_cell;
    int32_t n_parts;
    int8_t max_width_log2[LF_MAX_PARTS];
    int8_t block_nnz_log2[LF_MAX_PARTS];
} lf_cell_params;

/* Options of lf_cell_configure.
 *   max_parts         upper bound on P (<= LF_MAX_PARTS; 0 = LF_MAX_PARTS).
 *   block_mult_log2   k_p = e_p + block_mult_log2 ("one or multiple times
 *                     the maximum bucket width").
 *   force_parts       > 0: use this P instead of the predictor (section 5.2).
 *   force_width_log2  >= 0: skip Algorithm 3 and use this e_p for every
 *                     non-empty partition (clamped to its longest segment).
 *   force_format      0: predictor decides use_cell; 1: force CELL; 2: force CSR. */
typedef struct lf_configure_opts {
    int32_t max_parts;
    int32_t block_mult_log2;
    int32_t force_parts;
    int32_t force_width_log2;
    int32_t force_format;
} lf_configure_opts;

/* Statistics lf_cell_configure computes on the GPU, returned for inspection.
 * features: Table 2 -- n_rows, n_cols, nnz, mean, min, max and
 *   population std of the row lengths; features[7] = J (Table 3).
 * For every partition p < n_parts and natural bucket t = ceil_log2(l) of a
 * row segment of length l >= 1 (bucket rule P:L494-497, R1):
 *   H[p][t]    segments with ceil_log2(l) == t
 *   F[p][t]    sum over segments with ceil_log2(l) >= t of ceil(l / 2^t)
 *   Unat[p][t] distinct columns of the segments with ceil_log2(l) == t
 *   Utop[p][t] distinct columns of the segments with ceil_log2(l) >= t
 *   max_log2[p] ceil_log2 of the longest segment (-1: empty partition)
 *   cost[p][e] eq. 7 (R10) summed over the partition's buckets for
 *              max width 2^e, e = 0..max_log2[p]  (-1 elsewhere)
 *   chosen_log2[p] the e_p Algorithm 3 returned (R8). */
typedef struct lf_configure_stats {
    double features[8];
    int32_t n_parts;
    int32_t max_log2[LF_MAX_PARTS];
    int32_t chosen_log2[LF_MAX_PARTS];
    int64_t H[LF_MAX_PARTS][32];
    int64_t F[LF_MAX_PARTS][32];
    int64_t Unat[LF_MAX_PARTS][32];
    int64_t Utop[LF_MAX_PARTS][32];
    int64_t cost[LF_MAX_PARTS][32];
    double group_union_ratio; /* sampled: distinct columns / nonzeros of groups of 4 consecutive rows */
    int32_t spmm_grouped;     /* 1: lf_cell_build given these stats makes lf_spmm take the grouped path */
    int32_t spmm_tc;          /* 1: ... the tcgen05 windowed path (32 <= J <= 128) */
    double window_span_mean;  /* sampled groups of 128 consecutive rows: mean span (max - min column + 1) */
    double window_over_frac;  /* ... fraction of sampled groups whose span exceeds 256 B rows */
} lf_configure_stats;

/* One CELL bucket (Fig. 4).  Buckets are stored
 * partition-major, ascending width, empty buckets omitted (R7). */
typedef struct lf_bucket {
    int32_t part;           /* partition p                                  */
    int32_t width_log2;     /* t: bucket width W = 2^t                      */
    int32_t rows_per_block; /* 2^(k_p - t)                                  */
    int32_t pad_;
    int64_t n_rows;         /* CELL rows holding data (folded rows counted) */
    int64_t n_rows_pad;     /* rounded up to a multiple of rows_per_block   */
    int64_t row_off;        /* first CELL row of the bucket in row_ind      */
    int64_t slot_off;       /* first slot of the bucket in col_ind / val    */
} lf_bucket;

/* Read-only view of a built handle.  Layout (R1-R7): CELL row r of bucket b
 * is row_ind[b.row_off + q]; its slot w is col_ind/val[b.slot_off + q*W + w]
 * ("[i * W + j]").  row_ind = source row of A, or -1 for a
 * block-padding row (Fig. 4's "*", R5); padding slots hold col_ind = -1,
 * val = +0.0f.  A folded row occupies consecutive CELL rows (R4, R6). */
typedef struct lf_cell_arrays {
    int64_t n_rows;      /* I of A */
    int64_t n_cols;      /* K of A */
    int64_t nnz;
    int64_t n_cell_rows; /* total CELL rows, padding included */
    int64_t n_slots;     /* total slots, padding included     */
    int32_t n_buckets;
    int32_t pad_;
    const int32_t *row_ind; /* (device) [n_cell_rows] */
    const int32_t *col_ind; /* (device) [n_slots]     */
    const float *val;       /* (device) [n_slots]     */
    const lf_bucket *buckets; /* (host) [n_buckets], owned by the handle */
    lf_cell_params params;
} lf_cell_arrays;

typedef struct lf_cell lf_cell; /* opaque handle */

/* Automatic composition (section 5, Fig. 2): computes the
 * Table 2 features on the GPU, decides use_cell and P with lf_predict
 * (sections 5.1-5.2) unless both are forced, then computes the per-partition
 * statistics above and for each partition runs Algorithm 3 over eq. 7
 * (section 5.3) to pick e_p; k_p = e_p + block_mult_log2.
 *   A      (host struct of device pointers)   J >= 1   opts may be NULL
 *   out    (host) receives the parameters     stats (host) may be NULL
 * The statistics pass also yields the features, so with the predictor on
 * and nnz <= 2^25 it runs once for P = 1 before the prediction and again
 * only if another P is predicted; larger matrices read the features from
 * row_ptr first.  When the fixed CSR format is chosen (use_cell = 0) no
 * CELL statistics are computed (stats: features only, tables zero).
 * Synchronises stream s once or twice (small device-to-host copies).
 * Errors: LF_ERR_INVALID_ARG for bad sizes / pointers / options. */
LF_API lf_status lf_cell_configure(const lf_csr *A, int32_t J, const lf_configure_opts *opts, lf_cell_params *out,
                            lf_configure_stats *stats, lf_stream_t s);

/* LiteForm's predictors (sections 5.1-5.2), host only: from the
 * Table 2/3 features -- features[8] = n_rows, n_cols,
 * nnz, mean, min, max and population std of the row lengths, J, exactly as
 * lf_configure_stats.features -- decide
 *   *use_cell  1: CELL (Random Forest "CELL >= 1.1x faster than CSR",
 *              P:L676-678); 0: the fixed-format CSR kernel (lf_csr_spmm)
 *   *n_parts   column partitions P in {1, 2, 4, 8}, halved
 *              until <= max_parts (0 = LF_MAX_PARTS).
 * The forests were trained on B200 timings (scripts/train_predictor.py,
 * profiles/r1_predictor.md); the paper ships no weights.
 * Deterministic, no allocation, thread-safe.
 * Errors: LF_ERR_INVALID_ARG (NULL pointer, negative / non-finite feature,
 *         max_parts outside [0, LF_MAX_PARTS]). */
LF_API lf_status lf_predict(const double features[8], int32_t max_parts, int32_t *use_cell, int32_t *n_parts);

/* CSR -> CELL conversion on the GPU (section 4; canonical layout R1-R7; the
 * output is bit-identical to the oracle's).  Allocates the handle's arrays
 * (one pool) through al (NULL = the private pool below); the temporary scratch of
 * the conversion comes from the library's private stream-ordered pool on s.
 *   stats   (host, may be NULL) the statistics lf_cell_configure returned for
 *           the SAME A with params->n_parts partitions: the bucket sizes follow
 *           from them (bucket t < e_p holds H[p][t] rows, the max bucket
 *           F[p][e_p]), so the build enqueues everything asynchronously with
 *           no host synchronisation.  NULL: the sizes are counted on the GPU
 *           and s is synchronised once.  stats->spmm_tc = 1 makes the
 *           handle's lf_spmm take the tcgen05 windowed path (the per-group
 *           B-row windows are built here), else stats->spmm_grouped = 1 the
 *           grouped path (LF_TC=0/1 and LF_GROUPED=0/1 in the environment
 *           override them; LF_TC=1 at build time builds the windows).
 * The handle may be used on s immediately.
 * Errors: LF_ERR_INVALID_ARG (sizes, e_p > k_p, P out of range; stats for a
 *         different P, for a matrix with other n_rows / n_cols / nnz, or with
 *         tables that do not cover A: sum_p F[p][0] != nnz, e.g. the stats of
 *         a configure that chose the CSR format; with LF_VALIDATE=1 also bucket
 *         sizes counted on the GPU that differ from the stats), LF_ERR_INDEX_OVERFLOW (n_rows >= 2^28 or K > 2^31-1),
 *         LF_ERR_NO_MEMORY, LF_ERR_CUDA, LF_ERR_UNSORTED_CSR (LF_VALIDATE=1). */
LF_API lf_status lf_cell_build(const lf_csr *A, const lf_cell_params *params, const lf_configure_stats *stats,
                               const lf_allocator *al, lf_stream_t s, lf_cell **out);

/* C = A . B (eq. 3-4; Alg. 2 over every block),
 * overwriting C (beta = 0; rows of A with no entries become +0.0, R13).
 *   B (device) K x J, ldb >= J;   C (device) I x J, ldc >= J;   J >= 0.
 * The vectorised path needs J % 4 == 0 and 16-byte aligned B, C, ldb*4,
 * ldc*4; other shapes take the scalar path.  Asynchronous on s; no host
 * synchronisation.  The handle's arrays are immutable: concurrent calls on
 * different streams (and host threads) with different C are safe -- the
 * work-queue counter slot a launch uses is fenced behind that slot's previous
 * launch when it ran on another stream.  B must not alias C.
 * CUDA graphs: calls on the handle's build stream launch kernels only and can
 * be captured into a graph (a replay reuses the counter slots of the capture;
 * replays of one graph must not overlap).  Calls on other streams record and
 * wait on events of the build stream, so capture them only with the build
 * stream in the same capture. */
LF_API lf_status lf_spmm(const lf_cell *h, const float *B, int64_t ldb, int32_t J, float *C, int64_t ldc,
                  lf_stream_t s);

/* Options of lf_spmm_ex: the FUSED ROW EXCHANGE of row-sharded multi-GPU SpMM
 * (SURVEY 8(e), 8(f) NEXT-3).  With n_dst > 0 the kernels write every C row
 * i of this handle's A straight from registers into each destination C,
 * dst[d] + (row_base + i) * ldc -- the rank's own full C and its peers' C
 * buffers mapped over NVLink (peer / symmetric memory) -- instead of C: the
 * transfer overlaps the compute, and no separate all-gather follows.
 *   n_dst     0 (plain lf_spmm) or 1..LF_MAX_DST
 *   dst       (host) array of n_dst (device) pointers, each the base of a full
 *             I_total x ldc C; read during the call (copied into the launch's
 *             slot of the handle), may be freed when it returns
 *   row_base  first row of this handle's rows in every destination
 * The caller orders reads of a peer's rows after that peer's launch (e.g. a
 * barrier); rows written with red.add (several CELL rows per C row) are
 * pre-zeroed in every destination by the same launch. */
#define LF_MAX_DST 8
typedef struct lf_spmm_opts {
    int32_t n_dst;
    int32_t pad_;
    float *const *dst;
    int64_t row_base;
} lf_spmm_opts;

/* lf_spmm with options (opts may be NULL = lf_spmm).  C may be NULL when
 * n_dst > 0.  Errors as lf_spmm, plus LF_ERR_INVALID_ARG (n_dst outside
 * [0, LF_MAX_DST], NULL dst or destination, row_base < 0) and
 * LF_ERR_UNSUPPORTED (n_dst > 0 on a handle built with use_cell = 0). */
LF_API lf_status lf_spmm_ex(const lf_cell *h, const float *B, int64_t ldb, int32_t J, float *C, int64_t ldc,
                            const lf_spmm_opts *opts, lf_stream_t s);

/* Name of the SpMM kernel family lf_spmm runs for this handle at this J
 * with 16-byte aligned B / C and ldb = ldc = J (e.g. "cell_spmm_kernel",
 * "cell_spmm_grouped_kernel", "cell_spmm_tc_kernel", "csr_spmm_kernel";
 * "" for a NULL handle, J <= 0 or an empty matrix).  Host only; the string is
 * static.  For reports and tests: it launches nothing. */
LF_API const char *lf_spmm_kernel_name(const lf_cell *h, int32_t J);

/* Algorithm 1 on the GPU directly from CSR: the fixed-format
 * path the predictor can choose instead of CELL.  Same conventions as lf_spmm. */
LF_API lf_status lf_csr_spmm(const lf_csr *A, const float *B, int64_t ldb, int32_t J, float *C, int64_t ldc,
                      lf_stream_t s);

/* Fills *out with the handle's arrays (no copy; valid until destroy). */
LF_API lf_status lf_cell_view(const lf_cell *h, lf_cell_arrays *out);

/* Frees the handle and its arrays, stream-ordered on the build stream after
 * every lf_spmm of the handle on any stream (each other stream's last launch
 * is recorded by lf_spmm and waited for here); returns without blocking.
 * The build stream must still exist.  Not thread-safe against concurrent
 * lf_spmm calls on the same handle. */
LF_API lf_status lf_cell_destroy(lf_cell *h);

LF_API const char *lf_status_string(lf_status st);
LF_API const char *lf_last_error_detail(void);
LF_API int32_t lf_abi_version(void);

#ifdef __cplusplus
}
#endif

#endif /* LITEFORM_H */
