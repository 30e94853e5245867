/*
 * spmv.h -- C ABI of libspmv: six-format SpMV y <- alpha*A*x + beta*y, the
 * CSR -> format converters, per-matrix sparsity features and the multi-GPU row
 * partition, hand-written for B200 (sm_100a).
 *
 * Paper: Nisa, Siegel, Sukumaran Rajam, Vishnu, Sadayappan, "Effective Machine
 * Learning Based Format Selection and Performance Modeling for SpMV on GPUs",
 * IPDPSW 2018.  PAPER.md:<n> = line n of the text extraction; A<n> = reading n of
 * the ambiguity register (restated in DESIGN.md §3).
 *
 * General rules
 *  - Plain C types only.  "device" pointers are CUDA device memory on the ctx's
 *    device; "host" pointers are ordinary host memory.
 *  - Every call returns an spmv_status; nothing aborts and no C++ exception crosses
 *    the ABI.  On error, spmv_last_error() returns a thread-local detail string.
 *  - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *    All device work is stream-ordered on it.
 *  - Inputs are BORROWED for the duration of the call (stream-ordered) and never
 *    retained, unless stated.  A handle OWNS every device array it allocates.
 *  - No CPU fallback exists: without a usable sm_100 device every entry point
 *    that would touch the device returns SPMV_ERR_UNSUPPORTED or SPMV_ERR_CUDA.
 */
#ifndef SPMV_H
#define SPMV_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* exported symbols stay visible when the library is built with -fvisibility=hidden */
#if defined(__GNUC__)
#pragma GCC visibility push(default)
#endif

#define SPMV_ABI_VERSION 3

typedef enum {
    SPMV_OK = 0,
    SPMV_ERR_INVALID_ARG = 1,   /* null/inconsistent argument, x/y overlap, bad id   */
    SPMV_ERR_NOT_CANONICAL = 2, /* row_ptr not monotone / not [0..nnz], column out of
                                   range, unsorted or duplicate column in a row (A15) */
    SPMV_ERR_SIZE = 3,          /* ELL/HYB slots exceed the size guard (A4), or an
                                   index does not fit its type                        */
    SPMV_ERR_NO_MEMORY = 4,     /* allocator returned NULL                            */
    SPMV_ERR_CUDA = 5,          /* a CUDA runtime call or kernel launch failed        */
    SPMV_ERR_UNSUPPORTED = 6    /* device is not sm_100, or dtype/format mismatch     */
} spmv_status;

/* The six formats of the study, in the paper's Fig. 3 order,
 * plus the CSR-scalar kernel variant (a variant, not a label, A5). */
typedef enum {
    SPMV_COO = 0,        /* PAPER.md:89  (§II-A.1) */
    SPMV_ELL = 1,        /* PAPER.md:93  (§II-A.3) */
    SPMV_CSR = 2,        /* PAPER.md:91  (§II-A.2), CSR-vector kernel (A5) */
    SPMV_HYB = 3,        /* PAPER.md:95  (§II-A.4) */
    SPMV_MERGE = 4,      /* PAPER.md:103 (§II-A.6) */
    SPMV_CSR5 = 5,       /* PAPER.md:97-101 (§II-A.5) */
    SPMV_CSR_SCALAR = 6  /* PAPER.md:91, one thread per row */
} spmv_format;

typedef enum { SPMV_F32 = 0, SPMV_F64 = 1 } spmv_dtype;   /* value type (fp32 accumulates in fp64, A13) */
typedef enum { SPMV_I32 = 0, SPMV_I64 = 1 } spmv_itype;   /* row_ptr type (A17) */

/* Canonical CSR matrix, all pointers DEVICE, borrowed.
 * row_ptr[n_rows+1] (ptr_type), col_idx[nnz] int32, vals[nnz] (dtype).
 * Canonical = row_ptr[0]=0, monotone, row_ptr[n_rows]=nnz, columns strictly
 * increasing within a row and in [0, n_cols) (A15). */
typedef struct {
    int64_t n_rows, n_cols, nnz;
    spmv_itype ptr_type;
    const void *row_ptr;
    const int32_t *col_idx;
    const void *vals;
    spmv_dtype dtype;
} spmv_csr;

/* Device allocator used for every allocation of a ctx (handles, scratch).
 * alloc(bytes, device, stream, user) returns a device pointer or NULL;
 * free(ptr, bytes, device, stream, user) is stream-ordered.
 * NULL allocator in spmv_init => cudaMallocAsync / cudaFreeAsync. */
typedef struct {
    void *(*alloc)(size_t bytes, int device, void *stream, void *user);
    void (*free)(void *ptr, size_t bytes, int device, void *stream, void *user);
    void *user;
} spmv_allocator;

typedef struct spmv_ctx spmv_ctx;
typedef struct spmv_handle spmv_handle;

/* ---- context ------------------------------------------------------------- */

/* Bind to `device` (must be compute capability 10.0, else SPMV_ERR_UNSUPPORTED).
 * The allocator struct is copied.  *out receives a ctx owned by the caller. */
spmv_status spmv_init(int device, const spmv_allocator *alloc, spmv_ctx **out);
/* Release the ctx (handles created from it must be destroyed first). */
spmv_status spmv_finalize(spmv_ctx *ctx);
/* Device SM count and L2 size the library sized its grids for (host outputs). */
spmv_status spmv_device_info(const spmv_ctx *ctx, int *sm_count, int64_t *l2_bytes);

/* ---- features (Table II; §IV-A) ---------- */

/* The 17 features of the paper under the names of its Figs 4-5,
 * read per A8 (nnz_frac in percent, population sigma, a block = maximal run of
 * consecutive columns within a row, nnzb_* over all rows, snzb_* over all blocks),
 * computed from exact integer sums by the fixed fp64 formulas of A9; plus the
 * north_star extras (ELL padding ratio, HYB split widths). */
typedef struct {
    int64_t n_rows, n_cols, nnz_tot;
    double nnz_mu, nnz_frac;
    int64_t nnz_max;  double nnz_sigma;
    double nnzb_mu, nnzb_sigma, snzb_mu, snzb_sigma;
    int64_t nnzb_tot, nnzb_min, nnzb_max, snzb_min, snzb_max, nnz_min;
    int64_t ell_width, ell_slots;  double ell_pad_frac;
    int64_t hyb_width, hyb_coo_nnz, hyb_width_floor, hyb_width_cusp;  /* PAPER.md:95, A2 */
    int64_t n_empty_rows;
    uint64_t sum_len2, sum_nnzb2, sum_snzb2;              /* exact sums behind the sigmas */
} spmv_features_t;

/* One kernel launch reads row_ptr and col_idx once each (vals are not read; DESIGN.md
 * §4 "Features"), then one 112-byte device->host readback: BLOCKS on `stream`.  No
 * allocation after the ctx's first call (device state is ctx-owned and reset by the
 * kernel; concurrent callers on one ctx are serialised).  Returns
 * SPMV_ERR_NOT_CANONICAL for a non-canonical matrix (out_host is then unspecified). */
spmv_status spmv_features(spmv_ctx *ctx, const spmv_csr *A, void *stream,
                          spmv_features_t *out_host);

/* ---- conversion ------------------------------------------------------------ */

typedef struct {
    int hyb_rule;          /* 0 = ceil(nnz/n_rows) (default; "nnz_mu, which we
                              use", A2), 1 = floor, 2 = the max(4096, rows/3)-style rule   */
    int64_t hyb_width;     /* >= 0 overrides hyb_rule; < 0 = use the rule                 */
    int csr5_sigma;        /* 0 = A6 rule (B200 revision): 4 if ceil(nnz_mu) <= 3, 8 if it is 4,
                              12 above; else 4, 8, 12 or 16                                 */
    int merge_items;       /* merge-path items per CTA (0 = default); recorded in info     */
    int vector_width;      /* CSR-vector lanes per row (0 = A5 rule), power of two 1..32  */
    size_t max_bytes;      /* ELL/HYB guard (0 = min(1/2 free memory, max(8x the CSR bytes,
                              64 MiB)))                                                    */
    int alias_input;       /* 1 = COO/CSR handles reference the caller's col/vals (caller
                              keeps them alive and unchanged); MERGE/CSR5/ELL/HYB copy,
                              and COO copies unless both arrays are 32-byte aligned        */
    int index64;           /* 1 = int64 row pointers/offsets inside the handle even when
                              nnz <= INT32_MAX (exercises the > 2^31-nonzero path, A17)   */
    int64_t csr_chunk;     /* CSR long-row split (A25): rows longer than 2*csr_chunk are cut
                              into csr_chunk-nonzero chunks, each reduced by its own warp and
                              added by the fix-up; 0 = default 512, < 0 = never split     */
    int64_t hot_x;         /* A30 hot x columns: 0 = auto (the columns of the highest degrees,
                              at most L2/2 worth of x entries, packed densely every run, when
                              x exceeds twice the L2 and they hold >= 1/4 of the nonzeros),
                              > 0 = always, at most this many columns, < 0 = never.  Not for
                              handles that alias the input column array, nor CSR_SCALAR.  */
    const spmv_features_t *features;
                           /* optional HOST pointer: the spmv_features() result of THIS matrix
                              (same arrays, unchanged since).  The conversion then reuses it
                              (nnz_max, hyb_width_cusp) and skips its own feature/validation
                              pass; dimensions must match A (else SPMV_ERR_INVALID_ARG).
                              Features of another matrix are undefined behaviour.  NULL =
                              validate here (one feature pass, one readback).              */
} spmv_convert_opts;

/* Fill `opts` with the defaults (all rules as above). */
void spmv_convert_opts_default(spmv_convert_opts *opts);

/* Build a handle holding A in format `fmt` (CSR -> COO/ELL/HYB/merge-partition/
 * CSR5-tile descriptors, layouts DESIGN.md §4).  Validates A (the
 * feature pass's canonical check), does one blocking size readback, checks the size
 * guard (ELL/HYB: SPMV_ERR_SIZE, A4), allocates through the ctx allocator on
 * `stream`, launches the conversion on `stream` and returns.  opts may be NULL. */
spmv_status spmv_convert(spmv_ctx *ctx, spmv_format fmt, const spmv_csr *A,
                         const spmv_convert_opts *opts, void *stream, spmv_handle **out);

/* y <- alpha*A*x + beta*y (BLAS conventions, A14): beta == 0 => y is write-only;
 * A handle with hot columns (A30) first packs x[hot] into its own buffer (one small
 * kernel), so one handle must not run concurrently on two streams (as for the carries); 
 * alpha == 0 => A is not read.  alpha/beta are HOST scalars of the handle's dtype
 * (float* or double*), copied at call time.  x (n_cols) and y (n_rows) are DEVICE
 * arrays of the handle's dtype; they must not overlap (SPMV_ERR_INVALID_ARG).
 * Fully asynchronous on `stream` (CUDA-graph capturable); a handle runs on one
 * stream at a time (it owns per-run carry scratch).  Summation is deterministic:
 * fixed-order segmented sums, no floating-point atomics. */
spmv_status spmv_run(spmv_handle *h, const void *alpha, const void *x,
                     const void *beta, void *y, void *stream);

/* End-to-end variant for HOST x/y (pageable or pinned): copies x (and y when
 * beta != 0) host->device into handle-owned buffers, runs, copies y back, and
 * synchronizes `stream` before returning. */
spmv_status spmv_run_host(spmv_handle *h, const void *alpha, const void *x_host,
                          const void *beta, void *y_host, void *stream);

/* Label-collection variant of spmv_run_host (every format of a
 * matrix is timed on the same x, §IV-B): hs[0..k) are k >= 1 distinct handles of ONE
 * matrix (same ctx, dtype, n_rows and n_cols; any formats).  x_host (n_cols) and
 * y_in_host (n_rows; not read when beta == 0) are copied host->device ONCE; then for
 * each i, y_i = alpha*A_i*x + beta*y_in is computed from a device copy of y_in and
 * copied back into y_out_host[i] (n_rows values), the copy of result i overlapping run
 * i+1 (a second, library-created stream).  Host buffers: pinned or pageable, owned by
 * the caller, not retained.  Device buffers: x and y_in owned by hs[0], each result by
 * its handle (allocated on first use, freed by spmv_destroy).  Synchronizes before
 * returning; the handles must not be running elsewhere.  SPMV_ERR_INVALID_ARG for
 * k < 1, NULL pointers, a repeated handle or handles of different shapes. */
spmv_status spmv_run_host_multi(spmv_handle *const *hs, int k, const void *alpha, const void *x_host,
                                const void *beta, const void *y_in_host, void *const *y_out_host,
                                void *stream);

/* Number of kernel launches one spmv_run issues for this handle (host output). */
spmv_status spmv_run_launches(const spmv_handle *h, int *launches);

typedef struct {
    spmv_format format;
    spmv_dtype dtype;
    spmv_itype ptr_type;            /* index type used inside the handle */
    int64_t n_rows, n_cols, nnz;
    int64_t ell_width, ell_ld;      /* ELL / HYB-ELL part */
    int64_t hyb_coo_nnz;            /* HYB COO part */
    int64_t csr5_sigma, csr5_tiles, csr5_map_len;
    int64_t merge_items, merge_tiles;
    int64_t vector_width;
    int64_t csr_chunks;             /* CSR long-row chunks (A25); 0 = none */
    int64_t hot_cols;               /* A30: hot x columns packed per run; 0 = none */
    size_t device_bytes;            /* bytes owned by the handle */
    size_t bytes_per_run;           /* algorithmic bytes of one run with beta != 0
                                       (format's own storage + x + y read + y write),
                                       DESIGN.md §6 */
    size_t bytes_per_run_beta0;     /* same with beta == 0 (y not read) */
} spmv_handle_info;

spmv_status spmv_info(const spmv_handle *h, spmv_handle_info *out_host);

/* Arrays a handle can export for bit-exact tests (layouts: DESIGN.md §4). */
typedef enum {
    SPMV_ARR_ROW_PTR = 0,    /* CSR/MERGE/CSR5/CSR_SCALAR row_ptr (ptr_type)          */
    SPMV_ARR_COL = 1,        /* CSR/MERGE/COO col (int32); CSR5: lane-interleaved col */
    SPMV_ARR_VAL = 2,        /* as above, values (dtype)                               */
    SPMV_ARR_COO_ROW = 3,    /* COO / HYB-COO row (int32)                              */
    SPMV_ARR_ELL_COL = 4,    /* ELL / HYB-ELL, K*ld int32, col = -1 padding            */
    SPMV_ARR_ELL_VAL = 5,    /* ELL / HYB-ELL, K*ld dtype, +0.0 padding                */
    SPMV_ARR_HYB_COO_COL = 6,
    SPMV_ARR_HYB_COO_VAL = 7,
    SPMV_ARR_MERGE_COORD_ROW = 8,   /* int64 [tiles+1] */
    SPMV_ARR_MERGE_COORD_NZ = 9,    /* int64 [tiles+1] */
    SPMV_ARR_CSR5_TILE_PTR = 10,    /* int64 [tiles+1] */
    SPMV_ARR_CSR5_ROW_LO = 11,      /* int64 [tiles+1] */
    SPMV_ARR_CSR5_TILE_DESC = 12,   /* uint32 [tiles*32] */
    SPMV_ARR_CSR5_MAP_OFF = 13,     /* int64 [tiles] (-1 = no empty row in range) */
    SPMV_ARR_CSR5_SEG_MAP = 14,     /* int64 [map_len] */
    SPMV_ARR_CSR_CHUNK_ROW = 15,    /* CSR: int64 [chunks], row of each long-row chunk (A25) */
    SPMV_ARR_CSR_CHUNK_LO = 16,     /* CSR: int64 [chunks], first nonzero of each chunk      */
    SPMV_ARR_MERGE_TILE_CLASS = 17, /* MERGE: uint8 [tiles], 1 = row-sum tile (A28): fewer than
                                       64 row ends in the tile and every row's part inside the
                                       tile (the open row included) <= 32 nonzeros; else 0     */
    SPMV_ARR_MERGE_TILE_ORDER = 18, /* MERGE: int32 [tiles], the tile ids stably partitioned by
                                       class: class-1 tiles first (ascending), then class 0    */
    SPMV_ARR_HOT_COLS = 19          /* any format: int32 [n_hot], the hot columns (A30), ascending;
                                       exported column arrays are always decoded back to column
                                       indices                                                 */
} spmv_array_id;

/* Copy array `id` of the handle to host memory (blocking on `stream`).
 * *written = bytes of the array; SPMV_ERR_INVALID_ARG if the handle has no such
 * array or cap < size (then *written still reports the size). */
spmv_status spmv_export(const spmv_handle *h, spmv_array_id id, void *host_dst,
                        size_t cap, size_t *written, void *stream);

/* Free the handle's arrays (stream-ordered on `stream`) and the handle. */
spmv_status spmv_destroy(spmv_handle *h, void *stream);

/* ---- multi-GPU row partition (north_star) --------------------- */

/* nnz-balanced merge-path row splits: splits[k] = row coordinate of the merge path
 * of A's row ends with its nonzeros at diagonal floor(k*(n_rows+nnz)/nparts),
 * k = 0..nparts (row-aligned; a straddling row goes to the later part).
 * row_splits_host[nparts+1] is HOST output.  Blocks on `stream`. */
spmv_status spmv_partition(spmv_ctx *ctx, const spmv_csr *A, int nparts, void *stream,
                           int64_t *row_splits_host);

/* Size of shard `part`: rows = splits[part+1]-splits[part], nnz of those rows and the
 * gathered-x slot size S = max part rows (all host outputs; blocks on `stream`). */
spmv_status spmv_slice_size(spmv_ctx *ctx, const spmv_csr *A, const int64_t *row_splits_host,
                            int nparts, int part, void *stream,
                            int64_t *rows, int64_t *nnz, int64_t *slot);

/* Shard `part` of a SQUARE matrix into caller-allocated DEVICE arrays:
 * row_ptr_out[rows+1] int32 (rebased to 0; SPMV_ERR_SIZE if shard nnz > INT32_MAX),
 * col_out[nnz] int32 remapped to the gathered-x slot owner(j)*S + (j - splits[owner]),
 * vals_out[nnz] (A's dtype).  Asynchronous on `stream`. */
spmv_status spmv_slice_remap(spmv_ctx *ctx, const spmv_csr *A, const int64_t *row_splits_host,
                             int nparts, int part, void *stream,
                             int32_t *row_ptr_out, int32_t *col_out, void *vals_out);

/* Compressed exchange: only columns that some row of A references are
 * exchanged.  colmap_out[j] (DEVICE, int32[n_cols]) = owner(j)*S' + (number of referenced
 * columns of owner(j) before j) for a referenced column j, -1 for a column no row uses;
 * S' = max over parts of referenced columns per part (host output *slot).  Square A.
 * Identical on every rank for the same A.  Blocks on `stream` (one readback). */
spmv_status spmv_partition_colmap(spmv_ctx *ctx, const spmv_csr *A, const int64_t *row_splits_host,
                                  int nparts, void *stream, int32_t *colmap_out, int64_t *slot);

/* Shard `part` like spmv_slice_remap, with columns mapped through `colmap` (DEVICE,
 * from spmv_partition_colmap) instead of the dense slot layout.  Asynchronous. */
spmv_status spmv_slice_remap_colmap(spmv_ctx *ctx, const spmv_csr *A, const int64_t *row_splits_host,
                                    int nparts, int part, const int32_t *colmap, void *stream,
                                    int32_t *row_ptr_out, int32_t *col_out, void *vals_out);

/* Local positions of part `part`'s referenced columns, in order: idx_out[q] = j - splits[part]
 * for the q-th referenced column j of the part (DEVICE int32 output, capacity = part rows);
 * `slot` is S' from spmv_partition_colmap; *count (host) = number written.  Blocks on `stream`. */
spmv_status spmv_colmap_pack_index(spmv_ctx *ctx, const int32_t *colmap, const int64_t *row_splits_host,
                                   int nparts, int part, int64_t slot, void *stream, int32_t *idx_out,
                                   int64_t *count);

/* Overlap of the exchange with compute: shard `part` split by column
 * ownership.  which = 0: the OWN block -- columns in [splits[part], splits[part+1]), remapped
 * to j - splits[part] (they index the rank's own x slice, available before the exchange);
 * which = 1: the FOREIGN block -- all other columns, remapped to gathered-x slots (dense layout
 * when colmap == NULL, else through colmap with slot layout of spmv_partition_colmap).
 * Both blocks cover the same rows [splits[part], splits[part+1]).
 * row_ptr_out[rows+1] (DEVICE int32) is always written and *nnz_out (host) receives the
 * block's nonzero count; col_out/vals_out (DEVICE) may be NULL for this sizing call, else
 * they receive the block.  Blocks on `stream`. */
spmv_status spmv_slice_split(spmv_ctx *ctx, const spmv_csr *A, const int64_t *row_splits_host, int nparts,
                             int part, const int32_t *colmap, int which, void *stream, int32_t *row_ptr_out,
                             int32_t *col_out, void *vals_out, int64_t *nnz_out);

/* Halo exchange of a row partition: the receiver `part`
 * needs, from every other owner o, exactly the x entries of o's rows (= columns, square A)
 * that part's rows reference.  colmap_out[j] (DEVICE int32[n_cols]) = owner(j)*S +
 * (number of such columns of owner(j) below j) for every column j referenced by a row of
 * `part` and owned by another part, -1 otherwise, with S = max(1, max_o counts[o]) the
 * receiver's slot (host output *slot); counts_host[nparts] (HOST) receives the per-owner
 * counts (counts_host[part] = 0).  The receive buffer of `part` holds owner o's entries at
 * [o*S, o*S + counts[o]).  The sender's pack list for this receiver is
 * spmv_colmap_pack_index(colmap_out, ..., sender, S).  Identical on every rank.  Blocks on
 * `stream` (one readback). */
spmv_status spmv_halo_colmap(spmv_ctx *ctx, const spmv_csr *A, const int64_t *row_splits_host, int nparts,
                             int part, void *stream, int32_t *colmap_out, int64_t *counts_host, int64_t *slot);

/* dst[q] = src[idx[q]] for q < n (DEVICE arrays of `dtype`): the per-step packing of a
 * rank's x slice into its compressed slot.  Asynchronous. */
spmv_status spmv_gather(spmv_ctx *ctx, spmv_dtype dtype, const void *src, const int32_t *idx, int64_t n,
                        void *dst, void *stream);

/* dst[idx[q]] = src[q] for q < n (DEVICE arrays of `dtype`; the idx[q] distinct, else which
 * write lands is unspecified): the inverse of spmv_gather, used to put a compressed-row
 * block's results back into the rank's y slice (A33).  Asynchronous. */
spmv_status spmv_scatter(spmv_ctx *ctx, spmv_dtype dtype, const void *src, const int32_t *idx, int64_t n,
                         void *dst, void *stream);

/* Compressed rows of A (A33; DESIGN.md §7 -- a rank's foreign-column block of a banded
 * matrix holds a few thousand non-empty rows among millions): rows_out (DEVICE int32,
 * capacity n_rows) receives the indices of A's non-empty rows in increasing order and
 * rp_out (DEVICE, A's ptr_type, capacity n_rows + 1) their row starts followed by nnz, so
 * that (rp_out, A.col_idx, A.val) is the CSR of those rows; *count_host = their number.
 * Buffers owned by the caller.  Blocks on `stream` (one readback).  SPMV_ERR_INVALID_ARG
 * for NULL outputs or more than 2^31 - 1 rows. */
spmv_status spmv_compress_rows(spmv_ctx *ctx, const spmv_csr *A, void *stream, int32_t *rows_out,
                               void *rp_out, int64_t *count_host);

/* ---- diagnostics ----------------------------------------------------------- */
const char *spmv_status_str(spmv_status s);
const char *spmv_last_error(void);
int spmv_abi_version(void);

#if defined(__GNUC__)
#pragma GCC visibility pop
#endif

#ifdef __cplusplus
}
#endif
#endif /* SPMV_H */
