/*
 * oracle.h -- CPU ORACLE for the six-format SpMV study (TEST INFRASTRUCTURE ONLY).
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load this library.  The product path
 * (paper_conf_ipps_nisassvs18_b200/, libspmv.so) never includes, links or
 * calls anything here, and this file includes nothing from the product.
 *
 * Paper: Nisa et al., "Effective Machine Learning Based Format Selection and
 * Performance Modeling for SpMV on GPUs", IPDPSW 2018 (/root/reference/PAPER.md,
 * cited as PAPER.md:<line>).  Readings of ambiguous passages are the A1..A22
 * entries of SURVEY.md §8(c) and are listed in DESIGN.md §3.
 *
 * Conventions: every array is a host array owned by the caller.  row_ptr is
 * always int64 here (callers widen int32 row_ptrs), col is int32, values are
 * fp64 (fp32 data is passed widened, which is exact).  Functions return 0 on
 * success and a negative number on invalid input; they never abort.
 */
#ifndef SPMV_ORACLE_H
#define SPMV_ORACLE_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---- SpMV: y <- alpha*A*x + beta*y  (PAPER.md:89-103 all formats store the same A) */

/* CSR SpMV, long-double accumulation.  bound_out (nullable)
 * receives |alpha|*sum|a||x| + |beta||y_in| per row (A16).  beta == 0 => y_in
 * is not read (may be NULL); alpha == 0 => A is not read (A14). */
int ora_spmv_csr(int64_t n_rows, const int64_t *row_ptr, const int32_t *col,
                 const double *val, const double *x, double alpha, double beta,
                 const double *y_in, double *y_out, double *bound_out);

/* COO SpMV over triplets in stored order (c2.2); independent of ora_spmv_csr. */
int ora_spmv_coo(int64_t n_rows, int64_t nnz, const int32_t *row, const int32_t *col,
                 const double *val, const double *x, double alpha, double beta,
                 const double *y_in, double *y_out);

/* Canonical CSR check (A15): row_ptr[0]=0, monotone, row_ptr[n]=nnz, col strictly
 * increasing within each row and in [0,n_cols).  Returns 1 canonical, 0 not. */
int ora_is_canonical(int64_t n_rows, int64_t n_cols, int64_t nnz,
                     const int64_t *row_ptr, const int32_t *col);

/* ---- converters (layouts of SURVEY §8(a) a3-a7) */

/* COO: row_out[k] = r for k in [row_ptr[r], row_ptr[r+1]). */
int ora_csr2coo(int64_t n_rows, const int64_t *row_ptr, int32_t *row_out);

/* ELL (A3): K = max row length, ld = round_up(n_rows, 32),
 * entry (r,j) at j*ld + r, padding col=-1 val=+0.0.  Caller sizes arrays K*ld. */
int64_t ora_ell_width(int64_t n_rows, const int64_t *row_ptr);
int64_t ora_ell_ld(int64_t n_rows);
int ora_csr2ell(int64_t n_rows, const int64_t *row_ptr, const int32_t *col,
                const double *val, int64_t K, int64_t ld,
                int32_t *ell_col, double *ell_val);

/* HYB widths (A2): rule 0 = ceil(nnz/n_rows) (default, "nnz_mu, which
 * we use"), 1 = floor, 2 = the max(4096, rows/3)-style rule of [2] (A2 text). */
int64_t ora_hyb_width(int64_t n_rows, const int64_t *row_ptr, int rule);
/* Number of entries that overflow a width-Kh ELL into COO. */
int64_t ora_hyb_coo_nnz(int64_t n_rows, const int64_t *row_ptr, int64_t Kh);
/* HYB (A1): the first min(len,Kh) entries of each row go to a width-Kh
 * ELL (layout as above), the rest to a row-major COO. */
int ora_csr2hyb(int64_t n_rows, const int64_t *row_ptr, const int32_t *col,
                const double *val, int64_t Kh, int64_t ld,
                int32_t *ell_col, double *ell_val,
                int32_t *coo_row, int32_t *coo_col, double *coo_val);

/* Merge-path coordinates (A7) by a LINEAR WALK of the merge of
 * A = row ends row_ptr[1..n] with B = nnz indices 0..nnz-1, row end first on ties.
 * coord_row/coord_nz receive the coordinate at diagonal min(t*T, n_rows+nnz) for
 * t = 0..n_tiles, n_tiles = ceil((n_rows+nnz)/T). */
int64_t ora_merge_ntiles(int64_t n_rows, int64_t nnz, int64_t T);
int ora_merge_coords(int64_t n_rows, const int64_t *row_ptr, int64_t T,
                     int64_t *coord_row, int64_t *coord_nz);
/* Merge tile class (A28): cls[t] = 1 iff tile t consumes fewer than max_rows row
 * ends and no row takes more than max_len of its nonzeros (walk, as above). */
int ora_merge_class(int64_t n_rows, const int64_t *row_ptr, int64_t T,
                    int64_t max_rows, int64_t max_len, uint8_t *cls);

/* CSR long-row chunks (A25): a row with len > 2*C is reduced as
 * ceil(len/C) chunks of C nonzeros (the last one shorter), chunk j of row r starting at
 * row_ptr[r] + j*C; chunks listed by ascending row, then j.  Returns the number of
 * chunks (negative on bad input); chunk_row/chunk_lo (nullable) receive them. */
int64_t ora_compress_rows(int64_t n_rows, const int64_t *row_ptr, int64_t *rows_out, int64_t *rp_out);
int64_t ora_csr_chunks(int64_t n_rows, const int64_t *row_ptr, int64_t C,
                       int64_t *chunk_row, int64_t *chunk_lo);

/* CSR5 (encoding of SURVEY A6, restated in DESIGN.md §4.6).
 * omega = 32 lanes, sigma from ora_csr5_sigma.  n_tiles = floor(nnz/(omega*sigma)).
 * Outputs (caller-sized):
 *   tile_ptr[n_tiles+1]  row of element t*omega*sigma (n_rows if past the end)
 *   row_lo[n_tiles+1]    first row r with row_ptr[r] >= t*omega*sigma (n_rows if none)
 *   tile_desc[n_tiles*32] u32: bits 0..15 bit_flag, 16..24 y_offset, 25..29 seg_offset
 *   map_off[n_tiles]     -1, or offset into seg_map when the tile's row range holds
 *                        an empty row; seg_map[map_off+k] = row of the tile's k-th segment
 *   col_perm[nnz], val_perm[nnz]  full tiles lane-interleaved with vector width
 *                        v = 16/elem_bytes (col: 4 B; val: val_bytes), tail unchanged.
 * ora_csr5_map_len returns the seg_map length. */
int64_t ora_csr5_sigma(int64_t n_rows, int64_t nnz);
int64_t ora_csr5_map_len(int64_t n_rows, const int64_t *row_ptr, int64_t sigma);
int ora_csr5_encode(int64_t n_rows, const int64_t *row_ptr, const int32_t *col,
                    const double *val, int64_t sigma, int val_bytes,
                    int64_t *tile_ptr, int64_t *row_lo, uint32_t *tile_desc,
                    int64_t *map_off, int64_t *seg_map,
                    int32_t *col_perm, double *val_perm);
/* Decoder back to CSR from the CSR5 arrays alone (full tiles) plus, for the
 * tail, the row_ptr entries of rows starting in the tail (passed as row_ptr;
 * only entries r >= row_lo[n_tiles] are read).  Writes row_ptr_out[n_rows+1],
 * col_out[nnz], val_out[nnz].  Returns 0, or <0 if the descriptors are inconsistent. */
int ora_csr5_decode(int64_t n_rows, int64_t nnz, const int64_t *row_ptr_tail,
                    int64_t sigma, int val_bytes,
                    const int64_t *tile_ptr, const int64_t *row_lo,
                    const uint32_t *tile_desc, const int64_t *map_off,
                    const int64_t *seg_map, const int32_t *col_perm,
                    const double *val_perm,
                    int64_t *row_ptr_out, int32_t *col_out, double *val_out);

/* ---- features (Table II, §IV-A :193-209; A8, A9) */
typedef struct {
    int64_t n_rows, n_cols, nnz_tot;
    double nnz_mu, nnz_frac;                           /* set 1 */
    int64_t nnz_max;  double nnz_sigma;                /* set 2 */
    double nnzb_mu, nnzb_sigma, snzb_mu, snzb_sigma;   /* set 2 */
    int64_t nnzb_tot, nnzb_min, nnzb_max, snzb_min, snzb_max, nnz_min; /* set 3 */
    /* extras (north_star): ELL width/padding, HYB widths */
    int64_t ell_width, ell_slots; double ell_pad_frac;
    int64_t hyb_width, hyb_coo_nnz, hyb_width_floor, hyb_width_cusp;
    int64_t n_empty_rows;
    /* exact integer sums the finals are computed from (A9) */
    uint64_t sum_len2, sum_nnzb2, sum_snzb2;
} ora_features_t;

int ora_features(int64_t n_rows, int64_t n_cols, const int64_t *row_ptr,
                 const int32_t *col, ora_features_t *out);

/* ---- multi-GPU row partition: linear merge walk to each
 * diagonal floor(k*(n_rows+nnz)/P), row-aligned. splits_out[P+1]. */
int ora_partition(int64_t n_rows, const int64_t *row_ptr, int nparts, int64_t *splits_out);
/* Shard `part`: rows [s_part, s_part+1), row_ptr rebased, columns remapped to the
 * gathered-x slot owner(j)*S + (j - splits[owner(j)]), S = max part rows.
 * out_row_ptr[rows+1], out_col/out_val[shard nnz]. Requires a square matrix. */
int64_t ora_partition_slot(const int64_t *splits, int nparts);
int ora_slice_remap(int64_t n_rows, const int64_t *row_ptr, const int32_t *col,
                    const double *val, const int64_t *splits, int nparts, int part,
                    int64_t *out_row_ptr, int32_t *out_col, double *out_val);

/* Compressed exchange: colmap[j] = owner(j)*S' + (referenced columns of
 * owner(j) before j) for a column some row references, -1 otherwise; returns S' (max
 * referenced columns per part).  Square matrices. */
int64_t ora_hot_columns(int64_t n_cols, int64_t nnz, const int32_t *col, int64_t kmax, int32_t *hot_out);
int64_t ora_halo_colmap(int64_t n_rows, const int64_t *row_ptr, const int32_t *col, const int64_t *splits,
                        int nparts, int part, int32_t *colmap, int64_t *counts);
int64_t ora_partition_colmap(int64_t n_rows, const int64_t *row_ptr, const int32_t *col,
                             const int64_t *splits, int nparts, int32_t *colmap);
/* Shard `part` with columns mapped through colmap. */
int ora_slice_remap_colmap(int64_t n_rows, const int64_t *row_ptr, const int32_t *col,
                           const double *val, const int64_t *splits, int part, const int32_t *colmap,
                           int64_t *out_row_ptr, int32_t *out_col, double *out_val);

/* Own / foreign split of shard `part`: which = 0 keeps columns in the
 * part's own row range, remapped to j - splits[part]; which = 1 keeps the others,
 * remapped to the dense slot layout (colmap == NULL) or through colmap.  Returns the
 * block's nonzero count; out_* may be NULL to size only. */
int64_t ora_slice_split(int64_t n_rows, const int64_t *row_ptr, const int32_t *col, const double *val,
                        const int64_t *splits, int nparts, int part, const int32_t *colmap, int which,
                        int64_t *out_row_ptr, int32_t *out_col, double *out_val);

#ifdef __cplusplus
}
#endif
#endif
