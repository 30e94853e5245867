/*
 * oracle.c -- CPU ORACLE for the six-format SpMV study.  TEST INFRASTRUCTURE ONLY:
 * loaded by tests/, __graft_entry__.smoke() and bench.py's cpu_baseline leg,
 * never by the product path.  Plain loops in the paper's terms, no blocking,
 * no fusion, no reordering; every function cites the passage it follows.
 *
 * Compile: gcc -O2 -std=c11 -ffp-contract=off -fno-fast-math -fPIC -shared
 * (-ffp-contract=off so that a*b+c is never fused: the long-double products and
 * sums round exactly as written).
 *
 * Pins (tests/test_oracle_*.py): hand 4x4/5x5 examples (tests/golden/), identity /
 * diagonal / permutation and 5-point-Laplacian closed forms, dense brute force,
 * scipy.sparse, CSR == COO bit-exact, integer-exact regime, numpy brute-force
 * features, linear-walk == binary-search merge coordinates, CSR5 decode round trip.
 * Parity unpinned: none of the functions below (labels/timing live in Python).
 */
#include "oracle.h"
#include <math.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------ SpMV */

/* y_i <- alpha * sum_{k in row i} a_k x[col_k] + beta * y_i  (
 * the formats of PAPER.md:89-103 all represent this same product).  Long double
 * (x87, 64-bit mantissa) accumulation; fp64 products of fp32 data are exact. */
int ora_spmv_csr(int64_t n_rows, const int64_t *row_ptr, const int32_t *col,
                 const double *val, const double *x, double alpha, double beta,
                 const double *y_in, double *y_out, double *bound_out)
{
    if (n_rows < 0) return -1;
    for (int64_t i = 0; i < n_rows; ++i) {
        long double acc = 0.0L, absacc = 0.0L;
        if (alpha != 0.0) {                         /* A14: alpha == 0 => A not read */
            for (int64_t k = row_ptr[i]; k < row_ptr[i + 1]; ++k) {
                long double p = (long double)val[k] * (long double)x[col[k]];
                acc += p;
                absacc += fabsl(p);
            }
        }
        long double r = (long double)alpha * acc;
        long double b = 0.0L;
        if (beta != 0.0) {                          /* A14: beta == 0 => y not read */
            r += (long double)beta * (long double)y_in[i];
            b = fabsl((long double)beta * (long double)y_in[i]);
        }
        y_out[i] = (double)r;
        if (bound_out) bound_out[i] = (double)(fabsl((long double)alpha) * absacc + b);
    }
    return 0;
}

/* COO SpMV: product contributions per stored triplet, accumulated
 * per row in stored order, then the same finalisation as the CSR oracle (c2.2). */
int ora_spmv_coo(int64_t n_rows, int64_t nnz, const int32_t *row, const int32_t *col,
                 const double *val, const double *x, double alpha, double beta,
                 const double *y_in, double *y_out)
{
    if (n_rows < 0 || nnz < 0) return -1;
    long double *acc = (long double *)calloc((size_t)(n_rows > 0 ? n_rows : 1), sizeof(long double));
    if (!acc) return -2;
    if (alpha != 0.0)
        for (int64_t k = 0; k < nnz; ++k)
            acc[row[k]] += (long double)val[k] * (long double)x[col[k]];
    for (int64_t i = 0; i < n_rows; ++i) {
        long double r = (long double)alpha * acc[i];
        if (beta != 0.0) r += (long double)beta * (long double)y_in[i];
        y_out[i] = (double)r;
    }
    free(acc);
    return 0;
}

/* A15: canonical CSR (SuiteSparse-style). */
int ora_is_canonical(int64_t n_rows, int64_t n_cols, int64_t nnz,
                     const int64_t *row_ptr, const int32_t *col)
{
    if (n_rows < 0 || n_cols < 0 || nnz < 0) return 0;
    if (row_ptr[0] != 0 || row_ptr[n_rows] != nnz) return 0;
    for (int64_t i = 0; i < n_rows; ++i) {
        if (row_ptr[i + 1] < row_ptr[i]) return 0;
        for (int64_t k = row_ptr[i]; k < row_ptr[i + 1]; ++k) {
            if (col[k] < 0 || (int64_t)col[k] >= n_cols) return 0;
            if (k > row_ptr[i] && col[k] <= col[k - 1]) return 0;
        }
    }
    return 1;
}

/* ------------------------------------------------------------ converters */

/* COO: "three dense arrays ... row indices, column indices, values". */
int ora_csr2coo(int64_t n_rows, const int64_t *row_ptr, int32_t *row_out)
{
    for (int64_t r = 0; r < n_rows; ++r)
        for (int64_t k = row_ptr[r]; k < row_ptr[r + 1]; ++k)
            row_out[k] = (int32_t)r;
    return 0;
}

/* ELL width = "max nnz" of a row. */
int64_t ora_ell_width(int64_t n_rows, const int64_t *row_ptr)
{
    int64_t K = 0;
    for (int64_t r = 0; r < n_rows; ++r)
        if (row_ptr[r + 1] - row_ptr[r] > K) K = row_ptr[r + 1] - row_ptr[r];
    return K;
}

/* A3: leading dimension rounded up to a warp. */
int64_t ora_ell_ld(int64_t n_rows) { return (n_rows + 31) / 32 * 32; }

/* ELL: rows left-shifted, padded with zeroes, column-major. */
int ora_csr2ell(int64_t n_rows, const int64_t *row_ptr, const int32_t *col,
                const double *val, int64_t K, int64_t ld,
                int32_t *ell_col, double *ell_val)
{
    if (ld < n_rows) return -1;
    for (int64_t j = 0; j < K; ++j)
        for (int64_t r = 0; r < ld; ++r) {
            ell_col[j * ld + r] = -1;          /* A3 padding sentinel */
            ell_val[j * ld + r] = 0.0;
        }
    for (int64_t r = 0; r < n_rows; ++r) {
        int64_t len = row_ptr[r + 1] - row_ptr[r];
        if (len > K) return -2;
        for (int64_t j = 0; j < len; ++j) {
            ell_col[j * ld + r] = col[row_ptr[r] + j];
            ell_val[j * ld + r] = val[row_ptr[r] + j];
        }
    }
    return 0;
}

/* HYB split width (A2). */
int64_t ora_hyb_width(int64_t n_rows, const int64_t *row_ptr, int rule)
{
    if (n_rows <= 0) return 0;
    int64_t nnz = row_ptr[n_rows];
    if (rule == 0) return (nnz + n_rows - 1) / n_rows;   /* ceil(nnz_mu) -- paper's choice */
    if (rule == 1) return nnz / n_rows;                  /* floor reading */
    /* rule 2: [2]'s rule as reconstructed in A2: the smallest k such that the rows
     * longer than k are fewer than a third of all rows, or fewer than 4096;
     * else the maximum row length. */
    int64_t K = ora_ell_width(n_rows, row_ptr);
    for (int64_t k = 0; k < K; ++k) {
        int64_t longer = 0;
        for (int64_t r = 0; r < n_rows; ++r)
            if (row_ptr[r + 1] - row_ptr[r] > k) ++longer;
        if (3 * longer < n_rows || longer < 4096) return k;
    }
    return K;
}

int64_t ora_hyb_coo_nnz(int64_t n_rows, const int64_t *row_ptr, int64_t Kh)
{
    int64_t c = 0;
    for (int64_t r = 0; r < n_rows; ++r) {
        int64_t len = row_ptr[r + 1] - row_ptr[r];
        if (len > Kh) c += len - Kh;
    }
    return c;
}

/* HYB (read per A1): first Kh entries of a row in ELL, the rest in COO. */
int ora_csr2hyb(int64_t n_rows, const int64_t *row_ptr, const int32_t *col,
                const double *val, int64_t Kh, int64_t ld,
                int32_t *ell_col, double *ell_val,
                int32_t *coo_row, int32_t *coo_col, double *coo_val)
{
    if (ld < n_rows) return -1;
    for (int64_t j = 0; j < Kh; ++j)
        for (int64_t r = 0; r < ld; ++r) {
            ell_col[j * ld + r] = -1;
            ell_val[j * ld + r] = 0.0;
        }
    int64_t c = 0;
    for (int64_t r = 0; r < n_rows; ++r) {
        int64_t len = row_ptr[r + 1] - row_ptr[r];
        for (int64_t j = 0; j < len; ++j) {
            int64_t k = row_ptr[r] + j;
            if (j < Kh) {
                ell_col[j * ld + r] = col[k];
                ell_val[j * ld + r] = val[k];
            } else {
                coo_row[c] = (int32_t)r;
                coo_col[c] = col[k];
                coo_val[c] = val[k];
                ++c;
            }
        }
    }
    return 0;
}

/* CSR long-row chunks (A25): rows longer than 2*C nonzeros are cut into C-nonzero chunks,
 * listed by row, then chunk index; chunk j of row r starts at row_ptr[r] + j*C. */
int64_t ora_csr_chunks(int64_t n_rows, const int64_t *row_ptr, int64_t C,
                       int64_t *chunk_row, int64_t *chunk_lo)
{
    if (C <= 0 || n_rows < 0) return -1;
    int64_t k = 0;
    for (int64_t r = 0; r < n_rows; ++r) {
        int64_t len = row_ptr[r + 1] - row_ptr[r];
        if (len <= 2 * C) continue;
        for (int64_t start = row_ptr[r]; start < row_ptr[r + 1]; start += C) {
            if (chunk_row) chunk_row[k] = r;
            if (chunk_lo) chunk_lo[k] = start;
            ++k;
        }
    }
    return k;
}

/* Compressed rows (A33): the rows of A holding at least one nonzero, in
 * increasing order, and their row starts followed by nnz -- the CSR of those rows over the
 * same col/val arrays.  Returns their number. */
int64_t ora_compress_rows(int64_t n_rows, const int64_t *row_ptr, int64_t *rows_out, int64_t *rp_out)
{
    if (n_rows < 0) return -1;
    int64_t k = 0;
    for (int64_t r = 0; r < n_rows; ++r) {
        if (row_ptr[r + 1] > row_ptr[r]) {
            if (rows_out) rows_out[k] = r;
            if (rp_out) rp_out[k] = row_ptr[r];
            ++k;
        }
    }
    if (rp_out) rp_out[k] = n_rows > 0 ? row_ptr[n_rows] : 0;
    return k;
}

/* Merge-based CSR: "logically partitions the work ... into equal
 * sized sub-problems".  Work items = n_rows row ends + nnz nonzeros; tile t takes
 * diagonals [t*T, (t+1)*T). */
int64_t ora_merge_ntiles(int64_t n_rows, int64_t nnz, int64_t T)
{
    if (T <= 0) return -1;
    return (n_rows + nnz + T - 1) / T;
}

/* A7: walk the merge one item at a time; a row end A[i] = row_ptr[i+1] is consumed
 * before nonzero j when A[i] <= j.  Records (i, j) at every diagonal t*T. */
int ora_merge_coords(int64_t n_rows, const int64_t *row_ptr, int64_t T,
                     int64_t *coord_row, int64_t *coord_nz)
{
    int64_t nnz = row_ptr[n_rows];
    int64_t total = n_rows + nnz;
    int64_t n_tiles = ora_merge_ntiles(n_rows, nnz, T);
    if (n_tiles < 0) return -1;
    int64_t i = 0, j = 0, t = 0;
    for (int64_t d = 0; d <= total; ++d) {
        /* record every tile boundary that falls on this diagonal */
        while (t <= n_tiles && (t * T < total ? t * T : total) == d) {
            coord_row[t] = i;
            coord_nz[t] = j;
            ++t;
        }
        if (d == total) break;
        if (i < n_rows && row_ptr[i + 1] <= j) ++i;   /* consume a row end */
        else ++j;                                      /* consume a nonzero */
    }
    return t == n_tiles + 1 ? 0 : -2;
}

/* A28: class of merge tile t = 1 iff the tile consumes fewer than
 * max_rows row ends and no row receives more than max_len of the tile's nonzeros
 * (the row still open at the tile's end included).  Walks the merge path item by
 * item, counting the nonzeros the current row takes inside the current tile. */
int ora_merge_class(int64_t n_rows, const int64_t *row_ptr, int64_t T,
                    int64_t max_rows, int64_t max_len, uint8_t *cls)
{
    int64_t nnz = row_ptr[n_rows];
    int64_t total = n_rows + nnz;
    int64_t n_tiles = ora_merge_ntiles(n_rows, nnz, T);
    if (n_tiles < 0) return -1;
    int64_t i = 0, j = 0;
    for (int64_t t = 0; t < n_tiles; ++t) {
        int64_t d_end = (t + 1) * T < total ? (t + 1) * T : total;
        int64_t ends = 0, run = 0, run_max = 0;
        for (int64_t d = t * T; d < d_end; ++d) {
            if (i < n_rows && row_ptr[i + 1] <= j) { ++i; ++ends; run = 0; }
            else { ++j; ++run; if (run > run_max) run_max = run; }
        }
        cls[t] = (ends < max_rows && run_max <= max_len) ? 1 : 0;
    }
    return 0;
}

/* ------------------------------------------------------------------ CSR5 */

#define ORA_OMEGA 32

/* A6 (B200 rule): sigma = 4 for ceil(nnz_mu) <= 3, 8 for 4, 12 above
 * (multiples of 4 keep the lane runs 16-byte vectorizable; <= 16 fits the packing). */
int64_t ora_csr5_sigma(int64_t n_rows, int64_t nnz)
{
    if (n_rows <= 0) return 4;
    int64_t mu_ceil = (nnz + n_rows - 1) / n_rows;
    if (mu_ceil <= 3) return 4;
    if (mu_ceil == 4) return 8;
    return 12;
}

/* row_of[e] for every element: the row whose range contains e (a plain expansion). */
static int32_t *ora_rows_of(int64_t n_rows, const int64_t *row_ptr)
{
    int64_t nnz = row_ptr[n_rows];
    int32_t *ro = (int32_t *)malloc((size_t)(nnz > 0 ? nnz : 1) * sizeof(int32_t));
    if (ro) ora_csr2coo(n_rows, row_ptr, ro);
    return ro;
}

/* first r in [0, n_rows] with r == n_rows or row_ptr[r] >= e (linear scan from a hint) */
static int64_t ora_first_row_starting_at_or_after(int64_t n_rows, const int64_t *row_ptr,
                                                  int64_t e, int64_t from)
{
    int64_t r = from;
    while (r < n_rows && row_ptr[r] < e) ++r;
    return r;
}

int64_t ora_csr5_map_len(int64_t n_rows, const int64_t *row_ptr, int64_t sigma)
{
    int64_t nnz = row_ptr[n_rows], W = ORA_OMEGA * sigma;
    int64_t n_tiles = nnz / W, len = 0, lo = 0;
    for (int64_t t = 0; t < n_tiles; ++t) {
        int64_t a = ora_first_row_starting_at_or_after(n_rows, row_ptr, t * W, lo);
        int64_t b = ora_first_row_starting_at_or_after(n_rows, row_ptr, (t + 1) * W, a);
        int has_empty = 0, segs = 0;
        for (int64_t r = a; r < b; ++r) {
            if (row_ptr[r + 1] == row_ptr[r]) has_empty = 1; else ++segs;
        }
        if (has_empty) len += segs;
        lo = a;
    }
    return len;
}

/* CSR5: "partitioned into equally sized small 2D tiles"; tile_ptr
 * and tile_desc are the two extra arrays.  Per-element construction of the A6
 * encoding: tile t, lane l (0..31), step s (0..sigma-1) holds CSR element
 * e = t*32*sigma + l*sigma + s. */
int ora_csr5_encode(int64_t n_rows, const int64_t *row_ptr, const int32_t *col,
                    const double *val, int64_t sigma, int val_bytes,
                    int64_t *tile_ptr, int64_t *row_lo, uint32_t *tile_desc,
                    int64_t *map_off, int64_t *seg_map,
                    int32_t *col_perm, double *val_perm)
{
    if (sigma < 4 || sigma > 16 || sigma % 4 || (val_bytes != 4 && val_bytes != 8)) return -1;
    int64_t nnz = row_ptr[n_rows], W = ORA_OMEGA * sigma, n_tiles = nnz / W;
    int32_t *ro = ora_rows_of(n_rows, row_ptr);
    if (!ro) return -2;
    const int64_t vc = 4, vv = 16 / val_bytes;   /* 16-byte vectors per lane */

    /* tile_ptr: the row holding the tile's first element */
    for (int64_t t = 0; t < n_tiles; ++t) tile_ptr[t] = ro[t * W];
    tile_ptr[n_tiles] = (n_tiles * W < nnz) ? ro[n_tiles * W] : n_rows;

    /* row_lo: first row whose start lies at or after the tile's first element */
    int64_t lo = 0;
    for (int64_t t = 0; t <= n_tiles; ++t) {
        lo = ora_first_row_starting_at_or_after(n_rows, row_ptr, t * W, lo);
        row_lo[t] = lo;
    }

    int64_t moff = 0;
    for (int64_t t = 0; t < n_tiles; ++t) {
        uint32_t flag[ORA_OMEGA];
        for (int l = 0; l < ORA_OMEGA; ++l) {
            flag[l] = 0;
            for (int64_t s = 0; s < sigma; ++s) {
                int64_t e = t * W + l * sigma + s;
                if (e == row_ptr[ro[e]]) flag[l] |= 1u << s;   /* a row starts at e */
            }
        }
        uint32_t y_off = 0;
        for (int l = 0; l < ORA_OMEGA; ++l) {
            uint32_t seg = 0;
            while (l + (int)seg + 1 < ORA_OMEGA && flag[l + seg + 1] == 0) ++seg;
            tile_desc[t * ORA_OMEGA + l] = flag[l] | (y_off << 16) | (seg << 25);
            y_off += (uint32_t)__builtin_popcount(flag[l]);
        }
        /* empty rows in the emitted range [row_lo[t], row_lo[t+1]) => explicit map */
        int has_empty = 0;
        for (int64_t r = row_lo[t]; r < row_lo[t + 1]; ++r)
            if (row_ptr[r + 1] == row_ptr[r]) has_empty = 1;
        if (has_empty) {
            map_off[t] = moff;
            for (int64_t r = row_lo[t]; r < row_lo[t + 1]; ++r)
                if (row_ptr[r + 1] > row_ptr[r]) seg_map[moff++] = r;
        } else {
            map_off[t] = -1;
        }
        /* lane-interleaved copy of col/val */
        for (int l = 0; l < ORA_OMEGA; ++l)
            for (int64_t s = 0; s < sigma; ++s) {
                int64_t e = t * W + l * sigma + s;
                col_perm[t * W + (s / vc) * ORA_OMEGA * vc + l * vc + s % vc] = col[e];
                val_perm[t * W + (s / vv) * ORA_OMEGA * vv + l * vv + s % vv] = val[e];
            }
    }
    for (int64_t e = n_tiles * W; e < nnz; ++e) {   /* tail stays in CSR order */
        col_perm[e] = col[e];
        val_perm[e] = val[e];
    }
    free(ro);
    return 0;
}

int ora_csr5_decode(int64_t n_rows, int64_t nnz, const int64_t *row_ptr_tail,
                    int64_t sigma, int val_bytes,
                    const int64_t *tile_ptr, const int64_t *row_lo,
                    const uint32_t *tile_desc, const int64_t *map_off,
                    const int64_t *seg_map, const int32_t *col_perm,
                    const double *val_perm,
                    int64_t *row_ptr_out, int32_t *col_out, double *val_out)
{
    if (sigma < 4 || sigma > 16 || sigma % 4 || (val_bytes != 4 && val_bytes != 8)) return -1;
    int64_t W = ORA_OMEGA * sigma, n_tiles = nnz / W;
    const int64_t vc = 4, vv = 16 / val_bytes;
    for (int64_t r = 0; r <= n_rows; ++r) row_ptr_out[r] = -1;
    for (int64_t t = 0; t < n_tiles; ++t) {
        int64_t k = 0;                    /* segment counter within the tile */
        uint32_t y_expect = 0;
        for (int l = 0; l < ORA_OMEGA; ++l) {
            uint32_t d = tile_desc[t * ORA_OMEGA + l];
            uint32_t flag = d & 0xFFFFu, y_off = (d >> 16) & 0x1FFu, seg = (d >> 25) & 0x1Fu;
            if (y_off != y_expect) return -2;
            uint32_t seg_expect = 0;
            while (l + (int)seg_expect + 1 < ORA_OMEGA &&
                   (tile_desc[t * ORA_OMEGA + l + seg_expect + 1] & 0xFFFFu) == 0) ++seg_expect;
            if (seg != seg_expect) return -3;
            for (int64_t s = 0; s < sigma; ++s) {
                int64_t e = t * W + l * sigma + s;
                col_out[e] = col_perm[t * W + (s / vc) * ORA_OMEGA * vc + l * vc + s % vc];
                val_out[e] = val_perm[t * W + (s / vv) * ORA_OMEGA * vv + l * vv + s % vv];
                if (flag & (1u << s)) {
                    int64_t row = map_off[t] >= 0 ? seg_map[map_off[t] + k] : row_lo[t] + k;
                    if (row < row_lo[t] || row >= row_lo[t + 1]) return -4;
                    row_ptr_out[row] = e;
                    ++k;
                }
            }
            y_expect += (uint32_t)__builtin_popcount(flag);
        }
        if (map_off[t] < 0 && k != row_lo[t + 1] - row_lo[t]) return -5;
    }
    for (int64_t e = n_tiles * W; e < nnz; ++e) {
        col_out[e] = col_perm[e];
        val_out[e] = val_perm[e];
    }
    for (int64_t r = row_lo[n_tiles]; r < n_rows; ++r) row_ptr_out[r] = row_ptr_tail[r];
    row_ptr_out[n_rows] = nnz;
    for (int64_t r = n_rows - 1; r >= 0; --r)        /* empty rows start where the next one does */
        if (row_ptr_out[r] < 0) row_ptr_out[r] = row_ptr_out[r + 1];
    /* tile_ptr[t] must be the row holding element t*W */
    for (int64_t t = 0; t <= n_tiles; ++t) {
        int64_t e = t * W;
        if (e >= nnz) { if (tile_ptr[t] != n_rows) return -6; continue; }
        int64_t r = tile_ptr[t];
        if (r < 0 || r >= n_rows || !(row_ptr_out[r] <= e && e < row_ptr_out[r + 1])) return -7;
    }
    return 0;
}

/* -------------------------------------------------------------- features */

/* Table II with the names of Figs 4-5, read per
 * A8: nnz_frac in percent; sigma = population std; a block is a maximal run of
 * consecutive column indices within a row ("continuous nnz chunk"); nnzb_* over all
 * rows (empty rows have 0 blocks); snzb_* over all blocks.  Exact integer sums,
 * then the fixed fp64 formulas of A9. */
int ora_features(int64_t n_rows, int64_t n_cols, const int64_t *row_ptr,
                 const int32_t *col, ora_features_t *f)
{
    memset(f, 0, sizeof(*f));
    if (n_rows < 0 || n_cols < 0) return -1;
    int64_t nnz = n_rows > 0 ? row_ptr[n_rows] : 0;
    f->n_rows = n_rows; f->n_cols = n_cols; f->nnz_tot = nnz;

    uint64_t S1 = 0, S2 = 0, B1 = 0, B2 = 0, Z2 = 0;
    int64_t len_min = -1, len_max = 0, nb_min = -1, nb_max = 0, bs_min = -1, bs_max = 0;
    int64_t n_empty = 0;
    for (int64_t r = 0; r < n_rows; ++r) {
        int64_t len = row_ptr[r + 1] - row_ptr[r];
        S1 += (uint64_t)len;
        S2 += (uint64_t)len * (uint64_t)len;
        if (len_min < 0 || len < len_min) len_min = len;
        if (len > len_max) len_max = len;
        if (len == 0) ++n_empty;
        /* walk the row's blocks */
        int64_t nb = 0, run = 0;
        for (int64_t k = row_ptr[r]; k < row_ptr[r + 1]; ++k) {
            int starts_block = (k == row_ptr[r]) || (col[k] != col[k - 1] + 1);
            if (starts_block) {
                if (run > 0) {               /* close the previous block of this row */
                    Z2 += (uint64_t)run * (uint64_t)run;
                    if (bs_min < 0 || run < bs_min) bs_min = run;
                    if (run > bs_max) bs_max = run;
                }
                ++nb;
                run = 1;
            } else {
                ++run;
            }
        }
        if (run > 0) {
            Z2 += (uint64_t)run * (uint64_t)run;
            if (bs_min < 0 || run < bs_min) bs_min = run;
            if (run > bs_max) bs_max = run;
        }
        B1 += (uint64_t)nb;
        B2 += (uint64_t)nb * (uint64_t)nb;
        if (nb_min < 0 || nb < nb_min) nb_min = nb;
        if (nb > nb_max) nb_max = nb;
    }
    f->sum_len2 = S2; f->sum_nnzb2 = B2; f->sum_snzb2 = Z2;
    f->n_empty_rows = n_empty;
    f->nnz_max = len_max;
    f->nnz_min = len_min < 0 ? 0 : len_min;
    f->nnzb_tot = (int64_t)B1;
    f->nnzb_min = nb_min < 0 ? 0 : nb_min;
    f->nnzb_max = nb_max;
    f->snzb_min = bs_min < 0 ? 0 : bs_min;
    f->snzb_max = bs_max;

    if (n_rows > 0) {
        __int128 n = n_rows;
        f->nnz_mu = (double)nnz / (double)n_rows;
        f->nnz_sigma = sqrt((double)(n * (__int128)S2 - (__int128)S1 * (__int128)S1)) / (double)n_rows;
        f->nnzb_mu = (double)B1 / (double)n_rows;
        f->nnzb_sigma = sqrt((double)(n * (__int128)B2 - (__int128)B1 * (__int128)B1)) / (double)n_rows;
        if (n_cols > 0)
            f->nnz_frac = (double)((__int128)100 * nnz) / (double)((__int128)n_rows * n_cols);
    }
    if (B1 > 0) {
        __int128 nb = (__int128)B1;
        f->snzb_mu = (double)nnz / (double)B1;
        f->snzb_sigma = sqrt((double)(nb * (__int128)Z2 - (__int128)nnz * (__int128)nnz)) / (double)B1;
    }
    /* extras: ELL width/padding and HYB widths (A2) */
    f->ell_width = len_max;
    f->ell_slots = len_max * n_rows;
    f->ell_pad_frac = f->ell_slots > 0 ? (double)(f->ell_slots - nnz) / (double)f->ell_slots : 0.0;
    f->hyb_width = ora_hyb_width(n_rows, row_ptr, 0);
    f->hyb_coo_nnz = ora_hyb_coo_nnz(n_rows, row_ptr, f->hyb_width);
    f->hyb_width_floor = ora_hyb_width(n_rows, row_ptr, 1);
    f->hyb_width_cusp = ora_hyb_width(n_rows, row_ptr, 2);
    return 0;
}

/* ------------------------------------------------------------- partition */

/* SURVEY §8(a) a14 (north_star: "nnz-balanced merge-path splits"): the row
 * coordinate of the merge path at diagonal floor(k*(n_rows+nnz)/P), found by the
 * same linear walk as ora_merge_coords. */
int ora_partition(int64_t n_rows, const int64_t *row_ptr, int nparts, int64_t *splits)
{
    if (nparts <= 0) return -1;
    int64_t nnz = row_ptr[n_rows], total = n_rows + nnz;
    int64_t i = 0, j = 0, d = 0;
    for (int k = 0; k <= nparts; ++k) {
        int64_t target = (int64_t)(((__int128)k * total) / nparts);
        while (d < target) {
            if (i < n_rows && row_ptr[i + 1] <= j) ++i; else ++j;
            ++d;
        }
        splits[k] = i;
    }
    splits[nparts] = n_rows;   /* the walk ends at (n_rows, nnz) */
    return 0;
}

int64_t ora_partition_slot(const int64_t *splits, int nparts)
{
    int64_t S = 0;
    for (int k = 0; k < nparts; ++k)
        if (splits[k + 1] - splits[k] > S) S = splits[k + 1] - splits[k];
    return S;
}

int ora_slice_remap(int64_t n_rows, const int64_t *row_ptr, const int32_t *col,
                    const double *val, const int64_t *splits, int nparts, int part,
                    int64_t *out_row_ptr, int32_t *out_col, double *out_val)
{
    if (part < 0 || part >= nparts) return -1;
    int64_t S = ora_partition_slot(splits, nparts);
    int64_t r0 = splits[part], r1 = splits[part + 1];
    for (int64_t r = r0; r <= r1; ++r) out_row_ptr[r - r0] = row_ptr[r] - row_ptr[r0];
    for (int64_t k = row_ptr[r0]; k < row_ptr[r1]; ++k) {
        int64_t j = col[k];
        if (j < 0 || j >= n_rows) return -2;          /* square matrices only */
        int owner = 0;
        while (!(splits[owner] <= j && j < splits[owner + 1])) ++owner;
        out_col[k - row_ptr[r0]] = (int32_t)(owner * S + (j - splits[owner]));
        out_val[k - row_ptr[r0]] = val[k];
    }
    return 0;
}

/* Compressed exchange: a column is exchanged only if some row references it. */
int64_t ora_partition_colmap(int64_t n_rows, const int64_t *row_ptr, const int32_t *col,
                             const int64_t *splits, int nparts, int32_t *colmap)
{
    int64_t nnz = row_ptr[n_rows];
    unsigned char *used = (unsigned char *)calloc((size_t)(n_rows > 0 ? n_rows : 1), 1);
    if (!used) return -1;
    for (int64_t k = 0; k < nnz; ++k) used[col[k]] = 1;
    int64_t S = 0;
    for (int part = 0; part < nparts; ++part) {
        int64_t c = 0;
        for (int64_t j = splits[part]; j < splits[part + 1]; ++j) c += used[j];
        if (c > S) S = c;
    }
    for (int part = 0; part < nparts; ++part) {
        int64_t c = 0;
        for (int64_t j = splits[part]; j < splits[part + 1]; ++j)
            colmap[j] = used[j] ? (int32_t)(part * S + c++) : -1;
    }
    free(used);
    return S;
}

/* A30 hot columns (a handle's x layout): the degree of column c is its
 * number of nonzeros; the hot set is every column of degree >= t for the smallest t >= 1
 * such that at most kmax columns qualify, listed ascending.  Plain loops: degrees, a
 * count per degree value, then t.  Returns the number of hot columns (hot_out may be NULL). */
int64_t ora_hot_columns(int64_t n_cols, int64_t nnz, const int32_t *col, int64_t kmax, int32_t *hot_out)
{
    if (n_cols <= 0 || nnz <= 0 || kmax <= 0) return 0;
    int64_t *deg = (int64_t *)calloc((size_t)n_cols, sizeof(int64_t));
    if (!deg) return -1;
    int64_t dmax = 0;
    for (int64_t k = 0; k < nnz; ++k) deg[col[k]] += 1;
    for (int64_t c = 0; c < n_cols; ++c) if (deg[c] > dmax) dmax = deg[c];
    int64_t *cnt = (int64_t *)calloc((size_t)dmax + 2, sizeof(int64_t));     /* cnt[v] = #{deg == v} */
    if (!cnt) { free(deg); return -1; }
    for (int64_t c = 0; c < n_cols; ++c) cnt[deg[c]] += 1;
    int64_t t = dmax + 1, ge = 0;                                         /* ge = #{deg >= t} */
    while (t > 1 && ge + cnt[t - 1] <= kmax) { t -= 1; ge += cnt[t]; }
    int64_t K = 0;
    for (int64_t c = 0; c < n_cols; ++c)
        if (deg[c] >= t) { if (hot_out) hot_out[K] = (int32_t)c; ++K; }
    free(cnt);
    free(deg);
    return K;
}

/* Halo exchange: receiver `part` needs the columns its rows reference
 * that other parts own.  Plain loops: mark them, count per owner, S = max(1, max count),
 * colmap[j] = owner*S + (rank of j among the owner's marked columns), -1 elsewhere.
 * counts[o] = marked columns of owner o.  Returns S. */
int64_t ora_halo_colmap(int64_t n_rows, const int64_t *row_ptr, const int32_t *col, const int64_t *splits,
                        int nparts, int part, int32_t *colmap, int64_t *counts)
{
    unsigned char *used = (unsigned char *)calloc((size_t)(n_rows > 0 ? n_rows : 1), 1);
    if (!used) return -1;
    for (int64_t r = splits[part]; r < splits[part + 1]; ++r)
        for (int64_t k = row_ptr[r]; k < row_ptr[r + 1]; ++k) {
            int64_t j = col[k];
            if (j < splits[part] || j >= splits[part + 1]) used[j] = 1;
        }
    int64_t S = 1;
    for (int o = 0; o < nparts; ++o) {
        int64_t c = 0;
        for (int64_t j = splits[o]; j < splits[o + 1]; ++j) c += used[j];
        counts[o] = c;
        if (c > S) S = c;
    }
    for (int o = 0; o < nparts; ++o) {
        int64_t c = 0;
        for (int64_t j = splits[o]; j < splits[o + 1]; ++j)
            colmap[j] = used[j] ? (int32_t)(o * S + c++) : -1;
    }
    free(used);
    return S;
}

int ora_slice_remap_colmap(int64_t n_rows, const int64_t *row_ptr, const int32_t *col,
                           const double *val, const int64_t *splits, int part, const int32_t *colmap,
                           int64_t *out_row_ptr, int32_t *out_col, double *out_val)
{
    int64_t r0 = splits[part], r1 = splits[part + 1];
    if (r1 > n_rows) return -1;
    for (int64_t r = r0; r <= r1; ++r) out_row_ptr[r - r0] = row_ptr[r] - row_ptr[r0];
    for (int64_t k = row_ptr[r0]; k < row_ptr[r1]; ++k) {
        out_col[k - row_ptr[r0]] = colmap[col[k]];
        out_val[k - row_ptr[r0]] = val[k];
    }
    return 0;
}

/* Own / foreign split of a shard: plain row-by-row filter in stored order. */
int64_t ora_slice_split(int64_t n_rows, const int64_t *row_ptr, const int32_t *col, const double *val,
                        const int64_t *splits, int nparts, int part, const int32_t *colmap, int which,
                        int64_t *out_row_ptr, int32_t *out_col, double *out_val)
{
    int64_t r0 = splits[part], r1 = splits[part + 1];
    int64_t S = ora_partition_slot(splits, nparts), q = 0;
    if (r1 > n_rows) return -1;
    for (int64_t r = r0; r < r1; ++r) {
        if (out_row_ptr) out_row_ptr[r - r0] = q;
        for (int64_t k = row_ptr[r]; k < row_ptr[r + 1]; ++k) {
            int64_t j = col[k];
            int own = j >= r0 && j < r1;
            if (own != (which == 0)) continue;
            if (out_col) {
                if (which == 0) out_col[q] = (int32_t)(j - r0);
                else if (colmap) out_col[q] = colmap[j];
                else {
                    int owner = 0;
                    while (!(splits[owner] <= j && j < splits[owner + 1])) ++owner;
                    out_col[q] = (int32_t)(owner * S + (j - splits[owner]));
                }
                out_val[q] = val[k];
            }
            ++q;
        }
    }
    if (out_row_ptr) out_row_ptr[r1 - r0] = q;
    return q;
}
