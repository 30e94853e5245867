/*
 * matgen.c -- seeded synthetic sparse-matrix generators (INPUT GENERATION ONLY).
 *
 * Serves both the oracle tests and the CUDA path; holds none of the method's
 * arithmetic (no SpMV, no format conversion, no features).  Every random draw is
 * a counter-based hash of (seed, stream, counter), so results are identical
 * regardless of thread count or call order.  Recipes: DESIGN.md §5.
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#ifdef _OPENMP
#include <omp.h>
#endif

static inline uint64_t mg_mix(uint64_t z)
{
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
}

uint64_t mg_hash3(uint64_t seed, uint64_t a, uint64_t b)
{
    return mg_mix(mg_mix(mg_mix(seed + 0x9E3779B97F4A7C15ULL) ^ (a * 0xD1B54A32D192ED03ULL)) + b);
}

/* value kinds: 0 = uniform [-1,1) on a 2^-52 grid (fp64-exact),
 *              1 = uniform [-1,1) on a 2^-23 grid (fp32-exact),
 *              2 = integer regime {-2,-1,1,2},
 *              3 = constant 1.0 */
static inline double mg_value(uint64_t h, int kind)
{
    switch (kind) {
    case 0: return (double)(h >> 11) * 0x1p-52 - 1.0;
    case 1: return (double)(h >> 40) * 0x1p-23 - 1.0;
    case 2: { static const double t[4] = {-2.0, -1.0, 1.0, 2.0}; return t[h & 3]; }
    default: return 1.0;
    }
}

/* dense vector: out[i] = value(hash(seed, stream, i)) */
void mg_vector(uint64_t seed, uint64_t stream, int64_t n, int kind, double *out)
{
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) out[i] = mg_value(mg_hash3(seed, stream, (uint64_t)i), kind);
}

/* matrix values: val[k] = value(hash(seed, row, col)) -- position keyed, so the
 * same (i,j) always gets the same value (dedup-order invariant, A18). */
void mg_matrix_values(uint64_t seed, int64_t n_rows, const int64_t *row_ptr,
                      const int32_t *col, int kind, double *val)
{
#pragma omp parallel for schedule(dynamic, 4096)
    for (int64_t r = 0; r < n_rows; ++r)
        for (int64_t k = row_ptr[r]; k < row_ptr[r + 1]; ++k)
            val[k] = mg_value(mg_hash3(seed, (uint64_t)r, (uint64_t)col[k] + 0x100000000ULL), kind);
}

static int cmp_i32(const void *a, const void *b)
{
    int32_t x = *(const int32_t *)a, y = *(const int32_t *)b;
    return (x > y) - (x < y);
}

/* Rows with prescribed lengths; columns drawn uniformly without replacement from
 * [0, n_cols) by Floyd's algorithm on the row's own stream, then sorted.
 * row_ptr must already hold the exclusive prefix sum of the lengths. */
int mg_fill_random_rows(uint64_t seed, int64_t n_rows, int64_t n_cols,
                        const int64_t *row_ptr, int32_t *col)
{
    int bad = 0;
#pragma omp parallel for schedule(dynamic, 256) reduction(|:bad)
    for (int64_t r = 0; r < n_rows; ++r) {
        int64_t len = row_ptr[r + 1] - row_ptr[r];
        if (len > n_cols) { bad = 1; continue; }
        int32_t *c = col + row_ptr[r];
        if (len == n_cols) {                      /* dense row */
            for (int64_t j = 0; j < len; ++j) c[j] = (int32_t)j;
            continue;
        }
        /* Floyd: for j = n-len .. n-1 draw t in [0, j]; take t unless already
         * taken, else take j.  Membership: linear scan for short rows, an
         * open-addressing set for long ones. */
        int64_t m = 0, cap = 0;
        int32_t *set = NULL;
        if (len > 64) {
            cap = 1;
            while (cap < 2 * len) cap <<= 1;
            set = (int32_t *)malloc((size_t)cap * sizeof(int32_t));
            if (!set) { bad = 1; continue; }
            for (int64_t q = 0; q < cap; ++q) set[q] = -1;
        }
        for (int64_t j = n_cols - len; j < n_cols; ++j) {
            uint64_t h = mg_hash3(seed ^ 0x5A5A5A5A5A5A5A5AULL, (uint64_t)r, (uint64_t)j);
            int32_t t = (int32_t)(h % (uint64_t)(j + 1));
            int32_t v = t;
            if (!set) {
                for (int64_t q = 0; q < m; ++q) if (c[q] == t) { v = (int32_t)j; break; }
            } else {
                uint64_t slot = mg_mix((uint64_t)t) & (uint64_t)(cap - 1);
                while (set[slot] != -1 && set[slot] != t) slot = (slot + 1) & (uint64_t)(cap - 1);
                if (set[slot] == t) v = (int32_t)j;
                slot = mg_mix((uint64_t)v) & (uint64_t)(cap - 1);
                while (set[slot] != -1) slot = (slot + 1) & (uint64_t)(cap - 1);
                set[slot] = v;
            }
            c[m++] = v;
        }
        free(set);
        qsort(c, (size_t)len, sizeof(int32_t), cmp_i32);
    }
    return bad ? -1 : 0;
}

/* 5-point Laplacian on a g x g grid, natural ordering, no wraparound:
 * diagonal 4, neighbours -1 (cfg2). Arrays sized n+1 / 5n. Returns nnz. */
int64_t mg_laplacian5(int64_t g, int64_t *row_ptr, int32_t *col, double *val)
{
    int64_t n = g * g;
    /* row lengths are known in closed form; fill row_ptr serially-by-row-of-grid */
    row_ptr[0] = 0;
    for (int64_t i = 0; i < g; ++i)
        for (int64_t j = 0; j < g; ++j) {
            int64_t r = i * g + j;
            int64_t len = 1 + (i > 0) + (i < g - 1) + (j > 0) + (j < g - 1);
            row_ptr[r + 1] = row_ptr[r] + len;
        }
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < g; ++i)
        for (int64_t j = 0; j < g; ++j) {
            int64_t r = i * g + j, k = row_ptr[r];
            if (i > 0)     { col[k] = (int32_t)(r - g); val[k++] = -1.0; }
            if (j > 0)     { col[k] = (int32_t)(r - 1); val[k++] = -1.0; }
            col[k] = (int32_t)r; val[k++] = 4.0;
            if (j < g - 1) { col[k] = (int32_t)(r + 1); val[k++] = -1.0; }
            if (i < g - 1) { col[k] = (int32_t)(r + g); val[k++] = -1.0; }
        }
    return row_ptr[n];
}

/* R-MAT edge keys (row << scale | col), Graph500 quadrant probabilities given as
 * 32-bit thresholds: P(top-left)=a, P(top-right)=b, P(bottom-left)=c (A18).
 * One 64-bit hash per two levels (two 32-bit uniforms). */
void mg_rmat_keys(uint64_t seed, int scale, int64_t n_edges,
                  uint32_t ta, uint32_t tab, uint32_t tabc, uint64_t *keys)
{
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < n_edges; ++e) {
        uint64_t row = 0, colv = 0;
        uint64_t h = 0;
        for (int lvl = 0; lvl < scale; ++lvl) {
            uint32_t u;
            if ((lvl & 1) == 0) { h = mg_hash3(seed, (uint64_t)e, (uint64_t)(lvl >> 1)); u = (uint32_t)h; }
            else u = (uint32_t)(h >> 32);
            uint64_t rb, cb;
            if (u < ta) { rb = 0; cb = 0; }
            else if (u < tab) { rb = 0; cb = 1; }
            else if (u < tabc) { rb = 1; cb = 0; }
            else { rb = 1; cb = 1; }
            row = (row << 1) | rb;
            colv = (colv << 1) | cb;
        }
        keys[e] = (row << scale) | colv;
    }
}

/* LSD radix sort (8-bit digits) of keys < 2^bits, then in-place unique.
 * Returns the number of unique keys.  tmp has n entries. */
int64_t mg_sort_unique(uint64_t *keys, uint64_t *tmp, int64_t n, int bits)
{
    if (n <= 0) return 0;
    int passes = (bits + 7) / 8;
    int nt = 1;
#ifdef _OPENMP
    nt = omp_get_max_threads();
#endif
    int64_t *hist = (int64_t *)calloc((size_t)nt * 256, sizeof(int64_t));
    uint64_t *src = keys, *dst = tmp;
    for (int p = 0; p < passes; ++p) {
        int sh = 8 * p;
        memset(hist, 0, (size_t)nt * 256 * sizeof(int64_t));
#pragma omp parallel num_threads(nt)
        {
            int tid = 0;
#ifdef _OPENMP
            tid = omp_get_thread_num();
#endif
            int64_t lo = n * tid / nt, hi = n * (tid + 1) / nt;
            int64_t *h = hist + (size_t)tid * 256;
            for (int64_t i = lo; i < hi; ++i) h[(src[i] >> sh) & 255]++;
#pragma omp barrier
#pragma omp single
            {
                int64_t run = 0;
                for (int d = 0; d < 256; ++d)
                    for (int t = 0; t < nt; ++t) {
                        int64_t c = hist[(size_t)t * 256 + d];
                        hist[(size_t)t * 256 + d] = run;
                        run += c;
                    }
            }
            for (int64_t i = lo; i < hi; ++i) dst[h[(src[i] >> sh) & 255]++] = src[i];
        }
        uint64_t *s = src; src = dst; dst = s;
    }
    free(hist);
    if (src != keys) memcpy(keys, src, (size_t)n * sizeof(uint64_t));
    int64_t m = 1;
    for (int64_t i = 1; i < n; ++i)
        if (keys[i] != keys[m - 1]) keys[m++] = keys[i];
    return m;
}

/* sorted unique keys (row << shift | col) -> CSR (row_ptr[n_rows+1], col[m]) */
void mg_keys_to_csr(const uint64_t *keys, int64_t m, int shift, int64_t n_rows,
                    int64_t *row_ptr, int32_t *col)
{
    uint64_t mask = (shift >= 64) ? ~0ULL : ((1ULL << shift) - 1);
    memset(row_ptr, 0, (size_t)(n_rows + 1) * sizeof(int64_t));
    for (int64_t i = 0; i < m; ++i) row_ptr[(keys[i] >> shift) + 1]++;
    for (int64_t r = 0; r < n_rows; ++r) row_ptr[r + 1] += row_ptr[r];
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < m; ++i) col[i] = (int32_t)(keys[i] & mask);
}

/* Band / block structure filter (sweep families): row r keeps column j of the
 * candidate window iff hash(seed, r, j) < p (32-bit threshold).  Window:
 *   mode 0 (banded): [r*n_cols/n_rows - w, r*n_cols/n_rows + w]
 *   mode 1 (block-diagonal, block size w): the block of r, scaled to n_cols.
 * Pass row_ptr == NULL-col to count: fills lens[r]; else fills col using row_ptr. */
static inline void mg_window(int mode, int64_t r, int64_t n_rows, int64_t n_cols, int64_t w,
                             int64_t *lo, int64_t *hi)
{
    int64_t c = (int64_t)(((__int128)r * n_cols) / (n_rows > 0 ? n_rows : 1));
    if (mode == 0) { *lo = c - w; *hi = c + w + 1; }
    else {
        int64_t b = r / w;
        *lo = (int64_t)(((__int128)b * w * n_cols) / n_rows);
        *hi = (int64_t)(((__int128)(b + 1) * w * n_cols) / n_rows);
        if (*hi <= *lo) *hi = *lo + 1;
    }
    if (*lo < 0) *lo = 0;
    if (*hi > n_cols) *hi = n_cols;
}

void mg_window_rows(uint64_t seed, int mode, int64_t n_rows, int64_t n_cols, int64_t w,
                    uint32_t p_thresh, int64_t *lens, const int64_t *row_ptr, int32_t *col)
{
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t r = 0; r < n_rows; ++r) {
        int64_t lo, hi, cnt = 0;
        mg_window(mode, r, n_rows, n_cols, w, &lo, &hi);
        for (int64_t j = lo; j < hi; ++j) {
            uint32_t u = (uint32_t)mg_hash3(seed, (uint64_t)r, (uint64_t)j);
            if (u < p_thresh || p_thresh == 0xFFFFFFFFu) {
                if (col) col[row_ptr[r] + cnt] = (int32_t)j;
                ++cnt;
            }
        }
        if (lens) lens[r] = cnt;
    }
}

int mg_num_threads(void)
{
#ifdef _OPENMP
    return omp_get_max_threads();
#else
    return 1;
#endif
}
