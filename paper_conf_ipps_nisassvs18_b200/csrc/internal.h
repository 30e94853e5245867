// internal.h -- ctx/handle layout and the internal entry points of libspmv.
#pragma once
#include <mutex>
#include "common.cuh"

struct spmv_ctx {
    int device = 0;
    int sm_count = 148;
    int64_t l2_bytes = 0;
    spmv_allocator alloc{};
    bool has_alloc = false;
    // feature pass state (features.cu): device accumulators + per-warp records + the A2
    // histogram, allocated once and reset by the kernel itself; pinned result readback.
    // The pass blocks until done; the mutex serialises callers sharing the ctx.
    std::mutex feat_mu;
    void *feat_state = nullptr, *feat_recs = nullptr, *feat_hist = nullptr, *feat_host = nullptr;
    size_t feat_hist_bytes = 0;
};

namespace spmv {

constexpr int kMaxArrays = 20;

struct DevArray {
    void *p = nullptr;
    size_t bytes = 0;
    bool owned = true;
};

// scratch/array allocation through the ctx allocator (stream-ordered)
spmv_status dev_alloc(spmv_ctx *ctx, size_t bytes, cudaStream_t s, void **out);
void dev_free(spmv_ctx *ctx, void *p, size_t bytes, cudaStream_t s);

// RAII scratch buffer (freed stream-ordered at scope exit)
struct Scratch {
    spmv_ctx *ctx;
    cudaStream_t s;
    void *p = nullptr;
    size_t bytes = 0;
    Scratch(spmv_ctx *c, cudaStream_t st) : ctx(c), s(st) {}
    spmv_status alloc(size_t b) { bytes = b; return dev_alloc(ctx, b ? b : 16, s, &p); }
    template <typename T> T *as() const { return reinterpret_cast<T *>(p); }
    ~Scratch() { if (p) dev_free(ctx, p, bytes ? bytes : 16, s); }
};

// Integer results of the feature pass (exact sums; finals computed on the host, A9).
struct FeatureSums {
    unsigned long long bad;            // non-zero => not canonical (bit flags)
    unsigned long long n_empty;
    unsigned long long sum_len2;
    unsigned long long len_min, len_max;
    unsigned long long hyb_coo_ceil;   // sum max(len - ceil(mu), 0)
    unsigned long long nb_tot;         // total blocks
    unsigned long long sum_nb2;        // sum over rows of blocks^2
    unsigned long long nb_min, nb_max;
    unsigned long long sum_bs2;        // sum over blocks of size^2
    unsigned long long bs_min, bs_max;
};

// Run the feature pass (level 0: canonical check + row-length stats only;
// level 1: everything).  Blocking.  hist_cusp receives the A2 "cusp" width when
// level == 1.
spmv_status feature_pass(spmv_ctx *ctx, const spmv_csr *A, cudaStream_t s, int level,
                         FeatureSums *out, int64_t *hyb_cusp);
void finalize_features(const spmv_csr *A, const FeatureSums &fs, int64_t hyb_cusp,
                       spmv_features_t *f);
void feature_state_free(spmv_ctx *ctx);

}  // namespace spmv

struct spmv_handle {
    spmv_ctx *ctx = nullptr;
    spmv_format fmt = SPMV_CSR;
    spmv_dtype dtype = SPMV_F64;
    spmv_itype itype = SPMV_I32;
    int64_t n_rows = 0, n_cols = 0, nnz = 0;
    spmv::DevArray arr[spmv::kMaxArrays];
    // format parameters
    int64_t ell_K = 0, ell_ld = 0;
    int64_t hyb_coo_nnz = 0;
    int64_t sigma = 0, n_tiles = 0, map_len = 0;
    int64_t csr5_tail_row = 0;     // first row starting in the CSR5 tail (host copy of row_lo[n_tiles])
    int64_t merge_T = 0, merge_tiles = 0, merge_lean = 0;   // merge_lean: class-1 tiles (A28)
    bool coo_persist = false;                // COO: persistent tile loop (regular matrix, fp64)
    int64_t vec_w = 0;
    int64_t csr_chunk = 0, csr_chunks = 0;   // CSR long-row split (A25): chunk length, chunk count
    // per-run scratch: carries (row, value) of CTAs/tiles for the fix-up pass
    spmv::DevArray carry_row, carry_val;
    int64_t n_carry = 0;
    // spmv_run_host staging
    spmv::DevArray io_x, io_y;
    spmv::DevArray io_yin;                   // spmv_run_host_multi: the device copy of y_in (first handle)
    // CSR-vector dynamic batch scheduler: one u64 counter, zeroed before every run
    spmv::DevArray sched;
    // hot columns (A30): the x entries stored as -2 - slot are read from xhot[slot], packed
    // from x[arr[SPMV_ARR_HOT_COLS][slot]] at the start of every run (n_hot = 0: none)
    spmv::DevArray xhot;
    int64_t n_hot = 0;
    int launches = 0;
};

namespace spmv {
// convert.cu
spmv_status convert_impl(spmv_ctx *ctx, spmv_format fmt, const spmv_csr *A,
                         const spmv_convert_opts *opts, cudaStream_t s, spmv_handle *h);
// hot.cu (A30)
spmv_status hot_select(spmv_ctx *ctx, const spmv_csr *A, int64_t kmax, bool force, cudaStream_t s,
                       spmv_handle *h, Scratch &slot);
spmv_status hot_encode(spmv_ctx *ctx, spmv_handle *h, const Scratch &slot, cudaStream_t s);
// spmv_kernels.cu
spmv_status run_impl(spmv_handle *h, double alpha, double beta, const void *x, void *y,
                     cudaStream_t s);
int run_launch_count(const spmv_handle *h, bool alpha0);
// partition.cu
spmv_status partition_impl(spmv_ctx *ctx, const spmv_csr *A, int nparts, cudaStream_t s,
                           int64_t *splits);
spmv_status slice_size_impl(spmv_ctx *ctx, const spmv_csr *A, const int64_t *splits, int nparts,
                            int part, cudaStream_t s, int64_t *rows, int64_t *nnz, int64_t *slot);
spmv_status slice_remap_impl(spmv_ctx *ctx, const spmv_csr *A, const int64_t *splits, int nparts,
                             int part, cudaStream_t s, int32_t *rp_out, int32_t *col_out,
                             void *val_out);
spmv_status colmap_impl(spmv_ctx *ctx, const spmv_csr *A, const int64_t *splits, int nparts, cudaStream_t s,
                        int32_t *colmap, int64_t *slot);
spmv_status slice_remap_colmap_impl(spmv_ctx *ctx, const spmv_csr *A, const int64_t *splits, int nparts, int part,
                                    const int32_t *colmap, cudaStream_t s, int32_t *rp_out, int32_t *col_out,
                                    void *val_out);
spmv_status halo_colmap_impl(spmv_ctx *ctx, const spmv_csr *A, const int64_t *splits, int nparts, int part,
                             cudaStream_t s, int32_t *colmap, int64_t *counts, int64_t *slot);
spmv_status pack_index_impl(spmv_ctx *ctx, const int32_t *colmap, const int64_t *splits, int nparts, int part,
                            int64_t slot, cudaStream_t s, int32_t *idx, int64_t *count);
spmv_status gather_impl(spmv_ctx *ctx, spmv_dtype dt, const void *src, const int32_t *idx, int64_t n, void *dst,
                        cudaStream_t s);
spmv_status scatter_impl(spmv_ctx *ctx, spmv_dtype dt, const void *src, const int32_t *idx, int64_t n, void *dst,
                         cudaStream_t s);
spmv_status compress_rows_impl(spmv_ctx *ctx, const spmv_csr *A, cudaStream_t s, int32_t *rows_out, void *rp_out,
                               int64_t *count);
spmv_status split_impl(spmv_ctx *ctx, const spmv_csr *A, const int64_t *splits, int nparts, int part,
                       const int32_t *colmap, int which, cudaStream_t s, int32_t *rp_out, int32_t *col_out,
                       void *val_out, int64_t *nnz_out);
}  // namespace spmv
