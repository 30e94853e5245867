// partition.cu -- nnz-balanced multi-GPU row partition (north_star):
// row splits at merge-path diagonals floor(k*(n_rows+nnz)/P) (same path as the
// merge-based CSR of PAPER.md:103, A7), and the shard extraction that remaps
// columns to slots of the all-gathered x.
#include <algorithm>
#include <vector>

#include "internal.h"

namespace spmv {

namespace {

constexpr int kMaxParts = 64;

struct Splits {
    int64_t s[kMaxParts + 1];
    int nparts;
    int64_t slot;
};

template <typename IT>
__global__ void k_partition(const IT *rp, int64_t n, int64_t nnz, int nparts, int64_t *out) {
    int k = blockIdx.x * blockDim.x + threadIdx.x;
    if (k > nparts) return;
    int64_t d = (int64_t)(((__int128)k * (n + nnz)) / nparts);
    out[k] = merge_path_row(rp, n, nnz, d);
}

template <typename IT>
__global__ void k_rebase(const IT *rp, int64_t r0, int64_t rows, int *out) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= rows; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = (int)((int64_t)rp[r0 + i] - (int64_t)rp[r0]);
}

__global__ void k_remap(const int *col, int64_t k0, int64_t cnt, Splits sp, int *out) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < cnt; k += (int64_t)gridDim.x * blockDim.x) {
        int64_t j = col[k0 + k];
        int lo = 0, hi = sp.nparts - 1;          // owner = last k with s[k] <= j; then s[k+1] > j
        while (lo < hi) {
            int mid = (lo + hi + 1) >> 1;
            if (sp.s[mid] <= j) lo = mid; else hi = mid - 1;
        }
        out[k] = (int)(lo * sp.slot + (j - sp.s[lo]));
    }
}

template <typename IT>
spmv_status read_rp(const spmv_csr *A, int64_t r, cudaStream_t s, int64_t *v) {
    IT t;
    SPMV_CUDA_TRY(cudaMemcpyAsync(&t, (const IT *)A->row_ptr + r, sizeof(IT), cudaMemcpyDeviceToHost, s));
    SPMV_CUDA_TRY(cudaStreamSynchronize(s));
    *v = (int64_t)t;
    return SPMV_OK;
}

spmv_status rp_at(const spmv_csr *A, int64_t r, cudaStream_t s, int64_t *v) {
    return A->ptr_type == SPMV_I32 ? read_rp<int>(A, r, s, v) : read_rp<int64_t>(A, r, s, v);
}

spmv_status check_splits(const spmv_csr *A, const int64_t *sp, int nparts) {
    if (nparts > kMaxParts) { set_error("at most 64 parts"); return SPMV_ERR_INVALID_ARG; }
    if (sp[0] != 0 || sp[nparts] != A->n_rows) { set_error("splits must span [0, n_rows]"); return SPMV_ERR_INVALID_ARG; }
    for (int k = 0; k < nparts; ++k)
        if (sp[k + 1] < sp[k]) { set_error("splits must be non-decreasing"); return SPMV_ERR_INVALID_ARG; }
    return SPMV_OK;
}

}  // namespace

spmv_status partition_impl(spmv_ctx *ctx, const spmv_csr *A, int nparts, cudaStream_t s, int64_t *splits) {
    Scratch d(ctx, s);
    SPMV_TRY(d.alloc((nparts + 1) * 8));
    if (A->ptr_type == SPMV_I32)
        k_partition<int><<<ceil_div(nparts + 1, 128), 128, 0, s>>>((const int *)A->row_ptr, A->n_rows, A->nnz, nparts,
                                                                   d.as<int64_t>());
    else
        k_partition<int64_t><<<ceil_div(nparts + 1, 128), 128, 0, s>>>((const int64_t *)A->row_ptr, A->n_rows, A->nnz,
                                                                       nparts, d.as<int64_t>());
    SPMV_LAUNCH_CHECK();
    SPMV_CUDA_TRY(cudaMemcpyAsync(splits, d.p, (nparts + 1) * 8, cudaMemcpyDeviceToHost, s));
    SPMV_CUDA_TRY(cudaStreamSynchronize(s));
    return SPMV_OK;
}

spmv_status slice_size_impl(spmv_ctx *ctx, const spmv_csr *A, const int64_t *sp, int nparts, int part, cudaStream_t s,
                            int64_t *rows, int64_t *nnz, int64_t *slot) {
    (void)ctx;
    SPMV_TRY(check_splits(A, sp, nparts));
    int64_t a = 0, b = 0;
    SPMV_TRY(rp_at(A, sp[part], s, &a));
    SPMV_TRY(rp_at(A, sp[part + 1], s, &b));
    int64_t S = 0;
    for (int k = 0; k < nparts; ++k) S = std::max(S, sp[k + 1] - sp[k]);
    if (rows) *rows = sp[part + 1] - sp[part];
    if (nnz) *nnz = b - a;
    if (slot) *slot = S;
    return SPMV_OK;
}

spmv_status slice_remap_impl(spmv_ctx *ctx, const spmv_csr *A, const int64_t *sp, int nparts, int part,
                             cudaStream_t s, int32_t *rp_out, int32_t *col_out, void *val_out) {
    int64_t rows = 0, nnz = 0, S = 0;
    SPMV_TRY(slice_size_impl(ctx, A, sp, nparts, part, s, &rows, &nnz, &S));
    if (nnz > INT32_MAX || (int64_t)nparts * S > (int64_t)INT32_MAX + 1) {
        set_error("shard exceeds int32 indices");
        return SPMV_ERR_SIZE;
    }
    if (nnz > 0 && (!col_out || !val_out)) { set_error("NULL col/val out"); return SPMV_ERR_INVALID_ARG; }
    int64_t k0 = 0;
    SPMV_TRY(rp_at(A, sp[part], s, &k0));
    const int g = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div<int64_t>(rows + 1, 256), ctx->sm_count * 8));
    if (A->ptr_type == SPMV_I32)
        k_rebase<int><<<g, 256, 0, s>>>((const int *)A->row_ptr, sp[part], rows, rp_out);
    else
        k_rebase<int64_t><<<g, 256, 0, s>>>((const int64_t *)A->row_ptr, sp[part], rows, rp_out);
    SPMV_LAUNCH_CHECK();
    if (nnz > 0) {
        Splits spl{};
        for (int k = 0; k <= nparts; ++k) spl.s[k] = sp[k];
        spl.nparts = nparts;
        spl.slot = S;
        const int g2 = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div<int64_t>(nnz, 256), ctx->sm_count * 16));
        k_remap<<<g2, 256, 0, s>>>(A->col_idx, k0, nnz, spl, col_out);
        SPMV_LAUNCH_CHECK();
        const size_t V = A->dtype == SPMV_F64 ? 8 : 4;
        SPMV_CUDA_TRY(cudaMemcpyAsync(val_out, (const char *)A->vals + k0 * V, nnz * V, cudaMemcpyDeviceToDevice, s));
    }
    return SPMV_OK;
}

}  // namespace spmv
