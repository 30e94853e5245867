// partition.cu -- nnz-balanced multi-GPU row partition (north_star):
// row splits at merge-path diagonals floor(k*(n_rows+nnz)/P) (same path as the
// merge-based CSR of PAPER.md:103, A7), and the shard extraction that remaps
// columns to slots of the all-gathered x.
#include <algorithm>
#include <vector>

#include "internal.h"
#include "scan.h"

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

// ---- compressed exchange
__global__ void k_mark_used(const int *col, int64_t nnz, unsigned char *used) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nnz; k += (int64_t)gridDim.x * blockDim.x)
        used[__ldg(col + k)] = 1;                 // benign race: every writer stores 1
}
// halo: columns referenced by the rows [rp[r0], rp[r1]) of one part, outside its own range
__global__ void k_mark_foreign(const int *col, int64_t k0, int64_t k1, int64_t c0, int64_t c1, unsigned char *used) {
    for (int64_t k = k0 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < k1; k += (int64_t)gridDim.x * blockDim.x) {
        const int64_t j = __ldg(col + k);
        if (j < c0 || j >= c1) used[j] = 1;       // benign race: every writer stores 1
    }
}
__global__ void k_used_to_i64(const unsigned char *used, int64_t n, int64_t *out) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x)
        out[j] = used[j];
}
__global__ void k_colmap(const unsigned char *used, const int64_t *prefix, int64_t n, Splits sp, int *colmap) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
        if (!used[j]) { colmap[j] = -1; continue; }
        int lo = 0, hi = sp.nparts - 1;           // owner = last k with s[k] <= j
        while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (sp.s[mid] <= j) lo = mid; else hi = mid - 1;
        }
        colmap[j] = (int)(lo * sp.slot + (prefix[j] - prefix[sp.s[lo]]));
    }
}
__global__ void k_remap_colmap(const int *col, int64_t k0, int64_t cnt, const int *colmap, int *out) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < cnt; k += (int64_t)gridDim.x * blockDim.x)
        out[k] = colmap[col[k0 + k]];
}
__global__ void k_pack_index(const int *colmap, int64_t r0, int64_t r1, int64_t base, int *idx,
                             unsigned long long *count) {
    for (int64_t j = r0 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < r1; j += (int64_t)gridDim.x * blockDim.x) {
        const int c = colmap[j];
        if (c >= 0) {
            idx[c - base] = (int)(j - r0);
            atomicAdd(count, 1ull);
        }
    }
}
template <typename V>
__global__ void k_gather(const V *src, const int *idx, int64_t n, V *dst) {
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < n; q += (int64_t)gridDim.x * blockDim.x)
        dst[q] = src[__ldg(idx + q)];
}
template <typename V>
__global__ void k_scatter(const V *src, const int *idx, int64_t n, V *dst) {
    for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < n; q += (int64_t)gridDim.x * blockDim.x)
        dst[__ldg(idx + q)] = src[q];
}

// compressed rows (A33): flag[r] = row r has a nonzero; then rows_out[pos[r]] = r and
// rp_out[pos[r]] = rp[r] for those rows, rp_out[count] = rp[n]
template <typename IT>
__global__ void k_nonempty(const IT *rp, int64_t n, int64_t *flag) {
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x)
        flag[r] = (int64_t)rp[r + 1] > (int64_t)rp[r] ? 1 : 0;
}
template <typename IT>
__global__ void k_compress_rows(const IT *rp, int64_t n, const int64_t *pos, int32_t *rows_out, IT *rp_out) {
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r <= n; r += (int64_t)gridDim.x * blockDim.x) {
        if (r == n) {
            rp_out[pos[n]] = rp[n];
        } else if ((int64_t)rp[r + 1] > (int64_t)rp[r]) {
            rows_out[pos[r]] = (int32_t)r;
            rp_out[pos[r]] = rp[r];
        }
    }
}

// own / foreign split of a shard
template <typename IT>
__global__ void k_split_count(const IT *rp, const int *col, int64_t r0, int64_t rows, int64_t c0, int64_t c1,
                              int which, int64_t *cnt) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < rows; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t c = 0;
        for (int64_t k = rp[r0 + i]; k < (int64_t)rp[r0 + i + 1]; ++k) {
            const int64_t j = col[k];
            const bool own = j >= c0 && j < c1;
            c += (which == 0) == own;
        }
        cnt[i] = c;
    }
}
__global__ void k_i64_to_i32(const int64_t *in, int64_t n, int *out) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = (int)in[i];
}
template <typename IT, typename V>
__global__ void k_split_fill(const IT *rp, const int *col, const V *val, int64_t r0, int64_t rows, int64_t c0,
                             int64_t c1, int which, Splits sp, const int *colmap, const int *rp_out, int *col_out,
                             V *val_out) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < rows; i += (int64_t)gridDim.x * blockDim.x) {
        int64_t q = rp_out[i];
        for (int64_t k = rp[r0 + i]; k < (int64_t)rp[r0 + i + 1]; ++k) {
            const int64_t j = col[k];
            const bool own = j >= c0 && j < c1;
            if ((which == 0) != own) continue;
            int slot;
            if (which == 0) {
                slot = (int)(j - c0);
            } else if (colmap) {
                slot = colmap[j];
            } else {
                int lo = 0, hi = sp.nparts - 1;
                while (lo < hi) {
                    const int mid = (lo + hi + 1) >> 1;
                    if (sp.s[mid] <= j) lo = mid; else hi = mid - 1;
                }
                slot = (int)(lo * sp.slot + (j - sp.s[lo]));
            }
            col_out[q] = slot;
            val_out[q] = val[k];
            ++q;
        }
    }
}

int blocks_for(const spmv_ctx *ctx, int64_t n) {
    return (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div<int64_t>(n, 256), (int64_t)ctx->sm_count * 16));
}

}  // namespace

spmv_status colmap_impl(spmv_ctx *ctx, const spmv_csr *A, const int64_t *sp, int nparts, cudaStream_t s,
                        int32_t *colmap, int64_t *slot) {
    SPMV_TRY(check_splits(A, sp, nparts));
    const int64_t n = A->n_cols;
    Scratch used(ctx, s), u64(ctx, s), prefix(ctx, s);
    SPMV_TRY(used.alloc(std::max<int64_t>(n, 1)));
    SPMV_TRY(u64.alloc(std::max<int64_t>(n, 1) * 8));
    SPMV_TRY(prefix.alloc((n + 1) * 8));
    SPMV_CUDA_TRY(cudaMemsetAsync(used.p, 0, std::max<int64_t>(n, 1), s));
    if (A->nnz) {
        k_mark_used<<<blocks_for(ctx, A->nnz), 256, 0, s>>>(A->col_idx, A->nnz, used.as<unsigned char>());
        SPMV_LAUNCH_CHECK();
    }
    if (n) {
        k_used_to_i64<<<blocks_for(ctx, n), 256, 0, s>>>(used.as<unsigned char>(), n, u64.as<int64_t>());
        SPMV_LAUNCH_CHECK();
    }
    SPMV_TRY(exclusive_scan_i64(ctx, u64.as<int64_t>(), prefix.as<int64_t>(), n, s));
    std::vector<int64_t> at(nparts + 1);
    for (int k = 0; k <= nparts; ++k)
        SPMV_CUDA_TRY(cudaMemcpyAsync(&at[k], prefix.as<int64_t>() + sp[k], 8, cudaMemcpyDeviceToHost, s));
    SPMV_CUDA_TRY(cudaStreamSynchronize(s));
    int64_t S = 0;
    for (int k = 0; k < nparts; ++k) S = std::max(S, at[k + 1] - at[k]);
    if ((int64_t)nparts * S > (int64_t)INT32_MAX) { set_error("compressed slots exceed int32"); return SPMV_ERR_SIZE; }
    Splits spl{};
    for (int k = 0; k <= nparts; ++k) spl.s[k] = sp[k];
    spl.nparts = nparts;
    spl.slot = S;
    if (n) {
        k_colmap<<<blocks_for(ctx, n), 256, 0, s>>>(used.as<unsigned char>(), prefix.as<int64_t>(), n, spl, colmap);
        SPMV_LAUNCH_CHECK();
    }
    *slot = S;
    return SPMV_OK;
}

spmv_status halo_colmap_impl(spmv_ctx *ctx, const spmv_csr *A, const int64_t *sp, int nparts, int part,
                             cudaStream_t s, int32_t *colmap, int64_t *counts, int64_t *slot) {
    SPMV_TRY(check_splits(A, sp, nparts));
    const int64_t n = A->n_cols;
    Scratch used(ctx, s), u64(ctx, s), prefix(ctx, s);
    SPMV_TRY(used.alloc(std::max<int64_t>(n, 1)));
    SPMV_TRY(u64.alloc(std::max<int64_t>(n, 1) * 8));
    SPMV_TRY(prefix.alloc((n + 1) * 8));
    SPMV_CUDA_TRY(cudaMemsetAsync(used.p, 0, std::max<int64_t>(n, 1), s));
    int64_t k0 = 0, k1 = 0;
    SPMV_TRY(rp_at(A, sp[part], s, &k0));
    SPMV_TRY(rp_at(A, sp[part + 1], s, &k1));
    if (k1 > k0) {
        k_mark_foreign<<<blocks_for(ctx, k1 - k0), 256, 0, s>>>(A->col_idx, k0, k1, sp[part], sp[part + 1],
                                                               used.as<unsigned char>());
        SPMV_LAUNCH_CHECK();
    }
    if (n) {
        k_used_to_i64<<<blocks_for(ctx, n), 256, 0, s>>>(used.as<unsigned char>(), n, u64.as<int64_t>());
        SPMV_LAUNCH_CHECK();
    }
    SPMV_TRY(exclusive_scan_i64(ctx, u64.as<int64_t>(), prefix.as<int64_t>(), n, s));
    std::vector<int64_t> at(nparts + 1);
    for (int k = 0; k <= nparts; ++k)
        SPMV_CUDA_TRY(cudaMemcpyAsync(&at[k], prefix.as<int64_t>() + sp[k], 8, cudaMemcpyDeviceToHost, s));
    SPMV_CUDA_TRY(cudaStreamSynchronize(s));
    int64_t S = 1;
    for (int k = 0; k < nparts; ++k) {
        counts[k] = at[k + 1] - at[k];
        S = std::max(S, counts[k]);
    }
    if ((int64_t)nparts * S > (int64_t)INT32_MAX) { set_error("halo slots exceed int32"); return SPMV_ERR_SIZE; }
    Splits spl{};
    for (int k = 0; k <= nparts; ++k) spl.s[k] = sp[k];
    spl.nparts = nparts;
    spl.slot = S;
    if (n) {
        k_colmap<<<blocks_for(ctx, n), 256, 0, s>>>(used.as<unsigned char>(), prefix.as<int64_t>(), n, spl, colmap);
        SPMV_LAUNCH_CHECK();
    }
    *slot = S;
    return SPMV_OK;
}

spmv_status slice_remap_colmap_impl(spmv_ctx *ctx, const spmv_csr *A, const int64_t *sp, int nparts, int part,
                                    const int32_t *colmap, cudaStream_t s, int32_t *rp_out, int32_t *col_out,
                                    void *val_out) {
    int64_t rows = 0, nnz = 0, S = 0;
    SPMV_TRY(slice_size_impl(ctx, A, sp, nparts, part, s, &rows, &nnz, &S));
    if (nnz > INT32_MAX) { set_error("shard exceeds int32 indices"); return SPMV_ERR_SIZE; }
    if (nnz > 0 && (!col_out || !val_out)) { set_error("NULL col/val out"); return SPMV_ERR_INVALID_ARG; }
    int64_t k0 = 0;
    SPMV_TRY(rp_at(A, sp[part], s, &k0));
    if (A->ptr_type == SPMV_I32)
        k_rebase<int><<<blocks_for(ctx, rows + 1), 256, 0, s>>>((const int *)A->row_ptr, sp[part], rows, rp_out);
    else
        k_rebase<int64_t><<<blocks_for(ctx, rows + 1), 256, 0, s>>>((const int64_t *)A->row_ptr, sp[part], rows, rp_out);
    SPMV_LAUNCH_CHECK();
    if (nnz > 0) {
        k_remap_colmap<<<blocks_for(ctx, nnz), 256, 0, s>>>(A->col_idx, k0, nnz, colmap, col_out);
        SPMV_LAUNCH_CHECK();
        const size_t V = A->dtype == SPMV_F64 ? 8 : 4;
        SPMV_CUDA_TRY(cudaMemcpyAsync(val_out, (const char *)A->vals + k0 * V, nnz * V, cudaMemcpyDeviceToDevice, s));
    }
    return SPMV_OK;
}

spmv_status pack_index_impl(spmv_ctx *ctx, const int32_t *colmap, const int64_t *sp, int nparts, int part,
                            int64_t slot, cudaStream_t s, int32_t *idx, int64_t *count) {
    Scratch cnt(ctx, s);
    SPMV_TRY(cnt.alloc(8));
    SPMV_CUDA_TRY(cudaMemsetAsync(cnt.p, 0, 8, s));
    const int64_t r0 = sp[part], r1 = sp[part + 1];
    if (r1 > r0) {
        k_pack_index<<<blocks_for(ctx, r1 - r0), 256, 0, s>>>(colmap, r0, r1, (int64_t)part * slot, idx,
                                                             cnt.as<unsigned long long>());
        SPMV_LAUNCH_CHECK();
    }
    unsigned long long c = 0;
    SPMV_CUDA_TRY(cudaMemcpyAsync(&c, cnt.p, 8, cudaMemcpyDeviceToHost, s));
    SPMV_CUDA_TRY(cudaStreamSynchronize(s));
    *count = (int64_t)c;
    (void)nparts;
    return SPMV_OK;
}

spmv_status gather_impl(spmv_ctx *ctx, spmv_dtype dt, const void *src, const int32_t *idx, int64_t n, void *dst,
                        cudaStream_t s) {
    if (n <= 0) return SPMV_OK;
    if (dt == SPMV_F64) k_gather<double><<<blocks_for(ctx, n), 256, 0, s>>>((const double *)src, idx, n, (double *)dst);
    else k_gather<float><<<blocks_for(ctx, n), 256, 0, s>>>((const float *)src, idx, n, (float *)dst);
    SPMV_LAUNCH_CHECK();
    return SPMV_OK;
}

spmv_status scatter_impl(spmv_ctx *ctx, spmv_dtype dt, const void *src, const int32_t *idx, int64_t n, void *dst,
                         cudaStream_t s) {
    if (n <= 0) return SPMV_OK;
    if (dt == SPMV_F64) k_scatter<double><<<blocks_for(ctx, n), 256, 0, s>>>((const double *)src, idx, n, (double *)dst);
    else k_scatter<float><<<blocks_for(ctx, n), 256, 0, s>>>((const float *)src, idx, n, (float *)dst);
    SPMV_LAUNCH_CHECK();
    return SPMV_OK;
}

template <typename IT>
spmv_status compress_rows_t(spmv_ctx *ctx, const spmv_csr *A, cudaStream_t s, int32_t *rows_out, void *rp_out,
                            int64_t *count) {
    const int64_t n = A->n_rows;
    const IT *rp = (const IT *)A->row_ptr;
    Scratch flag(ctx, s), pos(ctx, s);
    SPMV_TRY(flag.alloc(std::max<int64_t>(n, 1) * 8));
    SPMV_TRY(pos.alloc((n + 1) * 8));
    if (n) {
        k_nonempty<IT><<<blocks_for(ctx, n), 256, 0, s>>>(rp, n, flag.as<int64_t>());
        SPMV_LAUNCH_CHECK();
    }
    SPMV_TRY(exclusive_scan_i64(ctx, flag.as<int64_t>(), pos.as<int64_t>(), n, s));
    k_compress_rows<IT><<<blocks_for(ctx, n + 1), 256, 0, s>>>(rp, n, pos.as<int64_t>(), rows_out, (IT *)rp_out);
    SPMV_LAUNCH_CHECK();
    SPMV_CUDA_TRY(cudaMemcpyAsync(count, pos.as<int64_t>() + n, 8, cudaMemcpyDeviceToHost, s));
    SPMV_CUDA_TRY(cudaStreamSynchronize(s));
    return SPMV_OK;
}

spmv_status compress_rows_impl(spmv_ctx *ctx, const spmv_csr *A, cudaStream_t s, int32_t *rows_out, void *rp_out,
                               int64_t *count) {
    if (A->ptr_type == SPMV_I32) return compress_rows_t<int>(ctx, A, s, rows_out, rp_out, count);
    return compress_rows_t<int64_t>(ctx, A, s, rows_out, rp_out, count);
}

template <typename IT, typename V>
spmv_status split_t(spmv_ctx *ctx, const spmv_csr *A, const int64_t *sp, int nparts, int part, const int32_t *colmap,
                    int which, cudaStream_t s, int32_t *rp_out, int32_t *col_out, void *val_out, int64_t *nnz_out) {
    const int64_t r0 = sp[part], rows = sp[part + 1] - sp[part];
    const IT *rp = (const IT *)A->row_ptr;
    Scratch cnt(ctx, s), off(ctx, s);
    SPMV_TRY(cnt.alloc(std::max<int64_t>(rows, 1) * 8));
    SPMV_TRY(off.alloc((rows + 1) * 8));
    if (rows) {
        k_split_count<IT><<<blocks_for(ctx, rows), 256, 0, s>>>(rp, A->col_idx, r0, rows, sp[part], sp[part + 1],
                                                                which, cnt.as<int64_t>());
        SPMV_LAUNCH_CHECK();
    }
    SPMV_TRY(exclusive_scan_i64(ctx, cnt.as<int64_t>(), off.as<int64_t>(), rows, s));
    int64_t nnz = 0;
    SPMV_CUDA_TRY(cudaMemcpyAsync(&nnz, off.as<int64_t>() + rows, 8, cudaMemcpyDeviceToHost, s));
    SPMV_CUDA_TRY(cudaStreamSynchronize(s));
    if (nnz > INT32_MAX) { set_error("split block exceeds int32 indices"); return SPMV_ERR_SIZE; }
    k_i64_to_i32<<<blocks_for(ctx, rows + 1), 256, 0, s>>>(off.as<int64_t>(), rows + 1, rp_out);
    SPMV_LAUNCH_CHECK();
    *nnz_out = nnz;
    if (!col_out || !val_out || nnz == 0 || rows == 0) return SPMV_OK;
    Splits spl{};
    int64_t S = 0;
    for (int k = 0; k <= nparts; ++k) spl.s[k] = sp[k];
    for (int k = 0; k < nparts; ++k) S = std::max(S, sp[k + 1] - sp[k]);
    spl.nparts = nparts;
    spl.slot = S;
    k_split_fill<IT, V><<<blocks_for(ctx, rows), 256, 0, s>>>(rp, A->col_idx, (const V *)A->vals, r0, rows, sp[part],
                                                              sp[part + 1], which, spl, colmap, rp_out, col_out,
                                                              (V *)val_out);
    SPMV_LAUNCH_CHECK();
    return SPMV_OK;
}

spmv_status split_impl(spmv_ctx *ctx, const spmv_csr *A, const int64_t *sp, int nparts, int part,
                       const int32_t *colmap, int which, cudaStream_t s, int32_t *rp_out, int32_t *col_out,
                       void *val_out, int64_t *nnz_out) {
    SPMV_TRY(check_splits(A, sp, nparts));
    const bool i32 = A->ptr_type == SPMV_I32, f64 = A->dtype == SPMV_F64;
    if (i32 && f64) return split_t<int, double>(ctx, A, sp, nparts, part, colmap, which, s, rp_out, col_out, val_out, nnz_out);
    if (i32) return split_t<int, float>(ctx, A, sp, nparts, part, colmap, which, s, rp_out, col_out, val_out, nnz_out);
    if (f64) return split_t<int64_t, double>(ctx, A, sp, nparts, part, colmap, which, s, rp_out, col_out, val_out, nnz_out);
    return split_t<int64_t, float>(ctx, A, sp, nparts, part, colmap, which, s, rp_out, col_out, val_out, nnz_out);
}

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
