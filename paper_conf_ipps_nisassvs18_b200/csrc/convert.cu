// convert.cu -- CSR -> {COO, ELL, HYB, merge-path partition, CSR5 tiles}
// (§II-A; layouts DESIGN.md §4, readings A1-A7).
//
// COO/ELL/HYB are written by one balanced "walk": thread t takes a fixed-length
// slice of the merge path of row ends and nonzeros (the same decomposition the
// merge-based SpMV uses), so long and short rows cost the same.
#include <algorithm>
#include <climits>

#include <cstdint>

#include "internal.h"
#include "kernels.h"
#include "scan.h"

namespace spmv {

namespace {

constexpr int kT = 256;
constexpr int kWalkItems = 16;

template <typename ITI, typename ITO>
__global__ void k_cast_rowptr(const ITI *in, ITO *out, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = (ITO)in[i];
}

// generic walk over merge-path slices: op(row, k, j_in_row) for every nonzero k
template <typename IT, typename Op>
__global__ void __launch_bounds__(kT) k_walk(const IT *__restrict__ rp, int64_t n, int64_t nnz, Op op) {
    int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x;
    int64_t total = n + nnz;
    int64_t d0 = t * kWalkItems;
    if (d0 >= total) return;
    int64_t d1 = d0 + kWalkItems < total ? d0 + kWalkItems : total;
    int64_t i = merge_path_row(rp, n, nnz, d0);
    int64_t k = d0 - i;
    int64_t row_start = i < n ? (int64_t)rp[i] : nnz;
    int64_t row_end = i < n ? (int64_t)rp[i + 1] : nnz;
    for (int64_t d = d0; d < d1; ++d) {
        if (i < n && row_end <= k) {          // consume a row end (A7 tie-break)
            ++i;
            row_start = row_end;
            row_end = i < n ? (int64_t)rp[i + 1] : nnz;
        } else {
            op(i, k, k - row_start);
            ++k;
        }
    }
}

struct OpCoo {
    int *row;
    __device__ void operator()(int64_t r, int64_t k, int64_t) const { row[k] = (int)r; }
};

template <typename V>
struct OpEll {
    const int *col; const V *val; int *ecol; V *eval; int64_t ld;
    __device__ void operator()(int64_t r, int64_t k, int64_t j) const {
        ecol[j * ld + r] = col[k];
        eval[j * ld + r] = val[k];
    }
};

template <typename V>
struct OpHyb {
    const int *col; const V *val; int *ecol; V *eval; int64_t ld, kh;
    const int64_t *coo_off; int *crow; int *ccol; V *cval;
    __device__ void operator()(int64_t r, int64_t k, int64_t j) const {
        if (j < kh) {
            ecol[j * ld + r] = col[k];
            eval[j * ld + r] = val[k];
        } else {
            int64_t c = coo_off[r] + (j - kh);
            crow[c] = (int)r;
            ccol[c] = col[k];
            cval[c] = val[k];
        }
    }
};

template <typename IT>
__global__ void k_hyb_overflow(const IT *rp, int64_t n, int64_t kh, int64_t *cnt) {
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
        int64_t len = (int64_t)rp[r + 1] - (int64_t)rp[r];
        cnt[r] = len > kh ? len - kh : 0;
    }
}

// CSR long-row split (A25): rows longer than 2C become ceil(len/C) chunks of C nonzeros
template <typename IT>
__global__ void k_chunk_count(const IT *rp, int64_t n, int64_t C, int64_t *cnt) {
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
        const int64_t len = (int64_t)rp[r + 1] - (int64_t)rp[r];
        cnt[r] = len > 2 * C ? (len + C - 1) / C : 0;
    }
}
template <typename IT>
__global__ void k_chunk_fill(const IT *rp, int64_t n, int64_t C, const int64_t *off, int64_t *crow, int64_t *clo) {
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
        const int64_t a = rp[r], len = (int64_t)rp[r + 1] - a;
        if (len <= 2 * C) continue;
        const int64_t o = off[r], m = (len + C - 1) / C;
        for (int64_t j = 0; j < m; ++j) { crow[o + j] = r; clo[o + j] = a + j * C; }
    }
}

// merge-path tile coordinates at diagonals min(t*T, n+nnz) (A7)
template <typename IT>
__global__ void k_merge_coords(const IT *rp, int64_t n, int64_t nnz, int64_t T, int64_t tiles,
                               int64_t *crow, int64_t *cnz) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t <= tiles; t += (int64_t)gridDim.x * blockDim.x) {
        int64_t d = t * T < n + nnz ? t * T : n + nnz;
        int64_t i = merge_path_row(rp, n, nnz, d);
        crow[t] = i;
        cnz[t] = d - i;
    }
}

// merge tile class (A28): 1 = row-sum tile -- fewer than kMergeLeanRows row ends and
// every in-tile row part (row r1's included) <= kMergeLeanLen nonzeros.  Row i's part
// is clip(rp[i+1]) - clip(rp[i]), clip to the tile's nonzero range [k0, k1].
template <typename IT>
__global__ void k_merge_class(const IT *rp, int64_t n, const int64_t *crow, const int64_t *cnz, int64_t tiles,
                              unsigned char *cls) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < tiles; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r0 = crow[t], r1 = crow[t + 1], k0 = cnz[t], k1 = cnz[t + 1];
        bool ok = r1 - r0 < kMergeLeanRows;
        int64_t lo = k0;                                  // clip(rp[r0]) = k0 (A7: rp[r0] <= k0)
        for (int64_t i = r0; ok && i <= r1; ++i) {
            int64_t hi = i < n ? (int64_t)rp[i + 1] : k1;
            hi = hi < k0 ? k0 : hi > k1 ? k1 : hi;
            ok = hi - lo <= kMergeLeanLen;
            lo = hi;
        }
        cls[t] = ok ? 1 : 0;
    }
}
__global__ void k_u8_to_i64(const unsigned char *a, int64_t n, int64_t *b) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        b[i] = a[i] != 0;
}
// stable partition of the tile ids by class (class 1 first); pre = exclusive prefix
// count of class-1 tiles, nl = their total
__global__ void k_merge_order(const unsigned char *cls, const int64_t *pre, int64_t tiles, int64_t nl, int *order) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < tiles; t += (int64_t)gridDim.x * blockDim.x)
        order[cls[t] ? pre[t] : nl + (t - pre[t])] = (int)t;
}

// ---- CSR5 (encoding A6) -----------------------------------

template <typename IT>
__global__ void k_rowstart_bits(const IT *rp, int64_t n, unsigned *bits) {
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
        int64_t a = rp[r], b = rp[r + 1];
        if (b > a) atomicOr(&bits[a >> 5], 1u << (a & 31));
    }
}

// one warp per tile: bit_flag / y_offset / seg_offset per lane, tile_ptr, row_lo
template <typename IT>
__global__ void __launch_bounds__(kT)
k_csr5_desc(const IT *rp, int64_t n, int64_t nnz, int sigma, int64_t n_tiles, int64_t n_words,
            const unsigned *bits, unsigned *desc, int64_t *tile_ptr, int64_t *row_lo, int64_t *segs) {
    const int lane = threadIdx.x & 31;
    const int64_t W = 32 * (int64_t)sigma;
    int64_t t = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    if (t > n_tiles) return;
    if (lane == 0) {
        int64_t e = t * W;
        tile_ptr[t] = e < nnz ? upper_bound_rp(rp, n, e) - 1 : n;
        row_lo[t] = lower_bound_rp(rp, n, e);
    }
    if (t == n_tiles) return;                          // warp-uniform
    int64_t e0 = t * W + (int64_t)lane * sigma;
    int64_t w0 = e0 >> 5;
    unsigned long long win = bits[w0];
    if (w0 + 1 < n_words) win |= (unsigned long long)bits[w0 + 1] << 32;
    unsigned flag = (unsigned)(win >> (e0 & 31)) & ((1u << sigma) - 1u);
    unsigned pc = __popc(flag);
    unsigned incl = pc;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        unsigned v = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += v;
    }
    unsigned y_off = incl - pc;
    unsigned fb = __ballot_sync(0xffffffffu, flag != 0u);
    unsigned later = lane == 31 ? 0u : (fb & ~((2u << lane) - 1u));
    unsigned seg = later ? (unsigned)(__ffs(later) - 1 - lane - 1) : (unsigned)(31 - lane);
    desc[t * 32 + lane] = flag | (y_off << 16) | (seg << 25);
    unsigned total = __shfl_sync(0xffffffffu, incl, 31);
    if (lane == 0) segs[t] = total;
}

// tiles whose emitted row range [row_lo[t], row_lo[t+1]) holds an empty row need a map
__global__ void k_csr5_map_count(const int64_t *row_lo, const int64_t *segs, int64_t n_tiles, int64_t *cnt) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n_tiles; t += (int64_t)gridDim.x * blockDim.x)
        cnt[t] = (row_lo[t + 1] - row_lo[t] != segs[t]) ? segs[t] : 0;
}

template <typename IT>
__global__ void __launch_bounds__(kT)
k_csr5_map_fill(const IT *rp, const int64_t *row_lo, const int64_t *cnt, const int64_t *off, int64_t n_tiles,
                int64_t *map_off, int64_t *seg_map) {
    const int lane = threadIdx.x & 31;
    int64_t t = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    if (t >= n_tiles) return;
    if (cnt[t] == 0) {
        if (lane == 0) map_off[t] = -1;
        return;
    }
    int64_t o = off[t];
    if (lane == 0) map_off[t] = o;
    for (int64_t r0 = row_lo[t]; r0 < row_lo[t + 1]; r0 += 32) {
        int64_t r = r0 + lane;
        bool ne = r < row_lo[t + 1] && (int64_t)rp[r + 1] > (int64_t)rp[r];
        unsigned b = __ballot_sync(0xffffffffu, ne);
        if (ne) seg_map[o + __popc(b & ((1u << lane) - 1u))] = r;
        o += __popc(b);
    }
}

// lane-interleaved copy: element e = t*W + l*sigma + s -> t*W + (s/v)*32*v + l*v + s%v
template <typename T>
__global__ void k_csr5_permute(const T *in, T *out, int64_t full, int sigma, int v) {
    const int64_t W = 32 * (int64_t)sigma;
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < full; e += (int64_t)gridDim.x * blockDim.x) {
        int64_t t = e / W;
        int rem = (int)(e - t * W);
        int l = rem / sigma, s = rem - l * sigma;
        out[t * W + (int64_t)(s / v) * 32 * v + l * v + (s % v)] = in[e];
    }
}

int grid_cap(const spmv_ctx *ctx, int64_t work) {
    int64_t g = ceil_div<int64_t>(work, kT);
    int64_t cap = (int64_t)ctx->sm_count * 16;
    return (int)std::max<int64_t>(1, std::min(g, cap));
}

// Handle arrays carry kArrayPad bytes of slack so that vector loads of a lane chunk
// shifted to 16-byte alignment (merge kernel) never leave the allocation.
constexpr size_t kArrayPad = 64;

spmv_status arr_alloc(spmv_handle *h, int id, size_t bytes, cudaStream_t s) {
    DevArray &a = h->arr[id];
    a.bytes = bytes;
    a.owned = true;
    if (bytes == 0) { a.p = nullptr; return SPMV_OK; }
    SPMV_TRY(dev_alloc(h->ctx, bytes + kArrayPad, s, &a.p));
    SPMV_CUDA_TRY(cudaMemsetAsync((char *)a.p + bytes, 0, kArrayPad, s));
    return SPMV_OK;
}

template <typename IT, typename V>
spmv_status convert_t(spmv_ctx *ctx, spmv_format fmt, const spmv_csr *A, const spmv_convert_opts *o,
                      cudaStream_t s, spmv_handle *h, const FeatureSums &fs, int64_t cusp) {
    const int64_t n = A->n_rows, nnz = A->nnz;
    const size_t VB = sizeof(V);
    const int *col = A->col_idx;
    const V *val = reinterpret_cast<const V *>(A->vals);
    h->itype = sizeof(IT) == 4 ? SPMV_I32 : SPMV_I64;

    // the handle's row_ptr in its own index type (needed by every format's conversion)
    const IT *rp = nullptr;
    Scratch rp_tmp(ctx, s);
    const bool same_type = (A->ptr_type == SPMV_I32) == (sizeof(IT) == 4);
    const bool keeps_rowptr = fmt == SPMV_CSR || fmt == SPMV_CSR_SCALAR || fmt == SPMV_MERGE || fmt == SPMV_CSR5;
    if (same_type && (o->alias_input || !keeps_rowptr)) {
        rp = reinterpret_cast<const IT *>(A->row_ptr);
        if (keeps_rowptr) {
            h->arr[SPMV_ARR_ROW_PTR] = DevArray{const_cast<void *>(A->row_ptr), (size_t)(n + 1) * sizeof(IT), false};
        }
    } else {
        IT *dst;
        if (keeps_rowptr) {
            SPMV_TRY(arr_alloc(h, SPMV_ARR_ROW_PTR, (n + 1) * sizeof(IT), s));
            dst = reinterpret_cast<IT *>(h->arr[SPMV_ARR_ROW_PTR].p);
        } else {
            SPMV_TRY(rp_tmp.alloc((n + 1) * sizeof(IT)));
            dst = rp_tmp.as<IT>();
        }
        if (same_type) {
            SPMV_CUDA_TRY(cudaMemcpyAsync(dst, A->row_ptr, (n + 1) * sizeof(IT), cudaMemcpyDeviceToDevice, s));
        } else if (A->ptr_type == SPMV_I32) {
            k_cast_rowptr<int, IT><<<grid_cap(ctx, n + 1), kT, 0, s>>>((const int *)A->row_ptr, dst, n + 1);
            SPMV_LAUNCH_CHECK();
        } else {
            k_cast_rowptr<int64_t, IT><<<grid_cap(ctx, n + 1), kT, 0, s>>>((const int64_t *)A->row_ptr, dst, n + 1);
            SPMV_LAUNCH_CHECK();
        }
        rp = dst;
    }

    auto copy_colval = [&](bool alias) -> spmv_status {
        if (alias) {
            h->arr[SPMV_ARR_COL] = DevArray{const_cast<int *>(col), (size_t)nnz * 4, false};
            h->arr[SPMV_ARR_VAL] = DevArray{const_cast<V *>(val), (size_t)nnz * VB, false};
            return SPMV_OK;
        }
        SPMV_TRY(arr_alloc(h, SPMV_ARR_COL, nnz * 4, s));
        SPMV_TRY(arr_alloc(h, SPMV_ARR_VAL, nnz * VB, s));
        if (nnz) {
            SPMV_CUDA_TRY(cudaMemcpyAsync(h->arr[SPMV_ARR_COL].p, col, nnz * 4, cudaMemcpyDeviceToDevice, s));
            SPMV_CUDA_TRY(cudaMemcpyAsync(h->arr[SPMV_ARR_VAL].p, val, nnz * VB, cudaMemcpyDeviceToDevice, s));
        }
        return SPMV_OK;
    };

    const int64_t walk_threads = ceil_div<int64_t>(n + nnz, kWalkItems);
    const unsigned walk_grid = (unsigned)std::max<int64_t>(1, ceil_div<int64_t>(walk_threads, kT));

    // size guard (A4): default min(1/2 free device memory, max(8x the CSR bytes, 64 MiB))
    size_t max_bytes = o->max_bytes;
    if (max_bytes == 0) {
        size_t fr = 0, tot = 0;
        SPMV_CUDA_TRY(cudaMemGetInfo(&fr, &tot));
        size_t csr_bytes = (size_t)nnz * (4 + VB) + (size_t)(n + 1) * sizeof(IT);
        max_bytes = std::min(fr / 2, std::max<size_t>(8 * csr_bytes, (size_t)64 << 20));
    }

    switch (fmt) {
    case SPMV_CSR:
    case SPMV_CSR_SCALAR: {
        SPMV_TRY(copy_colval(o->alias_input != 0));
        int64_t w = o->vector_width;
        if (w == 0) {   // A5: clamp(next_pow2(ceil(nnz_mu)), 2, 32)
            int64_t mu = n > 0 ? ceil_div<int64_t>(nnz, n) : 1;
            w = 2;
            while (w < mu && w < 32) w <<= 1;
        }
        h->vec_w = fmt == SPMV_CSR_SCALAR ? 1 : w;
        if (fmt == SPMV_CSR && o->csr_chunk >= 0) {
            // long rows (> 2C nonzeros) as C-nonzero chunks, one warp each, added by the fix-up (A25)
            const int64_t C = o->csr_chunk > 0 ? o->csr_chunk : kCsrChunk;
            h->csr_chunk = C;
            Scratch cnt(ctx, s), off(ctx, s);
            SPMV_TRY(cnt.alloc(std::max<int64_t>(n, 1) * 8));
            SPMV_TRY(off.alloc((n + 1) * 8));
            if (n) {
                k_chunk_count<IT><<<grid_cap(ctx, n), kT, 0, s>>>(rp, n, C, cnt.as<int64_t>());
                SPMV_LAUNCH_CHECK();
            }
            SPMV_TRY(exclusive_scan_i64(ctx, cnt.as<int64_t>(), off.as<int64_t>(), n, s));
            int64_t nch = 0;
            SPMV_CUDA_TRY(cudaMemcpyAsync(&nch, off.as<int64_t>() + n, 8, cudaMemcpyDeviceToHost, s));
            SPMV_CUDA_TRY(cudaStreamSynchronize(s));
            h->csr_chunks = nch;
            SPMV_TRY(arr_alloc(h, SPMV_ARR_CSR_CHUNK_ROW, nch * 8, s));
            SPMV_TRY(arr_alloc(h, SPMV_ARR_CSR_CHUNK_LO, nch * 8, s));
            if (nch) {
                k_chunk_fill<IT><<<grid_cap(ctx, n), kT, 0, s>>>(rp, n, C, off.as<int64_t>(),
                                                                  (int64_t *)h->arr[SPMV_ARR_CSR_CHUNK_ROW].p,
                                                                  (int64_t *)h->arr[SPMV_ARR_CSR_CHUNK_LO].p);
                SPMV_LAUNCH_CHECK();
            }
            h->n_carry = nch;
        }
        break;
    }
    case SPMV_COO: {
        // the COO kernel reads 32-byte lane chunks: alias only 32-byte aligned arrays
        const bool al32 = (((uintptr_t)col | (uintptr_t)val) & 31) == 0;
        SPMV_TRY(copy_colval(o->alias_input != 0 && al32));
        SPMV_TRY(arr_alloc(h, SPMV_ARR_COO_ROW, nnz * 4, s));
        if (nnz) {
            k_walk<IT><<<walk_grid, kT, 0, s>>>(rp, n, nnz, OpCoo{(int *)h->arr[SPMV_ARR_COO_ROW].p});
            SPMV_LAUNCH_CHECK();
        }
        h->n_carry = ceil_div<int64_t>(nnz, kCooItems);
        // persistent tiles for regular matrices in fp64 (no empty row, rows of at most 32;
        // spmv_kernels.cu k_coo PERSIST)
        h->coo_persist = sizeof(V) == 8 && fs.n_empty == 0 && fs.len_max <= 32 && n > 0;
        break;
    }
    case SPMV_ELL: {
        int64_t K = (int64_t)fs.len_max, ld = ceil_div<int64_t>(n, 32) * 32;
        unsigned __int128 need = (unsigned __int128)K * (unsigned __int128)ld * (4 + VB);
        if (need > (unsigned __int128)max_bytes || (unsigned __int128)K * ld > (unsigned __int128)INT64_MAX / 16) {
            set_error("ELL needs " + std::to_string((double)need) + " bytes > guard " + std::to_string(max_bytes) + " (A4)");
            return SPMV_ERR_SIZE;
        }
        h->ell_K = K;
        h->ell_ld = ld;
        SPMV_TRY(arr_alloc(h, SPMV_ARR_ELL_COL, K * ld * 4, s));
        SPMV_TRY(arr_alloc(h, SPMV_ARR_ELL_VAL, K * ld * VB, s));
        if (K * ld) {
            SPMV_CUDA_TRY(cudaMemsetAsync(h->arr[SPMV_ARR_ELL_COL].p, 0xFF, K * ld * 4, s));   // col = -1
            SPMV_CUDA_TRY(cudaMemsetAsync(h->arr[SPMV_ARR_ELL_VAL].p, 0, K * ld * VB, s));     // +0.0
        }
        if (nnz) {
            OpEll<V> op{col, val, (int *)h->arr[SPMV_ARR_ELL_COL].p, (V *)h->arr[SPMV_ARR_ELL_VAL].p, ld};
            k_walk<IT><<<walk_grid, kT, 0, s>>>(rp, n, nnz, op);
            SPMV_LAUNCH_CHECK();
        }
        break;
    }
    case SPMV_HYB: {
        int64_t kh;
        if (o->hyb_width >= 0) kh = o->hyb_width;
        else if (o->hyb_rule == 1) kh = n > 0 ? nnz / n : 0;
        else if (o->hyb_rule == 2) kh = cusp;
        else kh = n > 0 ? ceil_div<int64_t>(nnz, n) : 0;
        int64_t ld = ceil_div<int64_t>(n, 32) * 32;
        Scratch cnt(ctx, s), off(ctx, s);
        SPMV_TRY(cnt.alloc(std::max<int64_t>(n, 1) * 8));
        SPMV_TRY(off.alloc((n + 1) * 8));
        if (n) {
            k_hyb_overflow<IT><<<grid_cap(ctx, n), kT, 0, s>>>(rp, n, kh, cnt.as<int64_t>());
            SPMV_LAUNCH_CHECK();
        }
        SPMV_TRY(exclusive_scan_i64(ctx, cnt.as<int64_t>(), off.as<int64_t>(), n, s));
        int64_t ncoo = 0;
        SPMV_CUDA_TRY(cudaMemcpyAsync(&ncoo, off.as<int64_t>() + n, 8, cudaMemcpyDeviceToHost, s));
        SPMV_CUDA_TRY(cudaStreamSynchronize(s));
        unsigned __int128 need = (unsigned __int128)kh * ld * (4 + VB) + (unsigned __int128)ncoo * (8 + VB);
        if (need > (unsigned __int128)max_bytes) {
            set_error("HYB needs more bytes than the guard (A4)");
            return SPMV_ERR_SIZE;
        }
        h->ell_K = kh;
        h->ell_ld = ld;
        h->hyb_coo_nnz = ncoo;
        SPMV_TRY(arr_alloc(h, SPMV_ARR_ELL_COL, kh * ld * 4, s));
        SPMV_TRY(arr_alloc(h, SPMV_ARR_ELL_VAL, kh * ld * VB, s));
        SPMV_TRY(arr_alloc(h, SPMV_ARR_COO_ROW, ncoo * 4, s));
        SPMV_TRY(arr_alloc(h, SPMV_ARR_HYB_COO_COL, ncoo * 4, s));
        SPMV_TRY(arr_alloc(h, SPMV_ARR_HYB_COO_VAL, ncoo * VB, s));
        if (kh * ld) {
            SPMV_CUDA_TRY(cudaMemsetAsync(h->arr[SPMV_ARR_ELL_COL].p, 0xFF, kh * ld * 4, s));
            SPMV_CUDA_TRY(cudaMemsetAsync(h->arr[SPMV_ARR_ELL_VAL].p, 0, kh * ld * VB, s));
        }
        if (nnz) {
            OpHyb<V> op{col, val, (int *)h->arr[SPMV_ARR_ELL_COL].p, (V *)h->arr[SPMV_ARR_ELL_VAL].p, ld, kh,
                        off.as<int64_t>(), (int *)h->arr[SPMV_ARR_COO_ROW].p,
                        (int *)h->arr[SPMV_ARR_HYB_COO_COL].p, (V *)h->arr[SPMV_ARR_HYB_COO_VAL].p};
            k_walk<IT><<<walk_grid, kT, 0, s>>>(rp, n, nnz, op);
            SPMV_LAUNCH_CHECK();
        }
        h->n_carry = ceil_div<int64_t>(ncoo, kCooItems);
        break;
    }
    case SPMV_MERGE: {
        SPMV_TRY(copy_colval(false));   // padded copies: the kernel's shifted vector loads need the slack
        int64_t T = o->merge_items > 0 ? o->merge_items : kMergeItems;
        if (T != 128 && T != 256) {
            set_error("merge_items must be 128 or 256 (32 lanes x 4 or 8 items)");
            return SPMV_ERR_UNSUPPORTED;
        }
        int64_t tiles = ceil_div<int64_t>(n + nnz, T);
        if (tiles >= INT32_MAX) {   // the tile order is int32
            set_error("too many merge tiles");
            return SPMV_ERR_SIZE;
        }
        h->merge_T = T;
        h->merge_tiles = tiles;
        SPMV_TRY(arr_alloc(h, SPMV_ARR_MERGE_COORD_ROW, (tiles + 1) * 8, s));
        SPMV_TRY(arr_alloc(h, SPMV_ARR_MERGE_COORD_NZ, (tiles + 1) * 8, s));
        k_merge_coords<IT><<<grid_cap(ctx, tiles + 1), kT, 0, s>>>(
            rp, n, nnz, T, tiles, (int64_t *)h->arr[SPMV_ARR_MERGE_COORD_ROW].p,
            (int64_t *)h->arr[SPMV_ARR_MERGE_COORD_NZ].p);
        SPMV_LAUNCH_CHECK();
        SPMV_TRY(arr_alloc(h, SPMV_ARR_MERGE_TILE_CLASS, tiles, s));
        h->merge_lean = 0;
        if (tiles > 0) {
            k_merge_class<IT><<<grid_cap(ctx, tiles), kT, 0, s>>>(
                rp, n, (const int64_t *)h->arr[SPMV_ARR_MERGE_COORD_ROW].p,
                (const int64_t *)h->arr[SPMV_ARR_MERGE_COORD_NZ].p, tiles,
                (unsigned char *)h->arr[SPMV_ARR_MERGE_TILE_CLASS].p);
            SPMV_LAUNCH_CHECK();
            Scratch c64(ctx, s), pre(ctx, s);
            SPMV_TRY(c64.alloc(tiles * 8));
            SPMV_TRY(pre.alloc((tiles + 1) * 8));
            k_u8_to_i64<<<grid_cap(ctx, tiles), kT, 0, s>>>((const unsigned char *)h->arr[SPMV_ARR_MERGE_TILE_CLASS].p,
                                                            tiles, c64.as<int64_t>());
            SPMV_LAUNCH_CHECK();
            SPMV_TRY(exclusive_scan_i64(ctx, c64.as<int64_t>(), pre.as<int64_t>(), tiles, s));
            int64_t nl = 0;
            SPMV_CUDA_TRY(cudaMemcpyAsync(&nl, pre.as<int64_t>() + tiles, 8, cudaMemcpyDeviceToHost, s));
            SPMV_CUDA_TRY(cudaStreamSynchronize(s));
            SPMV_TRY(arr_alloc(h, SPMV_ARR_MERGE_TILE_ORDER, tiles * 4, s));
            k_merge_order<<<grid_cap(ctx, tiles), kT, 0, s>>>((const unsigned char *)h->arr[SPMV_ARR_MERGE_TILE_CLASS].p,
                                                              pre.as<int64_t>(), tiles, nl,
                                                              (int *)h->arr[SPMV_ARR_MERGE_TILE_ORDER].p);
            SPMV_LAUNCH_CHECK();
            h->merge_lean = (int64_t)nl;
        }
        h->n_carry = tiles;
        break;
    }
    case SPMV_CSR5: {
        int64_t sigma = o->csr5_sigma;
        if (sigma == 0) {   // A6 (B200 rule): ceil(mu) <= 3 -> 4, == 4 -> 8, >= 5 -> 12
            int64_t mu = n > 0 ? ceil_div<int64_t>(nnz, n) : 1;
            sigma = mu <= 3 ? 4 : (mu == 4 ? 8 : 12);
        }
        const int64_t W = 32 * sigma;
        const int64_t tiles = nnz / W;
        h->sigma = sigma;
        h->n_tiles = tiles;
        SPMV_TRY(arr_alloc(h, SPMV_ARR_COL, nnz * 4, s));
        SPMV_TRY(arr_alloc(h, SPMV_ARR_VAL, nnz * VB, s));
        SPMV_TRY(arr_alloc(h, SPMV_ARR_CSR5_TILE_PTR, (tiles + 1) * 8, s));
        SPMV_TRY(arr_alloc(h, SPMV_ARR_CSR5_ROW_LO, (tiles + 1) * 8, s));
        SPMV_TRY(arr_alloc(h, SPMV_ARR_CSR5_TILE_DESC, tiles * 32 * 4, s));
        SPMV_TRY(arr_alloc(h, SPMV_ARR_CSR5_MAP_OFF, tiles * 8, s));
        const int64_t n_words = ceil_div<int64_t>(nnz, 32);
        Scratch bits(ctx, s), segs(ctx, s), cnt(ctx, s), off(ctx, s);
        SPMV_TRY(bits.alloc(std::max<int64_t>(n_words, 1) * 4));
        SPMV_TRY(segs.alloc((tiles + 1) * 8));
        SPMV_TRY(cnt.alloc(std::max<int64_t>(tiles, 1) * 8));
        SPMV_TRY(off.alloc((tiles + 1) * 8));
        SPMV_CUDA_TRY(cudaMemsetAsync(bits.p, 0, std::max<int64_t>(n_words, 1) * 4, s));
        if (n) {
            k_rowstart_bits<IT><<<grid_cap(ctx, n), kT, 0, s>>>(rp, n, bits.as<unsigned>());
            SPMV_LAUNCH_CHECK();
        }
        k_csr5_desc<IT><<<(unsigned)ceil_div<int64_t>((tiles + 1) * 32, kT), kT, 0, s>>>(
            rp, n, nnz, (int)sigma, tiles, n_words, bits.as<unsigned>(),
            (unsigned *)h->arr[SPMV_ARR_CSR5_TILE_DESC].p, (int64_t *)h->arr[SPMV_ARR_CSR5_TILE_PTR].p,
            (int64_t *)h->arr[SPMV_ARR_CSR5_ROW_LO].p, segs.as<int64_t>());
        SPMV_LAUNCH_CHECK();
        int64_t map_len = 0;
        SPMV_CUDA_TRY(cudaMemcpyAsync(&h->csr5_tail_row, (int64_t *)h->arr[SPMV_ARR_CSR5_ROW_LO].p + tiles, 8,
                                      cudaMemcpyDeviceToHost, s));
        SPMV_CUDA_TRY(cudaStreamSynchronize(s));
        if (tiles) {
            k_csr5_map_count<<<grid_cap(ctx, tiles), kT, 0, s>>>((int64_t *)h->arr[SPMV_ARR_CSR5_ROW_LO].p,
                                                                 segs.as<int64_t>(), tiles, cnt.as<int64_t>());
            SPMV_LAUNCH_CHECK();
            SPMV_TRY(exclusive_scan_i64(ctx, cnt.as<int64_t>(), off.as<int64_t>(), tiles, s));
            SPMV_CUDA_TRY(cudaMemcpyAsync(&map_len, off.as<int64_t>() + tiles, 8, cudaMemcpyDeviceToHost, s));
            SPMV_CUDA_TRY(cudaStreamSynchronize(s));
        }
        h->map_len = map_len;
        SPMV_TRY(arr_alloc(h, SPMV_ARR_CSR5_SEG_MAP, map_len * 8, s));
        if (tiles) {
            k_csr5_map_fill<IT><<<(unsigned)ceil_div<int64_t>(tiles * 32, kT), kT, 0, s>>>(
                rp, (int64_t *)h->arr[SPMV_ARR_CSR5_ROW_LO].p, cnt.as<int64_t>(), off.as<int64_t>(), tiles,
                (int64_t *)h->arr[SPMV_ARR_CSR5_MAP_OFF].p, (int64_t *)h->arr[SPMV_ARR_CSR5_SEG_MAP].p);
            SPMV_LAUNCH_CHECK();
            k_csr5_permute<int><<<grid_cap(ctx, tiles * W), kT, 0, s>>>(col, (int *)h->arr[SPMV_ARR_COL].p,
                                                                        tiles * W, (int)sigma, 4);
            SPMV_LAUNCH_CHECK();
            k_csr5_permute<V><<<grid_cap(ctx, tiles * W), kT, 0, s>>>(val, (V *)h->arr[SPMV_ARR_VAL].p,
                                                                      tiles * W, (int)sigma, (int)(16 / VB));
            SPMV_LAUNCH_CHECK();
        }
        if (nnz > tiles * W) {
            int64_t off0 = tiles * W, cnt_tail = nnz - off0;
            SPMV_CUDA_TRY(cudaMemcpyAsync((int *)h->arr[SPMV_ARR_COL].p + off0, col + off0, cnt_tail * 4,
                                          cudaMemcpyDeviceToDevice, s));
            SPMV_CUDA_TRY(cudaMemcpyAsync((V *)h->arr[SPMV_ARR_VAL].p + off0, val + off0, cnt_tail * VB,
                                          cudaMemcpyDeviceToDevice, s));
        }
        h->n_carry = tiles + 1;
        break;
    }
    }
    if (fmt == SPMV_CSR) {
        h->sched.bytes = 16;
        SPMV_TRY(dev_alloc(ctx, h->sched.bytes, s, &h->sched.p));
    }
    if (h->n_carry > 0) {
        h->carry_row.bytes = h->n_carry * 8;
        h->carry_val.bytes = h->n_carry * 8;
        SPMV_TRY(dev_alloc(ctx, h->carry_row.bytes, s, &h->carry_row.p));
        SPMV_TRY(dev_alloc(ctx, h->carry_val.bytes, s, &h->carry_val.p));
    }
    SPMV_CUDA_TRY(cudaGetLastError());
    return SPMV_OK;
}

}  // namespace

spmv_status convert_impl(spmv_ctx *ctx, spmv_format fmt, const spmv_csr *A, const spmv_convert_opts *o,
                         cudaStream_t s, spmv_handle *h) {
    FeatureSums fs;
    int64_t cusp = 0;
    const bool need_cusp = fmt == SPMV_HYB && o->hyb_width < 0 && o->hyb_rule == 2;
    if (o->features) {
        // the caller's spmv_features result for this matrix: no second pass
        const spmv_features_t *f = o->features;
        if (f->n_rows != A->n_rows || f->n_cols != A->n_cols || f->nnz_tot != A->nnz) {
            set_error("opts.features do not describe this matrix");
            return SPMV_ERR_INVALID_ARG;
        }
        fs = FeatureSums{};
        fs.len_max = (unsigned long long)f->nnz_max;
        fs.n_empty = (unsigned long long)f->n_empty_rows;
        fs.hyb_coo_ceil = (unsigned long long)f->hyb_coo_nnz;
        cusp = f->hyb_width_cusp;
    } else {
        SPMV_TRY(feature_pass(ctx, A, s, need_cusp ? 1 : 0, &fs, need_cusp ? &cusp : nullptr));
    }
    if (fs.bad) {
        set_error("matrix is not canonical (flags " + std::to_string(fs.bad) + ")");
        return SPMV_ERR_NOT_CANONICAL;
    }
    const bool i64 = A->nnz > INT32_MAX || o->index64;
    spmv_status st;
    if (A->dtype == SPMV_F64) {
        st = i64 ? convert_t<int64_t, double>(ctx, fmt, A, o, s, h, fs, cusp)
                 : convert_t<int, double>(ctx, fmt, A, o, s, h, fs, cusp);
    } else {
        st = i64 ? convert_t<int64_t, float>(ctx, fmt, A, o, s, h, fs, cusp)
                 : convert_t<int, float>(ctx, fmt, A, o, s, h, fs, cusp);
    }
    if (st != SPMV_OK || o->hot_x < 0 || fmt == SPMV_CSR_SCALAR) return st;
    // A30: hot x columns packed densely -- only where the handle owns its column arrays
    for (int id : {(int)SPMV_ARR_COL, (int)SPMV_ARR_ELL_COL, (int)SPMV_ARR_HYB_COO_COL})
        if (h->arr[id].p && !h->arr[id].owned) return SPMV_OK;
    const size_t V = A->dtype == SPMV_F64 ? 8 : 4;
    const int64_t kmax = o->hot_x > 0 ? o->hot_x : (int64_t)(ctx->l2_bytes / 2 / V);
    Scratch slot(ctx, s);
    SPMV_TRY(hot_select(ctx, A, kmax, o->hot_x > 0, s, h, slot));
    return hot_encode(ctx, h, slot, s);
}

}  // namespace spmv
