// hot.cu -- A30: hot x columns packed densely (B200 memory layout for power-law gathers).
//
// Every format gathers x[col].  On a power-law matrix (R-MAT) most gathers go to a few
// hot columns, but each one costs its own 32-byte L2 sector (and 128-byte L1 line) holding
// three or seven cold neighbours; when x outgrows the 126 MB L2 (R-MAT 27: 1.07 GB) the
// hot columns are sparse in the cache and the gathers become DRAM sector reads.  A handle
// therefore picks the hot columns at conversion -- the smallest degree threshold t such
// that at most K columns have >= t nonzeros, K = half the L2 in x entries -- stores a hot
// column c as -2 - slot(c) in its column arrays, and every run first packs
// xhot[slot] = x[hot[slot]] (k_hot_gather, K entries) so that the kernels' hot gathers
// read a dense array: four fp64 (eight fp32) hot values per sector, L2-resident.  The
// products are unchanged (same x values, same summation order).  Measured with the
// column-stream probe (tools/hotset_probe.py): R-MAT 27 gathers 28.8 -> 11.8 ms; the
// kernels (tools/exp_hot.py): R-MAT 27 CSR5 24.3 -> 14.1 ms, merge 27.0 -> 21.2, CSR 23.0
// -> 21.3.  Auto mode applies it when x exceeds twice the L2 (on R-MAT 24, whose x about
// fits the L2, the indirection costs more than it saves) and the hot columns hold at
// least a quarter of the nonzeros (a Laplacian's columns all have 3-5 nonzeros: no
// threshold qualifies, nothing changes).
#include <algorithm>
#include <vector>

#include "internal.h"
#include "scan.h"

namespace spmv {

namespace {

constexpr int kT = 256;
constexpr int kBins = 65536;

int blocks(const spmv_ctx *ctx, int64_t n) {
    return (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div<int64_t>(n, kT), (int64_t)ctx->sm_count * 16));
}

__global__ void k_degree(const int *__restrict__ col, int64_t nnz, unsigned *__restrict__ deg) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < nnz; k += (int64_t)gridDim.x * blockDim.x)
        atomicAdd(deg + __ldg(col + k), 1u);
}

// hist[d >> 16] for d >= 1 (level 0); hist[d & 0xFFFF] for d >> 16 == hi (level 1)
__global__ void k_deg_hist(const unsigned *__restrict__ deg, int64_t n, int level, unsigned hi,
                           unsigned *__restrict__ hist) {
    for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < n; c += (int64_t)gridDim.x * blockDim.x) {
        const unsigned d = deg[c];
        if (d == 0) continue;
        if (level == 0) atomicAdd(hist + (d >> 16), 1u);
        else if ((d >> 16) == hi) atomicAdd(hist + (d & 0xFFFFu), 1u);
    }
}

__global__ void k_hot_flags(const unsigned *__restrict__ deg, int64_t n, unsigned t, int64_t *__restrict__ flag,
                            unsigned long long *__restrict__ cover) {
    unsigned long long s = 0;
    for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < n; c += (int64_t)gridDim.x * blockDim.x) {
        const unsigned d = deg[c];
        const bool h = d >= t;
        flag[c] = h;
        s += h ? d : 0u;
    }
    for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if ((threadIdx.x & 31) == 0 && s) atomicAdd(cover, s);
}

__global__ void k_hot_slots(const int64_t *__restrict__ flag, const int64_t *__restrict__ pre, int64_t n,
                            int *__restrict__ slot, int *__restrict__ hot) {
    for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < n; c += (int64_t)gridDim.x * blockDim.x) {
        if (flag[c]) {
            slot[c] = (int)pre[c];
            hot[pre[c]] = (int)c;
        } else {
            slot[c] = -1;
        }
    }
}

__global__ void k_hot_encode(int *__restrict__ col, int64_t n, const int *__restrict__ slot) {
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) {
        const int c = col[k];
        if (c >= 0) {
            const int sl = __ldg(slot + c);
            if (sl >= 0) col[k] = -2 - sl;
        }
    }
}

}  // namespace

// Degree threshold of the hot set: the smallest t >= 1 with #{c : deg(c) >= t} <= kmax.
spmv_status hot_select(spmv_ctx *ctx, const spmv_csr *A, int64_t kmax, bool force, cudaStream_t s,
                       spmv_handle *h, Scratch &slot) {
    const int64_t n = A->n_cols, nnz = A->nnz;
    h->n_hot = 0;
    if (n == 0 || nnz == 0 || kmax <= 0) return SPMV_OK;
    const size_t V = A->dtype == SPMV_F64 ? 8 : 4;
    // auto: only when x is well beyond the L2 (R-MAT 24's 134 MB x mostly stays in the 126 MB
    // L2 and the indirection measured 3-20 % slower there; R-MAT 27's 1.07 GB x 1.2-1.7x faster)
    if (!force && (double)n * V <= 2.0 * (double)ctx->l2_bytes) return SPMV_OK;
    Scratch deg(ctx, s), hist(ctx, s);
    SPMV_TRY(deg.alloc(n * 4));
    SPMV_TRY(hist.alloc(kBins * 4));
    SPMV_CUDA_TRY(cudaMemsetAsync(deg.p, 0, n * 4, s));
    k_degree<<<blocks(ctx, nnz), kT, 0, s>>>(A->col_idx, nnz, deg.as<unsigned>());
    SPMV_LAUNCH_CHECK();
    std::vector<unsigned> h1(kBins), h2(kBins);
    SPMV_CUDA_TRY(cudaMemsetAsync(hist.p, 0, kBins * 4, s));
    k_deg_hist<<<blocks(ctx, n), kT, 0, s>>>(deg.as<unsigned>(), n, 0, 0, hist.as<unsigned>());
    SPMV_LAUNCH_CHECK();
    SPMV_CUDA_TRY(cudaMemcpyAsync(h1.data(), hist.p, kBins * 4, cudaMemcpyDeviceToHost, s));
    SPMV_CUDA_TRY(cudaStreamSynchronize(s));
    int64_t referenced = 0;
    for (unsigned v : h1) referenced += v;
    unsigned t = 1;
    if (referenced > kmax) {
        // D = the (kmax+1)-th largest degree = max{v : #{deg >= v} >= kmax + 1}; t = D + 1
        int64_t above = 0;                       // #{deg >> 16 > b}
        int b = kBins - 1;
        for (; b >= 0; --b) {
            if (above + (int64_t)h1[b] >= kmax + 1) break;
            above += h1[b];
        }
        SPMV_CUDA_TRY(cudaMemsetAsync(hist.p, 0, kBins * 4, s));
        k_deg_hist<<<blocks(ctx, n), kT, 0, s>>>(deg.as<unsigned>(), n, 1, (unsigned)b, hist.as<unsigned>());
        SPMV_LAUNCH_CHECK();
        SPMV_CUDA_TRY(cudaMemcpyAsync(h2.data(), hist.p, kBins * 4, cudaMemcpyDeviceToHost, s));
        SPMV_CUDA_TRY(cudaStreamSynchronize(s));
        int lo = kBins - 1;
        for (; lo >= 0; --lo) {
            if (above + (int64_t)h2[lo] >= kmax + 1) break;
            above += h2[lo];
        }
        t = (((unsigned)b << 16) | (unsigned)lo) + 1u;
    }
    Scratch flag(ctx, s), pre(ctx, s), cover(ctx, s);
    SPMV_TRY(flag.alloc(n * 8));
    SPMV_TRY(pre.alloc((n + 1) * 8));
    SPMV_TRY(cover.alloc(8));
    SPMV_CUDA_TRY(cudaMemsetAsync(cover.p, 0, 8, s));
    k_hot_flags<<<blocks(ctx, n), kT, 0, s>>>(deg.as<unsigned>(), n, t, flag.as<int64_t>(),
                                              cover.as<unsigned long long>());
    SPMV_LAUNCH_CHECK();
    SPMV_TRY(exclusive_scan_i64(ctx, flag.as<int64_t>(), pre.as<int64_t>(), n, s));
    int64_t K = 0;
    unsigned long long cov = 0;
    SPMV_CUDA_TRY(cudaMemcpyAsync(&K, pre.as<int64_t>() + n, 8, cudaMemcpyDeviceToHost, s));
    SPMV_CUDA_TRY(cudaMemcpyAsync(&cov, cover.p, 8, cudaMemcpyDeviceToHost, s));
    SPMV_CUDA_TRY(cudaStreamSynchronize(s));
    if (K == 0 || (!force && (double)cov < 0.25 * (double)nnz)) return SPMV_OK;
    SPMV_TRY(slot.alloc(n * 4));
    DevArray &hc = h->arr[SPMV_ARR_HOT_COLS];
    hc.bytes = (size_t)K * 4;
    hc.owned = true;
    SPMV_TRY(dev_alloc(ctx, hc.bytes + 64, s, &hc.p));
    k_hot_slots<<<blocks(ctx, n), kT, 0, s>>>(flag.as<int64_t>(), pre.as<int64_t>(), n, slot.as<int>(),
                                              reinterpret_cast<int *>(hc.p));
    SPMV_LAUNCH_CHECK();
    h->xhot.bytes = (size_t)K * V;
    SPMV_TRY(dev_alloc(ctx, h->xhot.bytes, s, &h->xhot.p));
    h->n_hot = K;
    return SPMV_OK;
}

spmv_status hot_encode(spmv_ctx *ctx, spmv_handle *h, const Scratch &slot, cudaStream_t s) {
    if (h->n_hot == 0) return SPMV_OK;
    for (int id : {(int)SPMV_ARR_COL, (int)SPMV_ARR_ELL_COL, (int)SPMV_ARR_HYB_COO_COL}) {
        DevArray &a = h->arr[id];
        if (!a.p || !a.bytes) continue;
        k_hot_encode<<<blocks(ctx, a.bytes / 4), kT, 0, s>>>(reinterpret_cast<int *>(a.p), (int64_t)(a.bytes / 4),
                                                            slot.as<int>());
        SPMV_LAUNCH_CHECK();
    }
    return SPMV_OK;
}

}  // namespace spmv
