// features.cu -- the per-matrix sparsity features of Table II (PAPER.md:161-185,
// §IV-A), read per SURVEY A8/A9, plus the canonical-CSR check
// (A15) that spmv_convert relies on.
//
// "Sets 2 and 3 require a scan on the entire matrix, O(nnz)": one
// streaming pass over col_idx and two over row_ptr, all integer arithmetic with
// exact 64-bit sums; the fp64 finals are computed on the host from those sums with
// the fixed formulas of A9, so the result is bit-exact and run-to-run identical.
//
// Block ("continuous nnz chunk") structure is carried by two
// bitmaps over the nnz positions:
//   rs[w]   bit l set <=> position 32w+l starts a non-empty row   (F1, row pass)
//   flag[w] bit l set <=> position 32w+l starts a block           (F2, element pass)
// A block starts at a row start or wherever col[k] != col[k-1] + 1.  Every row start
// is a block start, so block sizes are the gaps between consecutive flags (F4) and
// the number of blocks of row r is F(row_ptr[r+1]) - F(row_ptr[r]) where F(p) counts
// the flags before p (F3 prefix, F5).
#include <climits>
#include <cmath>
#include <vector>

#include "internal.h"

namespace spmv {

namespace {

constexpr int kThreads = 256;
constexpr int kScanChunk = 2048;          // words per local-prefix chunk (256 thr x 8)
constexpr int kSharedHist = 2048;         // row-length histogram bins kept in smem

enum : unsigned long long {
    BAD_ROWPTR_ENDS = 1, BAD_ROWPTR_ORDER = 2, BAD_COL_RANGE = 4, BAD_COL_ORDER = 8
};

__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}
__device__ __forceinline__ unsigned long long warp_min_u64(unsigned long long v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) { unsigned long long t = __shfl_xor_sync(0xffffffffu, v, o); v = t < v ? t : v; }
    return v;
}
__device__ __forceinline__ unsigned long long warp_max_u64(unsigned long long v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) { unsigned long long t = __shfl_xor_sync(0xffffffffu, v, o); v = t > v ? t : v; }
    return v;
}

// block-level reduction of (sum..., min, max) into global atomics
template <int NS>
__device__ void block_commit(unsigned long long (&sums)[NS], unsigned long long *gsum[NS],
                             unsigned long long mn, unsigned long long *gmin,
                             unsigned long long mx, unsigned long long *gmax) {
    __shared__ unsigned long long s_sum[NS][kThreads / 32];
    __shared__ unsigned long long s_min[kThreads / 32], s_max[kThreads / 32];
    int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
#pragma unroll
    for (int i = 0; i < NS; ++i) sums[i] = warp_sum_u64(sums[i]);
    mn = warp_min_u64(mn);
    mx = warp_max_u64(mx);
    if (lane == 0) {
#pragma unroll
        for (int i = 0; i < NS; ++i) s_sum[i][wid] = sums[i];
        s_min[wid] = mn;
        s_max[wid] = mx;
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        for (int w = 1; w < kThreads / 32; ++w) {
#pragma unroll
            for (int i = 0; i < NS; ++i) s_sum[i][0] += s_sum[i][w];
            s_min[0] = s_min[w] < s_min[0] ? s_min[w] : s_min[0];
            s_max[0] = s_max[w] > s_max[0] ? s_max[w] : s_max[0];
        }
#pragma unroll
        for (int i = 0; i < NS; ++i)
            if (gsum[i] && s_sum[i][0]) atomicAdd(gsum[i], s_sum[i][0]);
        if (gmin) atomicMin(gmin, s_min[0]);
        if (gmax) atomicMax(gmax, s_max[0]);
    }
}

// F1: row pass -- row lengths (sum len^2, min, max, empty rows, HYB overflow),
// row_ptr validity, row-start bitmap, row-length histogram for the A2 "cusp" rule.
template <typename IT>
__global__ void __launch_bounds__(kThreads)
k_rows(const IT *__restrict__ rp, int64_t n_rows, int64_t nnz, int64_t kh,
       unsigned *__restrict__ rs_bits, unsigned long long *__restrict__ hist, int64_t hist_bins,
       FeatureSums *out) {
    __shared__ unsigned s_hist[kSharedHist];
    const bool use_hist = hist != nullptr;
    const int sh_bins = hist_bins < kSharedHist ? (int)hist_bins : kSharedHist;
    if (use_hist)
        for (int i = threadIdx.x; i < sh_bins; i += blockDim.x) s_hist[i] = 0;
    __syncthreads();
    unsigned long long bad = 0, len2 = 0, empty = 0, over = 0;
    unsigned long long mn = ULLONG_MAX, mx = 0;
    if (blockIdx.x == 0 && threadIdx.x == 0)
        if ((int64_t)rp[0] != 0 || (int64_t)rp[n_rows] != nnz) bad |= BAD_ROWPTR_ENDS;
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n_rows;
         r += (int64_t)gridDim.x * blockDim.x) {
        int64_t a = rp[r], b = rp[r + 1];
        int64_t len = b - a;
        if (len < 0 || a < 0 || b > nnz) { bad |= BAD_ROWPTR_ORDER; len = 0; }
        unsigned long long ul = (unsigned long long)len;
        len2 += ul * ul;
        mn = ul < mn ? ul : mn;
        mx = ul > mx ? ul : mx;
        empty += (len == 0);
        over += len > kh ? (unsigned long long)(len - kh) : 0ull;
        if (len > 0) atomicOr(&rs_bits[a >> 5], 1u << (a & 31));
        if (use_hist) {
            // rows of a warp mostly share a length bin: one shared atomic per distinct bin
            const int64_t bin = len < hist_bins - 1 ? len : hist_bins - 1;
            const unsigned active = __activemask();
            const unsigned same = __match_any_sync(active, (unsigned long long)bin);
            if ((threadIdx.x & 31) == __ffs(same) - 1) {
                if (bin < sh_bins) atomicAdd(&s_hist[bin], (unsigned)__popc(same));
                else atomicAdd(&hist[bin], (unsigned long long)__popc(same));
            }
        }
    }
    if (bad) atomicOr(&out->bad, bad);
    unsigned long long sums[3] = {len2, empty, over};
    unsigned long long *g[3] = {&out->sum_len2, &out->n_empty, &out->hyb_coo_ceil};
    block_commit<3>(sums, g, mn, &out->len_min, mx, &out->len_max);
    if (use_hist) {
        __syncthreads();
        for (int i = threadIdx.x; i < sh_bins; i += blockDim.x)
            if (s_hist[i]) atomicAdd(&hist[i], (unsigned long long)s_hist[i]);
    }
}

// F2: element pass -- column validity/order and the block-start bitmap.  A warp
// handles a chunk of 512 positions (16 words) per iteration: lane l loads its 16
// consecutive elements with four 16-byte loads, derives 16 flag bits, and lane pairs
// merge their half-words into the chunk's flag words.
constexpr int kLaneElems = 16;
constexpr int kChunkWords = kLaneElems;      // 32 lanes x 16 elements = 16 words

__global__ void __launch_bounds__(kThreads)
k_flags(const int *__restrict__ col, int64_t nnz, int64_t n_cols, int64_t n_words,
        const unsigned *__restrict__ rs_bits, unsigned *__restrict__ flag_bits, FeatureSums *out) {
    const int lane = threadIdx.x & 31;
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t n_warps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t pol = policy_evict_first();
    unsigned bad = 0;
    for (int64_t wb = warp * kChunkWords; wb < n_words; wb += n_warps * kChunkWords) {
        const int64_t k0 = wb * 32 + (int64_t)lane * kLaneElems;      // this lane's first position
        int c[kLaneElems];
        if (k0 + kLaneElems <= nnz && ((uintptr_t)(col + k0) & 15) == 0) {
#pragma unroll
            for (int q = 0; q < kLaneElems / 4; ++q) {
                const int4 v = ld_hint(reinterpret_cast<const int4 *>(col + k0) + q, pol);
                c[4 * q] = v.x; c[4 * q + 1] = v.y; c[4 * q + 2] = v.z; c[4 * q + 3] = v.w;
            }
        } else {
#pragma unroll
            for (int e = 0; e < kLaneElems; ++e) c[e] = k0 + e < nnz ? col[k0 + e] : 0;
        }
        const unsigned rw = (wb + (lane >> 1) < n_words) ? rs_bits[wb + (lane >> 1)] : 0u;
        const unsigned rs16 = (rw >> ((lane & 1) * 16)) & 0xFFFFu;
        int prev = __shfl_up_sync(0xffffffffu, c[kLaneElems - 1], 1);
        if (lane == 0) prev = (k0 > 0 && k0 < nnz) ? col[k0 - 1] : 0;
        unsigned f16 = 0;
#pragma unroll
        for (int e = 0; e < kLaneElems; ++e) {
            const int64_t k = k0 + e;
            const bool valid = k < nnz;
            const int pv = e == 0 ? prev : c[e - 1];
            const bool rowstart = (rs16 >> e) & 1u;
            const bool flag = valid && (rowstart || k == 0 || (int64_t)c[e] != (int64_t)pv + 1);
            if (valid && (c[e] < 0 || (int64_t)c[e] >= n_cols)) bad |= BAD_COL_RANGE;
            if (valid && k > 0 && !rowstart && c[e] <= pv) bad |= BAD_COL_ORDER;
            if (valid && k == 0 && !rowstart) bad |= BAD_ROWPTR_ORDER;
            f16 |= (unsigned)flag << e;
        }
        const unsigned hi = __shfl_down_sync(0xffffffffu, f16, 1);
        if (!(lane & 1) && wb + (lane >> 1) < n_words) flag_bits[wb + (lane >> 1)] = f16 | (hi << 16);
    }
    bad = __reduce_or_sync(0xffffffffu, bad);
    if (lane == 0 && bad) atomicOr(&out->bad, (unsigned long long)bad);
}

// F3a: per-chunk exclusive prefix of flag popcounts (kScanChunk words per block).
__global__ void __launch_bounds__(kThreads)
k_scan_local(const unsigned *__restrict__ flag_bits, int64_t n_words, unsigned *__restrict__ local,
             unsigned long long *__restrict__ totals) {
    __shared__ unsigned s_warp[kThreads / 32];
    const int64_t base = (int64_t)blockIdx.x * kScanChunk;
    constexpr int per = kScanChunk / kThreads;   // 8 consecutive words per thread
    unsigned cnt[per];
    unsigned tsum = 0;
#pragma unroll
    for (int i = 0; i < per; ++i) {
        int64_t w = base + threadIdx.x * per + i;
        cnt[i] = w < n_words ? __popc(flag_bits[w]) : 0u;
        tsum += cnt[i];
    }
    // block exclusive scan of tsum
    int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    unsigned incl = tsum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        unsigned t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
    }
    if (lane == 31) s_warp[wid] = incl;
    __syncthreads();
    unsigned woff = 0;
    for (int i = 0; i < wid; ++i) woff += s_warp[i];
    unsigned run = woff + incl - tsum;
#pragma unroll
    for (int i = 0; i < per; ++i) {
        int64_t w = base + threadIdx.x * per + i;
        if (w < n_words) local[w] = run;
        run += cnt[i];
    }
    if (threadIdx.x == kThreads - 1) totals[blockIdx.x] = run;
}

// F3b: exclusive scan of the chunk totals (one block, sequential over tiles of 256).
__global__ void __launch_bounds__(kThreads)
k_scan_totals(unsigned long long *totals, int64_t n) {
    __shared__ unsigned long long s_warp[kThreads / 32];
    __shared__ unsigned long long s_carry;
    if (threadIdx.x == 0) s_carry = 0;
    __syncthreads();
    int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    for (int64_t base = 0; base < n; base += kThreads) {
        int64_t i = base + threadIdx.x;
        unsigned long long v = i < n ? totals[i] : 0ull, incl = v;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            unsigned long long t = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += t;
        }
        if (lane == 31) s_warp[wid] = incl;
        __syncthreads();
        unsigned long long woff = 0;
        for (int k = 0; k < wid; ++k) woff += s_warp[k];
        unsigned long long carry = s_carry;
        if (i < n) totals[i] = carry + woff + incl - v;
        __syncthreads();
        if (threadIdx.x == kThreads - 1) s_carry = carry + woff + incl;
        __syncthreads();
    }
}

// F4: block sizes = gaps between consecutive block starts.  A warp takes 256 words
// (8192 positions) per iteration, lane l the 8 words [8l, 8l+8) loaded as two 16-byte
// vectors; a lane walks its flags in order (gap to the previous flag = one block), the
// block left open at the lane end closes at the first flag of a later lane (suffix
// minimum over lanes) or, past the chunk, at the next flagged word (forward scan).
constexpr int kLaneWords = 8;

__global__ void __launch_bounds__(kThreads)
k_block_sizes(const unsigned *__restrict__ flag_bits, int64_t n_words, int64_t nnz, FeatureSums *out) {
    const int lane = threadIdx.x & 31;
    const int64_t warp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t n_warps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    constexpr int64_t CW = 32 * kLaneWords;
    unsigned long long nb = 0, sz2 = 0, mn = ULLONG_MAX, mx = 0;
    auto take = [&](unsigned long long sz) {
        nb += 1;
        sz2 += sz * sz;
        mn = sz < mn ? sz : mn;
        mx = sz > mx ? sz : mx;
    };
    for (int64_t wb = warp * CW; wb < n_words; wb += n_warps * CW) {
        const int64_t w0 = wb + (int64_t)lane * kLaneWords;
        unsigned fw[kLaneWords];
        // flag_bits is padded to a multiple of CW words (zeros): vector loads stay inside
        const uint4 a = *reinterpret_cast<const uint4 *>(flag_bits + w0);
        const uint4 b = *reinterpret_cast<const uint4 *>(flag_bits + w0 + 4);
        fw[0] = a.x; fw[1] = a.y; fw[2] = a.z; fw[3] = a.w; fw[4] = b.x; fw[5] = b.y; fw[6] = b.z; fw[7] = b.w;
        int64_t first = -1, last = -1;
#pragma unroll
        for (int q = 0; q < kLaneWords; ++q) {
            unsigned w = fw[q];
            while (w) {
                const int64_t p = (w0 + q) * 32 + (__ffs(w) - 1);
                w &= w - 1;
                if (last >= 0) take((unsigned long long)(p - last));
                else first = p;
                last = p;
            }
        }
        // first flag strictly after this lane: suffix minimum of `first` over later lanes
        int64_t nxt = first >= 0 ? first : INT64_MAX;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const int64_t v = __shfl_down_sync(0xffffffffu, nxt, o);
            if (lane + o < 32 && v < nxt) nxt = v;
        }
        int64_t after = __shfl_down_sync(0xffffffffu, nxt, 1);
        if (lane == 31) after = INT64_MAX;
        // past the chunk: the next flagged word (warp-cooperative forward scan, rare)
        const bool need = __any_sync(0xffffffffu, last >= 0 && after == INT64_MAX);
        if (need) {
            int64_t beyond = nnz;
            for (int64_t base = wb + CW; base < n_words; base += 32) {
                const unsigned v = base + lane < n_words ? flag_bits[base + lane] : 0u;
                const unsigned bm = __ballot_sync(0xffffffffu, v != 0u);
                if (bm) {
                    const int src = __ffs(bm) - 1;
                    const unsigned fv = __shfl_sync(0xffffffffu, v, src);
                    beyond = (base + src) * 32 + (__ffs(fv) - 1);
                    break;
                }
            }
            if (after == INT64_MAX) after = beyond;
        }
        if (last >= 0) take((unsigned long long)(after - last));
    }
    unsigned long long sums[2] = {nb, sz2};
    unsigned long long *g[2] = {&out->nb_tot, &out->sum_bs2};
    block_commit<2>(sums, g, mn, &out->bs_min, mx, &out->bs_max);
}

__device__ __forceinline__ unsigned long long flags_before(int64_t p, int64_t n_words,
                                                           const unsigned *__restrict__ flag_bits,
                                                           const unsigned *__restrict__ local,
                                                           const unsigned long long *__restrict__ totals,
                                                           unsigned long long total_flags) {
    int64_t w = p >> 5;
    if (w >= n_words) return total_flags;
    unsigned m = (p & 31) ? (flag_bits[w] & ((1u << (p & 31)) - 1u)) : 0u;
    return totals[w / kScanChunk] + local[w] + __popc(m);
}

// F5: blocks per row (nnzb_*), over all rows including empty ones (A8).
template <typename IT>
__global__ void __launch_bounds__(kThreads)
k_row_blocks(const IT *__restrict__ rp, int64_t n_rows, int64_t n_words,
             const unsigned *__restrict__ flag_bits, const unsigned *__restrict__ local,
             const unsigned long long *__restrict__ totals, FeatureSums *out) {
    const unsigned long long total_flags = out->nb_tot;
    unsigned long long sum2 = 0, mn = ULLONG_MAX, mx = 0;
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n_rows;
         r += (int64_t)gridDim.x * blockDim.x) {
        unsigned long long fa = flags_before(rp[r], n_words, flag_bits, local, totals, total_flags);
        unsigned long long fb = flags_before(rp[r + 1], n_words, flag_bits, local, totals, total_flags);
        unsigned long long nb = fb - fa;
        sum2 += nb * nb;
        mn = nb < mn ? nb : mn;
        mx = nb > mx ? nb : mx;
    }
    unsigned long long sums[1] = {sum2};
    unsigned long long *g[1] = {&out->sum_nb2};
    block_commit<1>(sums, g, mn, &out->nb_min, mx, &out->nb_max);
}

int grid_for(const spmv_ctx *ctx, int64_t work, int per_block = kThreads) {
    int64_t g = ceil_div<int64_t>(work, per_block);
    int64_t cap = (int64_t)ctx->sm_count * 8;
    if (g > cap) g = cap;
    if (g < 1) g = 1;
    return (int)g;
}

template <typename IT>
spmv_status feature_pass_t(spmv_ctx *ctx, const spmv_csr *A, cudaStream_t s, int level,
                           FeatureSums *host, int64_t *hyb_cusp) {
    const IT *rp = reinterpret_cast<const IT *>(A->row_ptr);
    const int64_t n = A->n_rows, nnz = A->nnz;
    const int64_t n_words = ceil_div<int64_t>(nnz, 32);
    const int64_t n_chunks = ceil_div<int64_t>(n_words, kScanChunk);
    const int64_t kh = n > 0 ? ceil_div<int64_t>(nnz, n) : 0;
    const int64_t hist_bins = level ? nnz / 4096 + 2 : 0;

    Scratch sums(ctx, s), rs(ctx, s), flags(ctx, s), local(ctx, s), totals(ctx, s), hist(ctx, s);
    SPMV_TRY(sums.alloc(sizeof(FeatureSums)));
    SPMV_TRY(rs.alloc(n_words * 4));
    const int64_t n_words_pad = ceil_div<int64_t>(n_words, 256) * 256 + 256;   // F4 reads whole 256-word chunks
    SPMV_TRY(flags.alloc(n_words_pad * 4));
    if (level) {
        SPMV_TRY(local.alloc(n_words * 4));
        SPMV_TRY(totals.alloc(n_chunks * 8));
        SPMV_TRY(hist.alloc(hist_bins * 8));
        SPMV_CUDA_TRY(cudaMemsetAsync(hist.p, 0, hist_bins * 8, s));
    }
    FeatureSums init{};
    init.len_min = init.nb_min = init.bs_min = ULLONG_MAX;
    SPMV_CUDA_TRY(cudaMemcpyAsync(sums.p, &init, sizeof(init), cudaMemcpyHostToDevice, s));
    SPMV_CUDA_TRY(cudaMemsetAsync(rs.p, 0, n_words * 4, s));
    SPMV_CUDA_TRY(cudaMemsetAsync(flags.p, 0, n_words_pad * 4, s));
    FeatureSums *d = sums.as<FeatureSums>();

    if (n >= 0) {
        k_rows<IT><<<grid_for(ctx, n > 0 ? n : 1), kThreads, 0, s>>>(
            rp, n, nnz, kh, rs.as<unsigned>(), level ? hist.as<unsigned long long>() : nullptr,
            hist_bins, d);
        SPMV_LAUNCH_CHECK();
    }
    if (n_words > 0) {
        k_flags<<<grid_for(ctx, ceil_div<int64_t>(n_words, kChunkWords) * 32), kThreads, 0, s>>>(A->col_idx, nnz, A->n_cols, n_words,
                                                                rs.as<unsigned>(), flags.as<unsigned>(), d);
        SPMV_LAUNCH_CHECK();
    }
    if (level && n_words > 0) {
        k_scan_local<<<(unsigned)n_chunks, kThreads, 0, s>>>(flags.as<unsigned>(), n_words, local.as<unsigned>(),
                                                             totals.as<unsigned long long>());
        SPMV_LAUNCH_CHECK();
        k_scan_totals<<<1, kThreads, 0, s>>>(totals.as<unsigned long long>(), n_chunks);
        SPMV_LAUNCH_CHECK();
        k_block_sizes<<<grid_for(ctx, ceil_div<int64_t>(n_words, 32 * kLaneWords) * 32), kThreads, 0, s>>>(flags.as<unsigned>(), n_words, nnz, d);
        SPMV_LAUNCH_CHECK();
    }
    if (level && n > 0) {
        k_row_blocks<IT><<<grid_for(ctx, n), kThreads, 0, s>>>(rp, n, n_words, flags.as<unsigned>(),
                                                               local.as<unsigned>(),
                                                               totals.as<unsigned long long>(), d);
        SPMV_LAUNCH_CHECK();
    }
    SPMV_CUDA_TRY(cudaMemcpyAsync(host, d, sizeof(FeatureSums), cudaMemcpyDeviceToHost, s));
    std::vector<unsigned long long> h;
    if (level) {
        h.resize(hist_bins);
        SPMV_CUDA_TRY(cudaMemcpyAsync(h.data(), hist.p, hist_bins * 8, cudaMemcpyDeviceToHost, s));
    }
    SPMV_CUDA_TRY(cudaStreamSynchronize(s));
    if (n == 0) { host->len_min = 0; host->len_max = 0; }
    if (nnz == 0) { host->nb_tot = 0; host->sum_bs2 = 0; host->bs_min = 0; host->bs_max = 0; }
    if (level && n > 0 && nnz == 0) { host->nb_min = 0; host->nb_max = 0; host->sum_nb2 = 0; }
    if (hyb_cusp) {
        // A2 "cusp" width: smallest k with 3*#{len>k} < n_rows or #{len>k} < 4096,
        // else the maximum row length; #{len>k} is exact for k <= nnz/4096.
        int64_t kmax = (int64_t)host->len_max, longer = n, ans = kmax;
        for (int64_t k = 0; level && k < kmax; ++k) {
            longer -= (int64_t)h[k < hist_bins - 1 ? k : hist_bins - 1];
            if (3 * longer < n || longer < 4096) { ans = k; break; }
        }
        *hyb_cusp = n > 0 ? ans : 0;
    }
    return SPMV_OK;
}

}  // namespace

spmv_status feature_pass(spmv_ctx *ctx, const spmv_csr *A, cudaStream_t s, int level, FeatureSums *out,
                         int64_t *hyb_cusp) {
    if (A->ptr_type == SPMV_I32) return feature_pass_t<int>(ctx, A, s, level, out, hyb_cusp);
    return feature_pass_t<int64_t>(ctx, A, s, level, out, hyb_cusp);
}

// A9: fixed fp64 formulas from exact integer sums (identical rounding on every run).
void finalize_features(const spmv_csr *A, const FeatureSums &fs, int64_t hyb_cusp, spmv_features_t *f) {
    *f = spmv_features_t{};
    const int64_t n = A->n_rows, m = A->n_cols, nnz = A->nnz;
    f->n_rows = n;
    f->n_cols = m;
    f->nnz_tot = nnz;
    f->nnz_max = (int64_t)fs.len_max;
    f->nnz_min = n > 0 ? (int64_t)fs.len_min : 0;
    f->n_empty_rows = (int64_t)fs.n_empty;
    f->nnzb_tot = (int64_t)fs.nb_tot;
    f->nnzb_min = n > 0 ? (int64_t)fs.nb_min : 0;
    f->nnzb_max = n > 0 ? (int64_t)fs.nb_max : 0;
    f->snzb_min = fs.nb_tot ? (int64_t)fs.bs_min : 0;
    f->snzb_max = fs.nb_tot ? (int64_t)fs.bs_max : 0;
    f->sum_len2 = fs.sum_len2;
    f->sum_nnzb2 = fs.sum_nb2;
    f->sum_snzb2 = fs.sum_bs2;
    if (n > 0) {
        __int128 N = n;
        __int128 S1 = nnz, S2 = (__int128)fs.sum_len2, B1 = (__int128)fs.nb_tot, B2 = (__int128)fs.sum_nb2;
        f->nnz_mu = (double)nnz / (double)n;
        f->nnz_sigma = std::sqrt((double)(N * S2 - S1 * S1)) / (double)n;
        f->nnzb_mu = (double)fs.nb_tot / (double)n;
        f->nnzb_sigma = std::sqrt((double)(N * B2 - B1 * B1)) / (double)n;
        if (m > 0) f->nnz_frac = (double)((__int128)100 * nnz) / (double)((__int128)n * m);
    }
    if (fs.nb_tot > 0) {
        __int128 NB = (__int128)fs.nb_tot, Z2 = (__int128)fs.sum_bs2;
        f->snzb_mu = (double)nnz / (double)fs.nb_tot;
        f->snzb_sigma = std::sqrt((double)(NB * Z2 - (__int128)nnz * nnz)) / (double)fs.nb_tot;
    }
    f->ell_width = f->nnz_max;
    f->ell_slots = f->nnz_max * n;
    f->ell_pad_frac = f->ell_slots > 0 ? (double)(f->ell_slots - nnz) / (double)f->ell_slots : 0.0;
    f->hyb_width = n > 0 ? (nnz + n - 1) / n : 0;
    f->hyb_coo_nnz = (int64_t)fs.hyb_coo_ceil;
    f->hyb_width_floor = n > 0 ? nnz / n : 0;
    f->hyb_width_cusp = hyb_cusp;
}

}  // namespace spmv
