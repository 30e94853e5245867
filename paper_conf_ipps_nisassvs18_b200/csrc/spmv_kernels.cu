// spmv_kernels.cu -- y <- alpha*A*x + beta*y in the six formats of PAPER.md:89-103.
//
// Design rules:
//  * bandwidth-bound: no tensor cores; A (col/val) is streamed once through the
//    read-only path with an L2 evict-first policy, x is gathered through the
//    read-only path with an L2 evict-last policy;
//  * fp64 accumulation for both storage types (A13), one rounding per output;
//  * deterministic: every cross-thread / cross-CTA combination is a fixed-order
//    segmented sum, no floating-point atomics;
//  * BLAS semantics (A14): beta == 0 never reads y, alpha == 0 never reads A.
// Rows split across CTAs/tiles: the CTA holding the row's LAST element writes
// y = alpha*s + beta*y, earlier CTAs leave (row, partial) carries that k_fixup adds
// in carry order (one thread per run of equal rows).
#include <algorithm>

#include "internal.h"
#include "kernels.h"

namespace spmv {

namespace {

constexpr int kT = kRunThreads;
constexpr int kIPT = kItemsPerThread;
constexpr int kFold = 256;   // sequential steps per accumulator before folding (A13)

// ------------------------------------------------------------------ helpers

// Block-wide segmented scan over threads (kT threads): S(t) = v(t) + (head(t) ? 0 : S(t-1)).
// Returns the exclusive value S(t-1) (0 for t = 0); *incl receives S(t).
__device__ __forceinline__ double block_seg_scan(bool head, double v, double *incl) {
    __shared__ double s_S[kT / 32];
    __shared__ int s_H[kT / 32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    double S = v;
    bool H = head;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        double Sp = __shfl_up_sync(0xffffffffu, S, o);
        int Hp = __shfl_up_sync(0xffffffffu, (int)H, o);
        if (lane >= o) {
            if (!H) S += Sp;
            H = H || Hp;
        }
    }
    if (lane == 31) { s_S[wid] = S; s_H[wid] = H; }
    __syncthreads();
    double carry = 0.0;                     // combination of warps < wid
    for (int w = 0; w < wid; ++w) carry = s_H[w] ? s_S[w] : carry + s_S[w];
    double full = H ? S : S + carry;
    double ex = __shfl_up_sync(0xffffffffu, full, 1);
    if (lane == 0) ex = carry;
    __syncthreads();
    *incl = full;
    return ex;
}

template <typename V, bool B0>
__device__ __forceinline__ void y_write(V *y, int64_t r, double s, double alpha, double beta) {
    double out = alpha * s;
    if (!B0) out = fma(beta, (double)y[r], out);
    y[r] = (V)out;
}
template <typename V, bool B0>
__device__ __forceinline__ void y_beta(V *y, int64_t r, double beta) {
    y[r] = B0 ? (V)0 : (V)(beta * (double)y[r]);
}

// ------------------------------------------------------------------ alpha == 0

template <typename V, bool B0>
__global__ void k_scale(V *y, int64_t n, double beta) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        y_beta<V, B0>(y, i, beta);
}

// ------------------------------------------------------------------ CSR-vector (K3/G8)
// "assign a WARP to process a row".  A W-lane group per row (A5);
// lanes stride the row with four independent accumulators (folded every kFold
// steps into a running total), shuffle reduction.
template <typename V, typename IT, int W, bool B0>
__global__ void __launch_bounds__(kT)
k_csr_vector(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val,
             const V *__restrict__ x, V *__restrict__ y, int64_t n, double alpha, double beta) {
    constexpr int RPW = 32 / W;
    const int lane = threadIdx.x & 31;
    const int sub = lane & (W - 1);
    const int64_t gwarp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    for (int64_t base = gwarp * RPW; base < n; base += nwarps * RPW) {
        const int64_t r = base + lane / W;
        double tot = 0.0, a0 = 0.0, a1 = 0.0, a2 = 0.0, a3 = 0.0;
        if (r < n) {
            const int64_t b = (int64_t)__ldg(rp + r + 1);
            int64_t k = (int64_t)__ldg(rp + r) + sub;
            int it = 0;
            for (; k + 3 * W < b; k += 4 * W) {
                int c0 = ld_hint(col + k, pa), c1 = ld_hint(col + k + W, pa);
                int c2 = ld_hint(col + k + 2 * W, pa), c3 = ld_hint(col + k + 3 * W, pa);
                V v0 = ld_hint(val + k, pa), v1 = ld_hint(val + k + W, pa);
                V v2 = ld_hint(val + k + 2 * W, pa), v3 = ld_hint(val + k + 3 * W, pa);
                a0 += (double)v0 * (double)ld_x(x + c0, px);
                a1 += (double)v1 * (double)ld_x(x + c1, px);
                a2 += (double)v2 * (double)ld_x(x + c2, px);
                a3 += (double)v3 * (double)ld_x(x + c3, px);
                if (++it == kFold) {            // blocked summation keeps chains short (A13)
                    tot += (a0 + a1) + (a2 + a3);
                    a0 = a1 = a2 = a3 = 0.0;
                    it = 0;
                }
            }
            for (; k < b; k += W) a0 += (double)ld_hint(val + k, pa) * (double)ld_x(x + ld_hint(col + k, pa), px);
        }
        double s = tot + ((a0 + a1) + (a2 + a3));
#pragma unroll
        for (int o = W / 2; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
        if (sub == 0 && r < n) y_write<V, B0>(y, r, s, alpha, beta);
    }
}

// ------------------------------------------------------------------ CSR-scalar (K2)
// "assigning a thread to process each row -- the scalar CSR kernel".
template <typename V, typename IT, bool B0>
__global__ void __launch_bounds__(kT)
k_csr_scalar(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val,
             const V *__restrict__ x, V *__restrict__ y, int64_t n, double alpha, double beta) {
    const uint64_t px = policy_evict_last();
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
        double a0 = 0.0, a1 = 0.0;
        int64_t k = __ldg(rp + r), b = __ldg(rp + r + 1);
        for (; k + 1 < b; k += 2) {
            a0 += (double)__ldg(val + k) * (double)ld_x(x + __ldg(col + k), px);
            a1 += (double)__ldg(val + k + 1) * (double)ld_x(x + __ldg(col + k + 1), px);
        }
        if (k < b) a0 += (double)__ldg(val + k) * (double)ld_x(x + __ldg(col + k), px);
        y_write<V, B0>(y, r, a0 + a1, alpha, beta);
    }
}

// ------------------------------------------------------------------ ELL (K4/G9)
// column-major, "each row is processed by a single thread".
// Padding slots carry col = -1 and are skipped (A3).
template <typename V, bool B0>
__global__ void __launch_bounds__(kT)
k_ell(const int *__restrict__ ecol, const V *__restrict__ eval, int64_t K, int64_t ld,
      const V *__restrict__ x, V *__restrict__ y, int64_t n, double alpha, double beta) {
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
        double tot = 0.0, a0 = 0.0, a1 = 0.0, a2 = 0.0, a3 = 0.0;
        int64_t j = 0;
        int it = 0;
        for (; j + 3 < K; j += 4) {
            int c0 = ld_hint(ecol + j * ld + r, pa), c1 = ld_hint(ecol + (j + 1) * ld + r, pa);
            int c2 = ld_hint(ecol + (j + 2) * ld + r, pa), c3 = ld_hint(ecol + (j + 3) * ld + r, pa);
            V v0 = ld_hint(eval + j * ld + r, pa), v1 = ld_hint(eval + (j + 1) * ld + r, pa);
            V v2 = ld_hint(eval + (j + 2) * ld + r, pa), v3 = ld_hint(eval + (j + 3) * ld + r, pa);
            if (c0 >= 0) a0 += (double)v0 * (double)ld_x(x + c0, px);
            if (c1 >= 0) a1 += (double)v1 * (double)ld_x(x + c1, px);
            if (c2 >= 0) a2 += (double)v2 * (double)ld_x(x + c2, px);
            if (c3 >= 0) a3 += (double)v3 * (double)ld_x(x + c3, px);
            if (++it == kFold) {
                tot += (a0 + a1) + (a2 + a3);
                a0 = a1 = a2 = a3 = 0.0;
                it = 0;
            }
        }
        for (; j < K; ++j) {
            int c = ld_hint(ecol + j * ld + r, pa);
            V v = ld_hint(eval + j * ld + r, pa);
            if (c >= 0) a0 += (double)v * (double)ld_x(x + c, px);
        }
        y_write<V, B0>(y, r, tot + ((a0 + a1) + (a2 + a3)), alpha, beta);
    }
}

// ------------------------------------------------------------------ COO (K1/G7)
// "first all product contributions are computed for the non-zero
// elements, followed by a segmented reduction across threads".  CTA c owns nonzeros
// [c*T, (c+1)*T): staged products, thread-sequential segments of kIPT items, a
// block segmented scan for the thread carries, a CTA carry for the fix-up.
// ACCUM (HYB's COO part): y += alpha*s, no beta, no empty-row writes.
template <typename V, bool ACCUM, bool B0>
__global__ void __launch_bounds__(kT)
k_coo(const int *__restrict__ row, const int *__restrict__ col, const V *__restrict__ val, int64_t nnz,
      const V *__restrict__ x, V *__restrict__ y, int64_t n_rows, double alpha, double beta,
      int64_t *__restrict__ carry_row, double *__restrict__ carry_val) {
    __shared__ int s_row[kCooItems + 1];
    __shared__ double s_prod[kCooItems];
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    const int64_t k0 = (int64_t)blockIdx.x * kCooItems;
    const int cnt = (int)(nnz - k0 < kCooItems ? nnz - k0 : kCooItems);
#pragma unroll
    for (int u = 0; u < kIPT; ++u) {
        int i = threadIdx.x + u * kT;
        if (i < cnt) {
            int c = ld_hint(col + k0 + i, pa);
            V v = ld_hint(val + k0 + i, pa);
            s_row[i] = ld_hint(row + k0 + i, pa);
            s_prod[i] = (double)v * (double)ld_x(x + c, px);
        }
    }
    if (threadIdx.x == 0) s_row[cnt] = k0 + cnt < nnz ? row[k0 + cnt] : (int)n_rows;   // sentinel
    __syncthreads();
    if (!ACCUM && blockIdx.x == 0 && threadIdx.x == 0)      // leading empty rows [0, row[0])
        for (int r = 0; r < s_row[0]; ++r) y_beta<V, B0>(y, r, beta);

    const int i0 = threadIdx.x * kIPT;
    const int i1 = min(i0 + kIPT, cnt);
    bool has_end = false;
    double acc = 0.0, first_sum = 0.0;
    int first_row = -1;
    for (int i = i0; i < i1; ++i) {
        acc += s_prod[i];
        const int r = s_row[i], rn = s_row[i + 1];
        if (rn != r) {                                   // row r ends at element i
            if (!has_end) { first_sum = acc; first_row = r; has_end = true; }
            else if (ACCUM) y[r] = (V)((double)y[r] + alpha * acc);
            else y_write<V, B0>(y, r, acc, alpha, beta);
            if (!ACCUM)
                for (int g = r + 1; g < rn; ++g) y_beta<V, B0>(y, g, beta);   // empty rows in the gap
            acc = 0.0;
        }
    }
    double incl;
    const double carry_in = block_seg_scan(has_end || i0 >= cnt, i0 < cnt ? acc : 0.0, &incl);
    if (has_end) {
        const double s = first_sum + carry_in;
        if (ACCUM) y[first_row] = (V)((double)y[first_row] + alpha * s);
        else y_write<V, B0>(y, first_row, s, alpha, beta);
    }
    // CTA carry: the thread holding the last element
    if (i0 < cnt && i1 == cnt) {
        const bool open = s_row[cnt] == s_row[cnt - 1];
        carry_row[blockIdx.x] = open ? s_row[cnt - 1] : -1;
        carry_val[blockIdx.x] = open ? incl : 0.0;
    }
}

// ------------------------------------------------------------------ merge-based CSR (K7/G11)
// "logically partitions the work of processing a group of contiguous
// rows into equal sized sub-problems".  CTA t consumes merge-path diagonals
// [t*T, (t+1)*T) of (row ends) x (nonzeros) (coordinates precomputed at conversion,
// A7).  Row ends and products are staged in shared memory with coalesced loads
// (all x gathers of the tile in flight at once); each thread then consumes kIPT
// consecutive items of the path.
template <typename V, typename IT, bool B0>
__global__ void __launch_bounds__(kT)
k_merge(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val,
        const int64_t *__restrict__ crow, const int64_t *__restrict__ cnz, int64_t n_rows,
        const V *__restrict__ x, V *__restrict__ y, double alpha, double beta,
        int64_t *__restrict__ carry_row, double *__restrict__ carry_val) {
    __shared__ int s_end[kMergeItems];
    __shared__ double s_prod[kMergeItems];
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    const int64_t t = blockIdx.x;
    const int64_t r0 = crow[t], k0 = cnz[t], r1 = crow[t + 1], k1 = cnz[t + 1];
    const int nrows = (int)(r1 - r0), nnzt = (int)(k1 - k0), items = nrows + nnzt;
    for (int i = threadIdx.x; i < nrows; i += kT) s_end[i] = (int)((int64_t)__ldg(rp + r0 + 1 + i) - k0);
#pragma unroll
    for (int u = 0; u < kIPT; ++u) {
        int j = threadIdx.x + u * kT;
        if (j < nnzt) {
            int c = ld_hint(col + k0 + j, pa);
            V v = ld_hint(val + k0 + j, pa);
            s_prod[j] = (double)v * (double)ld_x(x + c, px);
        }
    }
    __syncthreads();
    // this thread's start on the tile's merge path: largest i with s_end[i-1] + i <= d
    const int d = threadIdx.x * kIPT;
    const int nit = max(0, min(kIPT, items - d));
    int lo = max(0, d - nnzt), hi = min(d, nrows);
    while (lo < hi) {
        int mid = (lo + hi + 1) >> 1;
        if (s_end[mid - 1] + mid <= d) lo = mid; else hi = mid - 1;
    }
    int i = lo, j = d - lo;
    bool has_end = false;
    double acc = 0.0, first_sum = 0.0;
    int64_t first_row = -1;
    for (int it = 0; it < nit; ++it) {
        if (i < nrows && s_end[i] <= j) {                // row r0+i ends (A7 tie-break)
            if (!has_end) { first_sum = acc; first_row = r0 + i; has_end = true; }
            else y_write<V, B0>(y, r0 + i, acc, alpha, beta);
            acc = 0.0;
            ++i;
        } else {
            acc += s_prod[j];
            ++j;
        }
    }
    double incl;
    const double carry_in = block_seg_scan(has_end || nit == 0, nit ? acc : 0.0, &incl);
    if (has_end) y_write<V, B0>(y, first_row, first_sum + carry_in, alpha, beta);
    // tile carry: nonzeros after the tile's last row end belong to row r1 (ends later)
    if (nit > 0 && d + nit == items) {
        const bool open = r1 < n_rows && k1 > (nrows ? k0 + s_end[nrows - 1] : k0);
        carry_row[t] = open ? r1 : -1;
        carry_val[t] = open ? incl : 0.0;
    }
    if (items == 0 && threadIdx.x == 0) carry_row[t] = -1;
}

// ------------------------------------------------------------------ CSR5 (K6/G12)
// equally sized 2-D tiles (32 lanes x sigma) with tile_ptr and
// tile_desc.  One warp per tile.  Lane l holds elements t*W + l*sigma + s stored
// lane-interleaved (A6) so each lane issues 16-byte loads.  Segments (rows) closed
// inside a lane are written directly; the segment a lane opens last is completed by
// a flag-segmented suffix sum of the next lanes' heads (shuffles; y_offset gives the
// segment index, the empty-row map or row_lo gives its row).  The tile's leading
// partial (row tile_ptr[t], started in an earlier tile) is the tile carry.
template <int SIGMA, typename V>
struct Csr5Vec;
template <int SIGMA>
struct Csr5Vec<SIGMA, double> {
    static __device__ __forceinline__ void load(const double *val, int64_t base, int lane, double (&v)[SIGMA], uint64_t pol) {
#pragma unroll
        for (int q = 0; q < SIGMA / 2; ++q) {
            double2 w = ld_hint(reinterpret_cast<const double2 *>(val + base + q * 64 + lane * 2), pol);
            v[2 * q] = w.x;
            v[2 * q + 1] = w.y;
        }
    }
};
template <int SIGMA>
struct Csr5Vec<SIGMA, float> {
    static __device__ __forceinline__ void load(const float *val, int64_t base, int lane, float (&v)[SIGMA], uint64_t pol) {
#pragma unroll
        for (int q = 0; q < SIGMA / 4; ++q) {
            float4 w = ld_hint(reinterpret_cast<const float4 *>(val + base + q * 128 + lane * 4), pol);
            v[4 * q] = w.x; v[4 * q + 1] = w.y; v[4 * q + 2] = w.z; v[4 * q + 3] = w.w;
        }
    }
};

template <int SIGMA, typename V, typename IT, bool B0>
__global__ void __launch_bounds__(kT)
k_csr5(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val,
       const int64_t *__restrict__ tile_ptr, const int64_t *__restrict__ row_lo,
       const unsigned *__restrict__ desc, const int64_t *__restrict__ map_off,
       const int64_t *__restrict__ seg_map, int64_t n_tiles, int64_t nnz,
       const V *__restrict__ x, V *__restrict__ y, double alpha, double beta,
       int64_t *__restrict__ carry_row, double *__restrict__ carry_val) {
    constexpr int64_t W = 32 * SIGMA;
    const int lane = threadIdx.x & 31;
    const int64_t t = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    if (t > n_tiles) return;
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    if (t == n_tiles) {
        // tail carry: the row holding element n_tiles*W when it started in a full tile
        const int64_t e = n_tiles * W;
        double s = 0.0;
        int64_t r = -1;
        if (e < nnz) {
            r = tile_ptr[n_tiles];
            if ((int64_t)rp[r] < e) {
                const int64_t end = rp[r + 1];
                for (int64_t k = e + lane; k < end; k += 32) s += (double)val[k] * (double)ld_x(x + col[k], px);
            } else {
                r = -1;
            }
        }
        s = warp_sum(s);
        if (lane == 0) { carry_row[n_tiles] = r; carry_val[n_tiles] = r >= 0 ? s : 0.0; }
        return;
    }
    const int64_t base = t * W;
    const unsigned d = __ldg(desc + t * 32 + lane);
    int c[SIGMA];
#pragma unroll
    for (int q = 0; q < SIGMA / 4; ++q) {
        int4 w = ld_hint(reinterpret_cast<const int4 *>(col + base + q * 128 + lane * 4), pa);
        c[4 * q] = w.x; c[4 * q + 1] = w.y; c[4 * q + 2] = w.z; c[4 * q + 3] = w.w;
    }
    V v[SIGMA];
    Csr5Vec<SIGMA, V>::load(val, base, lane, v, pa);
    double p[SIGMA];
#pragma unroll
    for (int s = 0; s < SIGMA; ++s) p[s] = (double)v[s] * (double)ld_x(x + c[s], px);

    const unsigned flag = d & 0xFFFFu;
    const int y_off = (int)((d >> 16) & 0x1FFu);
    const int64_t lo = __ldg(row_lo + t);
    const int64_t moff = __ldg(map_off + t);
    auto seg_row = [&](int idx) -> int64_t { return moff >= 0 ? __ldg(seg_map + moff + idx) : lo + idx; };

    double acc = 0.0, head = 0.0;
    int kseg = 0;
#pragma unroll
    for (int s = 0; s < SIGMA; ++s) {
        if ((flag >> s) & 1u) {
            if (kseg == 0) head = acc;
            else y_write<V, B0>(y, seg_row(y_off + kseg - 1), acc, alpha, beta);   // closed in-lane
            ++kseg;
            acc = 0.0;
        }
        acc += p[s];
    }
    if (kseg == 0) head = acc;
    // R[l] = head[l] + (lane l has a flag ? 0 : R[l+1])  (flag-segmented suffix sum)
    double R = head;
    bool F = kseg > 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        double Rn = __shfl_down_sync(0xffffffffu, R, o);
        int Fn = __shfl_down_sync(0xffffffffu, (int)F, o);
        if (!F) {
            if (lane + o < 32) { R += Rn; F = Fn; }
            else F = true;
        }
    }
    double Rnext = __shfl_down_sync(0xffffffffu, R, 1);
    if (lane == 31) Rnext = 0.0;
    if (kseg > 0) y_write<V, B0>(y, seg_row(y_off + kseg - 1), acc + Rnext, alpha, beta);
    if (lane == 0) {
        const bool lead = !(flag & 1u);
        carry_row[t] = lead ? __ldg(tile_ptr + t) : -1;
        carry_val[t] = lead ? R : 0.0;
    }
    if (moff >= 0) {                                     // empty rows of the tile's range
        const int64_t hi = __ldg(row_lo + t + 1);
        for (int64_t r = lo + lane; r < hi; r += 32)
            if (__ldg(rp + r + 1) == __ldg(rp + r)) y_beta<V, B0>(y, r, beta);
    }
}

// ------------------------------------------------------------------ fix-up (G13)
template <typename V>
__global__ void k_fixup(const int64_t *__restrict__ carry_row, const double *__restrict__ carry_val, int64_t n,
                        V *__restrict__ y, double alpha) {
    for (int64_t c = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; c < n; c += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = carry_row[c];
        if (r < 0 || (c > 0 && carry_row[c - 1] == r)) continue;
        double s = 0.0;
        for (int64_t q = c; q < n && carry_row[q] == r; ++q) s += carry_val[q];
        y[r] = (V)((double)y[r] + alpha * s);
    }
}

// ------------------------------------------------------------------ launch helpers

int grid_stride_blocks(const spmv_ctx *ctx, int64_t threads_needed, int per_sm) {
    int64_t g = ceil_div<int64_t>(threads_needed, kT);
    int64_t cap = (int64_t)ctx->sm_count * per_sm;
    return (int)std::max<int64_t>(1, std::min(g, cap));
}

template <typename V, bool B0>
spmv_status launch_scale(spmv_handle *h, V *y, double beta, cudaStream_t s) {
    if (h->n_rows == 0) return SPMV_OK;
    k_scale<V, B0><<<grid_stride_blocks(h->ctx, h->n_rows, 16), kT, 0, s>>>(y, h->n_rows, beta);
    SPMV_LAUNCH_CHECK();
    return SPMV_OK;
}

template <typename V>
spmv_status launch_fixup(spmv_handle *h, V *y, double alpha, cudaStream_t s) {
    if (h->n_carry == 0) return SPMV_OK;
    k_fixup<V><<<grid_stride_blocks(h->ctx, h->n_carry, 16), kT, 0, s>>>(
        (const int64_t *)h->carry_row.p, (const double *)h->carry_val.p, h->n_carry, y, alpha);
    SPMV_LAUNCH_CHECK();
    return SPMV_OK;
}

template <typename V, typename IT, bool B0>
spmv_status launch_csr_vector(const spmv_handle *h, const IT *rp, const int *col, const V *val, const V *x, V *y,
                              int64_t n, int w, double alpha, double beta, cudaStream_t s) {
    if (n == 0) return SPMV_OK;
    // 16 CTAs (4096 threads) per SM of grid-stride warps
    const int64_t threads = ceil_div<int64_t>(n, 32 / w) * 32;
    const int g = grid_stride_blocks(h->ctx, threads, 16);
#define SPMV_VEC(WW) k_csr_vector<V, IT, WW, B0><<<g, kT, 0, s>>>(rp, col, val, x, y, n, alpha, beta)
    switch (w) {
    case 1: case 2: SPMV_VEC(2); break;
    case 4: SPMV_VEC(4); break;
    case 8: SPMV_VEC(8); break;
    case 16: SPMV_VEC(16); break;
    default: SPMV_VEC(32); break;
    }
#undef SPMV_VEC
    SPMV_LAUNCH_CHECK();
    return SPMV_OK;
}

template <typename V, typename IT, bool B0>
spmv_status run_t(spmv_handle *h, double alpha, double beta, const V *x, V *y, cudaStream_t s) {
    if (alpha == 0.0) return launch_scale<V, B0>(h, y, beta, s);   // A14: A not read
    const int64_t n = h->n_rows;
    const IT *rp = (const IT *)h->arr[SPMV_ARR_ROW_PTR].p;
    const int *col = (const int *)h->arr[SPMV_ARR_COL].p;
    const V *val = (const V *)h->arr[SPMV_ARR_VAL].p;
    int64_t *crow = (int64_t *)h->carry_row.p;
    double *cval = (double *)h->carry_val.p;
    switch (h->fmt) {
    case SPMV_CSR:
        return launch_csr_vector<V, IT, B0>(h, rp, col, val, x, y, n, (int)h->vec_w, alpha, beta, s);
    case SPMV_CSR_SCALAR:
        if (n == 0) return SPMV_OK;
        k_csr_scalar<V, IT, B0><<<grid_stride_blocks(h->ctx, n, 16), kT, 0, s>>>(rp, col, val, x, y, n, alpha, beta);
        SPMV_LAUNCH_CHECK();
        return SPMV_OK;
    case SPMV_ELL:
        if (n == 0) return SPMV_OK;
        k_ell<V, B0><<<grid_stride_blocks(h->ctx, n, 16), kT, 0, s>>>(
            (const int *)h->arr[SPMV_ARR_ELL_COL].p, (const V *)h->arr[SPMV_ARR_ELL_VAL].p, h->ell_K, h->ell_ld,
            x, y, n, alpha, beta);
        SPMV_LAUNCH_CHECK();
        return SPMV_OK;
    case SPMV_HYB: {
        if (n == 0) return SPMV_OK;
        k_ell<V, B0><<<grid_stride_blocks(h->ctx, n, 16), kT, 0, s>>>(
            (const int *)h->arr[SPMV_ARR_ELL_COL].p, (const V *)h->arr[SPMV_ARR_ELL_VAL].p, h->ell_K, h->ell_ld,
            x, y, n, alpha, beta);
        SPMV_LAUNCH_CHECK();
        if (h->hyb_coo_nnz == 0) return SPMV_OK;
        k_coo<V, true, B0><<<(unsigned)h->n_carry, kT, 0, s>>>(
            (const int *)h->arr[SPMV_ARR_COO_ROW].p, (const int *)h->arr[SPMV_ARR_HYB_COO_COL].p,
            (const V *)h->arr[SPMV_ARR_HYB_COO_VAL].p, h->hyb_coo_nnz, x, y, n, alpha, beta, crow, cval);
        SPMV_LAUNCH_CHECK();
        return launch_fixup<V>(h, y, alpha, s);
    }
    case SPMV_COO:
        if (h->nnz == 0) return launch_scale<V, B0>(h, y, beta, s);
        k_coo<V, false, B0><<<(unsigned)h->n_carry, kT, 0, s>>>(
            (const int *)h->arr[SPMV_ARR_COO_ROW].p, col, val, h->nnz, x, y, n, alpha, beta, crow, cval);
        SPMV_LAUNCH_CHECK();
        return launch_fixup<V>(h, y, alpha, s);
    case SPMV_MERGE:
        if (h->merge_tiles == 0) return SPMV_OK;
        k_merge<V, IT, B0><<<(unsigned)h->merge_tiles, kT, 0, s>>>(
            rp, col, val, (const int64_t *)h->arr[SPMV_ARR_MERGE_COORD_ROW].p,
            (const int64_t *)h->arr[SPMV_ARR_MERGE_COORD_NZ].p, n, x, y, alpha, beta, crow, cval);
        SPMV_LAUNCH_CHECK();
        return launch_fixup<V>(h, y, alpha, s);
    case SPMV_CSR5: {
        const int64_t warps = h->n_tiles + 1;
        const unsigned g = (unsigned)ceil_div<int64_t>(warps * 32, kT);
#define SPMV_CSR5_LAUNCH(SG)                                                                                  \
    k_csr5<SG, V, IT, B0><<<g, kT, 0, s>>>(rp, col, val, (const int64_t *)h->arr[SPMV_ARR_CSR5_TILE_PTR].p,   \
                                           (const int64_t *)h->arr[SPMV_ARR_CSR5_ROW_LO].p,                    \
                                           (const unsigned *)h->arr[SPMV_ARR_CSR5_TILE_DESC].p,                \
                                           (const int64_t *)h->arr[SPMV_ARR_CSR5_MAP_OFF].p,                   \
                                           (const int64_t *)h->arr[SPMV_ARR_CSR5_SEG_MAP].p, h->n_tiles,       \
                                           h->nnz, x, y, alpha, beta, crow, cval)
        switch (h->sigma) {
        case 4: SPMV_CSR5_LAUNCH(4); break;
        case 8: SPMV_CSR5_LAUNCH(8); break;
        case 12: SPMV_CSR5_LAUNCH(12); break;
        default: SPMV_CSR5_LAUNCH(16); break;
        }
#undef SPMV_CSR5_LAUNCH
        SPMV_LAUNCH_CHECK();
        // rows that start in the tail (< one tile of nonzeros left): CSR-vector
        const int64_t r_tail = h->csr5_tail_row;
        if (r_tail < n)
            SPMV_TRY((launch_csr_vector<V, IT, B0>(h, rp + r_tail, col, val, x, y + r_tail, n - r_tail, 32, alpha,
                                                   beta, s)));
        return launch_fixup<V>(h, y, alpha, s);
    }
    }
    set_error("unknown format");
    return SPMV_ERR_INVALID_ARG;
}

template <typename V>
spmv_status run_v(spmv_handle *h, double alpha, double beta, const void *x, void *y, cudaStream_t s) {
    const V *xv = (const V *)x;
    V *yv = (V *)y;
    if (h->itype == SPMV_I32)
        return beta == 0.0 ? run_t<V, int, true>(h, alpha, beta, xv, yv, s) : run_t<V, int, false>(h, alpha, beta, xv, yv, s);
    return beta == 0.0 ? run_t<V, int64_t, true>(h, alpha, beta, xv, yv, s)
                       : run_t<V, int64_t, false>(h, alpha, beta, xv, yv, s);
}

}  // namespace

spmv_status run_impl(spmv_handle *h, double alpha, double beta, const void *x, void *y, cudaStream_t s) {
    return h->dtype == SPMV_F64 ? run_v<double>(h, alpha, beta, x, y, s) : run_v<float>(h, alpha, beta, x, y, s);
}

int run_launch_count(const spmv_handle *h, bool alpha0) {
    if (alpha0) return h->n_rows ? 1 : 0;
    switch (h->fmt) {
    case SPMV_CSR: case SPMV_CSR_SCALAR: case SPMV_ELL: return h->n_rows ? 1 : 0;
    case SPMV_HYB: return (h->n_rows ? 1 : 0) + (h->hyb_coo_nnz ? 2 : 0);
    case SPMV_COO: return h->nnz ? 2 : (h->n_rows ? 1 : 0);
    case SPMV_MERGE: return h->merge_tiles ? 2 : 0;
    case SPMV_CSR5: return 1 + (h->csr5_tail_row < h->n_rows ? 1 : 0) + 1;
    }
    return 0;
}

}  // namespace spmv
