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
// "assign a WARP to process a row".  A W-lane group per row (A5).
// One warp iteration covers R = (32/W)*U consecutive rows: their row pointers come
// from one coalesced load (+ shuffles), every group issues the first 2W elements of
// each of its U rows before any x gather, and y is prefetched with the row
// pointers, so a warp keeps ~2U independent loads per lane in flight even when
// rows are as short as the 5-point stencil's.  Rows longer than 2W continue in a
// four-accumulator loop folded every kFold steps (A13).
template <int W> struct VecCfg { static constexpr int U = W <= 8 ? 4 : (W == 16 ? 2 : 1); };

template <typename V, typename IT, int W, bool B0>
__global__ void __launch_bounds__(kT)
k_csr_vector(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val,
             const V *__restrict__ x, V *__restrict__ y, int64_t n, double alpha, double beta) {
    constexpr int G = 32 / W;
    constexpr int U = (VecCfg<W>::U * G > 32) ? 32 / G : VecCfg<W>::U;
    constexpr int R = G * U;                      // rows per warp iteration (<= 32)
    const int lane = threadIdx.x & 31;
    const int sub = lane & (W - 1);
    const int g = lane / W;
    const int64_t gwarp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    for (int64_t base = gwarp * R; base < n; base += nwarps * R) {
        const int64_t rp_lo = (int64_t)__ldg(rp + (base + lane < n ? base + lane : n));
        const int64_t rp_hi = (int64_t)__ldg(rp + (base + R < n ? base + R : n));
        double yv[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t r = base + u * G + g;
            yv[u] = (!B0 && sub == 0 && r < n) ? (double)y[r] : 0.0;
        }
        int64_t a[U], b[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int i = u * G + g;                         // row index within the batch
            a[u] = __shfl_sync(0xffffffffu, rp_lo, i);
            const int64_t nx = __shfl_sync(0xffffffffu, rp_lo, (i + 1) & 31);
            b[u] = i + 1 < R ? nx : rp_hi;
            if (base + i >= n) { a[u] = 0; b[u] = 0; }
        }
        // first 2W elements of every row, all loads issued together
        int c0[U], c1[U];
        V v0[U], v1[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t k = a[u] + sub;
            c0[u] = k < b[u] ? ld_hint(col + k, pa) : -1;
            v0[u] = k < b[u] ? ld_hint(val + k, pa) : (V)0;
            c1[u] = k + W < b[u] ? ld_hint(col + k + W, pa) : -1;
            v1[u] = k + W < b[u] ? ld_hint(val + k + W, pa) : (V)0;
        }
        double s[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            double t0 = c0[u] >= 0 ? (double)v0[u] * (double)ld_x(x + c0[u], px) : 0.0;
            double t1 = c1[u] >= 0 ? (double)v1[u] * (double)ld_x(x + c1[u], px) : 0.0;
            s[u] = t0 + t1;
        }
        // long rows: the rest with four accumulators
#pragma unroll
        for (int u = 0; u < U; ++u) {
            int64_t k = a[u] + sub + 2 * W;
            if (k >= b[u]) continue;
            double tot = 0.0, a0 = 0.0, a1 = 0.0, a2 = 0.0, a3 = 0.0;
            int it = 0;
            for (; k + 3 * W < b[u]; k += 4 * W) {
                int d0 = ld_hint(col + k, pa), d1 = ld_hint(col + k + W, pa);
                int d2 = ld_hint(col + k + 2 * W, pa), d3 = ld_hint(col + k + 3 * W, pa);
                V w0 = ld_hint(val + k, pa), w1 = ld_hint(val + k + W, pa);
                V w2 = ld_hint(val + k + 2 * W, pa), w3 = ld_hint(val + k + 3 * W, pa);
                a0 += (double)w0 * (double)ld_x(x + d0, px);
                a1 += (double)w1 * (double)ld_x(x + d1, px);
                a2 += (double)w2 * (double)ld_x(x + d2, px);
                a3 += (double)w3 * (double)ld_x(x + d3, px);
                if (++it == kFold) {                     // blocked summation (A13)
                    tot += (a0 + a1) + (a2 + a3);
                    a0 = a1 = a2 = a3 = 0.0;
                    it = 0;
                }
            }
            for (; k < b[u]; k += W) a0 += (double)ld_hint(val + k, pa) * (double)ld_x(x + ld_hint(col + k, pa), px);
            s[u] += tot + ((a0 + a1) + (a2 + a3));
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
#pragma unroll
            for (int o = W / 2; o > 0; o >>= 1) s[u] += __shfl_xor_sync(0xffffffffu, s[u], o);
        }
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t r = base + u * G + g;
            if (sub == 0 && r < n) {
                double o = alpha * s[u];
                if (!B0) o = fma(beta, yv[u], o);
                y[r] = (V)o;
            }
        }
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
        const double yv = B0 ? 0.0 : (double)y[r];
        double a0 = 0.0, a1 = 0.0;
        int64_t k = __ldg(rp + r), b = __ldg(rp + r + 1);
        for (; k + 1 < b; k += 2) {
            a0 += (double)__ldg(val + k) * (double)ld_x(x + __ldg(col + k), px);
            a1 += (double)__ldg(val + k + 1) * (double)ld_x(x + __ldg(col + k + 1), px);
        }
        if (k < b) a0 += (double)__ldg(val + k) * (double)ld_x(x + __ldg(col + k), px);
        double o = alpha * (a0 + a1);
        if (!B0) o = fma(beta, yv, o);
        y[r] = (V)o;
    }
}

// ------------------------------------------------------------------ ELL (K4/G9)
// column-major, "each row is processed by a single thread".
// Slots are consumed kEllBatch at a time with predicated loads (all in flight before
// the first x gather); y is loaded before the slots.  Padding carries col = -1 (A3).
constexpr int kEllBatch = 8;

template <typename V, bool B0>
__global__ void __launch_bounds__(kT)
k_ell(const int *__restrict__ ecol, const V *__restrict__ eval, int64_t K, int64_t ld,
      const V *__restrict__ x, V *__restrict__ y, int64_t n, double alpha, double beta) {
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
        const double yv = B0 ? 0.0 : (double)y[r];
        double tot = 0.0, part = 0.0;
        int nb = 0;
        for (int64_t j0 = 0; j0 < K; j0 += kEllBatch) {
            int c[kEllBatch];
            V v[kEllBatch];
#pragma unroll
            for (int u = 0; u < kEllBatch; ++u) {
                const bool in = j0 + u < K;
                c[u] = in ? ld_hint(ecol + (j0 + u) * ld + r, pa) : -1;
                v[u] = in ? ld_hint(eval + (j0 + u) * ld + r, pa) : (V)0;
            }
            double a0 = 0.0, a1 = 0.0;
#pragma unroll
            for (int u = 0; u < kEllBatch; u += 2) {
                if (c[u] >= 0) a0 += (double)v[u] * (double)ld_x(x + c[u], px);
                if (c[u + 1] >= 0) a1 += (double)v[u + 1] * (double)ld_x(x + c[u + 1], px);
            }
            part += a0 + a1;
            if (++nb == kFold) {                          // blocked summation (A13)
                tot += part;
                part = 0.0;
                nb = 0;
            }
        }
        tot += part;
        double o = alpha * tot;
        if (!B0) o = fma(beta, yv, o);
        y[r] = (V)o;
    }
}

// ------------------------------------------------------------------ COO (K1/G7)
// "first all product contributions are computed for the non-zero
// elements, followed by a segmented reduction across threads".  CTA c owns nonzeros
// [c*T, (c+1)*T): row ids and products staged in shared memory (coalesced loads, all
// x gathers of the chunk in flight), kIPT-item thread segments, a block segmented
// scan for the thread carries, a CTA carry for the fix-up.  The chunk writes the
// contiguous row window [R0, R1) (rows ending here + the empty rows before the next
// chunk's first row): y of the window is prefetched into registers during staging
// and written back coalesced; a window wider than kCooItems rows (huge gaps) spills
// to direct writes.  ACCUM (HYB's COO part): y += alpha*s for the rows present only.
template <typename V, bool ACCUM, bool B0>
__global__ void __launch_bounds__(kT)
k_coo(const int *__restrict__ row, const int *__restrict__ col, const V *__restrict__ val, int64_t nnz,
      const V *__restrict__ x, V *__restrict__ y, int64_t n_rows, double alpha, double beta,
      int64_t *__restrict__ carry_row, double *__restrict__ carry_val) {
    constexpr int kWin = (int)kCooItems;
    __shared__ int s_row[kCooItems + 1];
    __shared__ double s_prod[kCooItems];            // products, then per-row sums
    __shared__ unsigned s_mark[kCooItems / 32];
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    const int64_t k0 = (int64_t)blockIdx.x * kCooItems;
    const int cnt = (int)(nnz - k0 < kCooItems ? nnz - k0 : kCooItems);
    // row window of this chunk (uniform loads)
    const int64_t R0 = (!ACCUM && blockIdx.x == 0) ? 0 : (int64_t)__ldg(row + k0);
    const int64_t R1 = k0 + cnt < nnz ? (int64_t)__ldg(row + k0 + cnt) : n_rows;
    const int64_t L = R1 - R0;
    double yv[kIPT];
#pragma unroll
    for (int u = 0; u < kIPT; ++u) {
        const int i = threadIdx.x + u * kT;
        yv[u] = ((ACCUM || !B0) && i < L) ? (double)y[R0 + i] : 0.0;
    }
#pragma unroll
    for (int u = 0; u < kIPT; ++u) {
        const int i = threadIdx.x + u * kT;
        if (i < cnt) {
            const int c = ld_hint(col + k0 + i, pa);
            const V v = ld_hint(val + k0 + i, pa);
            s_row[i] = ld_hint(row + k0 + i, pa);
            s_prod[i] = (double)v * (double)ld_x(x + c, px);
        }
    }
    if (threadIdx.x < kCooItems / 32) s_mark[threadIdx.x] = 0u;
    if (threadIdx.x == 0) s_row[cnt] = (int)R1;
    __syncthreads();

    const int i0 = threadIdx.x * kIPT;
    const int i1 = min(i0 + kIPT, cnt);
    unsigned emask = 0;
    double ev[kIPT];
    double acc = 0.0;
#pragma unroll
    for (int it = 0; it < kIPT; ++it) {
        const int i = i0 + it;
        ev[it] = 0.0;
        if (i < i1) {
            acc += s_prod[i];
            const int r = s_row[i], rn = s_row[i + 1];
            if (rn != r) {                                 // row r ends at element i
                ev[it] = acc;
                emask |= 1u << it;
                acc = 0.0;
                if (!ACCUM)                                // empty rows beyond the staged window
                    for (int64_t gq = max((int64_t)r + 1, R0 + kWin); gq < rn; ++gq) y_beta<V, B0>(y, gq, beta);
            }
        }
    }
    double incl;
    const double carry_in = block_seg_scan(emask != 0 || i0 >= cnt, i0 < cnt ? acc : 0.0, &incl);
    bool first = true;
#pragma unroll
    for (int it = 0; it < kIPT; ++it) {
        if ((emask >> it) & 1u) {
            const double v = ev[it] + (first ? carry_in : 0.0);
            first = false;
            const int64_t r = s_row[i0 + it];
            const int64_t li = r - R0;
            if (li < kWin) {
                s_prod[li] = v;
                atomicOr(&s_mark[li >> 5], 1u << (li & 31));
            } else if (ACCUM) {
                y[r] = (V)((double)y[r] + alpha * v);
            } else {
                y_write<V, B0>(y, r, v, alpha, beta);
            }
        }
    }
    if (i0 < cnt && i1 == cnt) {                           // CTA carry: the row open at the chunk end
        const bool open = s_row[cnt] == s_row[cnt - 1];
        carry_row[blockIdx.x] = open ? s_row[cnt - 1] : -1;
        carry_val[blockIdx.x] = open ? incl : 0.0;
    }
    if (!ACCUM && blockIdx.x == 0)                         // leading empty rows beyond the window
        for (int64_t gq = kWin + threadIdx.x; gq < s_row[0]; gq += kT) y_beta<V, B0>(y, gq, beta);
    __syncthreads();
#pragma unroll
    for (int u = 0; u < kIPT; ++u) {
        const int i = threadIdx.x + u * kT;
        if (i < L && i < kWin) {
            const bool marked = (s_mark[i >> 5] >> (i & 31)) & 1u;
            if (ACCUM) {
                if (marked) y[R0 + i] = (V)(yv[u] + alpha * s_prod[i]);
            } else {
                double o = marked ? alpha * s_prod[i] : 0.0;
                if (!B0) o = marked ? fma(beta, yv[u], o) : beta * yv[u];
                y[R0 + i] = (V)o;
            }
        }
    }
}

// ------------------------------------------------------------------ merge-based CSR (K7/G11)
// "logically partitions the work of processing a group of contiguous
// rows into equal sized sub-problems".  CTA t consumes merge-path diagonals
// [t*T, (t+1)*T) of (row ends) x (nonzeros) (coordinates precomputed at conversion,
// A7).  Row ends and products are staged in shared memory with coalesced loads
// (all x gathers of the tile in flight at once); y of the tile's rows [r0, r1) is
// prefetched into registers at the same time.  Each thread consumes kIPT consecutive
// path items; after the block segmented scan the per-row sums go to shared memory
// and the tile writes y[r0, r1) coalesced.
template <typename V, typename IT, bool B0>
__global__ void __launch_bounds__(kT)
k_merge(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val,
        const int64_t *__restrict__ crow, const int64_t *__restrict__ cnz, int64_t n_rows,
        const V *__restrict__ x, V *__restrict__ y, double alpha, double beta,
        int64_t *__restrict__ carry_row, double *__restrict__ carry_val) {
    __shared__ int s_end[kMergeItems];
    __shared__ double s_prod[kMergeItems];          // products, then per-row sums
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    const int64_t t = blockIdx.x;
    const int64_t r0 = crow[t], k0 = cnz[t], r1 = crow[t + 1], k1 = cnz[t + 1];
    const int nrows = (int)(r1 - r0), nnzt = (int)(k1 - k0), items = nrows + nnzt;
    double yv[kIPT];
#pragma unroll
    for (int u = 0; u < kIPT; ++u) {
        const int i = threadIdx.x + u * kT;
        yv[u] = (!B0 && i < nrows) ? (double)y[r0 + i] : 0.0;
    }
#pragma unroll
    for (int u = 0; u < kIPT; ++u) {
        const int i = threadIdx.x + u * kT;
        if (i < nrows) s_end[i] = (int)((int64_t)__ldg(rp + r0 + 1 + i) - k0);
    }
#pragma unroll
    for (int u = 0; u < kIPT; ++u) {
        const int j = threadIdx.x + u * kT;
        if (j < nnzt) {
            const int c = ld_hint(col + k0 + j, pa);
            const V v = ld_hint(val + k0 + j, pa);
            s_prod[j] = (double)v * (double)ld_x(x + c, px);
        }
    }
    __syncthreads();
    // this thread's start on the tile's merge path: largest i with s_end[i-1] + i <= d
    const int d = threadIdx.x * kIPT;
    const int nit = max(0, min(kIPT, items - d));
    int lo = max(0, d - nnzt), hi = min(d, nrows);
    while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (s_end[mid - 1] + mid <= d) lo = mid; else hi = mid - 1;
    }
    int i = lo, j = d - lo;
    const int first_local = i;
    unsigned emask = 0;
    double ev[kIPT];
    double acc = 0.0;
#pragma unroll
    for (int it = 0; it < kIPT; ++it) {
        ev[it] = 0.0;
        if (it < nit) {
            if (i < nrows && s_end[i] <= j) {              // row r0+i ends (A7 tie-break)
                ev[it] = acc;
                emask |= 1u << it;
                acc = 0.0;
                ++i;
            } else {
                acc += s_prod[j];
                ++j;
            }
        }
    }
    double incl;
    const double carry_in = block_seg_scan(emask != 0 || nit == 0, nit ? acc : 0.0, &incl);
    // (the scan's barriers guarantee every walk is done: s_prod is free for row sums)
    int li = first_local;
    bool first = true;
#pragma unroll
    for (int it = 0; it < kIPT; ++it) {
        if ((emask >> it) & 1u) {
            s_prod[li] = ev[it] + (first ? carry_in : 0.0);
            first = false;
            ++li;
        }
    }
    // tile carry: nonzeros after the tile's last row end belong to row r1 (ends later)
    if (nit > 0 && d + nit == items) {
        const bool open = r1 < n_rows && k1 > (nrows ? k0 + s_end[nrows - 1] : k0);
        carry_row[t] = open ? r1 : -1;
        carry_val[t] = open ? incl : 0.0;
    }
    __syncthreads();
#pragma unroll
    for (int u = 0; u < kIPT; ++u) {
        const int q = threadIdx.x + u * kT;
        if (q < nrows) {
            double o = alpha * s_prod[q];
            if (!B0) o = fma(beta, yv[u], o);
            y[r0 + q] = (V)o;
        }
    }
}

// ------------------------------------------------------------------ CSR5 (K6/G12)
// equally sized 2-D tiles (32 lanes x sigma) with tile_ptr and
// tile_desc.  One warp per tile.  Lane l holds elements t*W + l*sigma + s stored
// lane-interleaved (A6) so each lane issues 16-byte loads.  Segments (rows) closed
// inside a lane are finished in-lane; the segment a lane opens last is completed by a
// flag-segmented suffix sum of the next lanes' heads (shuffles; y_offset gives the
// segment index, the empty-row map or row_lo gives its row).  The tile emits exactly
// the rows [row_lo[t], row_lo[t+1]): y of that window (up to kCsr5Win rows) is
// prefetched while the x gathers are in flight, the row sums are collected in a
// per-warp shared buffer and the window is written back coalesced (empty rows get
// beta*y).  The tile's leading partial (row tile_ptr[t], started in an earlier tile)
// is the tile carry.
constexpr int kCsr5Win = 128;

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
    constexpr int kQ = kCsr5Win / 32;
    __shared__ double s_acc[kT / 32][kCsr5Win];
    __shared__ unsigned s_mark[kT / 32][kCsr5Win / 32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
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
    const int64_t lo = __ldg(row_lo + t), hi = __ldg(row_lo + t + 1);
    const int64_t moff = __ldg(map_off + t);
    int c[SIGMA];
#pragma unroll
    for (int q = 0; q < SIGMA / 4; ++q) {
        int4 w = ld_hint(reinterpret_cast<const int4 *>(col + base + q * 128 + lane * 4), pa);
        c[4 * q] = w.x; c[4 * q + 1] = w.y; c[4 * q + 2] = w.z; c[4 * q + 3] = w.w;
    }
    V v[SIGMA];
    Csr5Vec<SIGMA, V>::load(val, base, lane, v, pa);
    const int64_t L = hi - lo;
    double yv[kQ];
#pragma unroll
    for (int q = 0; q < kQ; ++q) {
        const int i = lane + 32 * q;
        yv[q] = (!B0 && i < L) ? (double)y[lo + i] : 0.0;
    }
    if (lane < kCsr5Win / 32) s_mark[wid][lane] = 0u;
    double p[SIGMA];
#pragma unroll
    for (int s = 0; s < SIGMA; ++s) p[s] = (double)v[s] * (double)ld_x(x + c[s], px);
    __syncwarp();

    const unsigned flag = d & 0xFFFFu;
    const int y_off = (int)((d >> 16) & 0x1FFu);
    auto seg_row = [&](int idx) -> int64_t { return moff >= 0 ? __ldg(seg_map + moff + idx) : lo + idx; };
    auto emit = [&](int idx, double sum) {
        const int64_t r = seg_row(idx);
        const int64_t li = r - lo;
        if (li < kCsr5Win) {
            s_acc[wid][li] = sum;
            atomicOr(&s_mark[wid][li >> 5], 1u << (li & 31));
        } else {
            y_write<V, B0>(y, r, sum, alpha, beta);
        }
    };

    double acc = 0.0, head = 0.0;
    int kseg = 0;
#pragma unroll
    for (int s = 0; s < SIGMA; ++s) {
        if ((flag >> s) & 1u) {
            if (kseg == 0) head = acc;
            else emit(y_off + kseg - 1, acc);              // segment closed inside the lane
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
        const double Rn = __shfl_down_sync(0xffffffffu, R, o);
        const int Fn = __shfl_down_sync(0xffffffffu, (int)F, o);
        if (!F) {
            if (lane + o < 32) { R += Rn; F = Fn; }
            else F = true;
        }
    }
    double Rnext = __shfl_down_sync(0xffffffffu, R, 1);
    if (lane == 31) Rnext = 0.0;
    if (kseg > 0) emit(y_off + kseg - 1, acc + Rnext);
    if (lane == 0) {
        const bool lead = !(flag & 1u);
        carry_row[t] = lead ? __ldg(tile_ptr + t) : -1;
        carry_val[t] = lead ? R : 0.0;
    }
    __syncwarp();
    // write the window: segment rows alpha*s + beta*y, empty rows beta*y
#pragma unroll
    for (int q = 0; q < kQ; ++q) {
        const int i = lane + 32 * q;
        if (i < L) {
            const bool marked = (s_mark[wid][i >> 5] >> (i & 31)) & 1u;
            double o = marked ? alpha * s_acc[wid][i] : 0.0;
            if (!B0) o = marked ? fma(beta, yv[q], o) : beta * yv[q];
            y[lo + i] = (V)o;
        }
    }
    if (L > kCsr5Win && moff >= 0) {                       // empty rows beyond the window
        for (int64_t r = lo + kCsr5Win + lane; r < hi; r += 32)
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
