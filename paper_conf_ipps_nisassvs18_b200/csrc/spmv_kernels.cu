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
#include <climits>
#include <cstdlib>
#include <cstring>
#include <type_traits>

#include "internal.h"
#include "kernels.h"


namespace spmv {

namespace {

constexpr int kT = kRunThreads;
constexpr int kIPT = kItemsPerThread;
constexpr int kWIPT = kWarpItemsPerLane;
constexpr int kMinBlocks = 4;   // 4 CTAs x 256 threads per SM: <= 64 registers
constexpr int kFold = 256;
constexpr int kSubMax = 256;  // CSR-vector: longest remainder walked by a lane subgroup (else whole warp)
constexpr int kMergeRowsMB = 4;   // k_merge_rows CTAs per SM
constexpr int kCsrRowsMB = 4;     // k_csr_rows CTAs per SM   // sequential steps per accumulator before folding (A13)

// ------------------------------------------------------------------ helpers

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

// ------------------------------------------------------------------ PDL (CSR long rows)
// The CSR row kernel is launched programmatically dependent on k_csr_chunks (A25), which
// triggers its dependents at entry: the row kernel's CTAs fill the SMs beside the chunk
// CTAs (the two are independent), and each row-kernel thread waits for the chunk grid
// before exiting, so the fix-up launched after it sees the chunk carries.  Both are
// no-ops when the kernel is launched without the attribute.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

// ------------------------------------------------------------------ alpha == 0

// A30: xh[i] = x[hot[i]] -- the run's values of the handle's hot columns, packed densely
// so that the gathers to them hit L2 (and L1) four (fp64) / eight (fp32) per sector
template <typename V>
__global__ void k_hot_gather(const V *__restrict__ x, const int *__restrict__ hot, int64_t k, V *__restrict__ xh) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < k; i += (int64_t)gridDim.x * blockDim.x)
        xh[i] = __ldg(x + __ldg(hot + i));
}

template <typename V, bool B0>
__global__ void k_scale(V *y, int64_t n, double beta) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        y_beta<V, B0>(y, i, beta);
}

// ------------------------------------------------------------------ CSR-vector (K3/G8)
// "assign a WARP to process a row".  A W-lane group per row (A5).
// One warp iteration covers R = 32 consecutive rows (U rows per group): their row
// pointers come from one coalesced load (+ shuffles) issued one iteration ahead
// (software pipelined), and every group issues the first W elements of each of its U
// rows before any x gather, so a warp keeps U independent loads per lane in flight
// even when rows are as short as the 5-point stencil's.  Rows longer than W finish
// with the whole warp on one row at a time (8 loads per lane in flight, accumulators
// folded every kFold steps, A13) -- the paper's warp-per-row kernel for long rows.
// fp64 at W = 16: 16 rows per group (a 32-row batch, one claim of the dynamic scheduler at
// a time) -- R-MAT 24 CSR 1.81 -> 1.60 ms (U = 4: 1.81, 8: 1.72); fp32 keeps U = 4 (U = 8 /
// 16: 1.62 / 1.76 against 1.60 ms)
template <int W, typename V = double> struct VecCfg {
    static constexpr int U = W <= 8 ? 32 / (32 / W) : (W == 16 ? (sizeof(V) == 8 ? 16 : 4) : 2);
};

template <typename V, typename IT, int W, bool B0, int MB, bool CHUNKED, bool DYN = false, bool HOT = false>
__global__ void __launch_bounds__(kT, MB)
k_csr_vector(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val,
             const V *__restrict__ x, const V *__restrict__ xh, V *__restrict__ y, int64_t n, double alpha, double beta, int64_t long_len,
             unsigned long long *__restrict__ sched = nullptr) {
    constexpr int G = 32 / W;
    constexpr int U = (VecCfg<W, V>::U * G > 32) ? 32 / G : VecCfg<W, V>::U;
    constexpr int R = G * U;                      // rows per warp iteration (<= 32)
    const int lane = threadIdx.x & 31;
    const int sub = lane & (W - 1);
    const int g = lane / W;
    const int64_t gwarp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    // one batch of R rows: group g's U rows have nonzeros [a[u], b[u]); lane i < R holds
    // row i's range [my_a, my_e) (slot_ok: a live row) for the long-row walk; the writer
    // lane (sub < U) of each row writes y[my_row] (row_ok)
    auto batch = [&](const IT (&a)[U], const IT (&b)[U], const IT ra0, const IT rhi, const bool contiguous,
                     const bool slot_ok, const int64_t my_row, const bool row_ok) {
        // the y value this lane will write (writer lane sub == u of group g)
        const double yv = (!B0 && sub < U && row_ok) ? (double)y[my_row] : 0.0;
        // first W elements of every row, all loads issued together
        int c0[U];
        V v0[U];
#pragma unroll
        for (int u = 0; u < U; ++u) {
            const int64_t k = (int64_t)a[u] + sub;
            c0[u] = k < b[u] ? ld_hint(col + k, pa) : -1;
            v0[u] = k < b[u] ? ld_hint(val + k, pa) : (V)0;
        }
        double s[U];
#pragma unroll
        for (int u = 0; u < U; ++u) s[u] = c0[u] != -1 ? (double)v0[u] * (double)ldx<HOT>(x, xh, c0[u], px) : 0.0;
        // the group's U results: lane sub == u of group g writes row u*G + g
        double mine = 0.0;
        {
            // lane bits >= U do not index rows: plain butterflies over them; then a
            // transpose reduction over the low bits -- at offset o a lane keeps the half
            // of its partial sums selected by (sub & o) and adds the other half received
            // from lane sub ^ o, so lane sub ends with row (sub mod U)'s sum (U - 1
            // shuffles instead of a butterfly per row, U * log2(U))
#pragma unroll
            for (int o = W / 2; o >= U; o >>= 1) {
#pragma unroll
                for (int u = 0; u < U; ++u) s[u] += __shfl_xor_sync(0xffffffffu, s[u], o);
            }
#pragma unroll
            for (int o = U / 2; o > 0; o >>= 1) {
                const bool hi = (sub & o) != 0;
#pragma unroll
                for (int j = 0; j < o; ++j) {
                    const double send = hi ? s[j] : s[j + o];
                    const double keep = hi ? s[j + o] : s[j];
                    s[j] = keep + __shfl_xor_sync(0xffffffffu, send, o);
                }
            }
            mine = s[0];
        }
        // rows longer than W: the remainder is processed by the WHOLE warp, one row at a
        // time (the paper's warp-per-row vector kernel), 8 loads per lane in
        // flight, accumulators folded every kFold steps (A13); lane i holds row i's range
        {
            // lane i's row range, derived only here: contiguous batches hold row starts
            // (the batch end in rhi), compacted ones hold [start, end) directly
            const IT my_a = ra0;
            const IT nx = __shfl_sync(0xffffffffu, ra0, (lane + 1) & 31);
            const IT my_e = contiguous ? (lane + 1 < R ? nx : rhi) : rhi;
            const int64_t my_len = (int64_t)my_e - (int64_t)my_a;
            const bool is_long = slot_ok && my_len > W && (!CHUNKED || my_len <= long_len);
            // remainders of at most kSubMax: all such rows of the batch at once, a subgroup
            // of SW = 32 / next_pow2(count) lanes per row, 8 predicated loads per lane per
            // step -- one gather round trip for the batch instead of one per row (R-MAT's
            // many rows a little longer than W)
            const unsigned few = __ballot_sync(0xffffffffu, is_long && my_len - W <= kSubMax);
            unsigned more = __ballot_sync(0xffffffffu, is_long) & ~few;
            if (few) {
                const int nl = __popc(few);
                const int lg = nl > 1 ? 32 - __clz(nl - 1) : 0;
                const int SW = 32 >> lg;
                const int sg = lane >> (5 - lg), sl = lane & (SW - 1);
                const int ri = sg < nl ? (int)__fns(few, 0, sg + 1) : 0;
                const int64_t ra = (int64_t)__shfl_sync(0xffffffffu, my_a, ri) + W;
                const int64_t re = (int64_t)__shfl_sync(0xffffffffu, my_e, ri);
                const int64_t rb = sg < nl ? re : ra;
                double acc[8];
#pragma unroll
                for (int q = 0; q < 8; ++q) acc[q] = 0.0;
                for (int64_t k = ra + sl; k < rb; k += 8 * SW) {
                    int d[8];
                    V w[8];
#pragma unroll
                    for (int q = 0; q < 8; ++q) {
                        const bool in = k + q * SW < rb;
                        d[q] = in ? ld_hint(col + k + q * SW, pa) : -1;
                        w[q] = in ? ld_hint(val + k + q * SW, pa) : (V)0;
                    }
#pragma unroll
                    for (int q = 0; q < 8; ++q) if (d[q] != -1) acc[q] += (double)w[q] * (double)ldx<HOT>(x, xh, d[q], px);
                }
                double part = ((acc[0] + acc[1]) + (acc[2] + acc[3])) + ((acc[4] + acc[5]) + (acc[6] + acc[7]));
                for (int o = SW >> 1; o > 0; o >>= 1) part += __shfl_xor_sync(0xffffffffu, part, o);
                const int wi = g * U + (sub < U ? sub : 0);           // this lane's row (writer lanes)
                const bool wmine = sub < U && ((few >> wi) & 1u);
                const int src = (__popc(few & ((1u << wi) - 1u)) << (5 - lg)) & 31;
                const double got = __shfl_sync(0xffffffffu, part, src);
                if (wmine) mine += got;
            }
            while (more) {
                const int i = __ffs(more) - 1;
                more &= more - 1;
                const int64_t ra = (int64_t)__shfl_sync(0xffffffffu, my_a, i) + W;
                const int64_t rb = (int64_t)__shfl_sync(0xffffffffu, my_e, i);
                double tot = 0.0, acc[8];
#pragma unroll
                for (int q = 0; q < 8; ++q) acc[q] = 0.0;
                int it = 0;
                int64_t k = ra + lane;
                for (; k + 7 * 32 < rb; k += 8 * 32) {
                    int d[8];
                    V w[8];
#pragma unroll
                    for (int q = 0; q < 8; ++q) { d[q] = ld_hint(col + k + 32 * q, pa); w[q] = ld_hint(val + k + 32 * q, pa); }
#pragma unroll
                    for (int q = 0; q < 8; ++q) acc[q] += (double)w[q] * (double)ldx<HOT>(x, xh, d[q], px);
                    if (++it == kFold) {                 // blocked summation (A13)
#pragma unroll
                        for (int q = 0; q < 8; ++q) { tot += acc[q]; acc[q] = 0.0; }
                        it = 0;
                    }
                }
                for (; k < rb; k += 32) acc[0] += (double)ld_hint(val + k, pa) * (double)ldx<HOT>(x, xh, ld_hint(col + k, pa), px);
                double part = ((acc[0] + acc[1]) + (acc[2] + acc[3])) + ((acc[4] + acc[5]) + (acc[6] + acc[7]));
                part = warp_sum(tot + part);
                const int writer = (i / U) * W + i % U;   // lane holding row i's group sum
                if (lane == writer) mine += part;
            }
        }
        if (sub < U && row_ok) {
            double o = alpha * mine;
            if (!B0) o = fma(beta, yv, o);
            y[my_row] = (V)o;
        }
    };
    // DYN: warps take work from a global counter (zeroed before the launch), the next
    // claim requested one claim ahead -- balances skewed rows (a static grid stride left
    // R-MAT warps idle behind the slowest batch sequences).
    // fp32: a claim is a window of 64 rows whose rows with work (non-empty, not chunked)
    // are compacted into batches of R, so that a batch never spends its lanes on empty rows
    // (R-MAT: 57% of the rows); rows without work get beta*y (nothing to write when
    // beta == 1).  R-MAT 24 fp32 CSR 1.60 -> 1.40 ms.  fp64 keeps contiguous 32-row
    // batches, one per claim: compacted it measured 1.90 / 2.04 / 2.12 ms at 8 / 16 / 32-row
    // batches against 1.58.
    if constexpr (DYN && sizeof(V) == 4) {
        constexpr int WIN = 64;
        __shared__ int64_t s_row_all[kT / 32][WIN];
        __shared__ IT s_a_all[kT / 32][WIN], s_e_all[kT / 32][WIN];
        const int wid = threadIdx.x >> 5;
        int64_t *s_row = s_row_all[wid];
        IT *s_a = s_a_all[wid], *s_e = s_e_all[wid];
        unsigned long long g0 = 0, ng = 0;
        if (lane == 0) { g0 = atomicAdd(sched, 1ull); ng = atomicAdd(sched, 1ull); }
        int64_t wb = (int64_t)__shfl_sync(0xffffffffu, g0, 0) * WIN;
        IT q0 = 0, q1 = 0, q2 = 0;                    // row pointers of the next window (prefetched)
        auto load_win = [&](int64_t w0) {
            q0 = __ldg(rp + (w0 + lane < n ? w0 + lane : n));
            q1 = __ldg(rp + (w0 + 32 + lane < n ? w0 + 32 + lane : n));
            q2 = __ldg(rp + (w0 + WIN < n ? w0 + WIN : n));
        };
        if (wb < n) load_win(wb);
        while (wb < n) {
            const IT p0 = q0, p1 = q1, p2 = q2;
            const int64_t nb = (int64_t)__shfl_sync(0xffffffffu, ng, 0) * WIN;
            if (lane == 0) ng = atomicAdd(sched, 1ull);
            if (nb < n) load_win(nb);
            const IT n0 = __shfl_down_sync(0xffffffffu, p0, 1), n1 = __shfl_down_sync(0xffffffffu, p1, 1);
            const IT f1 = __shfl_sync(0xffffffffu, p1, 0);
            const IT e0 = lane == 31 ? f1 : n0, e1 = lane == 31 ? p2 : n1;
            const int64_t r0 = wb + lane, r1 = wb + 32 + lane;
            const int64_t l0 = (int64_t)e0 - (int64_t)p0, l1 = (int64_t)e1 - (int64_t)p1;
            const bool v0 = r0 < n, v1 = r1 < n;
            const bool w0 = v0 && l0 > 0 && (!CHUNKED || l0 <= long_len);
            const bool w1 = v1 && l1 > 0 && (!CHUNKED || l1 <= long_len);
            if (beta != 1.0) {                            // empty rows and chunked rows (A25)
                if (v0 && !w0) y_beta<V, B0>(y, r0, beta);
                if (v1 && !w1) y_beta<V, B0>(y, r1, beta);
            }
            const unsigned m0 = __ballot_sync(0xffffffffu, w0), m1 = __ballot_sync(0xffffffffu, w1);
            const int c0 = __popc(m0), T = c0 + __popc(m1);
            const unsigned lt = (1u << lane) - 1u;
            __syncwarp();                                 // the previous window's slots are consumed
            if (w0) { const int sl = __popc(m0 & lt); s_row[sl] = r0; s_a[sl] = p0; s_e[sl] = e0; }
            if (w1) { const int sl = c0 + __popc(m1 & lt); s_row[sl] = r1; s_a[sl] = p1; s_e[sl] = e1; }
            __syncwarp();
            for (int off = 0; off < T; off += R) {
                const bool ok = lane < R && off + lane < T;
                const int64_t my_r = ok ? s_row[off + lane] : 0;
                const IT my_a = ok ? s_a[off + lane] : (IT)0, my_e = ok ? s_e[off + lane] : (IT)0;
                IT a[U], b[U];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    a[u] = __shfl_sync(0xffffffffu, my_a, g * U + u);
                    b[u] = __shfl_sync(0xffffffffu, my_e, g * U + u);
                }
                const int ws = g * U + (sub < U ? sub : 0);
                const int64_t my_row = __shfl_sync(0xffffffffu, my_r, ws);
                batch(a, b, my_a, my_e, false, ok, my_row, sub < U && off + ws < T);
            }
            wb = nb;
        }
    } else {
        // claims of kDynGroup consecutive batches (fp64: 1 batch of 32 rows; R-MAT 24 with
        // 8-row batches: group 4 1.82 ms, 2 1.79, 8 1.84; 32-row batches: group 2 1.67, 1 1.60)
        constexpr int kDynGroup = sizeof(V) == 8 ? 1 : 4;
        unsigned long long ng = 0;
        int j = 0;
        int64_t base = gwarp * R;
        if constexpr (DYN) {
            unsigned long long g0 = 0;
            if (lane == 0) { g0 = atomicAdd(sched, 1ull); ng = atomicAdd(sched, 1ull); }
            base = (int64_t)__shfl_sync(0xffffffffu, g0, 0) * (kDynGroup * R);
        }
        IT nlo = 0, nhi = 0;                          // row pointers of the next batch (prefetched)
        if (base < n) {
            nlo = __ldg(rp + (base + lane < n ? base + lane : n));
            nhi = __ldg(rp + (base + R < n ? base + R : n));
        }
        while (base < n) {
            const IT rp_lo = nlo, rp_hi = nhi;
            int64_t nb = base + nwarps * R;
            if constexpr (DYN) {
                if (++j < kDynGroup) {
                    nb = base + R;
                } else {
                    j = 0;
                    nb = (int64_t)__shfl_sync(0xffffffffu, ng, 0) * (kDynGroup * R);
                    if (lane == 0) ng = atomicAdd(sched, 1ull);
                }
            }
            if (nb < n) {                             // issue the next batch's row pointers now
                nlo = __ldg(rp + (nb + lane < n ? nb + lane : n));
                nhi = __ldg(rp + (nb + R < n ? nb + R : n));
            }
            // group g owns the U consecutive rows g*U + u of the batch, so b[u] = a[u+1]:
            // U + 1 shuffles of the batch's row pointers (a row per group slot u*G + g took 2U)
            IT a[U], b[U];
            {
                IT e[U + 1];
#pragma unroll
                for (int u = 0; u <= U; ++u) {
                    const int i = g * U + u;
                    const IT t = __shfl_sync(0xffffffffu, rp_lo, i & 31);
                    e[u] = i < R ? t : rp_hi;
                }
#pragma unroll
                for (int u = 0; u < U; ++u) { a[u] = e[u]; b[u] = e[u + 1]; }
            }
#pragma unroll
            for (int u = 0; u < U; ++u) {
                if (base + g * U + u >= n) { a[u] = 0; b[u] = 0; }
                if (CHUNKED && (int64_t)b[u] - (int64_t)a[u] > long_len) b[u] = a[u];   // chunked long row (A25): beta*y here
            }
            const int64_t my_row = base + g * U + (sub < U ? sub : 0);
            batch(a, b, rp_lo, rp_hi, true, lane < R && base + lane < n, my_row, my_row < n);
            base = nb;
        }
    }
    // PDL after k_csr_chunks (chunked handles only): exit only once the chunk grid is
    // done.  Not compiled into the unchunked kernels: even with nothing to wait for it
    // cost LAP4096 7-15 %
    if constexpr (CHUNKED) pdl_wait();
}

// ------------------------------------------------------------------ CSR long-row chunks (A25)
// One warp per C-nonzero chunk of a long row (8 loads per lane in flight, blocked
// summation, A13); the chunk sum is the carry (row, value) that the fix-up adds in
// chunk order.  The row-batch kernel wrote beta*y for these rows.
template <typename V, typename IT, bool HOT = false>
__global__ void __launch_bounds__(kT)
k_csr_chunks(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val,
             const int64_t *__restrict__ crow, const int64_t *__restrict__ clo, int64_t nch, int64_t C,
             const V *__restrict__ x, const V *__restrict__ xh, int64_t *__restrict__ carry_row, double *__restrict__ carry_val) {
    pdl_trigger();
    const int lane = threadIdx.x & 31;
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    for (int64_t c = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; c < nch;
         c += ((int64_t)gridDim.x * blockDim.x) >> 5) {
        const int64_t r = __ldg(crow + c), lo = __ldg(clo + c);
        const int64_t re = (int64_t)__ldg(rp + r + 1);
        const int64_t hi = lo + C < re ? lo + C : re;
        double tot = 0.0, acc[8];
#pragma unroll
        for (int q = 0; q < 8; ++q) acc[q] = 0.0;
        int it = 0;
        int64_t k = lo + lane;
        for (; k + 7 * 32 < hi; k += 8 * 32) {
            int d[8];
            V w[8];
#pragma unroll
            for (int q = 0; q < 8; ++q) { d[q] = ld_hint(col + k + 32 * q, pa); w[q] = ld_hint(val + k + 32 * q, pa); }
#pragma unroll
            for (int q = 0; q < 8; ++q) acc[q] += (double)w[q] * (double)ldx<HOT>(x, xh, d[q], px);
            if (++it == kFold) {
#pragma unroll
                for (int q = 0; q < 8; ++q) { tot += acc[q]; acc[q] = 0.0; }
                it = 0;
            }
        }
        for (; k < hi; k += 32) acc[0] += (double)ld_hint(val + k, pa) * (double)ldx<HOT>(x, xh, ld_hint(col + k, pa), px);
        const double part = warp_sum(tot + (((acc[0] + acc[1]) + (acc[2] + acc[3])) + ((acc[4] + acc[5]) + (acc[6] + acc[7]))));
        if (lane == 0) { carry_row[c] = r; carry_val[c] = part; }
    }
}

// ------------------------------------------------------------------ CSR-scalar (K2)
// "assigning a thread to process each row -- the scalar CSR kernel".
template <typename V, typename IT, bool B0, bool HOT = false>
__global__ void __launch_bounds__(kT)
k_csr_scalar(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val,
             const V *__restrict__ x, const V *__restrict__ xh, V *__restrict__ y, int64_t n, double alpha, double beta) {
    const uint64_t px = policy_evict_last();
    for (int64_t r = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; r < n; r += (int64_t)gridDim.x * blockDim.x) {
        const double yv = B0 ? 0.0 : (double)y[r];
        double a0 = 0.0, a1 = 0.0;
        int64_t k = __ldg(rp + r), b = __ldg(rp + r + 1);
        for (; k + 1 < b; k += 2) {
            a0 += (double)__ldg(val + k) * (double)ldx<HOT>(x, xh, __ldg(col + k), px);
            a1 += (double)__ldg(val + k + 1) * (double)ldx<HOT>(x, xh, __ldg(col + k + 1), px);
        }
        if (k < b) a0 += (double)__ldg(val + k) * (double)ldx<HOT>(x, xh, __ldg(col + k), px);
        double o = alpha * (a0 + a1);
        if (!B0) o = fma(beta, yv, o);
        y[r] = (V)o;
    }
}

// ------------------------------------------------------------------ ELL (K4/G9)
// column-major, "each row is processed by a single thread".
// Slots are consumed BATCH at a time with predicated loads (all in flight before the
// first x gather); y is loaded before the slots.  RPT = 2: a thread owns two adjacent
// rows and reads each slot pair with one 8-byte (col) and one 16-/8-byte (val) load.
// Padding carries col = -1 (A3).
template <typename V, int RPT> struct EllVec;
template <typename V> struct EllVec<V, 1> {
    using CT = int;
    using VT = V;
};
template <> struct EllVec<double, 2> {
    using CT = int2;
    using VT = double2;
};
template <> struct EllVec<float, 2> {
    using CT = int2;
    using VT = float2;
};
template <> struct EllVec<double, 4> {
    using CT = int4;
    using VT = double4a;
};
template <> struct EllVec<float, 4> {
    using CT = int4;
    using VT = float4;
};
__device__ __forceinline__ int lane_of(const int &c, int) { return c; }
__device__ __forceinline__ int lane_of(const int2 &c, int r) { return r ? c.y : c.x; }
__device__ __forceinline__ int lane_of(const int4 &c, int r) { return r == 0 ? c.x : r == 1 ? c.y : r == 2 ? c.z : c.w; }
__device__ __forceinline__ double lane_of(const double4a &v, int r) { return r == 0 ? v.lo.x : r == 1 ? v.lo.y : r == 2 ? v.hi.x : v.hi.y; }
__device__ __forceinline__ float lane_of(const float4 &v, int r) { return r == 0 ? v.x : r == 1 ? v.y : r == 2 ? v.z : v.w; }

template <typename V> __device__ __forceinline__ V lane_of(const V &v, int) { return v; }
__device__ __forceinline__ double lane_of(const double2 &v, int r) { return r ? v.y : v.x; }
__device__ __forceinline__ float lane_of(const float2 &v, int r) { return r ? v.y : v.x; }

template <typename V, bool B0, int RPT, int BATCH, bool HOT = false>
__global__ void __launch_bounds__(kT)
k_ell(const int *__restrict__ ecol, const V *__restrict__ eval, int64_t K, int64_t ld,
      const V *__restrict__ x, const V *__restrict__ xh, V *__restrict__ y, int64_t n, double alpha, double beta) {
    using CT = typename EllVec<V, RPT>::CT;
    using VT = typename EllVec<V, RPT>::VT;
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    const int64_t nt = ceil_div<int64_t>(n, RPT);
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nt; t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r0 = t * RPT;
        double yv[RPT], tot[RPT], part[RPT];
#pragma unroll
        for (int q = 0; q < RPT; ++q) {
            yv[q] = (!B0 && r0 + q < n) ? (double)y[r0 + q] : 0.0;
            tot[q] = 0.0;
            part[q] = 0.0;
        }
        int nb = 0;
        for (int64_t j0 = 0; j0 < K; j0 += BATCH) {
            CT c[BATCH];
            VT v[BATCH];
#pragma unroll
            for (int u = 0; u < BATCH; ++u) {
                const bool in = j0 + u < K;
                if (in) {
                    c[u] = ld_hint(reinterpret_cast<const CT *>(ecol + (j0 + u) * ld + r0), pa);
                    v[u] = ld_hint(reinterpret_cast<const VT *>(eval + (j0 + u) * ld + r0), pa);
                } else {
                    c[u] = CT{};
                    v[u] = VT{};
                }
            }
#pragma unroll
            for (int q = 0; q < RPT; ++q) {
                double a0 = 0.0, a1 = 0.0;
#pragma unroll
                for (int u = 0; u < BATCH; u += 2) {
                    const int cu = lane_of(c[u], q);
                    if (j0 + u < K && cu != -1) a0 += (double)lane_of(v[u], q) * (double)ldx<HOT>(x, xh, cu, px);
                    if (u + 1 < BATCH) {
                        const int cw = lane_of(c[u + 1], q);
                        if (j0 + u + 1 < K && cw != -1) a1 += (double)lane_of(v[u + 1], q) * (double)ldx<HOT>(x, xh, cw, px);
                    }
                }
                part[q] += a0 + a1;
            }
            if (++nb == kFold) {                          // blocked summation (A13)
#pragma unroll
                for (int q = 0; q < RPT; ++q) { tot[q] += part[q]; part[q] = 0.0; }
                nb = 0;
            }
        }
#pragma unroll
        for (int q = 0; q < RPT; ++q) {
            if (r0 + q < n) {
                double o = alpha * (tot[q] + part[q]);
                if (!B0) o = fma(beta, yv[q], o);
                y[r0 + q] = (V)o;
            }
        }
    }
}

// ------------------------------------------------------------------ warp-tile helpers

// cp.async (LDGSTS): global -> shared without staging in registers
template <int B>
__device__ __forceinline__ void cp_async_n(void *smem, const void *gmem) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], %2;" ::"r"(s), "l"(gmem), "n"(B));
}
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_all;" ::: "memory"); }

// Flag-segmented suffix sum over the 32 lanes (CSR5's cross-lane step):
// R[l] = head[l] + (F[l] ? 0 : R[l+1]), F[l] = "lane l holds a segment start".
// Returns R[l+1] (0 for lane 31) in *Rnext and R[l].
__device__ __forceinline__ double seg_suffix(double head, bool flagged, double *Rnext) {
    const int lane = threadIdx.x & 31;
    // At the round with offset o a lane has stopped iff a flagged lane lies in
    // [lane, lane + o) or lane + o > 32 (induction over the rounds), so the stop state
    // comes from one ballot instead of a shuffle per round; the sums are unchanged.
    const unsigned fb = __ballot_sync(0xffffffffu, flagged);
    double R = head;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const double Rn = __shfl_down_sync(0xffffffffu, R, o);
        const bool F = lane + o > 32 || ((fb >> lane) & ((1u << o) - 1u)) != 0u;
        if (!F && lane + o < 32) R += Rn;
    }
    const double rn = __shfl_down_sync(0xffffffffu, R, 1);
    *Rnext = lane == 31 ? 0.0 : rn;
    return R;
}

// Per-warp output window: row sums land in shared memory, then the window
// [lo, lo+L) is written back coalesced (y prefetched in registers, kOutQ per lane).
constexpr int kOutWin = 128;
constexpr int kOutQ = kOutWin / 32;

// ------------------------------------------------------------------ COO (K1/G7)
// "first all product contributions are computed for the non-zero
// elements, followed by a segmented reduction across threads".  One warp owns a tile
// of 32 x kWIPT consecutive nonzeros, lane l the kWIPT consecutive elements
// [8l, 8l+8): row/col/val arrive with 16-byte vector loads straight into registers,
// all x gathers in flight together.  A new segment starts wherever the row id
// changes; segments closed inside a lane are finished in-lane, the last one a lane
// opens is completed by the flag-segmented suffix sum over lanes (as in CSR5).
// Rows that START in the tile are written by it (alpha*s + beta*y); a leading
// continuation of a row started in an earlier tile is the tile carry (fix-up); empty
// rows between the tile's rows and up to the next tile's first row get beta*y.  The
// tile's row window is staged in shared memory and written back coalesced.
// ACCUM (HYB's COO part): y += alpha*s for rows present, nothing else.
// 8 consecutive elements from a 32-byte aligned address, 256-bit loads
template <typename V> struct VecLoad8;
template <> struct VecLoad8<double> {
    static __device__ __forceinline__ void load(const double *p, double (&v)[8], uint64_t pol) {
        double a[4], b[4];
        ld256(p, a, pol);
        ld256(p + 4, b, pol);
#pragma unroll
        for (int q = 0; q < 4; ++q) { v[q] = a[q]; v[4 + q] = b[q]; }
    }
};
template <> struct VecLoad8<float> {
    static __device__ __forceinline__ void load(const float *p, float (&v)[8], uint64_t pol) { ld256(p, v, pol); }
};
__device__ __forceinline__ void load_int8(const int *p, int (&v)[8], uint64_t pol) { ld256(p, v, pol); }

// PERSIST (regular matrices, chosen at conversion: no empty row, rows of at most 32):
// warps loop over tiles on a grid of kCooPersistCtas CTAs/SM instead of one tile per warp --
// LAP4096 fp64 0.321 -> 0.307 ms; measured slower on R-MAT 24 (1.30 -> 1.36 ms) and fp32,
// so irregular matrices keep one tile per warp
constexpr int kCooPersistCtas = 8;
template <typename V, bool ACCUM, bool B0, bool HOT = false, bool PERSIST = false>
__global__ void __launch_bounds__(kT, kMinBlocks)
k_coo(const int *__restrict__ row, const int *__restrict__ col, const V *__restrict__ val, int64_t nnz,
      int64_t n_tiles, const V *__restrict__ x, const V *__restrict__ xh, V *__restrict__ y, int64_t n_rows, double alpha, double beta,
      int64_t *__restrict__ carry_row, double *__restrict__ carry_val) {
    static_assert(kWIPT == 8, "COO lane chunk is 8 elements");
    __shared__ double s_acc_all[kT / 32][kOutWin];
    __shared__ unsigned s_mark_all[kT / 32][kOutWin / 32];
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    double *s_acc = s_acc_all[wid];
    unsigned *s_mark = s_mark_all[wid];
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    auto tile = [&](const int64_t t) {
    const int64_t k0 = t * kCooItems;
    const int cnt = (int)(nnz - k0 < kCooItems ? nnz - k0 : kCooItems);
    const int64_t e0 = k0 + lane * 8;
    const int nv = max(0, min(8, cnt - lane * 8));           // valid elements of this lane
    int r[8], c[8];
    V v[8];
    if (cnt == (int)kCooItems) {
        load_int8(row + e0, r, pa);
        load_int8(col + e0, c, pa);
        VecLoad8<V>::load(val + e0, v, pa);
    } else {
#pragma unroll
        for (int s = 0; s < 8; ++s) {
            const bool in = s < nv;
            r[s] = in ? ld_hint(row + e0 + s, pa) : INT_MAX;
            c[s] = in ? ld_hint(col + e0 + s, pa) : 0;
            v[s] = in ? ld_hint(val + e0 + s, pa) : (V)0;
        }
    }
    // fp32: the x gathers before the y window loads (the products and the segmented sums
    // need them first): LAP4096 0.321 -> 0.305 ms; fp64 measured 3 % slower that way
    double p[8];
    if constexpr (sizeof(V) == 4) {
#pragma unroll
        for (int s = 0; s < 8; ++s) p[s] = s < nv ? (double)v[s] * (double)ldx<HOT>(x, xh, c[s], px) : 0.0;
    }
    // rows around the tile (uniform loads)
    const int rf = __shfl_sync(0xffffffffu, r[0], 0);                       // tile's first row
    const int before = k0 > 0 ? __ldg(row + k0 - 1) : -1;                  // row before the tile
    const int64_t nr = k0 + cnt < nnz ? (int64_t)__ldg(row + k0 + cnt) : n_rows;   // next tile's first row
    const int last_lane = (cnt - 1) >> 3;
    int rsel = r[0];             // the lane's last valid row = max (rows sorted; no local-memory index)
#pragma unroll
    for (int q = 1; q < 8; ++q)
        if (q < nv) rsel = max(rsel, r[q]);
    const int rl = __shfl_sync(0xffffffffu, rsel, last_lane);              // tile's last row
    const bool cont = before == rf;                                        // leading continuation
    const int64_t Wlo = (!ACCUM && t == 0) ? 0 : (int64_t)rf + (cont ? 1 : 0);
    const int64_t Whi = ACCUM ? (int64_t)rl + 1 : (nr == rl ? nr + 1 : nr);
    const int64_t L = Whi - Wlo;
    double yv[kOutQ];
#pragma unroll
    for (int q = 0; q < kOutQ; ++q) {
        const int i = lane + 32 * q;
        yv[q] = ((ACCUM || !B0) && i < L) ? (double)y[Wlo + i] : 0.0;
    }
    // window rows without a segment (empty rows) keep s = 0: y = alpha*0 + beta*y, as the
    // definition (c1) reads; only ACCUM (rows present only) needs the row marks
    if (ACCUM) {
        if (lane < kOutWin / 32) s_mark[lane] = 0u;
    } else {
#pragma unroll
        for (int q = 0; q < kOutQ; ++q) s_acc[lane + 32 * q] = 0.0;
    }
    if constexpr (sizeof(V) == 8) {
#pragma unroll
        for (int s = 0; s < 8; ++s) p[s] = s < nv ? (double)v[s] * (double)ldx<HOT>(x, xh, c[s], px) : 0.0;
    }
    // rows past the window (sparse stretches: R-MAT's empty rows): the warp first writes
    // beta*y to all of them, 128 rows per step, coalesced; the tile's segments there then
    // add alpha*s (one more rounding of beta*y than the window path, within the bound).
    // beta == 1 leaves every row without a segment as it is: nothing to write (a halo's
    // foreign block -- a few boundary rows in millions -- would otherwise walk them all)
    if (!ACCUM && L > kOutWin && beta != 1.0) {
        for (int64_t g0 = Wlo + kOutWin; g0 < Whi; g0 += kOutWin) {
            double t4[kOutQ];
#pragma unroll
            for (int q = 0; q < kOutQ; ++q) {
                const int64_t g = g0 + lane + 32 * q;
                t4[q] = (!B0 && g < Whi) ? (double)y[g] : 0.0;
            }
#pragma unroll
            for (int q = 0; q < kOutQ; ++q) {
                const int64_t g = g0 + lane + 32 * q;
                if (g < Whi) y[g] = B0 ? (V)0 : (V)(beta * t4[q]);
            }
        }
    }
    __syncwarp();

    auto emit = [&](int64_t rr, double sum) {
        const int64_t li = rr - Wlo;
        if (li >= 0 && li < kOutWin) {
            s_acc[li] = sum;
            if (ACCUM) atomicOr(&s_mark[li >> 5], 1u << (li & 31));
        } else {
            y[rr] = (V)((double)y[rr] + alpha * sum);
        }
    };
    int prev = __shfl_up_sync(0xffffffffu, r[7], 1);
    if (lane == 0) prev = before;
    double acc = 0.0, head = 0.0;
    int kseg = 0, cur = -1;
#pragma unroll
    for (int s = 0; s < 8; ++s) {
        if (s < nv) {
            const int pr = s == 0 ? prev : r[s - 1];
            if (r[s] != pr) {                                   // a segment (row) starts here
                if (kseg == 0) head = acc;
                else emit(cur, acc);                            // closed inside the lane
                ++kseg;
                cur = r[s];
                acc = 0.0;
            }
            acc += p[s];
        }
    }
    if (kseg == 0) head = acc;
    double Rnext;
    const double R = seg_suffix(head, kseg > 0 || nv == 0, &Rnext);
    if (kseg > 0) emit(cur, acc + Rnext);
    if (lane == 0) {
        carry_row[t] = cont ? rf : -1;
        carry_val[t] = cont ? R : 0.0;
    }
    __syncwarp();
#pragma unroll
    for (int q = 0; q < kOutQ; ++q) {
        const int i = lane + 32 * q;
        if (i < L) {
            if (ACCUM) {
                if ((s_mark[i >> 5] >> (i & 31)) & 1u) y[Wlo + i] = (V)(yv[q] + alpha * s_acc[i]);
            } else {
                double o = alpha * s_acc[i];
                if (!B0) o = fma(beta, yv[q], o);
                y[Wlo + i] = (V)o;
            }
        }
    }
    };
    const int64_t t0 = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    if constexpr (PERSIST) {
        for (int64_t t = t0; t < n_tiles; t += ((int64_t)gridDim.x * blockDim.x) >> 5) {
            tile(t);
            __syncwarp();
        }
    } else {
        if (t0 >= n_tiles) return;
        tile(t0);
    }
}

// Row walk over a chunk staged in shared memory (cols s_c, values s_v): positions
// [st, st + len) of one row, 8 slots per step with all x gathers of a step in flight.
// Called by all lanes with their own row, so at slot j the warp gathers x for
// consecutive rows (few L1 wavefronts on banded matrices, as ELL).
template <typename V, bool HOT = false>
__device__ __forceinline__ double row_walk(const int *s_c, const V *s_v, int st, int len, const V *__restrict__ x, const V *__restrict__ xh,
                                           uint64_t px) {
    double a0 = 0.0, a1 = 0.0;
    for (int k = 0; k < len; k += 8) {
        int cc[8];
        V vv[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const bool in = k + u < len;
            cc[u] = in ? s_c[st + k + u] : 0;
            vv[u] = in ? s_v[st + k + u] : (V)0;
        }
        double pp[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) pp[u] = k + u < len ? (double)vv[u] * (double)ldx<HOT>(x, xh, cc[u], px) : 0.0;
#pragma unroll
        for (int u = 0; u < 8; u += 2) { a0 += pp[u]; a1 += pp[u + 1]; }
    }
    return a0 + a1;
}
// the same walk reading col/val from global memory (rows of a batch that does not fit
// the shared-memory chunk)
template <typename V, bool HOT = false>
__device__ __forceinline__ double row_walk_global(const int *__restrict__ col, const V *__restrict__ val, int64_t a,
                                                  int len, const V *__restrict__ x, const V *__restrict__ xh, uint64_t pa, uint64_t px) {
    double a0 = 0.0, a1 = 0.0;
    for (int k = 0; k < len; k += 8) {
        int cc[8];
        V vv[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) {
            const bool in = k + u < len;
            cc[u] = in ? ld_hint(col + a + k + u, pa) : 0;
            vv[u] = in ? ld_hint(val + a + k + u, pa) : (V)0;
        }
        double pp[8];
#pragma unroll
        for (int u = 0; u < 8; ++u) pp[u] = k + u < len ? (double)vv[u] * (double)ldx<HOT>(x, xh, cc[u], px) : 0.0;
#pragma unroll
        for (int u = 0; u < 8; u += 2) { a0 += pp[u]; a1 += pp[u + 1]; }
    }
    return a0 + a1;
}
// positions [0, n) (n <= 256) of a 32-byte aligned global run into shared memory, in
// warp-contiguous 16-byte pieces (lane l: piece l + 32q); pieces starting at or past n
// are not read (a piece holding the last element stays inside that element's sector)
template <typename T>
__device__ __forceinline__ void stage_pieces(const T *__restrict__ g, T *s, int n, uint64_t pa) {
    constexpr int E = 16 / sizeof(T);                    // elements per piece
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int q = 0; q < 256 / (32 * E); ++q) {
        const int pos = (lane + 32 * q) * E;
        if (pos < n) {
            if constexpr (sizeof(T) == 8) {
                const double2 w = ld_hint(reinterpret_cast<const double2 *>(g + pos), pa);
                *reinterpret_cast<double2 *>(s + pos) = w;
            } else if constexpr (std::is_same<T, float>::value) {
                const float4 w = ld_hint(reinterpret_cast<const float4 *>(g + pos), pa);
                *reinterpret_cast<float4 *>(s + pos) = w;
            } else {
                const int4 w = ld_hint(reinterpret_cast<const int4 *>(g + pos), pa);
                *reinterpret_cast<int4 *>(s + pos) = w;
            }
        }
    }
}
// a lane's 8-element chunk into shared memory (16-byte stores)
template <typename V>
__device__ __forceinline__ void chunk_store(int *s_c, V *s_v, int pos, const int (&c)[8], const V (&v)[8]) {
    *reinterpret_cast<int4 *>(s_c + pos) = make_int4(c[0], c[1], c[2], c[3]);
    *reinterpret_cast<int4 *>(s_c + pos + 4) = make_int4(c[4], c[5], c[6], c[7]);
#pragma unroll
    for (int e = 0; e < 8; e += (int)(16 / sizeof(V))) {
        if constexpr (sizeof(V) == 8) *reinterpret_cast<double2 *>(s_v + pos + e) = make_double2(v[e], v[e + 1]);
        else *reinterpret_cast<float4 *>(s_v + pos + e) = make_float4(v[e], v[e + 1], v[e + 2], v[e + 3]);
    }
}

// ------------------------------------------------------------------ CSR row batches (A29)
// Short rows (vector width W <= 8, A5): a warp takes 32 consecutive rows, whose nonzeros
// [rp[b], rp[b+32]) are contiguous -- lane l loads the 32-byte aligned chunk of 8
// nonzeros starting at (rp[b] rounded down to 8) + 8l with 256-bit loads, the products
// go to shared memory in that order and lane i sums row b + i sequentially (<= 32
// terms, two accumulators).  The batch's row pointers arrive one batch ahead.  A batch
// whose rows do not fit (a row > 32 nonzeros, or > 256 - (rp[b] mod 8) nonzeros in
// all) is reduced row by row by the whole warp (the paper's warp-per-row vector
// kernel; blocked summation, A13).  CHUNKED: rows longer than long_len
// get beta*y here and their chunks arrive through the fix-up (A25).
template <typename V, typename IT, bool B0, int MB, bool CHUNKED, bool HOT = false>
__global__ void __launch_bounds__(kT, MB)
k_csr_rows(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val,
           const V *__restrict__ x, const V *__restrict__ xh, V *__restrict__ y, int64_t n, double alpha, double beta, int64_t long_len) {
    __shared__ __align__(16) double s_p_all[kT / 32][264 + 132];   // values, then cols
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    double *s_p = s_p_all[wid];
    const int64_t gwarp = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    const int64_t nwarps = ((int64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    int64_t b = gwarp * 32;
    IT nlo = 0, nhi = 0;                          // row pointers of the next batch (prefetched)
    if (b < n) {
        nlo = __ldg(rp + (b + lane < n ? b + lane : n));
        nhi = __ldg(rp + (b + 32 < n ? b + 32 : n));
    }
    for (; b < n; b += nwarps * 32) {
        const int64_t my_a = (int64_t)nlo;
        const int64_t hi = (int64_t)nhi;
        const int64_t nb = b + nwarps * 32;
        if (nb < n) {
            nlo = __ldg(rp + (nb + lane < n ? nb + lane : n));
            nhi = __ldg(rp + (nb + 32 < n ? nb + 32 : n));
        }
        const int64_t lo = __shfl_sync(0xffffffffu, my_a, 0);
        const int64_t nx = __shfl_down_sync(0xffffffffu, my_a, 1);
        const int64_t my_e = lane == 31 ? hi : nx;    // rows >= n: my_a = my_e = rp[n]
        const bool in_row = b + lane < n;
        const double yv = (!B0 && in_row) ? (double)y[b + lane] : 0.0;
        const int off = (int)(lo & 7);
        const int cnt = (int)(hi - lo < (1 << 20) ? hi - lo : (1 << 20));
        double sum = 0.0;
        if (__all_sync(0xffffffffu, my_e - my_a <= 32) && cnt + off <= 256) {
            const int j0 = lane * 8 - off;
            const int64_t base = lo - off + lane * 8;
            // chunk -> shared memory, then lane i walks row b + i: at slot j the 32 lanes
            // gather x for 32 consecutive rows (ELL-like locality: few L1 wavefronts; the
            // products-to-shared variant, lane chunks gathering, was 0.312 vs 0.297 ms)
            int *s_c = reinterpret_cast<int *>(s_p + 264);
            V *s_v = reinterpret_cast<V *>(s_p);
            // warp-contiguous 16-byte pieces: each load / store instruction covers 512
            // consecutive bytes (no shared-memory bank conflicts; lane chunks of 32 / 64 B
            // made the stores 2- / 4-way conflicted); pieces past the batch are skipped
            stage_pieces(col + (lo - off), s_c, cnt + off, pa);
            stage_pieces(val + (lo - off), s_v, cnt + off, pa);
            (void)j0; (void)base;
            __syncwarp();
            int len = (int)(my_e - my_a);
            if (CHUNKED && len > long_len) len = 0;            // A25: chunks via the fix-up
            sum = row_walk<V, HOT>(s_c, s_v, (int)(my_a - lo) + off, len, x, xh, px);
            __syncwarp();
        } else {
            // rows <= 32 nonzeros: lane i walks row b + i straight from global memory;
            // longer rows: the whole warp on each (8 loads per lane in flight)
            int64_t len = my_e - my_a;
            if (CHUNKED && len > long_len) len = 0;            // A25: chunks via the fix-up
            const bool lng = len > 32;
            if (!lng) sum = row_walk_global<V, HOT>(col, val, my_a, (int)len, x, xh, pa, px);
            unsigned lm = __ballot_sync(0xffffffffu, lng);
            while (lm) {
                const int i = __ffs(lm) - 1;
                lm &= lm - 1;
                const int64_t ra = __shfl_sync(0xffffffffu, my_a, i), rb = __shfl_sync(0xffffffffu, my_e, i);
                double tot = 0.0, acc[8];
#pragma unroll
                for (int q = 0; q < 8; ++q) acc[q] = 0.0;
                int it = 0;
                int64_t k = ra + lane;
                for (; k + 7 * 32 < rb; k += 8 * 32) {
                    int d[8];
                    V w[8];
#pragma unroll
                    for (int q = 0; q < 8; ++q) { d[q] = ld_hint(col + k + 32 * q, pa); w[q] = ld_hint(val + k + 32 * q, pa); }
#pragma unroll
                    for (int q = 0; q < 8; ++q) acc[q] += (double)w[q] * (double)ldx<HOT>(x, xh, d[q], px);
                    if (++it == kFold) {
#pragma unroll
                        for (int q = 0; q < 8; ++q) { tot += acc[q]; acc[q] = 0.0; }
                        it = 0;
                    }
                }
                for (; k < rb; k += 32) acc[0] += (double)ld_hint(val + k, pa) * (double)ldx<HOT>(x, xh, ld_hint(col + k, pa), px);
                const double part = warp_sum(tot + (((acc[0] + acc[1]) + (acc[2] + acc[3])) + ((acc[4] + acc[5]) + (acc[6] + acc[7]))));
                if (lane == i) sum = part;
            }
        }
        if (in_row) {
            double o = alpha * sum;
            if (!B0) o = fma(beta, yv, o);
            y[b + lane] = (V)o;
        }
    }
    // PDL after k_csr_chunks (chunked handles only): exit only once the chunk grid is
    // done.  Not compiled into the unchunked kernels: even with nothing to wait for it
    // cost LAP4096 7-15 %
    if constexpr (CHUNKED) pdl_wait();
}

// ------------------------------------------------------------------ merge-based CSR (K7/G11)
// "logically partitions the work of processing a group of contiguous
// rows into equal sized sub-problems".  Warp w owns merge-path diagonals
// [w*T, (w+1)*T) of (row ends) x (nonzeros), T = kMergeItems: rows [r0, r1) end in
// the tile and nonzeros [k0, k1) are consumed by it (coordinates precomputed at
// conversion, A7; only the row coordinate is read, the nonzero one is d - row).
// Lane l takes the 32-byte aligned chunk of 8 nonzeros [base + 8l, base + 8l + 8),
// base = k0 rounded down to 8 elements, with 256-bit loads (each sector requested
// once); positions outside the tile are masked, and the <= 7 positions past lane 31's
// chunk (tiles with < 8 row ends) are a short extra loop of lane 31.  Products stay in
// registers with all x gathers in flight.  The tile's row ends (coalesced, shared)
// mark segment starts as shared byte flags over chunk positions; each lane then reduces
// its chunk like a CSR5 lane (in-lane segments + flag-segmented suffix sum).
// Persistent warps prefetch the next tile's row coordinates.  Every row ending
// in the tile is written by it (empty rows: beta*y); row r0 may have begun in an
// earlier tile (its earlier parts arrive as carries); the part of row r1 inside the
// tile is the tile carry.  The row window is written back coalesced.
__device__ __forceinline__ int64_t ld_coord(const int64_t *p, uint64_t pol) {
    int64_t v;
    asm volatile("ld.global.nc.L2::cache_hint.s64 %0, [%1], %2;" : "=l"(v) : "l"(p), "l"(pol));
    return v;
}

// N consecutive elements starting at an arbitrary (element-aligned) address: the
// covering 16-byte vectors, then a shift by the address's offset inside a vector
template <typename V, int N> struct ShiftLoad;
template <int N> struct ShiftLoad<double, N> {          // N/2 + 1 double2, shift 0/1
    static __device__ __forceinline__ void load(const double *p, double (&v)[N], uint64_t pol) {
        const int m = (int)(((uintptr_t)p >> 3) & 1);
        const double2 *b = reinterpret_cast<const double2 *>(p - m);
        double w[N + 2];
#pragma unroll
        for (int q = 0; q < N / 2 + 1; ++q) { double2 t = ld_hint(b + q, pol); w[2 * q] = t.x; w[2 * q + 1] = t.y; }
#pragma unroll
        for (int s = 0; s < N; ++s) v[s] = m ? w[s + 1] : w[s];
    }
};
template <typename T, typename T4, int N>
__device__ __forceinline__ void shift_load4(const T *p, T (&v)[N], uint64_t pol) {   // N/4 + 1 x 16 B, shift 0..3
    const int m = (int)(((uintptr_t)p >> 2) & 3);
    const T4 *b = reinterpret_cast<const T4 *>(p - m);
    T w[N + 4];
#pragma unroll
    for (int q = 0; q < N / 4 + 1; ++q) { T4 t = ld_hint(b + q, pol); w[4*q] = t.x; w[4*q+1] = t.y; w[4*q+2] = t.z; w[4*q+3] = t.w; }
#pragma unroll
    for (int s = 0; s < N; ++s) v[s] = m == 0 ? w[s] : m == 1 ? w[s + 1] : m == 2 ? w[s + 2] : w[s + 3];
}
template <int N> struct ShiftLoad<float, N> {
    static __device__ __forceinline__ void load(const float *p, float (&v)[N], uint64_t pol) { shift_load4<float, float4, N>(p, v, pol); }
};
template <int N> struct ShiftLoad<int, N> {
    static __device__ __forceinline__ void load(const int *p, int (&v)[N], uint64_t pol) { shift_load4<int, int4, N>(p, v, pol); }
};

template <typename V, typename IT, bool B0, int LI, bool HOT = false>
__device__ __forceinline__ void
merge_tile(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val, int64_t t,
           int64_t r0, int64_t r1, int64_t k0, int64_t k1, const V *__restrict__ x, const V *__restrict__ xh, V *__restrict__ y,
           double alpha, double beta, int64_t *__restrict__ carry_row, double *__restrict__ carry_val,
           double *s_sum, int *s_end, uint2 *s_flag, uint64_t pa, uint64_t px) {
    constexpr int TI = 32 * LI;
    const int lane = threadIdx.x & 31;
    const int nrows = (int)(r1 - r0), nnzt = (int)(k1 - k0);
    // LI = 8: lane l owns the 32-byte aligned chunk [base + 8l, base + 8l + 8), base =
    // k0 - off: tile positions [8l - off, 8l - off + 8), those outside [0, nnzt) masked,
    // so no shifting; positions [256 - off, nnzt) (a tile with < 8 row ends) are one
    // more chunk, taken by lane 31.  LI = 4: shifted 16-byte loads (off = 0).
    const int off = LI == 8 ? (int)(k0 & 7) : 0;
    const int64_t base = k0 - off;
    const int j0 = lane * LI - off;                        // tile position of the lane's first element
    const bool any = j0 < nnzt;                            // the lane holds a tile element
    int c[LI];
    V v[LI];
    if constexpr (LI == 8) {
        if (any) {
            ld256(col + base + lane * LI, c, pa);
            VecLoad8<V>::load(val + base + lane * LI, v, pa);
        }
    } else if (any) {
        ShiftLoad<int, LI>::load(col + k0 + j0, c, pa);
        ShiftLoad<V, LI>::load(val + k0 + j0, v, pa);
    }
    double yv[kOutQ];
#pragma unroll
    for (int q = 0; q < kOutQ; ++q) {
        const int i = lane + 32 * q;
        yv[q] = (!B0 && i < nrows) ? (double)y[r0 + i] : 0.0;
    }
    for (int i = lane; i < nrows; i += 32) s_end[i] = (int)((int64_t)__ldg(rp + r0 + 1 + i) - k0);
    const bool r0_inside = (int64_t)__ldg(rp + r0) == k0;   // A7: rp[r0] <= k0 always
    // segment-start flags, one byte per chunk position (plain stores, no atomics)
    unsigned char *s_fb = reinterpret_cast<unsigned char *>(s_flag);
    for (int i = lane; i < TI / 8 + 1; i += 32) s_flag[i] = make_uint2(0u, 0u);
    double p[LI];
#pragma unroll
    for (int e = 0; e < LI; ++e)
        p[e] = (any && (unsigned)(j0 + e) < (unsigned)nnzt) ? (double)v[e] * (double)ldx<HOT>(x, xh, c[e], px) : 0.0;
    __syncwarp();
    // segment starts: local row i (1 <= i <= nrows) starts at s_end[i-1]; row 0 at 0 if
    // r0_inside.  The bitmap is indexed by chunk position (tile position + off).
    for (int i = lane; i <= nrows; i += 32) {
        const int st = i == 0 ? 0 : s_end[i - 1];
        const int en = i < nrows ? s_end[i] : nnzt;         // open row r1 runs past the tile
        if ((i > 0 || r0_inside) && st < nnzt && en > st) {
            s_fb[st + off] = 1;
        }
    }
    // where the open row r1 starts inside the tile (its segment is the tile carry), else -1
    const int open_start = nrows > 0 ? (s_end[nrows - 1] < nnzt ? s_end[nrows - 1] : -1) : (r0_inside && nnzt > 0 ? 0 : -1);
    __syncwarp();
    // bytes (0/1) of the lane's chunk -> bit mask: (b & 0x01010101) * 0x01020408 gathers the
    // four low bits into the top byte without carries
    auto pack4 = [](unsigned w) -> unsigned { return ((w & 0x01010101u) * 0x01020408u) >> 24; };
    unsigned fl = 0u;
    if (any) {
        if constexpr (LI == 8) {
            const uint2 w = s_flag[lane];
            fl = pack4(w.x) | (pack4(w.y) << 4);
        } else {
            fl = pack4(reinterpret_cast<const unsigned *>(s_flag)[lane]);
        }
    }
    double acc = 0.0, head = 0.0;
    int kseg = 0, cur = -1;
#pragma unroll
    for (int e = 0; e < LI; ++e) {
        if ((fl >> e) & 1u) {
            if (kseg == 0) head = acc;
            else s_sum[cur] = acc;                        // segment closed inside the lane
            ++kseg;
            cur = j0 + e;
            acc = 0.0;
        }
        acc += p[e];
    }
    if constexpr (LI == 8) {
        if (lane == 31 && j0 + LI < nnzt) {               // overflow chunk (rare: long rows)
            const uint2 w2 = s_flag[TI / 8];
            const unsigned fl2 = pack4(w2.x) | (pack4(w2.y) << 4);
#pragma unroll 1
            for (int pos = j0 + LI; pos < nnzt; ++pos) {
                const int e = pos - (j0 + LI);
                if ((fl2 >> e) & 1u) {
                    if (kseg == 0) head = acc;
                    else s_sum[cur] = acc;
                    ++kseg;
                    cur = pos;
                    acc = 0.0;
                }
                acc += (double)ld_hint(val + k0 + pos, pa) * (double)ldx<HOT>(x, xh, ld_hint(col + k0 + pos, pa), px);
            }
        }
    }
    if (kseg == 0) head = acc;
    const int nv = any ? 1 : 0;
    double Rnext;
    const double R = seg_suffix(head, kseg > 0 || nv == 0, &Rnext);
    const double lead = __shfl_sync(0xffffffffu, R, 0);  // nonzeros before the tile's first segment start
    double cv = 0.0;
    int cset = 0;
    if (kseg > 0) {
        const double tot = acc + Rnext;
        if (cur != open_start) s_sum[cur] = tot;
        else { cv = tot; cset = 1; }                      // row r1 started in this tile
    }
    if (lane == 0 && !r0_inside && nnzt > 0 && nrows == 0) { cv = lead; cset = 1; }   // middle of row r0 == r1
    const unsigned who = __ballot_sync(0xffffffffu, cset);
    if (lane == 0 && who == 0) { carry_row[t] = -1; carry_val[t] = 0.0; }
    if (cset) { carry_row[t] = r1; carry_val[t] = cv; }
    __syncwarp();
    // every row ending in the tile: its segment sum (row 0 begun earlier: the lead run)
    auto row_sum = [&](int i) -> double {
        const int st = i == 0 ? 0 : s_end[i - 1];
        if (i == 0 && !r0_inside) return lead;
        return s_end[i] > st ? s_sum[st] : 0.0;
    };
#pragma unroll
    for (int q = 0; q < kOutQ; ++q) {
        const int i = lane + 32 * q;
        if (i < nrows) {
            double o = alpha * row_sum(i);
            if (!B0) o = fma(beta, yv[q], o);
            y[r0 + i] = (V)o;
        }
    }
    for (int i = kOutWin + lane; i < nrows; i += 32) {        // rows beyond the prefetched window
        double o = alpha * row_sum(i);
        if (!B0) o = fma(beta, (double)y[r0 + i], o);
        y[r0 + i] = (V)o;
    }
}

// nonzero coordinate of merge-path diagonal min(t*TI, n+nnz) with row coordinate r (A7)
__device__ __forceinline__ int64_t merge_k(int64_t t, int TI, int64_t r, int64_t dmax) {
    const int64_t d = t * TI;
    return (d < dmax ? d : dmax) - r;
}

// one warp per tile
template <typename V, typename IT, bool B0, int LI, int MB = kMinBlocks, bool HOT = false>
__global__ void __launch_bounds__(kT, MB)
k_merge(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val,
        const int64_t *__restrict__ crow, int64_t n_tiles, int64_t dmax,
        const V *__restrict__ x, const V *__restrict__ xh, V *__restrict__ y, double alpha, double beta,
        int64_t *__restrict__ carry_row, double *__restrict__ carry_val) {
    constexpr int TI = 32 * LI;
    __shared__ double s_sum_all[kT / 32][TI];             // segment sum, keyed by its start position
    __shared__ int s_end_all[kT / 32][TI];                // local end of local row i
    __shared__ uint2 s_flag_all[kT / 32][TI / 8 + 1];     // segment-start byte flags over the lane chunks
    const int wid = threadIdx.x >> 5;
    const int64_t t = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5;
    if (t >= n_tiles) return;
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    const int64_t r0 = ld_coord(crow + t, px), r1 = ld_coord(crow + t + 1, px);
    merge_tile<V, IT, B0, LI, HOT>(rp, col, val, t, r0, r1, merge_k(t, TI, r0, dmax), merge_k(t + 1, TI, r1, dmax), x, xh, y,
                              alpha, beta, carry_row, carry_val, s_sum_all[wid], s_end_all[wid], s_flag_all[wid], pa,
                              px);
}

// row-pointer entry through a volatile load, so that it is issued where it is written
// (beside the tile's chunk loads) and not sunk behind the x gathers
__device__ __forceinline__ int64_t ld_rp(const int *p) {
    int v;
    asm volatile("ld.global.nc.s32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
__device__ __forceinline__ int64_t ld_rp(const int64_t *p) {
    int64_t v;
    asm volatile("ld.global.nc.s64 %0, [%1];" : "=l"(v) : "l"(p));
    return v;
}

// Persistent warps over positions [i0, i1) of the tile order (A28): warp w takes
// positions i0 + w, i0 + w + W, ...  Two-stage prefetch: while tile order[i] runs, the
// coordinates of order[i + W] and the id order[i + 2W] are in flight.
#define SPMV_MERGE_SCHEDULE(BODY)                                                                        \
    const int64_t W = ((int64_t)gridDim.x * blockDim.x) >> 5;                                          \
    int64_t i = i0 + ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);                         \
    if (i >= i1) return;                                                                               \
    int64_t t = __ldg(order + i);                                                                      \
    int64_t r0 = ld_coord(crow + t, px), r1 = ld_coord(crow + t + 1, px);                              \
    int64_t tb = i + W < i1 ? __ldg(order + i + W) : 0;                                                \
    while (true) {                                                                                     \
        int64_t q0 = 0, q1 = 0, tc = 0;                                                                \
        if (i + W < i1) { q0 = ld_coord(crow + tb, px); q1 = ld_coord(crow + tb + 1, px); }            \
        if (i + 2 * W < i1) tc = __ldg(order + i + 2 * W);                                             \
        BODY;                                                                                          \
        i += W;                                                                                        \
        if (i >= i1) break;                                                                            \
        t = tb; r0 = q0; r1 = q1; tb = tc;                                                             \
        __syncwarp();                                                                                  \
    }

// Segmented-sum tiles (any class).  LIST = false: tiles i0 + w, i0 + w + W, ... (the
// next tile's coordinates loaded while the current one runs); LIST = true: positions
// [i0, i1) of the tile order.
template <typename V, typename IT, bool B0, int LI, int MB, bool LIST, bool HOT = false>
__global__ void __launch_bounds__(kT, MB)
k_merge_persist(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val,
                const int64_t *__restrict__ crow, const int *__restrict__ order, int64_t i0, int64_t i1,
                int64_t dmax, const V *__restrict__ x, const V *__restrict__ xh, V *__restrict__ y, double alpha, double beta,
                int64_t *__restrict__ carry_row, double *__restrict__ carry_val) {
    constexpr int TI = 32 * LI;
    __shared__ double s_sum_all[kT / 32][TI];
    __shared__ int s_end_all[kT / 32][TI];
    __shared__ uint2 s_flag_all[kT / 32][TI / 8 + 1];
    const int wid = threadIdx.x >> 5;
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    auto body = [&](int64_t t, int64_t r0, int64_t r1) {
        merge_tile<V, IT, B0, LI, HOT>(rp, col, val, t, r0, r1, merge_k(t, TI, r0, dmax), merge_k(t + 1, TI, r1, dmax), x, xh, y,
                                  alpha, beta, carry_row, carry_val, s_sum_all[wid], s_end_all[wid], s_flag_all[wid],
                                  pa, px);
    };
    if constexpr (!LIST) {
        const int64_t W = ((int64_t)gridDim.x * blockDim.x) >> 5;
        int64_t t = i0 + ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
        if (t >= i1) return;
        int64_t r0 = ld_coord(crow + t, px), r1 = ld_coord(crow + t + 1, px);
        while (true) {
            const int64_t tn = t + W;
            int64_t q0 = 0, q1 = 0;
            if (tn < i1) { q0 = ld_coord(crow + tn, px); q1 = ld_coord(crow + tn + 1, px); }
            body(t, r0, r1);
            if (tn >= i1) break;
            t = tn; r0 = q0; r1 = q1;
            __syncwarp();
        }
    } else {
        SPMV_MERGE_SCHEDULE(body(t, r0, r1))
    }
}

// Class-1 (row-sum) tile, A28: fewer than 64 row ends and every in-tile row part <= 32
// nonzeros.  Lane l holds its 32-byte aligned chunk of 8 nonzeros (as merge_tile; loaded
// one tile ahead by the caller) and loads the ends of rows l and l + 32; the products go
// to shared memory in chunk order and lane i sums rows i and i + 32 sequentially (two
// accumulators) -- no segment flags, no cross-lane segmented scan.  Row i covers local
// positions [end(i-1), end(i)) (row 0 from 0: the earlier parts of a row begun in an
// earlier tile arrive as carries); row nrows is the open row r1, its part the tile carry.
template <typename V>
struct MergeChunk {
    int c[8];
    V v[8];
};
// PAIRS: lane l holds chunk positions 2l + 64q and 2l + 64q + 1 (q < 4), so each load,
// each product store and each x-gather instruction covers 64 consecutive positions
// (conflict-free 512-byte stores; gathers of ~13 consecutive rows).  Else lane l holds
// the 32-byte aligned run [8l, 8l + 8).
template <typename V, bool PAIRS>
__device__ __forceinline__ int chunk_pos(int lane, int e) {
    return PAIRS ? 2 * lane + 64 * (e >> 1) + (e & 1) : 8 * lane + e;
}
template <typename V, bool PAIRS>
__device__ __forceinline__ void merge_chunk_load(const int *__restrict__ col, const V *__restrict__ val, int64_t k0,
                                                 int64_t k1, MergeChunk<V> &ch, uint64_t pa) {
    const int lane = threadIdx.x & 31;
    const int off = (int)(k0 & 7);
    const int lim = (int)(k1 - k0) + off;                 // chunk positions < lim hold tile elements
    if constexpr (PAIRS) {
#pragma unroll
        for (int q = 0; q < 4; ++q) {
            const int pos = 2 * lane + 64 * q;
            if (pos < lim) {
                const int2 c2 = ld_hint(reinterpret_cast<const int2 *>(col + (k0 - off) + pos), pa);
                ch.c[2 * q] = c2.x;
                ch.c[2 * q + 1] = c2.y;
                if constexpr (sizeof(V) == 8) {
                    const double2 v2 = ld_hint(reinterpret_cast<const double2 *>(val + (k0 - off) + pos), pa);
                    ch.v[2 * q] = v2.x;
                    ch.v[2 * q + 1] = v2.y;
                } else {
                    const float2 v2 = ld_hint(reinterpret_cast<const float2 *>(val + (k0 - off) + pos), pa);
                    ch.v[2 * q] = v2.x;
                    ch.v[2 * q + 1] = v2.y;
                }
            }
        }
    } else if (lane * 8 < lim) {
        ld256(col + (k0 - off) + lane * 8, ch.c, pa);
        VecLoad8<V>::load(val + (k0 - off) + lane * 8, ch.v, pa);
    }
}

template <typename V, typename IT, bool B0, bool PAIRS, bool HOT = false>
__device__ __forceinline__ void
merge_rows_tile(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val, int64_t t,
                int64_t r0, int64_t r1, int64_t k0, int64_t k1, const MergeChunk<V> &ch, const V *__restrict__ x, const V *__restrict__ xh,
                V *__restrict__ y, double alpha, double beta, int64_t *__restrict__ carry_row,
                double *__restrict__ carry_val, double *s_p, uint64_t pa, uint64_t px) {
    constexpr int LI = 8;
    const int lane = threadIdx.x & 31;
    const int nrows = (int)(r1 - r0), nnzt = (int)(k1 - k0);
    const int off = (int)(k0 & 7);
    const int j0 = lane * LI - off;
    const bool any0 = j0 < nnzt;
    int e_[2];                          // local ends of rows lane, lane + 32 (>= nrows: nnzt)
#pragma unroll
    for (int q = 0; q < 2; ++q) {
        const int i = lane + 32 * q;
        e_[q] = i < nrows ? (int)(ld_rp(rp + r0 + 1 + i) - k0) : nnzt;
    }
    // wait for the row ends before issuing the x gathers (measured: LAP4096 0.320 -> 0.298 ms)
    const bool ends_in = __all_sync(0xffffffffu, e_[0] >= 0 && e_[1] >= 0);   // every lane (no short circuit)
    (void)any0;
    double yv[2];
#pragma unroll
    for (int q = 0; q < 2; ++q) {
        const int i = lane + 32 * q;
        yv[q] = (!B0 && i < nrows) ? (double)y[r0 + i] : 0.0;
    }
#pragma unroll
    for (int e = 0; e < LI; e += 2) {
        const int pe = chunk_pos<V, PAIRS>(lane, e);      // chunk position of element e (pe + 1 of e + 1)
        const double p0 = (ends_in && (unsigned)(pe - off) < (unsigned)nnzt) ? (double)ch.v[e] * (double)ldx<HOT>(x, xh, ch.c[e], px) : 0.0;
        const double p1 = (ends_in && (unsigned)(pe + 1 - off) < (unsigned)nnzt) ? (double)ch.v[e + 1] * (double)ldx<HOT>(x, xh, ch.c[e + 1], px) : 0.0;
        *reinterpret_cast<double2 *>(s_p + pe) = make_double2(p0, p1);
    }
    if (lane == 31) {                                     // positions past lane 31's chunk (< off row ends)
#pragma unroll 1
        for (int pos = j0 + LI; pos < nnzt; ++pos)
            s_p[pos + off] = (double)ld_hint(val + k0 + pos, pa) * (double)ldx<HOT>(x, xh, ld_hint(col + k0 + pos, pa), px);
    }
    int s0 = __shfl_up_sync(0xffffffffu, e_[0], 1);
    const int last0 = __shfl_sync(0xffffffffu, e_[0], 31);
    int s1 = __shfl_up_sync(0xffffffffu, e_[1], 1);
    if (lane == 0) { s0 = 0; s1 = last0; }
    __syncwarp();
#pragma unroll
    for (int q = 0; q < 2; ++q) {
        const int i = lane + 32 * q;
        if (i > nrows) break;
        const int st = q ? s1 : s0, en = e_[q];
        const double *ps = s_p + off + st;
        double a0 = 0.0, a1 = 0.0;
        int k = 0;
        for (; k + 1 < en - st; k += 2) { a0 += ps[k]; a1 += ps[k + 1]; }
        if (k < en - st) a0 += ps[k];
        const double sum = a0 + a1;
        if (i < nrows) {
            double o = alpha * sum;
            if (!B0) o = fma(beta, yv[q], o);
            y[r0 + i] = (V)o;
        } else {
            carry_row[t] = en > st ? r1 : -1;
            carry_val[t] = sum;
        }
    }
}

// Persistent warps over the class-1 tiles.  LIST = false: every tile is class 1, warp w
// takes tiles w, w + W, ... and the next tile's coordinates are loaded while the current
// one runs; LIST = true: positions [i0, i1) of the tile order (SPMV_MERGE_SCHEDULE).
// The identity schedule is measurably faster than the list (LAP4096: 0.298 vs 0.339 ms).
template <typename V, typename IT, bool B0, int MB, bool LIST, bool PAIRS = true, bool HOT = false>
__global__ void __launch_bounds__(kT, MB)
k_merge_rows(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val,
             const int64_t *__restrict__ crow, const int *__restrict__ order, int64_t i0, int64_t i1,
             int64_t dmax, const V *__restrict__ x, const V *__restrict__ xh, V *__restrict__ y, double alpha, double beta,
             int64_t *__restrict__ carry_row, double *__restrict__ carry_val) {
    __shared__ __align__(16) double s_p_all[kT / 32][256 + 8];
    const int wid = threadIdx.x >> 5;
    const uint64_t pa = policy_evict_first(), px = policy_evict_last();
    auto body = [&](int64_t t, int64_t r0, int64_t r1) {
        MergeChunk<V> ch;
        const int64_t k0 = merge_k(t, 256, r0, dmax), k1 = merge_k(t + 1, 256, r1, dmax);
        merge_chunk_load<V, PAIRS>(col, val, k0, k1, ch, pa);
        merge_rows_tile<V, IT, B0, PAIRS, HOT>(rp, col, val, t, r0, r1, k0, k1, ch, x, xh, y, alpha, beta, carry_row, carry_val,
                                   s_p_all[wid], pa, px);
    };
    if constexpr (!LIST) {
        const int64_t W = ((int64_t)gridDim.x * blockDim.x) >> 5;
        int64_t t = i0 + ((blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5);
        if (t >= i1) return;
        int64_t r0 = ld_coord(crow + t, px), r1 = ld_coord(crow + t + 1, px);
        while (true) {
            const int64_t tn = t + W;
            int64_t q0 = 0, q1 = 0;
            if (tn < i1) { q0 = ld_coord(crow + tn, px); q1 = ld_coord(crow + tn + 1, px); }
            body(t, r0, r1);
            if (tn >= i1) break;
            t = tn; r0 = q0; r1 = q1;
            __syncwarp();
        }
    } else {
        SPMV_MERGE_SCHEDULE(body(t, r0, r1))
    }
}
#undef SPMV_MERGE_SCHEDULE

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

template <int SIGMA, typename V, typename IT, bool B0, bool HOT = false>
__global__ void __launch_bounds__(kT)
k_csr5(const IT *__restrict__ rp, const int *__restrict__ col, const V *__restrict__ val,
       const int64_t *__restrict__ tile_ptr, const int64_t *__restrict__ row_lo,
       const unsigned *__restrict__ desc, const int64_t *__restrict__ map_off,
       const int64_t *__restrict__ seg_map, int64_t n_tiles, int64_t nnz,
       const V *__restrict__ x, const V *__restrict__ xh, V *__restrict__ y, double alpha, double beta,
       int64_t *__restrict__ carry_row, double *__restrict__ carry_val) {
    constexpr int64_t W = 32 * SIGMA;
    constexpr int kQ = kCsr5Win / 32;
    __shared__ double s_acc[kT / 32][kCsr5Win];
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
                for (int64_t k = e + lane; k < end; k += 32) s += (double)val[k] * (double)ldx<HOT>(x, xh, col[k], px);
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
    // empty window rows keep s = 0: y = alpha*0 + beta*y, as the definition (c1) reads
#pragma unroll
    for (int q = 0; q < kQ; ++q) s_acc[wid][lane + 32 * q] = 0.0;
    const unsigned flag = d & 0xFFFFu;
    const int y_off = (int)((d >> 16) & 0x1FFu);
    double p[SIGMA];
#pragma unroll
    for (int s = 0; s < SIGMA; ++s) p[s] = (double)v[s] * (double)ldx<HOT>(x, xh, c[s], px);
    __syncwarp();

    auto emit = [&](int idx, double sum) {
        const int64_t li = moff >= 0 ? __ldg(seg_map + moff + idx) - lo : idx;
        if (li < kCsr5Win) {
            s_acc[wid][li] = sum;
        } else {
            y_write<V, B0>(y, lo + li, sum, alpha, beta);
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
    double Rnext;
    const double R = seg_suffix(head, kseg > 0, &Rnext);
    if (kseg > 0) emit(y_off + kseg - 1, acc + Rnext);
    if (lane == 0) {
        const bool lead = !(flag & 1u);
        carry_row[t] = lead ? __ldg(tile_ptr + t) : -1;
        carry_val[t] = lead ? R : 0.0;
    }
    __syncwarp();
    // write the window: alpha*s + beta*y (s = 0 for empty rows)
#pragma unroll
    for (int q = 0; q < kQ; ++q) {
        const int i = lane + 32 * q;
        if (i < L) {
            double o = alpha * s_acc[wid][i];
            if (!B0) o = fma(beta, yv[q], o);
            y[lo + i] = (V)o;
        }
    }
    if (L > kCsr5Win && moff >= 0 && beta != 1.0) {
        // empty rows past the window (sparse stretches: R-MAT's empty rows) get beta*y,
        // 128 rows per step: their row pointers, then y, all loads of a step in flight
        // (beta == 1: they stay as they are, nothing to write)
        for (int64_t g0 = lo + kCsr5Win; g0 < hi; g0 += kCsr5Win) {
            bool e[kQ];
            double t4[kQ];
#pragma unroll
            for (int q = 0; q < kQ; ++q) {
                const int64_t g = g0 + lane + 32 * q;
                e[q] = g < hi && __ldg(rp + g + 1) == __ldg(rp + g);
            }
#pragma unroll
            for (int q = 0; q < kQ; ++q) t4[q] = (!B0 && e[q]) ? (double)y[g0 + lane + 32 * q] : 0.0;
#pragma unroll
            for (int q = 0; q < kQ; ++q)
                if (e[q]) y[g0 + lane + 32 * q] = B0 ? (V)0 : (V)(beta * t4[q]);
        }
    }
}

// ------------------------------------------------------------------ fix-up (G13)
// Carries are stored in tile order, so a row's carries are one contiguous run (a row
// spanning many tiles -- an R-MAT hub row -- gives a run of hundreds).  One warp per 32
// consecutive carries: a flag-segmented suffix sum gives each run's sum inside the
// chunk; the run's head lane adds alpha * sum to y.  A run that starts in the chunk and
// reaches its end is continued by the whole warp, 32 carries per step (coalesced loads,
// warp sums, added in chunk order), so no thread walks a long run serially.  Runs that
// began in an earlier chunk are left to the warp holding their head.
template <typename V>
__global__ void k_fixup(const int64_t *__restrict__ carry_row, const double *__restrict__ carry_val, int64_t n,
                        V *__restrict__ y, double alpha) {
    const int lane = threadIdx.x & 31;
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    for (int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; w * 32 < n; w += nw) {
        const int64_t c = w * 32 + lane;
        const int64_t key = c < n ? carry_row[c] : -1;
        const double val = c < n ? carry_val[c] : 0.0;
        const int64_t prev = w > 0 ? carry_row[w * 32 - 1] : -1;
        const int64_t kup = __shfl_up_sync(0xffffffffu, key, 1);
        const int64_t kdn = __shfl_down_sync(0xffffffffu, key, 1);
        const bool head = lane == 0 ? key != prev : key != kup;
        const bool last = lane == 31 || key != kdn;            // run ends at this lane (inside the chunk)
        double Rnext;
        const double R = seg_suffix(val, last, &Rnext);        // R[l] = val[l] + (last[l] ? 0 : R[l+1])
        // the chunk's final run may continue into the next chunks
        const int64_t k31 = __shfl_sync(0xffffffffu, key, 31);
        const bool open = k31 >= 0 && (w + 1) * 32 < n && carry_row[(w + 1) * 32] == k31;
        const unsigned hb = __ballot_sync(0xffffffffu, head && key == k31);
        const int h31 = 31 - __clz(hb);                        // head lane of the final run
        const bool own_final = open && hb != 0u && !(h31 == 0 && k31 == prev);
        double tail = 0.0;
        if (own_final) {                                        // warp-uniform
            for (int64_t q = (w + 1) * 32; q < n; q += 32) {
                const int64_t kq = q + lane < n ? carry_row[q + lane] : -1;
                const double vq = q + lane < n ? carry_val[q + lane] : 0.0;
                const unsigned m = __ballot_sync(0xffffffffu, kq == k31);
                const unsigned pre = ~m ? ((1u << __ffs(~m) - 1) - 1u) : 0xffffffffu;   // leading run of equal keys
                tail += warp_sum((pre >> lane) & 1u ? vq : 0.0);
                if (pre != 0xffffffffu) break;
            }
        }
        if (head && key >= 0 && !(lane == 0 && key == prev)) {
            const double sum = (lane == h31 && own_final) ? R + tail : R;
            y[key] = (V)((double)y[key] + alpha * sum);
        }
    }
}

// ------------------------------------------------------------------ launch helpers

// L1 / shared-memory split: the x gathers live in L1, so the tile kernels' shared memory
// costs x hits.  SPMV_CARVEOUT=<percent> sets the preferred shared-memory carveout of
// the tile kernels (experiments); unset = the driver's choice.
template <typename K>
void carveout(K *kernel) {
    static const int pct = [] { const char *e = getenv("SPMV_CARVEOUT"); return e ? atoi(e) : -1; }();
    if (pct >= 0) cudaFuncSetAttribute((const void *)kernel, cudaFuncAttributePreferredSharedMemoryCarveout, pct);
}

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
    k_fixup<V><<<grid_stride_blocks(h->ctx, ceil_div<int64_t>(h->n_carry, 32) * 32, 16), kT, 0, s>>>(
        (const int64_t *)h->carry_row.p, (const double *)h->carry_val.p, h->n_carry, y, alpha);
    SPMV_LAUNCH_CHECK();
    return SPMV_OK;
}

// ELL rows-per-thread x slot-batch variant; SPMV_ELL_VARIANT="RB" (e.g. 18, 24, 42) overrides the
// dtype default for tuning experiments (tools/exp.py)
template <typename V, bool B0, bool HOT>
spmv_status launch_ell(spmv_handle *h, const V *x, V *y, double alpha, double beta, cudaStream_t s) {
    const V *xh = reinterpret_cast<const V *>(h->xhot.p);
    const int64_t n = h->n_rows;
    if (n == 0) return SPMV_OK;
    static const int var = [] { const char *e = getenv("SPMV_ELL_VARIANT"); return e ? atoi(e) : 0; }();
    const int *c = (const int *)h->arr[SPMV_ARR_ELL_COL].p;
    const V *v = (const V *)h->arr[SPMV_ARR_ELL_VAL].p;
    switch (var) {
    case 14: k_ell<V, B0, 1, 4, HOT><<<grid_stride_blocks(h->ctx, n, 16), kT, 0, s>>>(c, v, h->ell_K, h->ell_ld, x, xh, y, n, alpha, beta); break;
    case 28: k_ell<V, B0, 2, 8, HOT><<<grid_stride_blocks(h->ctx, (n + 1) / 2, 16), kT, 0, s>>>(c, v, h->ell_K, h->ell_ld, x, xh, y, n, alpha, beta); break;
    case 42: k_ell<V, B0, 4, 2, HOT><<<grid_stride_blocks(h->ctx, (n + 3) / 4, 16), kT, 0, s>>>(c, v, h->ell_K, h->ell_ld, x, xh, y, n, alpha, beta); break;
    case 44: k_ell<V, B0, 4, 4, HOT><<<grid_stride_blocks(h->ctx, (n + 3) / 4, 16), kT, 0, s>>>(c, v, h->ell_K, h->ell_ld, x, xh, y, n, alpha, beta); break;
    case 18: k_ell<V, B0, 1, 8, HOT><<<grid_stride_blocks(h->ctx, n, 16), kT, 0, s>>>(c, v, h->ell_K, h->ell_ld, x, xh, y, n, alpha, beta); break;
    default:   // 16-byte value loads: fp64 2 rows x 4-slot batch, fp32 4 rows x 2-slot batch (measured best)
        if (sizeof(V) == 8)
            k_ell<V, B0, 2, 4, HOT><<<grid_stride_blocks(h->ctx, (n + 1) / 2, 16), kT, 0, s>>>(c, v, h->ell_K, h->ell_ld, x, xh, y, n, alpha, beta);
        else
            k_ell<V, B0, 4, 2, HOT><<<grid_stride_blocks(h->ctx, (n + 3) / 4, 16), kT, 0, s>>>(c, v, h->ell_K, h->ell_ld, x, xh, y, n, alpha, beta);
        break;
    }
    SPMV_LAUNCH_CHECK();
    return SPMV_OK;
}

// kT-thread launch of `k` on `s`; pdl = programmatic dependent launch on the kernel
// before it in the stream (cudaLaunchAttributeProgrammaticStreamSerialization)
template <typename... KArgs, typename... Args>
cudaError_t launch_k(void (*k)(KArgs...), unsigned grid, cudaStream_t s, bool pdl, Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = dim3(grid);
    cfg.blockDim = dim3(kT);
    cfg.dynamicSmemBytes = 0;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = pdl ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, k, static_cast<KArgs>(args)...);
}

// the CSR-vector dynamic batch counter for this run, or nullptr: W >= 16 with the
// handle's scheduler counter, and only for row counts worth it (a resident grid --
// 3 CTAs/SM -- with >= 4 groups per warp; small matrices keep the static stride, whose
// launch has no memset or atomics)
inline unsigned long long *csr_sched(const spmv_handle *h, int64_t n, int w) {
    static const bool dyn_on = [] { const char *e = getenv("SPMV_CSR_DYN"); return !e || atoi(e) != 0; }();
    const int64_t resident_warps = (int64_t)h->ctx->sm_count * 3 * (kT / 32);
    return (dyn_on && h->sched.p && w >= 16 && n >= resident_warps * 4 * 4 * 32) ? (unsigned long long *)h->sched.p
                                                                                 : nullptr;
}

template <typename V, typename IT, bool B0, bool HOT>
spmv_status launch_csr_vector(const spmv_handle *h, const IT *rp, const int *col, const V *val, const V *x, V *y,
                              int64_t n, int w, double alpha, double beta, cudaStream_t s,
                              int64_t long_len = INT64_MAX, bool pdl = false) {
    if (n == 0) return SPMV_OK;
    const V *xh = reinterpret_cast<const V *>(h->xhot.p);
    // W <= 8: 32-row batches (A29) when col/val are 32-byte aligned (the chunk loads)
    static const int rows_on = [] { const char *e = getenv("SPMV_CSR_ROWS"); return e ? atoi(e) : 1; }();
    const int wmax = rows_on >= 8 ? rows_on : 8;          // experiment knob: SPMV_CSR_ROWS=16/32 widens it
    if (w <= wmax && rows_on && ((((uintptr_t)col) | ((uintptr_t)val)) & 31) == 0) {
        const unsigned gr = (unsigned)std::min<int64_t>(ceil_div<int64_t>(n, kT), (int64_t)h->ctx->sm_count * kCsrRowsMB);
        if (long_len == INT64_MAX)
            SPMV_CUDA_TRY(launch_k(k_csr_rows<V, IT, B0, kCsrRowsMB, false, HOT>, gr, s, pdl, rp, col, val, x, xh, y, n, alpha, beta, long_len));
        else
            SPMV_CUDA_TRY(launch_k(k_csr_rows<V, IT, B0, kCsrRowsMB, true, HOT>, gr, s, pdl, rp, col, val, x, xh, y, n, alpha, beta, long_len));
        return SPMV_OK;
    }
    // 16 CTAs (4096 threads) per SM of grid-stride warps
    const int64_t threads = ceil_div<int64_t>(n, 32 / w) * 32;
    const int g = grid_stride_blocks(h->ctx, threads, 16);
    // W <= 8: 4 CTAs/SM (64 registers; LAP4096 0.442 -> 0.384 ms); wider groups keep
    // 3 CTAs/SM (80 registers; R-MAT 24 at W = 16: 4 CTAs/SM 11 % slower)
    unsigned long long *sch = csr_sched(h, n, w);
    if (sch && !pdl) SPMV_CUDA_TRY(cudaMemsetAsync(sch, 0, 8, s));   // pdl: zeroed before the chunk launch
    const int gd = sch ? (int)std::min<int64_t>(g, (int64_t)h->ctx->sm_count * 3) : g;
#define SPMV_VEC(WW)                                                                                           \
    if (sch && long_len == INT64_MAX)                                                                          \
        SPMV_CUDA_TRY(launch_k(k_csr_vector<V, IT, WW, B0, (WW <= 8 ? 4 : 3), false, true, HOT>, gd, s, pdl, rp, col, val, x, xh, y, n, alpha, beta, long_len, sch)); \
    else if (sch)                                                                                              \
        SPMV_CUDA_TRY(launch_k(k_csr_vector<V, IT, WW, B0, (WW <= 8 ? 4 : 3), true, true, HOT>, gd, s, pdl, rp, col, val, x, xh, y, n, alpha, beta, long_len, sch)); \
    else if (long_len == INT64_MAX)                                                                            \
        SPMV_CUDA_TRY(launch_k(k_csr_vector<V, IT, WW, B0, (WW <= 8 ? 4 : 3), false, false, HOT>, g, s, pdl, rp, col, val, x, xh, y, n, alpha, beta, long_len, nosch)); \
    else                                                                                                       \
        SPMV_CUDA_TRY(launch_k(k_csr_vector<V, IT, WW, B0, (WW <= 8 ? 4 : 3), true, false, HOT>, g, s, pdl, rp, col, val, x, xh, y, n, alpha, beta, long_len, nosch))
    unsigned long long *nosch = nullptr;
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

template <typename V, typename IT, bool B0, bool HOT>
spmv_status run_t(spmv_handle *h, double alpha, double beta, const V *x, V *y, cudaStream_t s) {
    if (alpha == 0.0) return launch_scale<V, B0>(h, y, beta, s);   // A14: A not read
    const int64_t n = h->n_rows;
    // hot columns (A30): this run's x values of the handle's hot set, packed densely
    const V *xh = reinterpret_cast<const V *>(h->xhot.p);
    if (h->n_hot > 0) {
        k_hot_gather<V><<<grid_stride_blocks(h->ctx, h->n_hot, 4), kT, 0, s>>>(
            x, (const int *)h->arr[SPMV_ARR_HOT_COLS].p, h->n_hot, reinterpret_cast<V *>(h->xhot.p));
        SPMV_LAUNCH_CHECK();
    }
    const IT *rp = (const IT *)h->arr[SPMV_ARR_ROW_PTR].p;
    const int *col = (const int *)h->arr[SPMV_ARR_COL].p;
    const V *val = (const V *)h->arr[SPMV_ARR_VAL].p;
    int64_t *crow = (int64_t *)h->carry_row.p;
    double *cval = (double *)h->carry_val.p;
    switch (h->fmt) {
    case SPMV_CSR:
    {
        if (h->csr_chunks == 0) return launch_csr_vector<V, IT, B0, HOT>(h, rp, col, val, x, y, n, (int)h->vec_w, alpha, beta, s);
        // long-row chunks first, the row kernel programmatically dependent on them (PDL):
        // the two are independent and run side by side; the chunk grid is one resident
        // wave of chunk_ctas (2) CTAs/SM so that the row kernel's CTAs start at once beside it
        static const bool pdl_on = [] { const char *e = getenv("SPMV_CSR_PDL"); return !e || atoi(e) != 0; }();
        static const int chunk_ctas = [] { const char *e = getenv("SPMV_CSR_CHUNK_CTAS"); return e ? std::max(1, atoi(e)) : 2; }();
        if (pdl_on) {
            if (unsigned long long *sch = csr_sched(h, n, (int)h->vec_w)) SPMV_CUDA_TRY(cudaMemsetAsync(sch, 0, 8, s));
        } else {
            SPMV_TRY((launch_csr_vector<V, IT, B0, HOT>(h, rp, col, val, x, y, n, (int)h->vec_w, alpha, beta, s,
                                                   2 * h->csr_chunk)));
        }
        const int64_t warps = h->csr_chunks;
        const unsigned gc = (unsigned)std::min<int64_t>(ceil_div<int64_t>(warps, kT / 32),
                                                        (int64_t)h->ctx->sm_count * (pdl_on ? chunk_ctas : 16));
        k_csr_chunks<V, IT, HOT><<<gc, kT, 0, s>>>(rp, col, val, (const int64_t *)h->arr[SPMV_ARR_CSR_CHUNK_ROW].p,
                                              (const int64_t *)h->arr[SPMV_ARR_CSR_CHUNK_LO].p, h->csr_chunks,
                                              h->csr_chunk, x, xh, crow, cval);
        SPMV_LAUNCH_CHECK();
        if (pdl_on)
            SPMV_TRY((launch_csr_vector<V, IT, B0, HOT>(h, rp, col, val, x, y, n, (int)h->vec_w, alpha, beta, s,
                                                   2 * h->csr_chunk, true)));
        return launch_fixup<V>(h, y, alpha, s);
    }
    case SPMV_CSR_SCALAR:
        if (n == 0) return SPMV_OK;
        k_csr_scalar<V, IT, B0, HOT><<<grid_stride_blocks(h->ctx, n, 16), kT, 0, s>>>(rp, col, val, x, xh, y, n, alpha, beta);
        SPMV_LAUNCH_CHECK();
        return SPMV_OK;
    case SPMV_ELL:
        if (n == 0) return SPMV_OK;
        return launch_ell<V, B0, HOT>(h, x, y, alpha, beta, s);
    case SPMV_HYB: {
        if (n == 0) return SPMV_OK;
        SPMV_TRY((launch_ell<V, B0, HOT>(h, x, y, alpha, beta, s)));
        if (h->hyb_coo_nnz == 0) return SPMV_OK;
        k_coo<V, true, B0, HOT><<<(unsigned)ceil_div<int64_t>(h->n_carry, kT / 32), kT, 0, s>>>(
            (const int *)h->arr[SPMV_ARR_COO_ROW].p, (const int *)h->arr[SPMV_ARR_HYB_COO_COL].p,
            (const V *)h->arr[SPMV_ARR_HYB_COO_VAL].p, h->hyb_coo_nnz, h->n_carry, x, xh, y, n, alpha, beta, crow, cval);
        SPMV_LAUNCH_CHECK();
        return launch_fixup<V>(h, y, alpha, s);
    }
    case SPMV_COO:
        if (h->nnz == 0) return launch_scale<V, B0>(h, y, beta, s);
        if (h->coo_persist) {
            carveout(k_coo<V, false, B0, HOT, true>);
            const unsigned gp = (unsigned)std::min<int64_t>(ceil_div<int64_t>(h->n_carry, kT / 32),
                                                            (int64_t)h->ctx->sm_count * kCooPersistCtas);
            k_coo<V, false, B0, HOT, true><<<gp, kT, 0, s>>>(
                (const int *)h->arr[SPMV_ARR_COO_ROW].p, col, val, h->nnz, h->n_carry, x, xh, y, n, alpha, beta, crow, cval);
        } else {
            carveout(k_coo<V, false, B0, HOT>);
            k_coo<V, false, B0, HOT><<<(unsigned)ceil_div<int64_t>(h->n_carry, kT / 32), kT, 0, s>>>(
                (const int *)h->arr[SPMV_ARR_COO_ROW].p, col, val, h->nnz, h->n_carry, x, xh, y, n, alpha, beta, crow, cval);
        }
        SPMV_LAUNCH_CHECK();
        return launch_fixup<V>(h, y, alpha, s);
    case SPMV_MERGE:
        if (h->merge_tiles == 0) return SPMV_OK;
    {
        const unsigned g = (unsigned)ceil_div<int64_t>(h->merge_tiles, kT / 32);
        const int64_t *cr = (const int64_t *)h->arr[SPMV_ARR_MERGE_COORD_ROW].p;
        const int64_t dmax = n + h->nnz;
        // T = 256: persistent, 3 CTAs/SM (80 registers), next tile's coordinates prefetched --
        // measured 2 % faster than one tile per warp at 4 CTAs/SM (LAP4096, R-MAT 24);
        // T = 128: one tile per warp at 6 CTAs/SM
        if (h->merge_T == 128) {
            k_merge<V, IT, B0, 4, 6, HOT><<<g, kT, 0, s>>>(rp, col, val, cr, h->merge_tiles, dmax, x, xh, y, alpha, beta, crow, cval);
        } else {
            // T = 256 (A28): all tiles class 1 -> the row-sum kernel over all tiles; most
            // (>= half) class 1 -> the row-sum kernel over the class-1 part of the tile order,
            // then the segmented-sum kernel over the rest; else the segmented-sum kernel over
            // all tiles (it handles any tile; the order's indirection costs more than the
            // row-sum tiles save when they are few)
            const int *ord = (const int *)h->arr[SPMV_ARR_MERGE_TILE_ORDER].p;
            const int64_t nl = h->merge_lean, nt = h->merge_tiles;
            const unsigned gr = (unsigned)std::min<int64_t>(ceil_div<int64_t>(nl, kT / 32), (int64_t)h->ctx->sm_count * kMergeRowsMB);
            static const bool pairs = [] { const char *e = getenv("SPMV_MERGE_PAIRS"); return !e || atoi(e) != 0; }();
            if (nl == nt && !pairs) {
                carveout(k_merge_rows<V, IT, B0, kMergeRowsMB, false, false, HOT>);
                k_merge_rows<V, IT, B0, kMergeRowsMB, false, false, HOT><<<gr, kT, 0, s>>>(rp, col, val, cr, ord, 0, nt, dmax, x, xh, y,
                                                                               alpha, beta, crow, cval);
            } else if (nl == nt) {
                carveout(k_merge_rows<V, IT, B0, kMergeRowsMB, false, true, HOT>);
                k_merge_rows<V, IT, B0, kMergeRowsMB, false, true, HOT><<<gr, kT, 0, s>>>(rp, col, val, cr, ord, 0, nt, dmax, x, xh, y,
                                                                               alpha, beta, crow, cval);
            } else if (2 * nl >= nt) {
                carveout(k_merge_rows<V, IT, B0, kMergeRowsMB, true, true, HOT>);
                k_merge_rows<V, IT, B0, kMergeRowsMB, true, true, HOT><<<gr, kT, 0, s>>>(rp, col, val, cr, ord, 0, nl, dmax, x, xh, y,
                                                                              alpha, beta, crow, cval);
                SPMV_LAUNCH_CHECK();
                const unsigned gp = (unsigned)std::min<int64_t>(ceil_div<int64_t>(nt - nl, kT / 32), (int64_t)h->ctx->sm_count * 3);
                carveout(k_merge_persist<V, IT, B0, 8, 3, true, HOT>);
                k_merge_persist<V, IT, B0, 8, 3, true, HOT><<<gp, kT, 0, s>>>(rp, col, val, cr, ord, nl, nt, dmax, x, xh, y, alpha,
                                                                         beta, crow, cval);
            } else {
                const unsigned gp = (unsigned)std::min<int64_t>(g, (int64_t)h->ctx->sm_count * 3);
                carveout(k_merge_persist<V, IT, B0, 8, 3, false, HOT>);
                k_merge_persist<V, IT, B0, 8, 3, false, HOT><<<gp, kT, 0, s>>>(rp, col, val, cr, ord, 0, nt, dmax, x, xh, y, alpha,
                                                                          beta, crow, cval);
            }
        }
    }
        SPMV_LAUNCH_CHECK();
        return launch_fixup<V>(h, y, alpha, s);
    case SPMV_CSR5: {
        const int64_t warps = h->n_tiles + 1;
        const unsigned g = (unsigned)ceil_div<int64_t>(warps * 32, kT);
#define SPMV_CSR5_LAUNCH(SG)                                                                                  \
    carveout(k_csr5<SG, V, IT, B0, HOT>);                                                                          \
    k_csr5<SG, V, IT, B0, HOT><<<g, kT, 0, s>>>(rp, col, val, (const int64_t *)h->arr[SPMV_ARR_CSR5_TILE_PTR].p,   \
                                           (const int64_t *)h->arr[SPMV_ARR_CSR5_ROW_LO].p,                    \
                                           (const unsigned *)h->arr[SPMV_ARR_CSR5_TILE_DESC].p,                \
                                           (const int64_t *)h->arr[SPMV_ARR_CSR5_MAP_OFF].p,                   \
                                           (const int64_t *)h->arr[SPMV_ARR_CSR5_SEG_MAP].p, h->n_tiles,       \
                                           h->nnz, x, xh, y, alpha, beta, crow, cval)
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
            SPMV_TRY((launch_csr_vector<V, IT, B0, HOT>(h, rp + r_tail, col, val, x, y + r_tail, n - r_tail, 32, alpha,
                                                   beta, s)));
        return launch_fixup<V>(h, y, alpha, s);
    }
    }
    set_error("unknown format");
    return SPMV_ERR_INVALID_ARG;
}

// beta == 0 (y write-only, A14) and hot columns (A30) are compile-time kernel variants
template <typename V, typename IT>
spmv_status run_b(spmv_handle *h, double alpha, double beta, const V *x, V *y, cudaStream_t s) {
    if (h->n_hot > 0)
        return beta == 0.0 ? run_t<V, IT, true, true>(h, alpha, beta, x, y, s) : run_t<V, IT, false, true>(h, alpha, beta, x, y, s);
    return beta == 0.0 ? run_t<V, IT, true, false>(h, alpha, beta, x, y, s) : run_t<V, IT, false, false>(h, alpha, beta, x, y, s);
}

template <typename V>
spmv_status run_v(spmv_handle *h, double alpha, double beta, const void *x, void *y, cudaStream_t s) {
    const V *xv = (const V *)x;
    V *yv = (V *)y;
    if (h->itype == SPMV_I32)
        return run_b<V, int>(h, alpha, beta, xv, yv, s);
    return run_b<V, int64_t>(h, alpha, beta, xv, yv, s);
}

}  // namespace

spmv_status run_impl(spmv_handle *h, double alpha, double beta, const void *x, void *y, cudaStream_t s) {
    return h->dtype == SPMV_F64 ? run_v<double>(h, alpha, beta, x, y, s) : run_v<float>(h, alpha, beta, x, y, s);
}

int run_launch_count(const spmv_handle *h, bool alpha0) {
    if (alpha0) return h->n_rows ? 1 : 0;
    switch (h->fmt) {
    case SPMV_CSR: return h->n_rows ? 1 + (h->csr_chunks ? 2 : 0) : 0;
    case SPMV_CSR_SCALAR: case SPMV_ELL: return h->n_rows ? 1 : 0;
    case SPMV_HYB: return (h->n_rows ? 1 : 0) + (h->hyb_coo_nnz ? 2 : 0);
    case SPMV_COO: return h->nnz ? 2 : (h->n_rows ? 1 : 0);
    case SPMV_MERGE:
        if (!h->merge_tiles) return 0;
        if (h->merge_T == 128) return 2;
        return (h->merge_lean == h->merge_tiles || 2 * h->merge_lean < h->merge_tiles ? 1 : 2) + 1;
    case SPMV_CSR5: return 1 + (h->csr5_tail_row < h->n_rows ? 1 : 0) + 1;
    }
    return 0;
}

}  // namespace spmv
