// features.cu -- the per-matrix sparsity features of Table II (PAPER.md:161-185,
// §IV-A), read per SURVEY A8/A9, plus the canonical-CSR check
// (A15) that spmv_convert relies on.
//
// "Sets 2 and 3 require a scan on the entire matrix, O(nnz)": ONE
// kernel launch reads row_ptr and col_idx once each (vals are never read), with
// exact 64-bit integer sums; the fp64 finals are computed on the host from those
// sums with the fixed formulas of A9, so the result is bit-exact and run-to-run
// identical.  One 112-byte device->host copy returns the result.
//
// Work split (rows + nonzeros balanced, as the merge-path split of A7): the merge
// of the row STARTS row_ptr[0..n) with the nonzero indices is cut into equal
// diagonal ranges, one per warp.  A warp finds its two end coordinates with a
// 32-ary warp-cooperative search (g(i) = row_ptr[i-1] + i, largest i with
// g(i) <= d) and then walks its range in sub-spans of kSub diagonal items:
//   phase R  the rows whose start falls in the sub-span (row_ptr read once,
//            coalesced): row-length sums/min/max, empty rows, HYB overflow, the
//            A2 row-length histogram, row_ptr validity, and a row-start bitmap of
//            the sub-span's nonzero positions in shared memory;
//   phase E  the sub-span's nonzeros, 16 per lane per 512-position chunk (four
//            16-byte loads): column range/order checks and the block starts
//            ("continuous nnz chunk": a block starts at a row
//            start or wherever col[k] != col[k-1] + 1).  Block sizes are the gaps
//            between consecutive block starts; a row's block count is the number
//            of block starts between its start and the next row start.  Both are
//            closed in-lane in position order, with warp scans carrying the last
//            block start / row start across lanes and chunks.
// A block or row still open at the end of a warp's range is recorded (WarpRec);
// the last CTA to finish closes them in one forward pass over the records
// (at most one open block and one open row per warp), writes the result and
// resets the accumulators for the next call.  No global bitmaps, no second pass.
#include <climits>
#include <cmath>
#include <mutex>
#include <vector>

#include "internal.h"

namespace spmv {

namespace {

constexpr int kThreads = 256;
constexpr int kWarps = kThreads / 32;
constexpr int kCtasPerSm = 2;
constexpr int kSub = 8192;                      // diagonal items per sub-span
constexpr int kChunk = 512;                     // nonzero positions per warp chunk (16 per lane)
constexpr int kBmWords = (kSub + kChunk) / 32;  // row-start bitmap words per warp (+ alignment slack)
constexpr int kSharedHist = 1024;               // row-length histogram bins kept in shared memory
constexpr int kRowW = 4;                        // diagonal weight of a row start (a row costs ~4 nonzeros)

enum : unsigned { BAD_ROWPTR_ENDS = 1, BAD_ROWPTR_ORDER = 2, BAD_COL_RANGE = 4, BAD_COL_ORDER = 8 };

__device__ __forceinline__ unsigned long long warp_sum_u64(unsigned long long v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}
__device__ __forceinline__ unsigned warp_min_u32(unsigned v) { return __reduce_min_sync(0xffffffffu, v); }
__device__ __forceinline__ unsigned warp_max_u32(unsigned v) { return __reduce_max_sync(0xffffffffu, v); }

// exclusive prefix sum / max over lanes
__device__ __forceinline__ unsigned excl_sum(unsigned v, int lane) {
    unsigned s = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        unsigned t = __shfl_up_sync(0xffffffffu, s, o);
        if (lane >= o) s += t;
    }
    return s - v;
}
__device__ __forceinline__ int incl_max(int v, int lane) {
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        int t = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o && t > v) v = t;
    }
    return v;
}

// Warp-cooperative 32-ary merge-path search for two diagonals at once (A7 with the
// row starts as the first list, each row start weighing kRowW items): largest i in
// [max(0, (d-nnz)/kRowW), min(n, d/kRowW)] with g(i) <= d, g(0) = 0,
// g(i) = row_ptr[i-1] + kRowW*i.  Every lane returns both results.  On a non-monotone
// row_ptr the result is still some i in range (the caller only needs termination
// there; the row walk flags the matrix).
template <typename IT>
__device__ __forceinline__ void mp_search2(const IT *__restrict__ rp, int64_t n, int64_t nnz, const int64_t (&d)[2],
                                           int lane, int64_t (&out)[2]) {
    int64_t lo[2], hi[2];
#pragma unroll
    for (int t = 0; t < 2; ++t) {
        lo[t] = d[t] - nnz > 0 ? (d[t] - nnz) / kRowW : 0;
        hi[t] = d[t] / kRowW < n ? d[t] / kRowW : n;
        if (hi[t] < lo[t]) hi[t] = lo[t];
    }
    while (hi[0] > lo[0] || hi[1] > lo[1]) {
        int64_t q[2];
        bool ok[2];
#pragma unroll
        for (int t = 0; t < 2; ++t) {
            const int64_t len = hi[t] - lo[t];
            q[t] = lo[t] + 1 + ((int64_t)lane * len) / 32;
            ok[t] = true;
            if (len > 0) ok[t] = (int64_t)__ldg(rp + q[t] - 1) + kRowW * q[t] <= d[t];
        }
#pragma unroll
        for (int t = 0; t < 2; ++t) {
            const unsigned m = __ballot_sync(0xffffffffu, ok[t]);
            const int j = m == 0xffffffffu ? 32 : __ffs(~m) - 1;     // leading lanes with g(q) <= d
            const int64_t qa = __shfl_sync(0xffffffffu, q[t], j > 0 ? j - 1 : 0);
            const int64_t qb = __shfl_sync(0xffffffffu, q[t], j < 32 ? j : 31);
            if (hi[t] > lo[t]) {
                if (j == 0) hi[t] = lo[t];
                else if (j == 32) lo[t] = qa;
                else { lo[t] = qa; hi[t] = qb - 1; }
            }
        }
    }
    out[0] = lo[0];
    out[1] = lo[1];
}

}  // namespace

// Per-warp record for the cross-warp fix-up (one block and one row may stay open).
struct WarpRec {
    long long first_flag;        // first block start in the warp's range (-1: none)
    long long last_flag;         // last block start (-1: none)
    unsigned long long nflags;   // block starts in the range
    unsigned long long head_nb;  // block starts before the first row start of the range
    long long has_rs;            // a row starts inside the range
    unsigned long long open_tail;// block starts from the start of the row still open at the end
    long long has_open;          // a row starting in the range ends past it
};

// Device state of the feature pass, owned by the ctx: atomically accumulated sums
// (reset by the last CTA of every launch), the done counter and the result.
struct FeatureState {
    FeatureSums acc;
    unsigned long long done;
    FeatureSums result;
    long long cusp;
};

namespace {

// records and histogram are written by other CTAs: read them at L2 (no stale L1 lines)
__device__ __forceinline__ WarpRec load_rec(const WarpRec *p) {
    WarpRec r;
    r.first_flag = __ldcg(&p->first_flag);
    r.last_flag = __ldcg(&p->last_flag);
    r.nflags = __ldcg(&p->nflags);
    r.head_nb = __ldcg(&p->head_nb);
    r.has_rs = __ldcg(&p->has_rs);
    r.open_tail = __ldcg(&p->open_tail);
    r.has_open = __ldcg(&p->has_open);
    return r;
}

__device__ __forceinline__ void init_sums(FeatureSums &s) {
    s.bad = 0; s.n_empty = 0; s.sum_len2 = 0; s.len_min = ULLONG_MAX; s.len_max = 0; s.hyb_coo_ceil = 0;
    s.nb_tot = 0; s.sum_nb2 = 0; s.nb_min = ULLONG_MAX; s.nb_max = 0; s.sum_bs2 = 0;
    s.bs_min = ULLONG_MAX; s.bs_max = 0;
}

template <typename IT>
__global__ void __launch_bounds__(kThreads, kCtasPerSm)
k_features(const IT *__restrict__ rp, const int *__restrict__ col, int64_t n, int64_t nnz, int64_t n_cols,
           int64_t kh, int64_t per_warp, WarpRec *__restrict__ recs, unsigned long long *__restrict__ hist,
           int64_t hist_bins, FeatureState *st) {
    using P = IT;                       // nonzero positions: 32-bit arithmetic for int32 row_ptr
    constexpr P kNone = sizeof(P) == 4 ? (P)INT_MIN : (P)LLONG_MIN;
    // per warp: the sub-span's row-start bits, its block-start bits (flags) and the
    // exclusive prefix of flag popcounts per word
    __shared__ unsigned s_bm[kWarps][kBmWords];
    __shared__ unsigned s_fl[kWarps][kBmWords];
    __shared__ unsigned s_pf[kWarps][kBmWords];
    __shared__ unsigned s_hist[kSharedHist];
    __shared__ bool s_last;
    const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    const bool use_hist = hist != nullptr;
    const int sh_bins = hist_bins < kSharedHist ? (int)hist_bins : kSharedHist;
    if (use_hist)
        for (int i = threadIdx.x; i < sh_bins; i += kThreads) s_hist[i] = 0;
    unsigned *bm = s_bm[wid];
    unsigned *fl = s_fl[wid];
    unsigned *pf = s_pf[wid];
    const uint64_t pol = policy_evict_first();
    constexpr int kCap = kBmWords * 32;
    const bool col_aligned = (reinterpret_cast<uintptr_t>(col) & 15) == 0;

    const int64_t items = (int64_t)kRowW * n + nnz;
    const int64_t W = (int64_t)gridDim.x * kWarps;
    const int64_t w = (int64_t)blockIdx.x * kWarps + wid;
    int64_t dd[2], ii[2];
    dd[0] = w * per_warp < items ? w * per_warp : items;
    dd[1] = dd[0] + per_warp < items ? dd[0] + per_warp : items;
    mp_search2(rp, n, nnz, dd, lane, ii);
    const int64_t d0 = dd[0], d1 = dd[1];
    const int64_t i0 = w == 0 ? 0 : ii[0];
    const int64_t i1 = w == W - 1 ? n : ii[1];
    auto clampk = [&](int64_t k) { return (P)(k < 0 ? 0 : (k > nnz ? nnz : k)); };
    // coordinate (i, k): i row starts and k = min(d - kRowW*i, row_ptr[i]) nonzeros consumed
    const int64_t rpi0 = (int64_t)__ldg(rp + i0), rpi1 = (int64_t)__ldg(rp + i1);
    const P k0 = w == 0 ? (P)0 : clampk(d0 - kRowW * i0 < rpi0 ? d0 - kRowW * i0 : rpi0);
    P k1 = w == W - 1 ? (P)nnz : clampk(d1 - kRowW * i1 < rpi1 ? d1 - kRowW * i1 : rpi1);
    if (k1 < k0) k1 = k0;

    unsigned bad = 0;
    if (w == 0 && lane == 0)
        if ((int64_t)rp[0] != 0 || (int64_t)rp[n] != nnz) bad |= BAD_ROWPTR_ENDS;

    // per-lane accumulators
    unsigned long long len2 = 0, over = 0, nb2 = 0, sz2 = 0;
    unsigned len_mn = UINT_MAX, len_mx = 0, n_empty = 0, nb_mn = UINT_MAX, nb_mx = 0, sz_mn = UINT_MAX, sz_mx = 0;
    // P-typed (32-bit for int32 row_ptr) copies of the bounds the row pass compares with
    const P nnzP = (P)nnz, khP = (P)(kh < nnz ? kh : nnz);
    const P hbinP = (P)(hist_bins - 1 < nnz ? (hist_bins - 1 > 0 ? hist_bins - 1 : 0) : nnz);
    // warp-uniform state
    P c_lastflag = kNone;           // position of the last block start so far (kNone: none)
    unsigned c_F = 0;               // block starts so far in the warp's range
    long long head_nb = -1;         // flags before the first row start of the range (-1: none yet)
    long long c_Frs = -1;           // flags before the last row start so far (-1: none yet)
    P my_first_flag = kNone;        // set by the single lane that meets the range's first block start

    // the range's first nonzero starts a row owned (row-walk-wise) by the previous warp:
    // its row-start bit is set here, so its block count is this warp's
    bool pending_rs = i0 > 0 && k0 < k1 && (int64_t)__ldg(rp + i0 - 1) == (int64_t)k0;

    // row_ptr window of R1 (rows wrb .. wrb+127, four per lane, + row wrb+128), kept across sub-spans
    const bool rp_vec = (reinterpret_cast<uintptr_t>(rp) & 15) == 0;
    auto load_win = [&](int64_t rb, IT (&a)[4], IT &a4) {
        const int64_t q = rb + 4 * lane;
        if (rp_vec && q + 3 <= n) {
            if constexpr (sizeof(IT) == 4) {
                const int4 t = __ldg(reinterpret_cast<const int4 *>(rp + q));
                a[0] = t.x; a[1] = t.y; a[2] = t.z; a[3] = t.w;
            } else {
                const longlong2 t0 = __ldg(reinterpret_cast<const longlong2 *>(rp + q));
                const longlong2 t1 = __ldg(reinterpret_cast<const longlong2 *>(rp + q) + 1);
                a[0] = t0.x; a[1] = t0.y; a[2] = t1.x; a[3] = t1.y;
            }
        } else {
#pragma unroll
            for (int u = 0; u < 4; ++u) a[u] = __ldg(rp + (q + u < n ? q + u : n));
        }
        a4 = __ldg(rp + (rb + 128 < n ? rb + 128 : n));
    };
    IT wa[4] = {0, 0, 0, 0}, wa4 = 0;
    int64_t wrb = 0;
    bool have_win = false;
    int64_t r = i0, dcur = d0;
    P kcur = k0;
    while (true) {
        const int64_t dsub = dcur + kSub < d1 ? dcur + kSub : d1;
        const bool last = dsub == d1;
        const P base = kcur & ~(P)15;
        const int kc_rel = (int)(kcur - base);
        int prevc = 0;                  // col[kcur-1]: latency hidden by phase R1
        if (kcur > 0 && kcur < k1) prevc = __ldg(col + kcur - 1);
        for (int i = lane; i < kBmWords; i += 32) { bm[i] = 0u; fl[i] = 0u; }
        __syncwarp();
        if (pending_rs && lane == 0) atomicOr(&bm[kc_rel >> 5], 1u << (kc_rel & 31));

        // ---- R1: rows r with g(r+1) = row_ptr[r] + kRowW*(r+1) <= dsub (every row < i1 when
        //      last), taken strictly in order: lengths (sums, min/max, empty, HYB overflow,
        //      histogram), row_ptr validity, and row-start bits of their start positions.
        //      Relative form: row_ptr[r] - base <= lim - kRowW*(r - r_start).
        //      Windows of 128 rows from wrb = r & ~3, four consecutive rows per lane (one
        //      16-byte load): the next window is loaded while this one is processed, and the
        //      window a stop leaves open carries over to the next sub-span (shuffles).
        const int64_t r_start = r;
        const int64_t lim64 = dsub - kRowW * (r_start + 1) - (int64_t)base;
        const int lim = last ? INT_MAX : (int)(lim64 < INT_MIN ? INT_MIN : (lim64 > INT_MAX ? INT_MAX : lim64));
        const int64_t jmax64 = i1 - r_start;
        const int jmax = (int)(jmax64 < INT_MAX - 1024 ? jmax64 : INT_MAX - 1024);
        if (r < i1) {
            if (!have_win) {
                wrb = r & ~(int64_t)3;
                load_win(wrb, wa, wa4);
                have_win = true;
            }
            while (true) {
                IT na[4], na4;
                load_win(wrb + 128, na, na4);
                const int off = (int)(r - wrb);
                const int jb = (int)(wrb - r_start) + 4 * lane;
                P av[4], bv[4];
#pragma unroll
                for (int u = 0; u < 4; ++u) av[u] = (P)wa[u];
                const P nx = __shfl_down_sync(0xffffffffu, av[0], 1);
                bv[0] = av[1]; bv[1] = av[2]; bv[2] = av[3];
                bv[3] = lane == 31 ? (P)wa4 : nx;
                int fb = 4;                                  // the lane's first unwanted row
#pragma unroll
                for (int u = 3; u >= 0; --u) {
                    const int j = jb + u;
                    const bool want = 4 * lane + u < off ||
                                      (j < jmax && (last || av[u] - base <= (P)(lim - kRowW * j)));
                    if (!want) fb = u;
                }
                const unsigned fm = __ballot_sync(0xffffffffu, fb < 4);
                const int fl0 = fm ? __ffs(fm) - 1 : 0;
                const int fbf = __shfl_sync(0xffffffffu, fb, fl0);
                const int cutoff = fm ? 4 * fl0 + fbf : 128;
                unsigned cw = UINT_MAX, cm = 0;              // row-start bits of the lane's rows
                int hcnt = 0;
                unsigned hbin0 = 0, binv[4];
                bool huni = true;
#pragma unroll
                for (int u = 0; u < 4; ++u) {
                    const int idx = 4 * lane + u;
                    binv[u] = UINT_MAX;
                    if (idx >= off && idx < cutoff) {
                        const P arel = av[u] - base;
                        if (arel >= (P)kc_rel && arel < (P)kCap) {
                            const unsigned wd = (unsigned)arel >> 5, bit = 1u << ((unsigned)arel & 31);
                            if (wd != cw) {
                                if (cm) atomicOr(&bm[cw], cm);
                                cw = wd;
                                cm = 0;
                            }
                            cm |= bit;
                        }
                        P len = bv[u] - av[u];
                        if (len < 0 || av[u] < 0 || bv[u] > nnzP) { bad |= BAD_ROWPTR_ORDER; len = 0; }
                        const unsigned ul = (unsigned)len;
                        len2 += (unsigned long long)ul * ul;
                        len_mn = min(len_mn, ul);
                        len_mx = max(len_mx, ul);
                        n_empty += len == 0;
                        over += (unsigned)(len > khP ? len - khP : (P)0);
                        if (use_hist && len > 0) {                // empty rows: n_empty (bin 0)
                            const unsigned bin = (unsigned)(len < hbinP ? len : hbinP);
                            binv[u] = bin;
                            if (hcnt == 0) hbin0 = bin;
                            else huni = huni && bin == hbin0;
                            ++hcnt;
                        }
                    }
                }
                if (cm) atomicOr(&bm[cw], cm);
                if (use_hist) {
                    const unsigned hm = __ballot_sync(0xffffffffu, hcnt > 0);
                    if (hm) {
                        const int lead = __ffs(hm) - 1;
                        const unsigned b0 = __shfl_sync(0xffffffffu, hbin0, lead);
                        if (__all_sync(0xffffffffu, hcnt == 0 || (huni && hbin0 == b0))) {  // one bin
                            const unsigned tot = __reduce_add_sync(0xffffffffu, (unsigned)hcnt);
                            if (lane == lead) {
                                if ((int)b0 < sh_bins) atomicAdd(&s_hist[b0], tot);
                                else atomicAdd(&hist[b0], (unsigned long long)tot);
                            }
                        } else {
#pragma unroll
                            for (int u = 0; u < 4; ++u) {
                                if (binv[u] == UINT_MAX) continue;
                                if ((int)binv[u] < sh_bins) atomicAdd(&s_hist[binv[u]], 1u);
                                else atomicAdd(&hist[binv[u]], 1ull);
                            }
                        }
                    }
                }
                r = wrb + cutoff;
                if (cutoff < 128) {
                    // carry: the window from r & ~3 = rows of this window and the next
                    const int sh = cutoff >> 2;
                    const int src = (lane + sh) & 31;
                    const bool hi = lane + sh >= 32;
#pragma unroll
                    for (int u = 0; u < 4; ++u) {
                        const IT x0 = __shfl_sync(0xffffffffu, wa[u], src);
                        const IT x1 = __shfl_sync(0xffffffffu, na[u], src);
                        wa[u] = hi ? x1 : x0;
                    }
                    wa4 = __shfl_sync(0xffffffffu, na[0], sh);
                    wrb += 4 * sh;
                    break;
                }
                wrb += 128;
#pragma unroll
                for (int u = 0; u < 4; ++u) wa[u] = na[u];
                wa4 = na4;
                if (r >= i1) break;
            }
        }
        const int64_t r_end = r;
        P knext = k1;
        if (!last) {
            int64_t rpe;
            if (have_win) {                                // window at wrb = r_end & ~3
                const int cu = (int)(r_end - wrb);
                const IT sel = cu == 0 ? wa[0] : cu == 1 ? wa[1] : cu == 2 ? wa[2] : wa[3];
                rpe = (int64_t)__shfl_sync(0xffffffffu, sel, 0);
            } else {
                rpe = (int64_t)__ldg(rp + (r_end < n ? r_end : n));
            }
            const int64_t kk = dsub - kRowW * r_end;
            knext = clampk(kk < rpe ? kk : rpe);
            if (knext < kcur) knext = kcur;
            if (knext > k1) knext = k1;
        }
        const int kn_rel = (int)(knext - base);
        __syncwarp();
        // a row start exactly at knext belongs to the next sub-span's first position
        const bool pending_next = knext < k1 && kn_rel < kCap && ((bm[kn_rel >> 5] >> (kn_rel & 31)) & 1u);
        __syncwarp();

        // ---- E: nonzeros [kcur, knext), 16 per lane per 512-position chunk from `base`:
        //      checks, block starts (written over the row-start bits), block sizes
        const unsigned F_sub = c_F;
        // a lane's 16 columns of the chunk at relative position cr (next chunk prefetched)
        auto load16 = [&](int cr, int (&v)[16]) {
            const P q0 = base + (P)(cr + lane * 16);
            if (col_aligned && (int64_t)q0 + 16 <= nnz) {
#pragma unroll
                for (int q = 0; q < 4; ++q) {
                    const int4 t = ld_hint(reinterpret_cast<const int4 *>(col + q0) + q, pol);
                    v[4 * q] = t.x; v[4 * q + 1] = t.y; v[4 * q + 2] = t.z; v[4 * q + 3] = t.w;
                }
            } else {
#pragma unroll
                for (int e = 0; e < 16; ++e) v[e] = (int64_t)q0 + e < nnz ? __ldg(col + q0 + e) : 0;
            }
        };
        int cn[16];
        if (kn_rel > 0) load16(0, cn);
        for (int cr = 0; cr < kn_rel; cr += kChunk) {
            const int off = cr + lane * 16;                          // relative position of the lane's first
            const P p0 = base + (P)off;
            int c[16];
#pragma unroll
            for (int e = 0; e < 16; ++e) c[e] = cn[e];
            if (cr + kChunk < kn_rel) load16(cr + kChunk, cn);
            const unsigned rs16 = (bm[off >> 5] >> (off & 31)) & 0xFFFFu;
            int pv = __shfl_up_sync(0xffffffffu, c[15], 1);
            if (lane == 0) pv = prevc;
            prevc = __shfl_sync(0xffffffffu, c[15], 31);
            const int lo_e = min(max(kc_rel - off, 0), 16);
            const int hi_e = min(max(kn_rel - off, 0), 16);
            const unsigned v16 = hi_e > lo_e ? (((1u << hi_e) - 1u) & ~((1u << lo_e) - 1u)) : 0u;
            unsigned fr = 0, ob = 0, cmax = 0;
#pragma unroll
            for (int e = 0; e < 16; ++e) {
                const int u = c[e] - (e == 0 ? pv : c[e - 1]) - 1;   // 0: the next column
                fr |= (unsigned)(u != 0) << e;                        // a block starts
                ob |= ((unsigned)u >> 31) << e;                      // not increasing: only at a row start
                cmax = max(cmax, (unsigned)c[e]);
            }
            const unsigned rsv = rs16 & v16;
            const unsigned f16 = (fr | rsv) & v16;
            if (ob & ~rsv & v16) bad |= BAD_COL_ORDER;
            if (v16 && (unsigned long long)cmax >= (unsigned long long)n_cols) bad |= BAD_COL_RANGE;
            const unsigned f_up = __shfl_up_sync(0xffffffffu, f16, 1);
            {
                const unsigned hi = __shfl_down_sync(0xffffffffu, f16, 1);
                if (!(lane & 1)) fl[off >> 5] = f16 | (hi << 16);
            }
            // block sizes = gaps between consecutive block starts.  A start whose previous
            // position is a start closes a block of size 1 (bit test, no loop); the others
            // (block >= 2, or the range's first start) walk back to the previous start.
            unsigned fprev = (f16 << 1) | (f_up >> 15);
            if (lane == 0) {
                const int q0 = max(off, kc_rel);                     // first valid position of lane 0
                fprev = (f16 << 1) | ((c_lastflag == base + (P)q0 - 1) ? 1u << (q0 - off) : 0u);
            }
            const unsigned s1 = f16 & fprev;
            const unsigned c1 = __popc(s1);
            sz2 += c1;
            if (c1) { sz_mn = 1u; sz_mx = max(sz_mx, 1u); }
            const int rel_last = f16 ? off + 31 - __clz(f16) : INT_MIN;
            const int incl = incl_max(rel_last, lane);
            const int before = __shfl_up_sync(0xffffffffu, incl, 1);
            int lastf_in;                                            // sub-span-relative previous start
            if (lane > 0 && before != INT_MIN) lastf_in = before;
            else if (c_lastflag != kNone) {
                const int64_t dl = (int64_t)c_lastflag - (int64_t)base;
                lastf_in = (int)(dl > (int64_t)INT_MIN + 1 ? dl : (int64_t)INT_MIN + 1);
            } else lastf_in = INT_MIN;
            unsigned rem = f16 & ~s1;
            while (rem) {
                const int e = __ffs(rem) - 1;
                rem &= rem - 1u;
                const unsigned below = f16 & ((1u << e) - 1u);
                const int pf_ = below ? off + 31 - __clz(below) : lastf_in;
                if (pf_ == INT_MIN) {
                    my_first_flag = p0 + (P)e;
                } else {
                    const unsigned sz = (unsigned)(off + e - pf_);
                    sz2 += (unsigned long long)sz * sz;
                    sz_mn = min(sz_mn, sz);
                    sz_mx = max(sz_mx, sz);
                }
            }
            const int last_in_chunk = __shfl_sync(0xffffffffu, incl, 31);
            if (last_in_chunk != INT_MIN) c_lastflag = base + (P)last_in_chunk;
            c_F += __reduce_add_sync(0xffffffffu, (unsigned)__popc(f16));
        }
        __syncwarp();

        // ---- P: exclusive prefix of the flag popcounts per bitmap word (words up to knext)
        {
            const int wk = kn_rel >> 5;
            constexpr int per = (kBmWords + 31) / 32;
            unsigned cnt[per], tot = 0;
#pragma unroll
            for (int j = 0; j < per; ++j) {
                const int wi = lane * per + j;
                cnt[j] = (wi < kBmWords && wi <= wk) ? __popc(fl[wi]) : 0u;
                tot += cnt[j];
            }
            unsigned run = excl_sum(tot, lane);
#pragma unroll
            for (int j = 0; j < per; ++j) {
                const int wi = lane * per + j;
                if (wi < kBmWords) pf[wi] = run;
                run += cnt[j];
            }
        }
        __syncwarp();
        // ---- B: blocks per row.  A (non-empty) row's block count is the number of block
        //      starts from its start to the next row start, F(next) - F(start) with F(p) =
        //      flags before p.  The sub-span's T row starts (valid positions) are dealt to
        //      the lanes in order, T/32 each: lane l closes rows [lT/32, (l+1)T/32).
        {
            constexpr int per = (kBmWords + 31) / 32;
            const int wk = kn_rel >> 5;
            auto vmask = [&](int wi) -> unsigned {                   // valid positions [kc_rel, kn_rel)
                const int lo = kc_rel - 32 * wi, hi = kn_rel - 32 * wi;
                return (hi >= 32 ? 0xffffffffu : (hi <= 0 ? 0u : (1u << hi) - 1u)) &
                       (lo <= 0 ? 0xffffffffu : (lo >= 32 ? 0u : ~((1u << lo) - 1u)));
            };
            unsigned cnt = 0;
#pragma unroll
            for (int j = 0; j < per; ++j) {
                const int wi = lane * per + j;
                if (wi < kBmWords && wi <= wk) cnt += __popc(bm[wi] & vmask(wi));
            }
            const unsigned ex = excl_sum(cnt, lane);
            const unsigned T = __shfl_sync(0xffffffffu, ex + cnt, 31);
            if (T > 0) {
                const unsigned s0 = (unsigned)(((unsigned long long)lane * T) >> 5);
                const unsigned s1 = (unsigned)(((unsigned long long)(lane + 1) * T) >> 5);
                // owner of row start s0: the last lane o with ex_o <= s0
                int o = 0;
#pragma unroll
                for (int step = 16; step > 0; step >>= 1) {
                    const unsigned e2 = __shfl_sync(0xffffffffu, ex, o + step);
                    if (e2 <= s0) o += step;
                }
                const unsigned exo = __shfl_sync(0xffffffffu, ex, o);
                long long F_first = -1, F_last = -1;
                if (s1 > s0) {
                    unsigned Fl = 0;                                  // F of the previous row start
                    bool have = false;
                    // the (s0 - ex_o)-th row start inside lane o's words
                    unsigned skip = s0 - exo;
                    int wi = o * per;
                    unsigned m = bm[wi] & vmask(wi);
                    while (__popc(m) <= skip) { skip -= __popc(m); ++wi; m = bm[wi] & vmask(wi); }
                    for (; skip; --skip) m &= m - 1u;
                    F_first = (long long)(F_sub + pf[wi] + __popc(fl[wi] & ((1u << (__ffs(m) - 1)) - 1u)));
                    for (unsigned k = s0; k < s1; ++k) {
                        const int b = __ffs(m) - 1;
                        const unsigned Fp = F_sub + pf[wi] + __popc(fl[wi] & ((1u << b) - 1u));
                        const unsigned nb = Fp - Fl;                  // the previous row's block count
                        if (have) {
                            nb2 += (unsigned long long)nb * nb;
                            nb_mn = min(nb_mn, nb);
                            nb_mx = max(nb_mx, nb);
                        }
                        have = true;
                        Fl = Fp;
                        m &= m - 1u;
                        if (k + 1 < s1)
                            while (!m) { ++wi; m = bm[wi] & vmask(wi); }
                    }
                    F_last = (long long)Fl;
                }
                // the last row of a lane ends at the next working lane's first row start
                const unsigned workm = __ballot_sync(0xffffffffu, s1 > s0);
                const unsigned later = workm & ~((2u << lane) - 1u);
                const long long F_next = __shfl_sync(0xffffffffu, F_first, later ? __ffs(later) - 1 : 0);
                if (s1 > s0 && later) {
                    const unsigned nb = (unsigned)(F_next - F_last);
                    nb2 += (unsigned long long)nb * nb;
                    nb_mn = min(nb_mn, nb);
                    nb_mx = max(nb_mx, nb);
                }
                // the first row start closes the row left open before the sub-span
                const int firstw = __ffs(workm) - 1, lastw = 31 - __clz(workm);
                const long long F0 = __shfl_sync(0xffffffffu, F_first, firstw);
                const long long FL = __shfl_sync(0xffffffffu, F_last, lastw);
                if (c_Frs >= 0) {
                    if (lane == 0) {
                        const unsigned nb = (unsigned)(F0 - c_Frs);
                        nb2 += (unsigned long long)nb * nb;
                        nb_mn = min(nb_mn, nb);
                        nb_mx = max(nb_mx, nb);
                    }
                } else if (head_nb < 0) {
                    head_nb = F0;                                     // the range's first row start
                }
                c_Frs = FL;
            }
        }
        __syncwarp();
        pending_rs = pending_next;
        kcur = knext;
        dcur = dsub;
        if (last) break;
    }

    // ---- warp record for the fix-up
    {
        const unsigned fm = __ballot_sync(0xffffffffu, my_first_flag != kNone);
        const long long ff = fm ? (long long)__shfl_sync(0xffffffffu, my_first_flag, __ffs(fm) - 1) : -1;
        if (lane == 0) {
            WarpRec rec;
            rec.first_flag = ff;
            rec.last_flag = c_lastflag != kNone ? (long long)c_lastflag : -1;
            rec.nflags = c_F;
            rec.has_rs = head_nb >= 0;
            rec.head_nb = head_nb >= 0 ? (unsigned long long)head_nb : 0ull;
            rec.has_open = c_Frs >= 0;                 // the last row start's row runs to the end
            rec.open_tail = c_Frs >= 0 ? (unsigned long long)(c_F - (unsigned)c_Frs) : 0ull;
            recs[w] = rec;
        }
    }

    // ---- commit the CTA's sums
    __shared__ unsigned long long s_u64[6][kWarps];
    __shared__ unsigned s_u32[7][kWarps];
    {
        unsigned long long v64[6] = {len2, over, nb2, sz2, (unsigned long long)n_empty, (unsigned long long)c_F};
#pragma unroll
        for (int i = 0; i < 5; ++i) v64[i] = warp_sum_u64(v64[i]);
        unsigned v32[7] = {warp_min_u32(len_mn), warp_max_u32(len_mx), warp_min_u32(nb_mn), warp_max_u32(nb_mx),
                           warp_min_u32(sz_mn), warp_max_u32(sz_mx), __reduce_or_sync(0xffffffffu, bad)};
        if (lane == 0) {
#pragma unroll
            for (int i = 0; i < 6; ++i) s_u64[i][wid] = v64[i];
#pragma unroll
            for (int i = 0; i < 7; ++i) s_u32[i][wid] = v32[i];
        }
    }
    __syncthreads();
    if (threadIdx.x == 0) {
        unsigned long long t64[6] = {0, 0, 0, 0, 0, 0};
        unsigned mn[3] = {UINT_MAX, UINT_MAX, UINT_MAX}, mx[3] = {0, 0, 0}, bd = 0;
        for (int k = 0; k < kWarps; ++k) {
            for (int i = 0; i < 6; ++i) t64[i] += s_u64[i][k];
            for (int i = 0; i < 3; ++i) {
                mn[i] = min(mn[i], s_u32[2 * i][k]);
                mx[i] = max(mx[i], s_u32[2 * i + 1][k]);
            }
            bd |= s_u32[6][k];
        }
        FeatureSums &A = st->acc;
        if (t64[0]) atomicAdd(&A.sum_len2, t64[0]);
        if (t64[1]) atomicAdd(&A.hyb_coo_ceil, t64[1]);
        if (t64[2]) atomicAdd(&A.sum_nb2, t64[2]);
        if (t64[3]) atomicAdd(&A.sum_bs2, t64[3]);
        if (t64[4]) atomicAdd(&A.n_empty, t64[4]);
        if (t64[5]) atomicAdd(&A.nb_tot, t64[5]);
        if (mn[0] != UINT_MAX) atomicMin(&A.len_min, (unsigned long long)mn[0]);
        if (mx[0]) atomicMax(&A.len_max, (unsigned long long)mx[0]);
        if (mn[1] != UINT_MAX) atomicMin(&A.nb_min, (unsigned long long)mn[1]);
        if (mx[1]) atomicMax(&A.nb_max, (unsigned long long)mx[1]);
        if (mn[2] != UINT_MAX) atomicMin(&A.bs_min, (unsigned long long)mn[2]);
        if (mx[2]) atomicMax(&A.bs_max, (unsigned long long)mx[2]);
        if (bd) atomicOr(&A.bad, (unsigned long long)bd);
    }
    if (use_hist) {
        __syncthreads();
        for (int i = threadIdx.x; i < sh_bins; i += kThreads)
            if (s_hist[i]) atomicAdd(&hist[i], (unsigned long long)s_hist[i]);
    }
    // ---- the last CTA closes the open blocks/rows and writes the result
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) s_last = atomicAdd(&st->done, 1ull) == gridDim.x - 1;
    __syncthreads();
    if (!s_last) return;
    __threadfence();
    unsigned long long fsz2 = 0, fnb2 = 0, fsz_mn = ULLONG_MAX, fsz_mx = 0, fnb_mn = ULLONG_MAX, fnb_mx = 0;
    for (int64_t v = threadIdx.x; v < W; v += kThreads) {
        const WarpRec rv = load_rec(recs + v);
        if (rv.last_flag >= 0) {                 // open block: closes at the next block start
            long long end = nnz;
            for (int64_t u = v + 1; u < W; ++u) {
                const long long f = __ldcg(&recs[u].first_flag);
                if (f >= 0) { end = f; break; }
            }
            const unsigned long long sz = (unsigned long long)(end - rv.last_flag);
            fsz2 += sz * sz;
            fsz_mn = sz < fsz_mn ? sz : fsz_mn;
            fsz_mx = sz > fsz_mx ? sz : fsz_mx;
        }
        if (rv.has_open) {                       // open row: closes at the next row start
            unsigned long long nb = rv.open_tail;
            for (int64_t u = v + 1; u < W; ++u) {
                if (__ldcg(&recs[u].has_rs)) { nb += __ldcg(&recs[u].head_nb); break; }
                nb += __ldcg(&recs[u].nflags);
            }
            fnb2 += nb * nb;
            fnb_mn = nb < fnb_mn ? nb : fnb_mn;
            fnb_mx = nb > fnb_mx ? nb : fnb_mx;
        }
    }
    __shared__ unsigned long long s_f[6][kWarps];
    {
        unsigned long long a = warp_sum_u64(fsz2), b = warp_sum_u64(fnb2);
        unsigned long long c1 = fsz_mn, c2 = fsz_mx, c3 = fnb_mn, c4 = fnb_mx;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) {
            unsigned long long t;
            t = __shfl_xor_sync(0xffffffffu, c1, o); c1 = t < c1 ? t : c1;
            t = __shfl_xor_sync(0xffffffffu, c2, o); c2 = t > c2 ? t : c2;
            t = __shfl_xor_sync(0xffffffffu, c3, o); c3 = t < c3 ? t : c3;
            t = __shfl_xor_sync(0xffffffffu, c4, o); c4 = t > c4 ? t : c4;
        }
        if (lane == 0) { s_f[0][wid] = a; s_f[1][wid] = b; s_f[2][wid] = c1; s_f[3][wid] = c2; s_f[4][wid] = c3; s_f[5][wid] = c4; }
    }
    __syncthreads();
    __shared__ long long s_cusp;
    if (threadIdx.x == 0) {
        FeatureSums R;
        volatile FeatureSums &A = st->acc;
        R.bad = A.bad; R.n_empty = A.n_empty; R.sum_len2 = A.sum_len2; R.len_min = A.len_min; R.len_max = A.len_max;
        R.hyb_coo_ceil = A.hyb_coo_ceil; R.nb_tot = A.nb_tot; R.sum_nb2 = A.sum_nb2; R.nb_min = A.nb_min;
        R.nb_max = A.nb_max; R.sum_bs2 = A.sum_bs2; R.bs_min = A.bs_min; R.bs_max = A.bs_max;
        for (int k = 0; k < kWarps; ++k) {
            R.sum_bs2 += s_f[0][k];
            R.sum_nb2 += s_f[1][k];
            R.bs_min = s_f[2][k] < R.bs_min ? s_f[2][k] : R.bs_min;
            R.bs_max = s_f[3][k] > R.bs_max ? s_f[3][k] : R.bs_max;
            R.nb_min = s_f[4][k] < R.nb_min ? s_f[4][k] : R.nb_min;
            R.nb_max = s_f[5][k] > R.nb_max ? s_f[5][k] : R.nb_max;
        }
        if (R.n_empty > 0) R.nb_min = 0;        // an empty row has no block (A8: all rows)
        st->result = R;
        s_cusp = (long long)R.len_max;
    }
    __syncthreads();
    if (use_hist) {
        // A2 "cusp" width: smallest k < nnz_max with 3*#{len>k} < n or #{len>k} < 4096, else
        // nnz_max; #{len>k} = n - sum_{j<=k} hist[j], exact for k < hist_bins - 1 and the
        // answer is < hist_bins - 1 by construction (hist_bins = nnz/4096 + 2).
        const long long kmax = s_cusp;
        const unsigned long long empty_rows = st->result.n_empty;
        __shared__ unsigned long long s_scan[kWarps];
        __shared__ unsigned long long s_run;
        __shared__ long long s_ans;
        if (threadIdx.x == 0) { s_run = 0; s_ans = kmax; }
        __syncthreads();
        for (long long b0 = 0; b0 < kmax && b0 < hist_bins; b0 += kThreads) {
            const long long k = b0 + threadIdx.x;
            const unsigned long long hv = k == 0 ? (unsigned long long)empty_rows : (k < hist_bins ? __ldcg(hist + k) : 0ull);
            unsigned long long incl = hv;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const unsigned long long t = __shfl_up_sync(0xffffffffu, incl, o);
                if (lane >= o) incl += t;
            }
            if (lane == 31) s_scan[wid] = incl;
            __syncthreads();
            unsigned long long woff = 0;
            for (int j = 0; j < wid; ++j) woff += s_scan[j];
            const unsigned long long cum = s_run + woff + incl;     // sum_{j<=k} hist[j]
            const long long longer = n - (long long)cum;
            const bool hit = k < kmax && k < hist_bins && (3 * longer < n || longer < 4096);
            const unsigned hb = __ballot_sync(0xffffffffu, hit);
            if (hb && lane == __ffs(hb) - 1) atomicMin((unsigned long long *)&s_ans, (unsigned long long)k);
            __syncthreads();
            if (threadIdx.x == kThreads - 1) s_run += woff + incl;
            __syncthreads();
            if (s_ans < kmax) break;
        }
        if (threadIdx.x == 0) st->cusp = n > 0 ? s_ans : 0;
        for (long long k = threadIdx.x; k < hist_bins; k += kThreads) hist[k] = 0ull;
    }
    if (threadIdx.x == 0) {
        init_sums(st->acc);
        st->done = 0;
    }
}

__global__ void k_features_state_init(FeatureState *st) {
    init_sums(st->acc);
    st->done = 0;
    st->cusp = 0;
}

template <typename IT>
spmv_status feature_pass_t(spmv_ctx *ctx, const spmv_csr *A, cudaStream_t s, int level,
                           FeatureSums *host, int64_t *hyb_cusp) {
    const IT *rp = reinterpret_cast<const IT *>(A->row_ptr);
    const int64_t n = A->n_rows, nnz = A->nnz;
    const int64_t items = (int64_t)kRowW * n + nnz;
    const int64_t hist_bins = level ? nnz / 4096 + 2 : 0;
    std::lock_guard<std::mutex> lock(ctx->feat_mu);

    // ctx-owned state, allocated once (and the histogram grown on demand)
    const int64_t max_ctas = (int64_t)ctx->sm_count * kCtasPerSm;
    if (!ctx->feat_state) {
        SPMV_TRY(dev_alloc(ctx, sizeof(FeatureState), nullptr, &ctx->feat_state));
        SPMV_TRY(dev_alloc(ctx, max_ctas * kWarps * sizeof(WarpRec), nullptr, &ctx->feat_recs));
        SPMV_CUDA_TRY(cudaMallocHost(&ctx->feat_host, sizeof(FeatureState)));
        k_features_state_init<<<1, 1, 0, nullptr>>>(reinterpret_cast<FeatureState *>(ctx->feat_state));
        SPMV_LAUNCH_CHECK();
        SPMV_CUDA_TRY(cudaStreamSynchronize(nullptr));
    }
    if (hist_bins * 8 > (int64_t)ctx->feat_hist_bytes) {
        if (ctx->feat_hist) dev_free(ctx, ctx->feat_hist, ctx->feat_hist_bytes, nullptr);
        ctx->feat_hist = nullptr;
        ctx->feat_hist_bytes = 0;
        SPMV_TRY(dev_alloc(ctx, hist_bins * 8, nullptr, &ctx->feat_hist));
        ctx->feat_hist_bytes = hist_bins * 8;
        SPMV_CUDA_TRY(cudaMemsetAsync(ctx->feat_hist, 0, hist_bins * 8, nullptr));
        SPMV_CUDA_TRY(cudaStreamSynchronize(nullptr));
    }
    // grid: up to kCtasPerSm resident CTAs per SM, each warp >= one sub-span of work
    int64_t ctas = ceil_div<int64_t>(items > 0 ? items : 1, (int64_t)kWarps * kSub);
    if (ctas > max_ctas) ctas = max_ctas;
    if (ctas < 1) ctas = 1;
    const int64_t W = ctas * kWarps;
    const int64_t per_warp = ceil_div<int64_t>(items > 0 ? items : 1, W);
    FeatureState *st = reinterpret_cast<FeatureState *>(ctx->feat_state);
    k_features<IT><<<(unsigned)ctas, kThreads, 0, s>>>(
        rp, A->col_idx, n, nnz, A->n_cols, n > 0 ? ceil_div<int64_t>(nnz, n) : 0, per_warp,
        reinterpret_cast<WarpRec *>(ctx->feat_recs), level ? reinterpret_cast<unsigned long long *>(ctx->feat_hist) : nullptr,
        hist_bins, st);
    SPMV_LAUNCH_CHECK();
    FeatureState *hs = reinterpret_cast<FeatureState *>(ctx->feat_host);
    SPMV_CUDA_TRY(cudaMemcpyAsync(&hs->result, &st->result, sizeof(FeatureSums) + sizeof(long long),
                                  cudaMemcpyDeviceToHost, s));
    SPMV_CUDA_TRY(cudaStreamSynchronize(s));
    *host = hs->result;
    if (n == 0) { host->len_min = 0; host->len_max = 0; }
    if (nnz == 0) { host->nb_tot = 0; host->sum_bs2 = 0; host->bs_min = 0; host->bs_max = 0; }
    if (n > 0 && nnz == 0) { host->nb_min = 0; host->nb_max = 0; host->sum_nb2 = 0; }
    if (hyb_cusp) *hyb_cusp = level ? hs->cusp : 0;
    return SPMV_OK;
}

}  // namespace

spmv_status feature_pass(spmv_ctx *ctx, const spmv_csr *A, cudaStream_t s, int level, FeatureSums *out,
                         int64_t *hyb_cusp) {
    if (A->ptr_type == SPMV_I32) return feature_pass_t<int>(ctx, A, s, level, out, hyb_cusp);
    return feature_pass_t<int64_t>(ctx, A, s, level, out, hyb_cusp);
}

void feature_state_free(spmv_ctx *ctx) {
    if (ctx->feat_state) dev_free(ctx, ctx->feat_state, sizeof(FeatureState), nullptr);
    if (ctx->feat_recs) dev_free(ctx, ctx->feat_recs, (size_t)ctx->sm_count * kCtasPerSm * kWarps * sizeof(WarpRec), nullptr);
    if (ctx->feat_hist) dev_free(ctx, ctx->feat_hist, ctx->feat_hist_bytes, nullptr);
    if (ctx->feat_host) cudaFreeHost(ctx->feat_host);
    ctx->feat_state = ctx->feat_recs = ctx->feat_hist = ctx->feat_host = nullptr;
    ctx->feat_hist_bytes = 0;
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
