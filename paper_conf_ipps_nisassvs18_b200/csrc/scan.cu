// scan.cu -- device exclusive prefix sum over int64 (conversion helper: HYB COO
// offsets, CSR5 empty-row map offsets).  Three phases: per-block sums, a single
// block scanning the block sums, per-block rescan with the block offset.
#include "internal.h"
#include "scan.h"

namespace spmv {

namespace {
constexpr int kT = 256;
constexpr int kPer = 8;                 // items per thread
constexpr int kTile = kT * kPer;

__device__ __forceinline__ long long block_excl_scan(long long v, long long *total) {
    __shared__ long long s_w[kT / 32];
    int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
    long long incl = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        long long t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
    }
    if (lane == 31) s_w[wid] = incl;
    __syncthreads();
    long long off = 0, tot = 0;
#pragma unroll
    for (int i = 0; i < kT / 32; ++i) {
        if (i < wid) off += s_w[i];
        tot += s_w[i];
    }
    __syncthreads();
    *total = tot;
    return off + incl - v;
}

__global__ void __launch_bounds__(kT) k_block_sums(const int64_t *in, int64_t n, int64_t *sums) {
    int64_t base = (int64_t)blockIdx.x * kTile + threadIdx.x * kPer;
    long long s = 0;
#pragma unroll
    for (int i = 0; i < kPer; ++i) s += base + i < n ? in[base + i] : 0;
    long long tot;
    block_excl_scan(s, &tot);
    if (threadIdx.x == 0) sums[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(kT) k_scan_sums(int64_t *sums, int64_t nb) {
    __shared__ long long carry;
    if (threadIdx.x == 0) carry = 0;
    __syncthreads();
    for (int64_t base = 0; base < nb; base += kT) {
        int64_t i = base + threadIdx.x;
        long long v = i < nb ? sums[i] : 0, tot;
        long long ex = block_excl_scan(v, &tot);
        long long c = carry;
        if (i < nb) sums[i] = c + ex;
        __syncthreads();
        if (threadIdx.x == 0) carry = c + tot;
        __syncthreads();
    }
    if (threadIdx.x == 0) sums[nb] = carry;
}

__global__ void __launch_bounds__(kT) k_rescan(const int64_t *in, int64_t n, const int64_t *sums, int64_t *out) {
    int64_t base = (int64_t)blockIdx.x * kTile + threadIdx.x * kPer;
    long long v[kPer], s = 0;
#pragma unroll
    for (int i = 0; i < kPer; ++i) { v[i] = base + i < n ? in[base + i] : 0; s += v[i]; }
    long long tot;
    long long run = block_excl_scan(s, &tot) + sums[blockIdx.x];
#pragma unroll
    for (int i = 0; i < kPer; ++i) {
        if (base + i < n) out[base + i] = run;
        run += v[i];
    }
}

__global__ void k_copy_total(const int64_t *sums, int64_t nb, int64_t *out, int64_t n) { out[n] = sums[nb]; }
}  // namespace

spmv_status exclusive_scan_i64(spmv_ctx *ctx, const int64_t *in, int64_t *out, int64_t n, cudaStream_t s) {
    if (n <= 0) {
        SPMV_CUDA_TRY(cudaMemsetAsync(out, 0, sizeof(int64_t), s));
        return SPMV_OK;
    }
    int64_t nb = ceil_div<int64_t>(n, kTile);
    Scratch sums(ctx, s);
    SPMV_TRY(sums.alloc((nb + 1) * sizeof(int64_t)));
    k_block_sums<<<(unsigned)nb, kT, 0, s>>>(in, n, sums.as<int64_t>());
    SPMV_LAUNCH_CHECK();
    k_scan_sums<<<1, kT, 0, s>>>(sums.as<int64_t>(), nb);
    SPMV_LAUNCH_CHECK();
    k_rescan<<<(unsigned)nb, kT, 0, s>>>(in, n, sums.as<int64_t>(), out);
    SPMV_LAUNCH_CHECK();
    k_copy_total<<<1, 1, 0, s>>>(sums.as<int64_t>(), nb, out, n);
    SPMV_LAUNCH_CHECK();
    return SPMV_OK;
}

}  // namespace spmv
