// common.cuh -- internal helpers of libspmv (sm_100a).  Not part of the ABI.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>
#include <stddef.h>
#include <string>
#include "../../include/spmv.h"

namespace spmv {

// ---------------------------------------------------------------- errors
void set_error(const std::string &msg);
const char *get_error();

#define SPMV_CUDA_TRY(expr)                                                        \
    do {                                                                           \
        cudaError_t _e = (expr);                                                   \
        if (_e != cudaSuccess) {                                                   \
            ::spmv::set_error(std::string(#expr) + ": " + cudaGetErrorString(_e)); \
            return SPMV_ERR_CUDA;                                                  \
        }                                                                          \
    } while (0)

#define SPMV_LAUNCH_CHECK()                                                        \
    do {                                                                           \
        cudaError_t _e = cudaGetLastError();                                       \
        if (_e != cudaSuccess) {                                                   \
            ::spmv::set_error(std::string("kernel launch: ") + cudaGetErrorString(_e)); \
            return SPMV_ERR_CUDA;                                                  \
        }                                                                          \
    } while (0)

#define SPMV_TRY(expr)                                   \
    do {                                                 \
        spmv_status _s = (expr);                         \
        if (_s != SPMV_OK) return _s;                    \
    } while (0)

static inline cudaStream_t as_stream(void *s) { return reinterpret_cast<cudaStream_t>(s); }

// ---------------------------------------------------------------- device loads
// A (col/val) is streamed once per SpMV: read-only path, no L1 allocation and an
// L2 evict-first policy so that the gathered x keeps its L2 residency (north_star:
// "x gathered through L2/read-only paths"); x itself is loaded through the
// read-only path with an L2 evict-last policy.  sm_100 accepts the eviction
// qualifier directly only on 256-bit loads; narrower loads carry a createpolicy
// cache-policy operand instead.
__device__ __forceinline__ uint64_t policy_evict_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t policy_evict_last() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}

#define SPMV_LD_HINT(T, PT, REG)                                                        \
    __device__ __forceinline__ T ld_hint(const T *p, uint64_t pol) {                     \
        T v;                                                                            \
        asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint." PT " %0, [%1], %2;"  \
                     : "=" REG(v) : "l"(p), "l"(pol));                                   \
        return v;                                                                       \
    }
SPMV_LD_HINT(int, "s32", "r")
SPMV_LD_HINT(float, "f32", "f")
SPMV_LD_HINT(double, "f64", "d")
SPMV_LD_HINT(int64_t, "s64", "l")
#undef SPMV_LD_HINT

__device__ __forceinline__ int4 ld_hint(const int4 *p, uint64_t pol) {
    int4 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.s32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ int2 ld_hint(const int2 *p, uint64_t pol) {
    int2 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.s32 {%0,%1}, [%2], %3;"
                 : "=r"(v.x), "=r"(v.y) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ float4 ld_hint(const float4 *p, uint64_t pol) {
    float4 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.f32 {%0,%1,%2,%3}, [%4], %5;"
                 : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ float2 ld_hint(const float2 *p, uint64_t pol) {
    float2 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f32 {%0,%1}, [%2], %3;"
                 : "=f"(v.x), "=f"(v.y) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ double2 ld_hint(const double2 *p, uint64_t pol) {
    double2 v;
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v2.f64 {%0,%1}, [%2], %3;"
                 : "=d"(v.x), "=d"(v.y) : "l"(p), "l"(pol));
    return v;
}
// four doubles (two 16-byte loads) -- ELL's 4-rows-per-thread slot pairs
struct double4a { double2 lo, hi; };
__device__ __forceinline__ double4a ld_hint(const double4a *p, uint64_t pol) {
    double4a r;
    r.lo = ld_hint(reinterpret_cast<const double2 *>(p), pol);
    r.hi = ld_hint(reinterpret_cast<const double2 *>(p) + 1, pol);
    return r;
}
// 256-bit (32-byte aligned) streaming loads: one instruction covers a whole sector per
// lane, so a lane's 8-element chunk is requested from L2 once (two 16-byte loads of one
// sector would be two requests -- with L1::no_allocate the second goes to L2 again)
__device__ __forceinline__ void ld256(const int *p, int (&v)[8], uint64_t pol) {
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
                 : "l"(p), "l"(pol));
}
__device__ __forceinline__ void ld256(const float *p, float (&v)[8], uint64_t pol) {
    int w[8];
    ld256(reinterpret_cast<const int *>(p), w, pol);
#pragma unroll
    for (int i = 0; i < 8; ++i) v[i] = __int_as_float(w[i]);
}
__device__ __forceinline__ void ld256(const double *p, double (&v)[4], uint64_t pol) {
    long long w[4];
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.b64 {%0,%1,%2,%3}, [%4], %5;"
                 : "=l"(w[0]), "=l"(w[1]), "=l"(w[2]), "=l"(w[3]) : "l"(p), "l"(pol));
#pragma unroll
    for (int i = 0; i < 4; ++i) v[i] = __longlong_as_double(w[i]);
}

// x gathers: read-only path, keep in L1 (neighbouring gathers hit), L2 evict-last
__device__ __forceinline__ float ld_x(const float *p, uint64_t pol) {
    float v;
    asm volatile("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ double ld_x(const double *p, uint64_t pol) {
    double v;
    asm volatile("ld.global.nc.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(pol));
    return v;
}
__device__ __forceinline__ int ld_x(const int *p, uint64_t pol) {
    int v;
    asm volatile("ld.global.nc.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
    return v;
}

// A30 hot columns: a handle may store the column of a hot x entry as -2 - slot (-1 stays
// the "no element" sentinel of ELL padding and partial loads); its value is then
// xh[slot], the run's densely packed copy of the hot x entries
template <bool HOT, typename V>
__device__ __forceinline__ const V *xp(const V *x, const V *xh, int c) {
    if constexpr (HOT) return c >= 0 ? x + c : xh + (-2 - c);
    else return x + c;
}


// x gather of column c (HOT, A30: from the packed hot entries when c <= -2).  Marking the
// cold gathers evict_first instead of evict_last was measured slower on R-MAT 27 (CSR5
// 14.1 -> 14.3 ms, merge 21.2 -> 22.0), so both keep the evict_last policy of x.
template <bool HOT, typename V>
__device__ __forceinline__ V ldx(const V *x, const V *xh, int c, uint64_t px) {
    return ld_x(xp<HOT>(x, xh, c), px);
}

// plain read-only loads for metadata (row_ptr, descriptors)
template <typename T> __device__ __forceinline__ T ldg(const T *p) { return __ldg(p); }

// ---------------------------------------------------------------- y update
// y_r <- alpha*s + beta*y_r with beta == 0 => y not read (A14).  Accumulation is
// fp64 for both dtypes (A13); one rounding to the storage type at the end.
template <typename V>
__device__ __forceinline__ void y_store(V *y, int64_t r, double s, double alpha, double beta, bool beta0) {
    double out = alpha * s;
    if (!beta0) out = fma(beta, (double)y[r], out);
    y[r] = (V)out;
}

// ---------------------------------------------------------------- misc
template <typename T> __host__ __device__ __forceinline__ T ceil_div(T a, T b) { return (a + b - 1) / b; }

// warp-wide sum of a double (full mask; all 32 lanes must participate)
__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}

// binary search: largest i in [lo, hi] with key(i) <= d, where key is strictly
// increasing.  Used for merge-path coordinates (A7): key(i) = row_ptr[i] + i.
template <typename IT>
__device__ __forceinline__ int64_t merge_path_row(const IT *row_ptr, int64_t n_rows, int64_t nnz, int64_t d) {
    int64_t lo = d - nnz > 0 ? d - nnz : 0;      // at most nnz nonzeros can precede
    int64_t hi = d < n_rows ? d : n_rows;
    while (lo < hi) {                             // invariant: answer in [lo, hi]
        int64_t mid = (lo + hi + 1) >> 1;
        if ((int64_t)row_ptr[mid] + mid <= d) lo = mid; else hi = mid - 1;
    }
    return lo;
}

// upper_bound over row_ptr[0..n_rows]: number of i in [0, n_rows] with row_ptr[i] <= e
template <typename IT>
__device__ __forceinline__ int64_t upper_bound_rp(const IT *row_ptr, int64_t n_rows, int64_t e) {
    int64_t lo = 0, hi = n_rows + 1;
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if ((int64_t)row_ptr[mid] <= e) lo = mid + 1; else hi = mid;
    }
    return lo;
}
// lower_bound over row_ptr[0..n_rows): first r in [0, n_rows] with r == n_rows or row_ptr[r] >= e
template <typename IT>
__device__ __forceinline__ int64_t lower_bound_rp(const IT *row_ptr, int64_t n_rows, int64_t e) {
    int64_t lo = 0, hi = n_rows;
    while (lo < hi) {
        int64_t mid = (lo + hi) >> 1;
        if ((int64_t)row_ptr[mid] < e) lo = mid + 1; else hi = mid;
    }
    return lo;
}

}  // namespace spmv
