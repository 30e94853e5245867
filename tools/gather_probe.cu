// gather_probe.cu -- the practical ceiling of a matrix's column stream on this GPU.
//
// Not part of libspmv: a measurement tool (tools/gather_probe.py) that times, over a
// matrix's own col/val arrays, (a) streaming col+val alone and (b) streaming col+val
// plus the x[col] gather, with NO row handling.  (b) is the time any SpMV kernel of
// the six formats needs at least for this column stream (same loads, same gathers,
// nothing else), so "format time / probe time" separates the gather cost the
// matrix's structure imposes from the kernel's own overheads.
#include <cuda_runtime.h>
#include <stdint.h>

namespace {

__device__ __forceinline__ uint64_t pol_first() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ uint64_t pol_last() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
    return p;
}
__device__ __forceinline__ void ld8i(const int *p, int (&v)[8], uint64_t pol) {
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
                 : "l"(p), "l"(pol));
}
__device__ __forceinline__ void ld4d(const double *p, double (&v)[4], uint64_t pol) {
    long long w[4];
    asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.b64 {%0,%1,%2,%3}, [%4], %5;"
                 : "=l"(w[0]), "=l"(w[1]), "=l"(w[2]), "=l"(w[3]) : "l"(p), "l"(pol));
#pragma unroll
    for (int i = 0; i < 4; ++i) v[i] = __longlong_as_double(w[i]);
}
template <int MODE>
__device__ __forceinline__ double gx(const double *p, uint64_t pol) {
    double v;
    if (MODE == 1)        // L1 allocate, L2 evict-last (what the SpMV kernels use)
        asm volatile("ld.global.nc.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(pol));
    else if (MODE == 2)   // no L1 allocation
        asm volatile("ld.global.nc.L1::no_allocate.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(pol));
    else                  // plain ld.global (coherent path)
        asm volatile("ld.global.f64 %0, [%1];" : "=d"(v) : "l"(p));
    return v;
}

// one warp per 256 consecutive nonzeros (lane: 8 consecutive), grid-stride over chunks.
// MODE 0: stream col+val only.  MODE 1..3: + x gather (see gx).
template <int MODE>
__global__ void __launch_bounds__(256, 4)
k_probe(const int *__restrict__ col, const double *__restrict__ val, int64_t nnz, const double *__restrict__ x,
        double *__restrict__ out) {
    const int lane = threadIdx.x & 31;
    const uint64_t pa = pol_first(), px = pol_last();
    const int64_t nw = ((int64_t)gridDim.x * blockDim.x) >> 5;
    double s = 0.0;
    for (int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; w * 256 < nnz; w += nw) {
        const int64_t e0 = w * 256 + lane * 8;
        int c[8];
        double v[8];
        if (e0 + 8 <= nnz) {
            ld8i(col + e0, c, pa);
            double a[4], b[4];
            ld4d(val + e0, a, pa);
            ld4d(val + e0 + 4, b, pa);
#pragma unroll
            for (int q = 0; q < 4; ++q) { v[q] = a[q]; v[4 + q] = b[q]; }
        } else {
#pragma unroll
            for (int q = 0; q < 8; ++q) {
                const bool in = e0 + q < nnz;
                c[q] = in ? col[e0 + q] : -1;
                v[q] = in ? val[e0 + q] : 0.0;
            }
        }
#pragma unroll
        for (int q = 0; q < 8; ++q) {
            if (MODE == 0) s += v[q] + (double)c[q];
            else if (c[q] >= 0) s += v[q] * gx<MODE>(x + c[q], px);
        }
    }
    if (s == 1.2345e300) out[0] = s;   // keep the loads live; never true for the probe inputs
}

}  // namespace

extern "C" int probe_run(int mode, const int *col, const double *val, int64_t nnz, const double *x, double *out,
                         int sm_count, void *stream) {
    cudaStream_t s = (cudaStream_t)stream;
    int64_t warps = (nnz + 255) / 256;
    int64_t blocks = (warps + 7) / 8;
    if (blocks > (int64_t)sm_count * 16) blocks = (int64_t)sm_count * 16;
    if (blocks < 1) blocks = 1;
    switch (mode) {
    case 0: k_probe<0><<<(unsigned)blocks, 256, 0, s>>>(col, val, nnz, x, out); break;
    case 1: k_probe<1><<<(unsigned)blocks, 256, 0, s>>>(col, val, nnz, x, out); break;
    case 2: k_probe<2><<<(unsigned)blocks, 256, 0, s>>>(col, val, nnz, x, out); break;
    default: k_probe<3><<<(unsigned)blocks, 256, 0, s>>>(col, val, nnz, x, out); break;
    }
    return (int)cudaGetLastError();
}
