/*
 * matgen_gpu.cu -- GPU twins of matgen.c's generators (INPUT GENERATION ONLY).
 *
 * "Generated on the GPU (counter-based RNG -> radix
 * sort -> unique).  Each rank builds identically and keeps its shard."  Every output
 * is bit-identical to the host generator (same counter-based hash, same key layout,
 * same value formula), so the oracle tests built on matgen.c pin these too
 * (tests/test_gpu_matgen.py compares them element by element).  Holds none of the
 * method's arithmetic (no SpMV, conversion, feature or partition code); the radix
 * sort and unique are CUB library primitives.
 *
 * All pointers are device pointers allocated by the caller; every call is
 * asynchronous on `stream` unless stated.
 */
#include <cub/cub.cuh>
#include <stdint.h>

namespace {

__device__ __forceinline__ uint64_t mix(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
}

__device__ __forceinline__ uint64_t hash3(uint64_t seed, uint64_t a, uint64_t b) {
    return mix(mix(mix(seed + 0x9E3779B97F4A7C15ULL) ^ (a * 0xD1B54A32D192ED03ULL)) + b);
}

/* matgen.c mg_value: 0 = [-1,1) on 2^-52, 1 = [-1,1) on 2^-23, 2 = {-2,-1,1,2}, 3 = 1 */
__device__ __forceinline__ double value(uint64_t h, int kind) {
    switch (kind) {
    case 0: return (double)(h >> 11) * 0x1p-52 - 1.0;
    case 1: return (double)(h >> 40) * 0x1p-23 - 1.0;
    case 2: { const double t[4] = {-2.0, -1.0, 1.0, 2.0}; return t[h & 3]; }
    default: return 1.0;
    }
}

__global__ void k_rmat_keys(uint64_t seed, int scale, int64_t n_edges, uint32_t ta, uint32_t tab, uint32_t tabc,
                            uint64_t *keys) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < n_edges;
         e += (int64_t)gridDim.x * blockDim.x) {
        uint64_t row = 0, colv = 0, h = 0;
        for (int lvl = 0; lvl < scale; ++lvl) {
            uint32_t u;
            if ((lvl & 1) == 0) { h = hash3(seed, (uint64_t)e, (uint64_t)(lvl >> 1)); u = (uint32_t)h; }
            else u = (uint32_t)(h >> 32);
            uint64_t rb, cb;
            if (u < ta) { rb = 0; cb = 0; }
            else if (u < tab) { rb = 0; cb = 1; }
            else if (u < tabc) { rb = 1; cb = 0; }
            else { rb = 1; cb = 1; }
            row = (row << 1) | rb;
            colv = (colv << 1) | cb;
        }
        keys[e] = (row << scale) | colv;
    }
}

/* row_ptr[r] = first key index of row >= r: thread i writes the rows in (row(i-1), row(i)];
 * the virtual key m (row n) closes the trailing empty rows. */
__global__ void k_keys_row_ptr(const uint64_t *keys, int64_t m, int shift, int64_t n_rows, int64_t *row_ptr) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i <= m; i += (int64_t)gridDim.x * blockDim.x) {
        const int64_t r = i < m ? (int64_t)(keys[i] >> shift) : n_rows;
        const int64_t rp = i > 0 ? (int64_t)(keys[i - 1] >> shift) : -1;
        for (int64_t q = rp + 1; q <= r; ++q) row_ptr[q] = i;
    }
}

__global__ void k_keys_col(const uint64_t *keys, int64_t k0, int64_t k1, uint64_t mask, int32_t *col) {
    for (int64_t k = k0 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < k1; k += (int64_t)gridDim.x * blockDim.x)
        col[k - k0] = (int32_t)(keys[k] & mask);
}

/* matgen.c mg_matrix_values: val(i, j) = value(hash(seed, i, j + 2^32)) -- position keyed */
template <typename V>
__global__ void k_keys_values(uint64_t seed, const uint64_t *keys, int64_t k0, int64_t k1, int shift, int kind, V *val) {
    const uint64_t mask = (1ULL << shift) - 1;
    for (int64_t k = k0 + blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < k1; k += (int64_t)gridDim.x * blockDim.x) {
        const uint64_t key = keys[k];
        val[k - k0] = (V)value(hash3(seed, key >> shift, (key & mask) + 0x100000000ULL), kind);
    }
}

template <typename V>
__global__ void k_vector(uint64_t seed, uint64_t stream_id, int64_t i0, int64_t n, int kind, V *out) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        out[i] = (V)value(hash3(seed, stream_id, (uint64_t)(i0 + i)), kind);
}

unsigned grid_for(int64_t n) {
    int64_t g = (n + 255) / 256;
    if (g > 148 * 32) g = 148 * 32;
    return (unsigned)(g < 1 ? 1 : g);
}

int ok(cudaError_t e) { return e == cudaSuccess ? 0 : -(int)e; }

}  // namespace

extern "C" {

/* R-MAT edge keys (row << scale | col), identical to mg_rmat_keys. */
int mgg_rmat_keys(uint64_t seed, int scale, int64_t n_edges, uint32_t ta, uint32_t tab, uint32_t tabc,
                  uint64_t *keys, void *stream) {
    k_rmat_keys<<<grid_for(n_edges), 256, 0, (cudaStream_t)stream>>>(seed, scale, n_edges, ta, tab, tabc, keys);
    return ok(cudaGetLastError());
}

/* Scratch bytes mgg_sort_unique needs for n keys (radix sort + unique, the larger). */
int64_t mgg_sort_unique_temp_bytes(int64_t n, int bits) {
    size_t a = 0, b = 0;
    cub::DoubleBuffer<uint64_t> db(nullptr, nullptr);
    cub::DeviceRadixSort::SortKeys(nullptr, a, db, n, 0, bits);
    cub::DeviceSelect::Unique(nullptr, b, (const uint64_t *)nullptr, (uint64_t *)nullptr, (int64_t *)nullptr, n);
    return (int64_t)(a > b ? a : b);
}

/* Sort keys[0..n) (< 2^bits) and drop duplicates; the unique keys end up in `keys`
 * (tmp is an n-key scratch buffer, temp the CUB scratch of mgg_sort_unique_temp_bytes).
 * Blocks on `stream`; returns the number of unique keys (< 0: CUDA error). */
int64_t mgg_sort_unique(uint64_t *keys, uint64_t *tmp, int64_t n, int bits, void *temp, int64_t temp_bytes,
                        int64_t *count_dev, void *stream) {
    cudaStream_t s = (cudaStream_t)stream;
    if (n <= 0) return 0;
    cub::DoubleBuffer<uint64_t> db(keys, tmp);
    size_t tb = (size_t)temp_bytes;
    if (cudaError_t e = cub::DeviceRadixSort::SortKeys(temp, tb, db, n, 0, bits, s)) return -(int64_t)e;
    uint64_t *src = db.Current(), *dst = src == keys ? tmp : keys;
    tb = (size_t)temp_bytes;
    if (cudaError_t e = cub::DeviceSelect::Unique(temp, tb, src, dst, count_dev, n, s)) return -(int64_t)e;
    int64_t m = 0;
    if (cudaError_t e = cudaMemcpyAsync(&m, count_dev, sizeof(m), cudaMemcpyDeviceToHost, s)) return -(int64_t)e;
    if (cudaError_t e = cudaStreamSynchronize(s)) return -(int64_t)e;
    if (dst != keys)
        if (cudaError_t e = cudaMemcpyAsync(keys, dst, (size_t)m * 8, cudaMemcpyDeviceToDevice, s)) return -(int64_t)e;
    return m;
}

/* sorted unique keys -> row_ptr[n_rows+1] (int64), identical to mg_keys_to_csr. */
int mgg_keys_row_ptr(const uint64_t *keys, int64_t m, int shift, int64_t n_rows, int64_t *row_ptr, void *stream) {
    k_keys_row_ptr<<<grid_for(m + 1), 256, 0, (cudaStream_t)stream>>>(keys, m, shift, n_rows, row_ptr);
    return ok(cudaGetLastError());
}

/* col[k - k0] = low `shift` bits of keys[k], k in [k0, k1). */
int mgg_keys_col(const uint64_t *keys, int64_t k0, int64_t k1, int shift, int32_t *col, void *stream) {
    if (k1 <= k0) return 0;
    k_keys_col<<<grid_for(k1 - k0), 256, 0, (cudaStream_t)stream>>>(keys, k0, k1, (1ULL << shift) - 1, col);
    return ok(cudaGetLastError());
}

/* val[k - k0] for k in [k0, k1): the position-keyed values of mg_matrix_values (fp64 or
 * rounded to fp32 when f32 != 0). */
int mgg_keys_values(uint64_t seed, const uint64_t *keys, int64_t k0, int64_t k1, int shift, int kind, int f32,
                    void *val, void *stream) {
    if (k1 <= k0) return 0;
    if (f32)
        k_keys_values<float><<<grid_for(k1 - k0), 256, 0, (cudaStream_t)stream>>>(seed, keys, k0, k1, shift, kind, (float *)val);
    else
        k_keys_values<double><<<grid_for(k1 - k0), 256, 0, (cudaStream_t)stream>>>(seed, keys, k0, k1, shift, kind, (double *)val);
    return ok(cudaGetLastError());
}

/* out[i] = value(hash(seed, stream_id, i0 + i)), i < n: mg_vector's entries i0.. */
int mgg_vector(uint64_t seed, uint64_t stream_id, int64_t i0, int64_t n, int kind, int f32, void *out, void *stream) {
    if (n <= 0) return 0;
    if (f32)
        k_vector<float><<<grid_for(n), 256, 0, (cudaStream_t)stream>>>(seed, stream_id, i0, n, kind, (float *)out);
    else
        k_vector<double><<<grid_for(n), 256, 0, (cudaStream_t)stream>>>(seed, stream_id, i0, n, kind, (double *)out);
    return ok(cudaGetLastError());
}

}  // extern "C"
