// api.cu -- the C ABI of include/spmv.h: ctx, handle lifetime, dispatch, export.
#include <cstring>
#include <new>
#include <string>
#include <vector>

#include <nvtx3/nvToolsExt.h>

#include "internal.h"

namespace spmv {

// NVTX ranges (SURVEY §5 tracing): visible in Nsight Systems / ncu --nvtx, free otherwise
struct NvtxRange {
    explicit NvtxRange(const char *name) { nvtxRangePushA(name); }
    ~NvtxRange() { nvtxRangePop(); }
};
static const char *kRunNames[] = {"spmv_run:coo", "spmv_run:ell", "spmv_run:csr", "spmv_run:hyb",
                                  "spmv_run:merge", "spmv_run:csr5", "spmv_run:csr_scalar"};
static const char *kConvNames[] = {"spmv_convert:coo", "spmv_convert:ell", "spmv_convert:csr", "spmv_convert:hyb",
                                   "spmv_convert:merge", "spmv_convert:csr5", "spmv_convert:csr_scalar"};

static thread_local std::string g_err;
void set_error(const std::string &msg) { g_err = msg; }
const char *get_error() { return g_err.c_str(); }

spmv_status dev_alloc(spmv_ctx *ctx, size_t bytes, cudaStream_t s, void **out) {
    *out = nullptr;
    if (bytes == 0) bytes = 16;
    if (ctx->has_alloc) {
        *out = ctx->alloc.alloc(bytes, ctx->device, (void *)s, ctx->alloc.user);
        if (!*out) {
            set_error("allocator returned NULL for " + std::to_string(bytes) + " bytes");
            return SPMV_ERR_NO_MEMORY;
        }
        return SPMV_OK;
    }
    cudaError_t e = cudaMallocAsync(out, bytes, s);
    if (e != cudaSuccess) {
        cudaGetLastError();
        set_error(std::string("cudaMallocAsync: ") + cudaGetErrorString(e));
        *out = nullptr;
        return e == cudaErrorMemoryAllocation ? SPMV_ERR_NO_MEMORY : SPMV_ERR_CUDA;
    }
    return SPMV_OK;
}

void dev_free(spmv_ctx *ctx, void *p, size_t bytes, cudaStream_t s) {
    if (!p) return;
    if (bytes == 0) bytes = 16;
    if (ctx->has_alloc) ctx->alloc.free(p, bytes, ctx->device, (void *)s, ctx->alloc.user);
    else cudaFreeAsync(p, s);
}

// Every entry point that touches the device runs on the ctx's device and leaves the
// caller's current device as it found it.
struct DeviceGuard {
    int prev = -1;
    cudaError_t err = cudaSuccess;
    explicit DeviceGuard(int dev) {
        if (cudaGetDevice(&prev) != cudaSuccess) { cudaGetLastError(); prev = -1; }
        if (prev != dev) err = cudaSetDevice(dev);
    }
    ~DeviceGuard() {
        int cur = -1;
        if (prev >= 0 && cudaGetDevice(&cur) == cudaSuccess && cur != prev) cudaSetDevice(prev);
    }
};
#define SPMV_ON_DEVICE(dev)                                                        \
    DeviceGuard _dg(dev);                                                          \
    if (_dg.err != cudaSuccess) {                                                  \
        set_error(std::string("cudaSetDevice: ") + cudaGetErrorString(_dg.err));   \
        return SPMV_ERR_CUDA;                                                      \
    }

static spmv_status check_csr(const spmv_csr *A) {
    if (!A) { set_error("A is NULL"); return SPMV_ERR_INVALID_ARG; }
    if (A->n_rows < 0 || A->n_cols < 0 || A->nnz < 0) { set_error("negative dimension"); return SPMV_ERR_INVALID_ARG; }
    if (A->n_rows > INT32_MAX || A->n_cols > (int64_t)INT32_MAX + 1) {
        set_error("n_rows/n_cols exceed the int32 index range (A17)");
        return SPMV_ERR_SIZE;
    }
    if (A->ptr_type != SPMV_I32 && A->ptr_type != SPMV_I64) { set_error("bad ptr_type"); return SPMV_ERR_INVALID_ARG; }
    if (A->dtype != SPMV_F32 && A->dtype != SPMV_F64) { set_error("bad dtype"); return SPMV_ERR_INVALID_ARG; }
    if (A->ptr_type == SPMV_I32 && A->nnz > INT32_MAX) { set_error("nnz > INT32_MAX with int32 row_ptr"); return SPMV_ERR_SIZE; }
    if (!A->row_ptr) { set_error("row_ptr is NULL"); return SPMV_ERR_INVALID_ARG; }
    if (A->nnz > 0 && (!A->col_idx || !A->vals)) { set_error("col_idx/vals NULL with nnz > 0"); return SPMV_ERR_INVALID_ARG; }
    return SPMV_OK;
}

}  // namespace spmv

using namespace spmv;

extern "C" {

int spmv_abi_version(void) { return SPMV_ABI_VERSION; }

const char *spmv_status_str(spmv_status s) {
    switch (s) {
    case SPMV_OK: return "SPMV_OK";
    case SPMV_ERR_INVALID_ARG: return "SPMV_ERR_INVALID_ARG";
    case SPMV_ERR_NOT_CANONICAL: return "SPMV_ERR_NOT_CANONICAL";
    case SPMV_ERR_SIZE: return "SPMV_ERR_SIZE";
    case SPMV_ERR_NO_MEMORY: return "SPMV_ERR_NO_MEMORY";
    case SPMV_ERR_CUDA: return "SPMV_ERR_CUDA";
    case SPMV_ERR_UNSUPPORTED: return "SPMV_ERR_UNSUPPORTED";
    }
    return "SPMV_ERR_UNKNOWN";
}

const char *spmv_last_error(void) { return get_error(); }

spmv_status spmv_init(int device, const spmv_allocator *alloc, spmv_ctx **out) {
    if (!out) { set_error("out is NULL"); return SPMV_ERR_INVALID_ARG; }
    *out = nullptr;
    int n = 0;
    cudaError_t e = cudaGetDeviceCount(&n);
    if (e != cudaSuccess || n == 0) {
        cudaGetLastError();
        set_error(std::string("no CUDA device: ") + cudaGetErrorString(e));
        return SPMV_ERR_UNSUPPORTED;
    }
    if (device < 0 || device >= n) { set_error("device out of range"); return SPMV_ERR_INVALID_ARG; }
    cudaDeviceProp prop;
    SPMV_CUDA_TRY(cudaGetDeviceProperties(&prop, device));
    if (prop.major != 10 || prop.minor != 0) {
        set_error("libspmv is built for sm_100a (B200); device is sm_" + std::to_string(prop.major) +
                  std::to_string(prop.minor));
        return SPMV_ERR_UNSUPPORTED;
    }
    SPMV_ON_DEVICE(device);
    spmv_ctx *c = new (std::nothrow) spmv_ctx();
    if (!c) return SPMV_ERR_NO_MEMORY;
    c->device = device;
    c->sm_count = prop.multiProcessorCount;
    c->l2_bytes = prop.l2CacheSize;
    if (alloc && alloc->alloc && alloc->free) {
        c->alloc = *alloc;
        c->has_alloc = true;
    }
    *out = c;
    return SPMV_OK;
}

spmv_status spmv_finalize(spmv_ctx *ctx) {
    if (!ctx) return SPMV_OK;
    {
        DeviceGuard dg(ctx->device);
        feature_state_free(ctx);
    }
    delete ctx;
    return SPMV_OK;
}

spmv_status spmv_device_info(const spmv_ctx *ctx, int *sm_count, int64_t *l2_bytes) {
    if (!ctx) return SPMV_ERR_INVALID_ARG;
    if (sm_count) *sm_count = ctx->sm_count;
    if (l2_bytes) *l2_bytes = ctx->l2_bytes;
    return SPMV_OK;
}

spmv_status spmv_features(spmv_ctx *ctx, const spmv_csr *A, void *stream, spmv_features_t *out) {
    NvtxRange nv("spmv_features");
    if (!ctx || !out) { set_error("NULL ctx/out"); return SPMV_ERR_INVALID_ARG; }
    SPMV_TRY(check_csr(A));
    SPMV_ON_DEVICE(ctx->device);
    FeatureSums fs;
    int64_t cusp = 0;
    SPMV_TRY(feature_pass(ctx, A, as_stream(stream), 1, &fs, &cusp));
    if (fs.bad) {
        set_error("matrix is not canonical (flags " + std::to_string(fs.bad) + ")");
        return SPMV_ERR_NOT_CANONICAL;
    }
    finalize_features(A, fs, cusp, out);
    return SPMV_OK;
}

void spmv_convert_opts_default(spmv_convert_opts *o) {
    if (!o) return;
    std::memset(o, 0, sizeof(*o));
    o->hyb_rule = 0;
    o->hyb_width = -1;
}

spmv_status spmv_convert(spmv_ctx *ctx, spmv_format fmt, const spmv_csr *A,
                         const spmv_convert_opts *opts, void *stream, spmv_handle **out) {
    if (!ctx || !out) { set_error("NULL ctx/out"); return SPMV_ERR_INVALID_ARG; }
    *out = nullptr;
    SPMV_TRY(check_csr(A));
    if ((int)fmt < 0 || (int)fmt > (int)SPMV_CSR_SCALAR) { set_error("bad format"); return SPMV_ERR_INVALID_ARG; }
    NvtxRange nv(kConvNames[fmt]);
    spmv_convert_opts o;
    spmv_convert_opts_default(&o);
    if (opts) o = *opts;
    if (o.csr5_sigma && (o.csr5_sigma < 4 || o.csr5_sigma > 16 || o.csr5_sigma % 4)) {
        set_error("csr5_sigma must be 4, 8, 12 or 16");
        return SPMV_ERR_INVALID_ARG;
    }
    if (o.vector_width && (o.vector_width > 32 || (o.vector_width & (o.vector_width - 1)))) {
        set_error("vector_width must be a power of two <= 32");
        return SPMV_ERR_INVALID_ARG;
    }
    SPMV_ON_DEVICE(ctx->device);
    spmv_handle *h = new (std::nothrow) spmv_handle();
    if (!h) return SPMV_ERR_NO_MEMORY;
    h->ctx = ctx;
    h->fmt = fmt;
    h->dtype = A->dtype;
    h->n_rows = A->n_rows;
    h->n_cols = A->n_cols;
    h->nnz = A->nnz;
    spmv_status st = convert_impl(ctx, fmt, A, &o, as_stream(stream), h);
    if (st != SPMV_OK) {
        spmv_destroy(h, stream);
        return st;
    }
    *out = h;
    return SPMV_OK;
}

static bool overlaps(const void *a, size_t na, const void *b, size_t nb) {
    const char *x = (const char *)a, *y = (const char *)b;
    return na && nb && x < y + nb && y < x + na;
}

spmv_status spmv_run(spmv_handle *h, const void *alpha, const void *x, const void *beta, void *y,
                     void *stream) {
    if (!h || !alpha || !beta) { set_error("NULL handle/alpha/beta"); return SPMV_ERR_INVALID_ARG; }
    size_t V = h->dtype == SPMV_F64 ? 8 : 4;
    if ((h->n_cols > 0 && !x) || (h->n_rows > 0 && !y)) { set_error("NULL x/y"); return SPMV_ERR_INVALID_ARG; }
    if (overlaps(x, h->n_cols * V, y, h->n_rows * V)) { set_error("x and y overlap"); return SPMV_ERR_INVALID_ARG; }
    double a, b;
    if (h->dtype == SPMV_F64) { a = *(const double *)alpha; b = *(const double *)beta; }
    else { a = *(const float *)alpha; b = *(const float *)beta; }
    SPMV_ON_DEVICE(h->ctx->device);
    NvtxRange nv(kRunNames[h->fmt]);
    return run_impl(h, a, b, x, y, as_stream(stream));
}

spmv_status spmv_run_host(spmv_handle *h, const void *alpha, const void *x_host, const void *beta,
                          void *y_host, void *stream) {
    if (!h || !alpha || !beta) { set_error("NULL handle/alpha/beta"); return SPMV_ERR_INVALID_ARG; }
    size_t V = h->dtype == SPMV_F64 ? 8 : 4;
    cudaStream_t s = as_stream(stream);
    SPMV_ON_DEVICE(h->ctx->device);
    size_t bx = (size_t)h->n_cols * V, by = (size_t)h->n_rows * V;
    if (!h->io_x.p && bx) { SPMV_TRY(dev_alloc(h->ctx, bx, s, &h->io_x.p)); h->io_x.bytes = bx; }
    if (!h->io_y.p && by) { SPMV_TRY(dev_alloc(h->ctx, by, s, &h->io_y.p)); h->io_y.bytes = by; }
    double b = h->dtype == SPMV_F64 ? *(const double *)beta : *(const float *)beta;
    if (bx) SPMV_CUDA_TRY(cudaMemcpyAsync(h->io_x.p, x_host, bx, cudaMemcpyHostToDevice, s));
    if (by && b != 0.0) SPMV_CUDA_TRY(cudaMemcpyAsync(h->io_y.p, y_host, by, cudaMemcpyHostToDevice, s));
    SPMV_TRY(spmv_run(h, alpha, h->io_x.p, beta, h->io_y.p, stream));
    if (by) SPMV_CUDA_TRY(cudaMemcpyAsync(y_host, h->io_y.p, by, cudaMemcpyDeviceToHost, s));
    SPMV_CUDA_TRY(cudaStreamSynchronize(s));
    return SPMV_OK;
}

spmv_status spmv_run_host_multi(spmv_handle *const *hs, int k, const void *alpha, const void *x_host,
                                const void *beta, const void *y_in_host, void *const *y_out_host, void *stream) {
    if (!hs || k < 1 || !alpha || !beta || !y_out_host) { set_error("NULL handles/alpha/beta/y_out or k < 1"); return SPMV_ERR_INVALID_ARG; }
    spmv_handle *H = hs[0];
    if (!H) { set_error("NULL handle"); return SPMV_ERR_INVALID_ARG; }
    for (int i = 0; i < k; ++i) {
        const spmv_handle *h = hs[i];
        if (!h || h->ctx != H->ctx || h->dtype != H->dtype || h->n_rows != H->n_rows || h->n_cols != H->n_cols) {
            set_error("spmv_run_host_multi: handle " + std::to_string(i) + " is not of the first handle's ctx/dtype/shape");
            return SPMV_ERR_INVALID_ARG;
        }
        for (int j = 0; j < i; ++j)
            if (hs[j] == h) { set_error("spmv_run_host_multi: a handle appears twice"); return SPMV_ERR_INVALID_ARG; }
        if (H->n_rows && !y_out_host[i]) { set_error("spmv_run_host_multi: NULL y_out"); return SPMV_ERR_INVALID_ARG; }
    }
    const size_t V = H->dtype == SPMV_F64 ? 8 : 4;
    const double b = H->dtype == SPMV_F64 ? *(const double *)beta : *(const float *)beta;
    if (H->n_rows && b != 0.0 && !y_in_host) { set_error("spmv_run_host_multi: NULL y_in with beta != 0"); return SPMV_ERR_INVALID_ARG; }
    cudaStream_t s = as_stream(stream);
    SPMV_ON_DEVICE(H->ctx->device);
    const size_t bx = (size_t)H->n_cols * V, by = (size_t)H->n_rows * V;
    if (!H->io_x.p && bx) { SPMV_TRY(dev_alloc(H->ctx, bx, s, &H->io_x.p)); H->io_x.bytes = bx; }
    if (!H->io_yin.p && by && b != 0.0) { SPMV_TRY(dev_alloc(H->ctx, by, s, &H->io_yin.p)); H->io_yin.bytes = by; }
    for (int i = 0; i < k; ++i)
        if (!hs[i]->io_y.p && by) { SPMV_TRY(dev_alloc(H->ctx, by, s, &hs[i]->io_y.p)); hs[i]->io_y.bytes = by; }
    // x and y_in cross PCIe once; each run starts from a device copy of y_in; run i's result
    // goes back on a second stream while run i+1 computes
    if (bx) SPMV_CUDA_TRY(cudaMemcpyAsync(H->io_x.p, x_host, bx, cudaMemcpyHostToDevice, s));
    if (by && b != 0.0) SPMV_CUDA_TRY(cudaMemcpyAsync(H->io_yin.p, y_in_host, by, cudaMemcpyHostToDevice, s));
    cudaStream_t c = nullptr;
    SPMV_CUDA_TRY(cudaStreamCreateWithFlags(&c, cudaStreamNonBlocking));
    std::vector<cudaEvent_t> ev((size_t)k, nullptr);
    spmv_status st = SPMV_OK;
    for (int i = 0; i < k && st == SPMV_OK; ++i) {
        spmv_handle *h = hs[i];
        if (by && b != 0.0 && cudaMemcpyAsync(h->io_y.p, H->io_yin.p, by, cudaMemcpyDeviceToDevice, s) != cudaSuccess) {
            set_error(std::string("spmv_run_host_multi: y_in copy: ") + cudaGetErrorString(cudaGetLastError()));
            st = SPMV_ERR_CUDA;
            break;
        }
        st = spmv_run(h, alpha, H->io_x.p, beta, h->io_y.p, stream);
        if (st != SPMV_OK || !by) continue;
        if (cudaEventCreateWithFlags(&ev[i], cudaEventDisableTiming) != cudaSuccess || cudaEventRecord(ev[i], s) != cudaSuccess ||
            cudaStreamWaitEvent(c, ev[i], 0) != cudaSuccess ||
            cudaMemcpyAsync(y_out_host[i], h->io_y.p, by, cudaMemcpyDeviceToHost, c) != cudaSuccess) {
            set_error(std::string("spmv_run_host_multi: y copy-back: ") + cudaGetErrorString(cudaGetLastError()));
            st = SPMV_ERR_CUDA;
        }
    }
    const cudaError_t e1 = cudaStreamSynchronize(c), e2 = cudaStreamSynchronize(s);
    for (cudaEvent_t e : ev)
        if (e) cudaEventDestroy(e);
    cudaStreamDestroy(c);
    if (st == SPMV_OK && (e1 != cudaSuccess || e2 != cudaSuccess)) {
        set_error(std::string("spmv_run_host_multi: ") + cudaGetErrorString(e1 != cudaSuccess ? e1 : e2));
        st = SPMV_ERR_CUDA;
    }
    return st;
}

spmv_status spmv_run_launches(const spmv_handle *h, int *launches) {
    if (!h || !launches) return SPMV_ERR_INVALID_ARG;
    *launches = run_launch_count(h, false);
    return SPMV_OK;
}

spmv_status spmv_info(const spmv_handle *h, spmv_handle_info *o) {
    if (!h || !o) return SPMV_ERR_INVALID_ARG;
    std::memset(o, 0, sizeof(*o));
    o->format = h->fmt;
    o->dtype = h->dtype;
    o->ptr_type = h->itype;
    o->n_rows = h->n_rows;
    o->n_cols = h->n_cols;
    o->nnz = h->nnz;
    o->ell_width = h->ell_K;
    o->ell_ld = h->ell_ld;
    o->hyb_coo_nnz = h->hyb_coo_nnz;
    o->csr5_sigma = h->sigma;
    o->csr5_tiles = h->n_tiles;
    o->csr5_map_len = h->map_len;
    o->merge_items = h->merge_T;
    o->merge_tiles = h->merge_tiles;
    o->vector_width = h->vec_w;
    o->csr_chunks = h->csr_chunks;
    o->hot_cols = h->n_hot;
    size_t dev = 0, fmt_bytes = 0;
    for (int i = 0; i < kMaxArrays; ++i) {
        if (h->arr[i].owned) dev += h->arr[i].bytes;
        // the merge kernels derive the nonzero coordinate as d - row (A7) and take the tile
        // class from the tile order: both kept for export, not read by a run
        if (i != SPMV_ARR_MERGE_COORD_NZ && i != SPMV_ARR_MERGE_TILE_CLASS) fmt_bytes += h->arr[i].bytes;
    }
    dev += h->carry_row.bytes + h->carry_val.bytes + h->sched.bytes + h->xhot.bytes;
    o->device_bytes = dev;
    // algorithmic bytes per run: the format's own arrays + x + y
    size_t V = h->dtype == SPMV_F64 ? 8 : 4;
    size_t xy = (size_t)h->n_cols * V + (size_t)h->n_rows * V;
    // A30: the per-run hot pack reads x[hot] (counted in x), writes xhot, the kernels read it
    // back; the hot-column list itself is counted with the format's arrays
    const size_t hot = (size_t)h->n_hot * V * 2;
    o->bytes_per_run_beta0 = fmt_bytes + xy + hot;
    o->bytes_per_run = fmt_bytes + xy + hot + (size_t)h->n_rows * V;
    return SPMV_OK;
}

spmv_status spmv_export(const spmv_handle *h, spmv_array_id id, void *dst, size_t cap, size_t *written,
                        void *stream) {
    if (!h || (int)id < 0 || (int)id >= kMaxArrays) { set_error("bad handle/array id"); return SPMV_ERR_INVALID_ARG; }
    const DevArray &a = h->arr[id];
    if (written) *written = a.bytes;
    if (!a.p && a.bytes) { set_error("array not present"); return SPMV_ERR_INVALID_ARG; }
    if (!a.p) {
        // present-but-empty arrays have bytes == 0; absent arrays are flagged by bytes==0 and p==NULL
        bool present = false;
        switch (h->fmt) {
        case SPMV_COO: present = id == SPMV_ARR_COO_ROW || id == SPMV_ARR_COL || id == SPMV_ARR_VAL; break;
        case SPMV_CSR: present = id <= SPMV_ARR_VAL || id == SPMV_ARR_CSR_CHUNK_ROW || id == SPMV_ARR_CSR_CHUNK_LO; break;
        case SPMV_CSR_SCALAR: present = id <= SPMV_ARR_VAL; break;
        case SPMV_ELL: present = id == SPMV_ARR_ELL_COL || id == SPMV_ARR_ELL_VAL; break;
        case SPMV_HYB: present = id == SPMV_ARR_ELL_COL || id == SPMV_ARR_ELL_VAL || id == SPMV_ARR_COO_ROW ||
                                 id == SPMV_ARR_HYB_COO_COL || id == SPMV_ARR_HYB_COO_VAL; break;
        case SPMV_MERGE: present = id <= SPMV_ARR_VAL || id == SPMV_ARR_MERGE_COORD_ROW ||
                                   id == SPMV_ARR_MERGE_COORD_NZ || id == SPMV_ARR_MERGE_TILE_CLASS ||
                                   id == SPMV_ARR_MERGE_TILE_ORDER; break;
        case SPMV_CSR5: present = id <= SPMV_ARR_VAL || (id >= SPMV_ARR_CSR5_TILE_PTR && id <= SPMV_ARR_CSR5_SEG_MAP); break;
        }
        if (id == SPMV_ARR_HOT_COLS) present = true;            // A30: empty when no hot columns
        if (!present) { set_error("handle has no such array"); return SPMV_ERR_INVALID_ARG; }
        return SPMV_OK;
    }
    if (cap < a.bytes || !dst) { set_error("destination too small"); return SPMV_ERR_INVALID_ARG; }
    cudaStream_t s = as_stream(stream);
    SPMV_ON_DEVICE(h->ctx->device);
    SPMV_CUDA_TRY(cudaMemcpyAsync(dst, a.p, a.bytes, cudaMemcpyDeviceToHost, s));
    SPMV_CUDA_TRY(cudaStreamSynchronize(s));
    if (h->n_hot > 0 && (id == SPMV_ARR_COL || id == SPMV_ARR_ELL_COL || id == SPMV_ARR_HYB_COO_COL)) {
        // A30: column arrays are exported as column indices (-2 - slot -> hot[slot])
        std::vector<int32_t> hot((size_t)h->n_hot);
        SPMV_CUDA_TRY(cudaMemcpyAsync(hot.data(), h->arr[SPMV_ARR_HOT_COLS].p, hot.size() * 4,
                                      cudaMemcpyDeviceToHost, s));
        SPMV_CUDA_TRY(cudaStreamSynchronize(s));
        int32_t *c = static_cast<int32_t *>(dst);
        for (size_t k = 0; k < a.bytes / 4; ++k)
            if (c[k] <= -2) c[k] = hot[(size_t)(-2 - c[k])];
    }
    return SPMV_OK;
}

spmv_status spmv_destroy(spmv_handle *h, void *stream) {
    if (!h) return SPMV_OK;
    cudaStream_t s = as_stream(stream);
    DeviceGuard dg(h->ctx->device);
    for (int i = 0; i < kMaxArrays; ++i)
        if (h->arr[i].owned && h->arr[i].p) dev_free(h->ctx, h->arr[i].p, h->arr[i].bytes + 64, s);
    dev_free(h->ctx, h->carry_row.p, h->carry_row.bytes, s);
    dev_free(h->ctx, h->carry_val.p, h->carry_val.bytes, s);
    dev_free(h->ctx, h->io_x.p, h->io_x.bytes, s);
    dev_free(h->ctx, h->sched.p, h->sched.bytes, s);
    dev_free(h->ctx, h->xhot.p, h->xhot.bytes, s);
    dev_free(h->ctx, h->io_y.p, h->io_y.bytes, s);
    dev_free(h->ctx, h->io_yin.p, h->io_yin.bytes, s);
    delete h;
    return SPMV_OK;
}

spmv_status spmv_partition(spmv_ctx *ctx, const spmv_csr *A, int nparts, void *stream, int64_t *splits) {
    NvtxRange nv("spmv_partition");
    if (!ctx || !splits || nparts <= 0) { set_error("bad ctx/splits/nparts"); return SPMV_ERR_INVALID_ARG; }
    SPMV_TRY(check_csr(A));
    SPMV_ON_DEVICE(ctx->device);
    return partition_impl(ctx, A, nparts, as_stream(stream), splits);
}

spmv_status spmv_slice_size(spmv_ctx *ctx, const spmv_csr *A, const int64_t *splits, int nparts, int part,
                            void *stream, int64_t *rows, int64_t *nnz, int64_t *slot) {
    if (!ctx || !splits || nparts <= 0 || part < 0 || part >= nparts) { set_error("bad args"); return SPMV_ERR_INVALID_ARG; }
    SPMV_TRY(check_csr(A));
    SPMV_ON_DEVICE(ctx->device);
    return slice_size_impl(ctx, A, splits, nparts, part, as_stream(stream), rows, nnz, slot);
}

spmv_status spmv_slice_remap(spmv_ctx *ctx, const spmv_csr *A, const int64_t *splits, int nparts, int part,
                             void *stream, int32_t *rp_out, int32_t *col_out, void *val_out) {
    if (!ctx || !splits || nparts <= 0 || part < 0 || part >= nparts || !rp_out) { set_error("bad args"); return SPMV_ERR_INVALID_ARG; }
    SPMV_TRY(check_csr(A));
    if (A->n_rows != A->n_cols) { set_error("slice_remap needs a square matrix"); return SPMV_ERR_INVALID_ARG; }
    SPMV_ON_DEVICE(ctx->device);
    return slice_remap_impl(ctx, A, splits, nparts, part, as_stream(stream), rp_out, col_out, val_out);
}

spmv_status spmv_partition_colmap(spmv_ctx *ctx, const spmv_csr *A, const int64_t *splits, int nparts, void *stream,
                                  int32_t *colmap_out, int64_t *slot) {
    if (!ctx || !splits || nparts <= 0 || !colmap_out || !slot) { set_error("bad args"); return SPMV_ERR_INVALID_ARG; }
    SPMV_TRY(check_csr(A));
    if (A->n_rows != A->n_cols) { set_error("partition_colmap needs a square matrix"); return SPMV_ERR_INVALID_ARG; }
    SPMV_ON_DEVICE(ctx->device);
    return colmap_impl(ctx, A, splits, nparts, as_stream(stream), colmap_out, slot);
}

spmv_status spmv_slice_remap_colmap(spmv_ctx *ctx, const spmv_csr *A, const int64_t *splits, int nparts, int part,
                                    const int32_t *colmap, void *stream, int32_t *rp_out, int32_t *col_out,
                                    void *val_out) {
    if (!ctx || !splits || nparts <= 0 || part < 0 || part >= nparts || !rp_out || !colmap) {
        set_error("bad args");
        return SPMV_ERR_INVALID_ARG;
    }
    SPMV_TRY(check_csr(A));
    if (A->n_rows != A->n_cols) { set_error("slice_remap needs a square matrix"); return SPMV_ERR_INVALID_ARG; }
    SPMV_ON_DEVICE(ctx->device);
    return slice_remap_colmap_impl(ctx, A, splits, nparts, part, colmap, as_stream(stream), rp_out, col_out, val_out);
}

spmv_status spmv_halo_colmap(spmv_ctx *ctx, const spmv_csr *A, const int64_t *splits, int nparts, int part,
                             void *stream, int32_t *colmap_out, int64_t *counts_host, int64_t *slot) {
    if (!ctx || !splits || nparts <= 0 || part < 0 || part >= nparts || !colmap_out || !counts_host || !slot) {
        set_error("bad args");
        return SPMV_ERR_INVALID_ARG;
    }
    SPMV_TRY(check_csr(A));
    if (A->n_rows != A->n_cols) { set_error("halo_colmap needs a square matrix"); return SPMV_ERR_INVALID_ARG; }
    SPMV_ON_DEVICE(ctx->device);
    return halo_colmap_impl(ctx, A, splits, nparts, part, as_stream(stream), colmap_out, counts_host, slot);
}

spmv_status spmv_colmap_pack_index(spmv_ctx *ctx, const int32_t *colmap, const int64_t *splits, int nparts, int part,
                                   int64_t slot, void *stream, int32_t *idx_out, int64_t *count) {
    if (!ctx || !colmap || !splits || nparts <= 0 || part < 0 || part >= nparts || !count || slot < 0) {
        set_error("bad args");
        return SPMV_ERR_INVALID_ARG;
    }
    if (splits[part + 1] > splits[part] && !idx_out) { set_error("NULL idx_out"); return SPMV_ERR_INVALID_ARG; }
    SPMV_ON_DEVICE(ctx->device);
    return pack_index_impl(ctx, colmap, splits, nparts, part, slot, as_stream(stream), idx_out, count);
}

spmv_status spmv_slice_split(spmv_ctx *ctx, const spmv_csr *A, const int64_t *splits, int nparts, int part,
                             const int32_t *colmap, int which, void *stream, int32_t *rp_out, int32_t *col_out,
                             void *val_out, int64_t *nnz_out) {
    if (!ctx || !splits || nparts <= 0 || part < 0 || part >= nparts || !rp_out || !nnz_out || (which != 0 && which != 1)) {
        set_error("bad args");
        return SPMV_ERR_INVALID_ARG;
    }
    SPMV_TRY(check_csr(A));
    if (A->n_rows != A->n_cols) { set_error("slice_split needs a square matrix"); return SPMV_ERR_INVALID_ARG; }
    SPMV_ON_DEVICE(ctx->device);
    return split_impl(ctx, A, splits, nparts, part, colmap, which, as_stream(stream), rp_out, col_out, val_out, nnz_out);
}

spmv_status spmv_gather(spmv_ctx *ctx, spmv_dtype dtype, const void *src, const int32_t *idx, int64_t n, void *dst,
                        void *stream) {
    if (!ctx || n < 0 || (n > 0 && (!src || !idx || !dst))) { set_error("bad args"); return SPMV_ERR_INVALID_ARG; }
    if (dtype != SPMV_F32 && dtype != SPMV_F64) { set_error("bad dtype"); return SPMV_ERR_INVALID_ARG; }
    SPMV_ON_DEVICE(ctx->device);
    return gather_impl(ctx, dtype, src, idx, n, dst, as_stream(stream));
}

spmv_status spmv_scatter(spmv_ctx *ctx, spmv_dtype dtype, const void *src, const int32_t *idx, int64_t n, void *dst,
                         void *stream) {
    if (!ctx || n < 0 || (n > 0 && (!src || !idx || !dst))) { set_error("bad args"); return SPMV_ERR_INVALID_ARG; }
    if (dtype != SPMV_F32 && dtype != SPMV_F64) { set_error("bad dtype"); return SPMV_ERR_INVALID_ARG; }
    SPMV_ON_DEVICE(ctx->device);
    return scatter_impl(ctx, dtype, src, idx, n, dst, as_stream(stream));
}

spmv_status spmv_compress_rows(spmv_ctx *ctx, const spmv_csr *A, void *stream, int32_t *rows_out, void *rp_out,
                               int64_t *count_host) {
    if (!ctx || !count_host || !rp_out || (A && A->n_rows > 0 && !rows_out)) { set_error("bad args"); return SPMV_ERR_INVALID_ARG; }
    SPMV_TRY(check_csr(A));
    if (A->n_rows > INT32_MAX) { set_error("compress_rows: more than 2^31 - 1 rows"); return SPMV_ERR_INVALID_ARG; }
    SPMV_ON_DEVICE(ctx->device);
    return compress_rows_impl(ctx, A, as_stream(stream), rows_out, rp_out, count_host);
}

}  // extern "C"
