// scan.h -- internal device scan helper.
#pragma once
#include "internal.h"

namespace spmv {
// out[0..n] = exclusive prefix sums of in[0..n), out[n] = total.  Stream-ordered.
spmv_status exclusive_scan_i64(spmv_ctx *ctx, const int64_t *in, int64_t *out, int64_t n, cudaStream_t s);
}  // namespace spmv
