// kernels.h -- compile-time tile sizes shared by conversion and run.
#pragma once
#include <stdint.h>

namespace spmv {
constexpr int kRunThreads = 256;           // CTA size of the tiled kernels
constexpr int kItemsPerThread = 8;         // sequential items per thread (COO / merge)
constexpr int64_t kCooItems = kRunThreads * kItemsPerThread;     // nonzeros per COO CTA
constexpr int64_t kMergeItems = kRunThreads * kItemsPerThread;   // merge-path items per CTA
}  // namespace spmv
