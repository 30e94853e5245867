// kernels.h -- compile-time tile sizes shared by conversion and run.
#pragma once
#include <stdint.h>

namespace spmv {
constexpr int kRunThreads = 256;           // CTA size of the tiled kernels
constexpr int kItemsPerThread = 8;         // sequential items per thread (COO / merge)
constexpr int kWarpItemsPerLane = 8;      // sequential items per lane (warp-tile COO / merge)
constexpr int64_t kCooItems = 32 * kWarpItemsPerLane;     // nonzeros per COO warp tile
constexpr int64_t kMergeItems = 32 * kWarpItemsPerLane;   // merge-path items per warp tile
constexpr int64_t kMergeLeanRows = 64;    // merge row-sum tiles (A28): < 64 row ends and
constexpr int64_t kMergeLeanLen = 32;     // in-tile row parts <= 32 nonzeros
constexpr int64_t kCsrChunk = 512;         // CSR long-row chunk (A25): rows > 2*kCsrChunk are split
                                           // (R-MAT 24: 6.6 -> 3.6 ms; 128..1024 within 15 %)
}  // namespace spmv
