"""B200-native six-format SpMV (COO, ELL, CSR, HYB, merge-path CSR, CSR5), CSR->format
converters, sparsity features and nnz-balanced multi-GPU partition -- the hot path of
Nisa et al., IPDPSW 2018.  The compute lives in libspmv.so (CUDA, sm_100a)
behind the C ABI of include/spmv.h; this package is a thin binding over it.
"""
from .spmv import (CSR, FORMATS, PAPER_FEATURES, PAPER_FORMATS, Context, Handle, SpmvError,  # noqa: F401
                   context, convert, features, lib, partition, run_host_multi, slice_remap, spmv_convert,
                   spmv_destroy, spmv_export, spmv_features, spmv_info, spmv_partition, spmv_run,
                   spmv_slice_remap)

__all__ = ["CSR", "FORMATS", "PAPER_FEATURES", "PAPER_FORMATS", "Context", "Handle", "SpmvError",
           "context", "convert", "features", "lib", "partition", "run_host_multi", "slice_remap", "spmv_convert",
           "spmv_destroy", "spmv_export", "spmv_features", "spmv_info", "spmv_partition", "spmv_run",
           "spmv_slice_remap"]
