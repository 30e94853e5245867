"""Small workload that launches every libspmv kernel, for
compute-sanitizer: features, all converters, every format's SpMV in fp64/fp32 with
beta = 0 (NaN y) and beta != 0, alpha = 0, the int64 index path, the CSR long-row
chunks, A30 hot columns in every format, the GPU R-MAT generator, partition / slice
remap / colmap / halo colmap / gather / own-foreign split.

usage: compute-sanitizer --tool memcheck python tools/sanitize_workload.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import matgen  # noqa: E402
import paper_conf_ipps_nisassvs18_b200 as sp  # noqa: E402
from paper_conf_ipps_nisassvs18_b200 import spmv as S  # noqa: E402
from test_gpu_parity import edge_cases  # noqa: E402

FORMATS = ("coo", "ell", "csr", "hyb", "merge", "csr5", "csr_scalar")
CASES = ("1x1", "rect_7x3", "nnz0_rows5", "empty_runs", "tile_bounds", "u2048", "rmat12", "sparse_rows",
         "dense_row_1x5000")


def main():
    torch.cuda.set_device(0)
    n_launch = 0
    for kind, dt in (("f64", torch.float64), ("f32", torch.float32)):
        cases = edge_cases(kind)
        # merge tile schedules (A28) and the CSR batch kernel's staged / unstaged batches (A29)
        cases["lap64"] = matgen.laplacian5(64)
        rng = np.random.default_rng(28)
        lens = rng.integers(3, 8, 6000)
        lens[[500, 4000]] = [900, 300]
        cases["mixed_long"] = matgen.from_lengths(lens, 6000, seed=2801, kind=kind)
        for name in CASES + ("lap64", "mixed_long"):
            A = cases[name]
            dA = sp.CSR.from_host(A, dtype=dt)
            sp.features(dA)
            x = torch.from_numpy(matgen.vector(A.n_cols, 3, 1, kind)).cuda().to(dt)
            for fmt in FORMATS:
                for opts in ({}, {"index64": 1}, {"csr_chunk": 7} if fmt == "csr" else None):
                    if opts is None:
                        continue
                    try:
                        h = sp.convert(dA, fmt, **opts)
                    except sp.SpmvError:
                        continue
                    for alpha, beta in ((1.0, 0.0), (1.5, -0.5), (0.0, 2.0)):
                        y = (torch.full((A.n_rows,), float("nan"), dtype=dt, device="cuda") if beta == 0.0 else
                             torch.from_numpy(matgen.vector(A.n_rows, 3, 2, kind)).cuda().to(dt))
                        h.run(alpha, x, beta, y)
                        n_launch += h.launches()
                    h.destroy()
        torch.cuda.synchronize()
    # A30 hot columns forced on every format (the per-run pack + the HOT kernel variants)
    A = matgen.rmat(13, seed=13)
    dA = sp.CSR.from_host(A)
    x = torch.from_numpy(matgen.vector(A.n_cols, 6, 1)).cuda()
    for fmt in ("coo", "ell", "csr", "hyb", "merge", "csr5"):
        try:
            h = sp.convert(dA, fmt, hot_x=64)
        except sp.SpmvError:
            continue
        for beta in (0.0, 1.0):
            y = torch.zeros(A.n_rows, dtype=torch.float64, device="cuda")
            h.run(1.0, x, beta, y)
            n_launch += h.launches()
        h.export("col") if fmt not in ("ell", "hyb") else h.export("ell_col")
        h.destroy()
    # the GPU R-MAT generator (input generation: keys, sort/unique, CSR, values, vectors)
    from matgen import gpu
    gpu.rmat(12, seed=14)
    gpu.vector(1000, 1, 1)
    torch.cuda.synchronize()
    # CSR-vector with the dynamic batch scheduler (W >= 16, >= 1.8M rows): R-MAT scale 21
    A = matgen.rmat(21, seed=21)
    dA = sp.CSR.from_host(A)
    h = sp.convert(dA, "csr")
    xr = torch.from_numpy(matgen.vector(A.n_cols, 5, 1)).cuda()
    yr = torch.from_numpy(matgen.vector(A.n_rows, 5, 2)).cuda()
    h.run(1.0, xr, 1.0, yr)
    n_launch += h.launches()
    h.destroy()
    del dA
    torch.cuda.synchronize()
    # multi-GPU plumbing on one device: partition, remap, colmap, gather, own/foreign split
    A = matgen.rmat(12, seed=12)
    dA = sp.CSR.from_host(A)
    splits = sp.partition(dA, 3)
    for part in range(3):
        sp.slice_remap(dA, splits, part)
        colmap, slot = S.spmv_partition_colmap(dA, splits)
        sl = S.spmv_slice_remap_colmap(dA, splits, part, colmap, slot)
        idx = S.spmv_colmap_pack_index(colmap, splits, part, slot)
        src = torch.from_numpy(matgen.vector(A.n_cols, 4, 1)).cuda()
        dst = torch.empty(idx.numel(), dtype=torch.float64, device="cuda")
        S.spmv_gather(src, idx, dst)
        for which in (0, 1):
            S.spmv_slice_split(dA, splits, part, which)
        # halo exchange plumbing: the foreign block through a HaloPlan colmap
        from paper_conf_ipps_nisassvs18_b200.dist import HaloPlan
        plan = HaloPlan(dA, splits, part)
        fb = S.spmv_slice_split(dA, splits, part, 1, plan.colmap, plan.S)
        hf = sp.convert(fb, "csr")
        hf.run(1.0, torch.zeros(plan.recv_len, dtype=torch.float64, device="cuda"), 1.0,
               torch.zeros(fb.n_rows, dtype=torch.float64, device="cuda"))
        hf.destroy()
        del sl
    torch.cuda.synchronize()
    print(f"sanitize workload done: {n_launch} SpMV launches")


if __name__ == "__main__":
    main()
