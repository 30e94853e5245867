"""Per-rank local work of the halo-exchange step (HaloSpMV, dist.py) on ONE GPU, no
process group: for a P-way split of CONFIG, rank RANK's own-column block and
foreign-column block are built exactly as HaloSpMV builds them (the foreign block both
over all rows and compressed to its non-empty rows, A33) and each format's runs are timed
apart (CUDA events, mean of reps).  Shows what the foreign pass costs next
to the own pass in strong scaling.  usage: python tools/halo_local_time.py CONFIG P RANK"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ipps_nisassvs18_b200 as sp  # noqa: E402
from paper_conf_ipps_nisassvs18_b200.dist import HaloPlan  # noqa: E402
from paper_conf_ipps_nisassvs18_b200.spmv import (CSR, partition, spmv_compress_rows, spmv_gather,  # noqa: E402
                                                   spmv_scatter, spmv_slice_split)


def t_run(h, x, y, reps=50, rows=None, yc=None):
    def once():
        if rows is None:
            h.run(1.0, x, 1.0, y)
        else:                                   # A33: gather, compressed-row SpMV, scatter
            spmv_gather(y, rows, yc)
            h.run(1.0, x, 1.0, yc)
            spmv_scatter(yc, rows, y)
    s = torch.cuda.current_stream()
    for _ in range(5):
        once()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(reps):
        once()
    b.record(s)
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


def main():
    config, P, rank = sys.argv[1], int(sys.argv[2]), int(sys.argv[3])
    dA, _ = bench.device_matrix(config, "f64", torch.float64)
    splits = partition(dA, P)
    plan = HaloPlan(dA, splits, rank)
    rows = int(splits[rank + 1] - splits[rank])
    own_A = spmv_slice_split(dA, splits, rank, 0)
    for_A = spmv_slice_split(dA, splits, rank, 1, plan.colmap, plan.S)
    x = torch.ones(rows, dtype=torch.float64, device="cuda")
    xr = torch.ones(max(plan.recv_len, 1), dtype=torch.float64, device="cuda")
    y = torch.zeros(rows, dtype=torch.float64, device="cuda")
    frows, rp_c = spmv_compress_rows(for_A)
    Fc = CSR(rp_c, for_A.col, for_A.val, (frows.numel(), for_A.n_cols))
    yc = torch.zeros(frows.numel(), dtype=torch.float64, device="cuda")
    for f in sp.PAPER_FORMATS:
        try:
            ho, hf, hc = sp.convert(own_A, f), sp.convert(for_A, f), sp.convert(Fc, f)
        except sp.SpmvError as e:
            print(json.dumps({"fmt": f, "skip": e.status}))
            continue
        print(json.dumps({"config": config, "P": P, "rank": rank, "fmt": f, "rows": rows,
                          "own_nnz": own_A.nnz, "foreign_nnz": for_A.nnz,
                          "foreign_rows": frows.numel(), "own_ms": round(t_run(ho, x, y), 4),
                          "foreign_full_ms": round(t_run(hf, xr, y), 4),
                          "foreign_compressed_ms": round(t_run(hc, xr, y, rows=frows, yc=yc), 4)}), flush=True)


if __name__ == "__main__":
    main()
