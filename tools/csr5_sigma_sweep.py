"""CSR5 sigma sweep (A6 reading, tuned on B200): time CSR5 with sigma in {4, 8, 12, 16} on
sweep matrices above a size threshold and on named configs; one JSON line per matrix.

usage: python tools/csr5_sigma_sweep.py [--count 400] [--min-nnz 1000000] [--configs lap4096 rmat22]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import matgen  # noqa: E402
import paper_conf_ipps_nisassvs18_b200 as sp  # noqa: E402
from paper_conf_ipps_nisassvs18_b200 import harness  # noqa: E402


def measure(A, tag, reps):
    dA = sp.CSR.from_host(A)
    x = torch.from_numpy(matgen.vector(A.n_cols, 1, 1)).cuda()
    y = torch.from_numpy(matgen.vector(A.n_rows, 1, 2)).cuda()
    out = {"tag": tag, "nnz": A.nnz, "n_rows": A.n_rows, "mu": A.nnz / max(A.n_rows, 1)}
    for s in (4, 8, 12, 16):
        h = sp.convert(dA, "csr5", csr5_sigma=s)
        out[f"s{s}"] = harness.time_handle(h, x, y.clone(), reps=reps, warmup=3, per_call=False)["t_mean_ms"]
        h.destroy()
    print(json.dumps(out), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--count", type=int, default=400)
    ap.add_argument("--min-nnz", type=int, default=1_000_000)
    ap.add_argument("--configs", nargs="*", default=["lap4096", "rmat22"])
    ap.add_argument("--reps", type=int, default=30)
    a = ap.parse_args()
    for c in a.configs:
        measure(bench.build_matrix(c, "f64"), c, a.reps)
    for i in range(a.count):
        p = matgen.sweep_params(i)
        if p["nnz_target"] < a.min_nnz:
            continue
        A, p = matgen.sweep_matrix(i)
        measure(A, f"sweep{i}:{p['family']}", a.reps)


if __name__ == "__main__":
    main()
