"""Tuning experiments: time one format on one config with given convert options.

usage: python tools/exp.py CONFIG FORMAT[:key=val,...] [FORMAT...] [--dtype f32] [--reps 50]
e.g.   python tools/exp.py rmat24 csr5 csr5:csr5_sigma=8 merge
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import matgen  # noqa: E402
import paper_conf_ipps_nisassvs18_b200 as sp  # noqa: E402
from paper_conf_ipps_nisassvs18_b200 import harness  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config")
    ap.add_argument("formats", nargs="+")
    ap.add_argument("--dtype", default="f64")
    ap.add_argument("--reps", type=int, default=50)
    a = ap.parse_args()
    dt = torch.float64 if a.dtype == "f64" else torch.float32
    t0 = time.time()
    A = bench.build_matrix(a.config, a.dtype)
    dA = sp.CSR.from_host(A, dtype=dt)
    x = torch.from_numpy(matgen.vector(A.n_cols, 1, 1, a.dtype)).cuda().to(dt)
    y = torch.from_numpy(matgen.vector(A.n_rows, 1, 2, a.dtype)).cuda().to(dt)
    print(f"# {a.config} n={A.n_rows} nnz={A.nnz} gen {time.time() - t0:.1f}s", flush=True)
    peak, _ = bench.measured_peak()
    for spec in a.formats:
        fmt, _, opt = spec.partition(":")
        opts = {}
        for kv in filter(None, opt.split(",")):
            k, v = kv.split("=")
            opts[k] = int(v) if v.lstrip("-").isdigit() else v
        try:
            h = sp.convert(dA, fmt, **opts)
        except sp.SpmvError as e:
            print(json.dumps({"spec": spec, "error": e.name}))
            continue
        t = harness.time_handle(h, x, y, reps=a.reps, warmup=5)
        info = h.info()
        gbs = info["bytes_per_run"] / (t["t_mean_ms"] * 1e-3) / 1e9
        print(json.dumps({"spec": spec, "ms": round(t["t_mean_ms"], 4), "ms_min": round(t["t_min_ms"], 4),
                          "gbs": round(gbs, 1), "frac": round(gbs / peak, 4),
                          "gflops": round(2 * A.nnz / (t["t_mean_ms"] * 1e-3) / 1e9, 1)}), flush=True)
        h.destroy()


if __name__ == "__main__":
    main()
