"""BASELINE configs[4] on one GPU: R-MAT scale 27, edge factor 16 (~2.1e9 nonzeros), fp64,
CSR / merge / CSR5.  Parity at full size in the launch configuration bench.py times:

  * integer regime (values and x in {+-1, +-2}, alpha = 2, beta = -1): every format must
    equal the oracle bit for bit on EVERY row (P5, order-independent);
  * uniform values: every format within 1e-12 * bound of the oracle on every row.

Then each format is timed (5 warm-ups, mean of 20 runs, alpha = beta = 1).
Writes one JSON line to stdout (and --out).  Needs ~80 GB of host RAM and ~120 GB of
HBM; refuses to start with less free host memory than --min-host-gb.
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=int, default=27)
    ap.add_argument("--formats", default="csr,merge,csr5")
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--min-host-gb", type=float, default=110.0)
    ap.add_argument("--out", default="")
    a = ap.parse_args()
    import psutil
    avail = psutil.virtual_memory().available / 2 ** 30
    if avail < a.min_host_gb:
        print(json.dumps({"skipped": f"only {avail:.0f} GB host memory available"}))
        return
    import numpy as np
    import torch

    import matgen
    import oracle
    import paper_conf_ipps_nisassvs18_b200 as sp
    from paper_conf_ipps_nisassvs18_b200 import harness

    rec = {"config": f"rmat{a.scale}", "formats": {}}
    t0 = time.time()
    A = matgen.rmat(a.scale, seed=matgen.SEEDS["rmat27"], kind="int")
    rec["gen_s"] = round(time.time() - t0, 1)
    rec.update(n_rows=A.n_rows, nnz=A.nnz, index_type="int64" if A.nnz > 2 ** 31 - 1 else "int32")
    x_i = matgen.vector(A.n_cols, 5, 1, "int")
    y_i = np.round(matgen.vector(A.n_rows, 5, 2, "f64") * 8)
    t0 = time.time()
    ref_i = oracle.spmv_csr(A, x_i, 2.0, -1.0, y_i)
    rec["oracle_int_s"] = round(time.time() - t0, 1)
    dA = sp.CSR.from_host(A)
    f = sp.features(dA)
    rec["features"] = {k: f[k] for k in sp.PAPER_FEATURES}
    fmts = a.formats.split(",")
    for fmt in fmts:
        h = sp.convert(dA, fmt)
        xd = torch.from_numpy(x_i).cuda()
        yd = torch.from_numpy(y_i).cuda()
        h.run(2.0, xd, -1.0, yd)
        torch.cuda.synchronize()
        rec["formats"][fmt] = {"int_bit_exact": bool(np.array_equal(yd.cpu().numpy(), ref_i)),
                               "ptr_type": h.info()["ptr_type"]}
        h.destroy()
        del xd, yd
    # uniform values (same structure): tolerance check + timing
    del ref_i
    A = matgen.set_values(A, matgen.SEEDS["rmat27"] + 11, "f64")
    dA = sp.CSR.from_host(A)
    x = matgen.vector(A.n_cols, 1, 1)
    y = matgen.vector(A.n_rows, 1, 2)
    t0 = time.time()
    ref, bound = oracle.spmv_csr(A, x, 1.0, 1.0, y, with_bound=True)
    rec["oracle_s"] = round(time.time() - t0, 1)
    xd = torch.from_numpy(x).cuda()
    import bench
    peak, _ = bench.measured_peak()
    for fmt in fmts:
        h = sp.convert(dA, fmt)
        yd = torch.from_numpy(y).cuda()
        h.run(1.0, xd, 1.0, yd)
        torch.cuda.synchronize()
        ok, ratio, nbad = oracle.check_tolerance(yd.cpu().numpy(), ref, bound, 1e-12)
        t = harness.time_handle(h, xd, yd, reps=a.reps, warmup=5)
        by = h.info()["bytes_per_run"]
        rec["formats"][fmt].update(tol_ok=ok, max_ratio=ratio, n_bad=nbad, ms=t["t_mean_ms"],
                                   gflops=2 * A.nnz / (t["t_mean_ms"] * 1e-3) / 1e9,
                                   gbs=by / (t["t_mean_ms"] * 1e-3) / 1e9,
                                   frac_of_measured_peak=by / (t["t_mean_ms"] * 1e-3) / 1e9 / peak)
        h.destroy()
        del yd
    line = json.dumps(rec)
    print(line, flush=True)
    if a.out:
        with open(a.out, "w") as fh:
            fh.write(line + "\n")


if __name__ == "__main__":
    main()
