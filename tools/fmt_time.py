"""Warm time of chosen formats on one config (harness.time_handle, mean of reps) with the
roofline fraction against the measured peak, under the current environment (kernel
switches such as SPMV_COO_PIPE are read by libspmv).  Checks every format against the
first one run.  usage: python tools/fmt_time.py CONFIG [f64|f32] [fmt,fmt,...] [--tag T]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ipps_nisassvs18_b200 as sp  # noqa: E402
from matgen import gpu  # noqa: E402
from paper_conf_ipps_nisassvs18_b200 import harness  # noqa: E402


def main():
    args = [a for a in sys.argv[1:] if not a.startswith("--")]
    tag = sys.argv[sys.argv.index("--tag") + 1] if "--tag" in sys.argv else ""
    if tag in args:
        args.remove(tag)
    config = args[0]
    dname = args[1] if len(args) > 1 else "f64"
    fmts = (args[2] if len(args) > 2 else "coo,ell,csr,hyb,merge,csr5").split(",")
    dtype = torch.float64 if dname == "f64" else torch.float32
    dA, _ = bench.device_matrix(config, dname, dtype)
    x = gpu.vector(dA.n_cols, 1, 1, dname, dtype)
    y = gpu.vector(dA.n_rows, 1, 2, dname, dtype)
    peak, _ = bench.measured_peak()
    ref = None
    for f in fmts:
        try:
            h = sp.convert(dA, f)
        except Exception as e:  # noqa: BLE001 (ELL infeasible)
            print(json.dumps({"config": config, "fmt": f, "skipped": str(e)[:80]}))
            continue
        yy = y.clone()
        h.run(1.0, x, 1.0, yy)
        torch.cuda.synchronize()
        if ref is None:
            ref = yy
        err = float(((yy.double() - ref.double()).abs().max() / ref.double().abs().max().clamp_min(1e-300)).item())
        t = harness.time_handle(h, x, y.clone(), reps=50, warmup=10)
        by = h.info()["bytes_per_run"]
        ms = t["t_mean_ms"]
        print(json.dumps({"config": config, "dtype": dname, "fmt": f, "tag": tag, "ms": round(ms, 4),
                          "frac": round(by / (ms * 1e-3) / 1e9 / peak, 4), "rel_diff_vs_first": err}), flush=True)
        h.destroy()


if __name__ == "__main__":
    main()
