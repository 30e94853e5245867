"""A/B of A30 hot columns: each format's SpMV time with hot_x = -1 (off) and 0 (auto).
usage: python tools/exp_hot.py CONFIG [f64|f32] [formats]"""
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
    config = sys.argv[1]
    dname = sys.argv[2] if len(sys.argv) > 2 else "f64"
    dtype = torch.float64 if dname == "f64" else torch.float32
    dA, _ = bench.device_matrix(config, dname, dtype)
    fm = (sys.argv[3] if len(sys.argv) > 3 else bench.RMAT_FORMATS.get(config, "coo,ell,csr,hyb,merge,csr5")).split(",")
    x = gpu.vector(dA.n_cols, 1, 1, dname, dtype)
    y = gpu.vector(dA.n_rows, 1, 2, dname, dtype)
    peak, _ = bench.measured_peak()
    for f in fm:
        rec = {"config": config, "dtype": dname, "format": f}
        for label, hx in (("off", -1), ("auto", 0)):
            try:
                h = sp.convert(dA, f, hot_x=hx)
            except sp.SpmvError as e:
                rec[label] = e.name
                continue
            t = harness.time_handle(h, x, y, reps=20, per_call=False)["t_mean_ms"]
            info = h.info()
            rec[label] = {"ms": round(t, 4), "hot": info["hot_cols"],
                          "frac": round(info["bytes_per_run"] / t / 1e6 / peak, 3)}
            h.destroy()
            torch.cuda.empty_cache()
        print(json.dumps(rec), flush=True)


if __name__ == "__main__":
    main()
