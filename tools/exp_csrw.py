"""CSR group-width / chunk-length sweep on one config: warm time of the CSR handle for
vector_width W in the list (0 = A5 rule) and csr_chunk C, checked against W = A5.
usage: python tools/exp_csrw.py CONFIG [f64|f32] W,W,... [C,C,...]"""
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
    config, dname = sys.argv[1], sys.argv[2]
    ws = [int(w) for w in sys.argv[3].split(",")]
    cs = [int(c) for c in sys.argv[4].split(",")] if len(sys.argv) > 4 else [0]
    dtype = torch.float64 if dname == "f64" else torch.float32
    dA, _ = bench.device_matrix(config, dname, dtype)
    x = gpu.vector(dA.n_cols, 1, 1, dname, dtype)
    y0 = gpu.vector(dA.n_rows, 1, 2, dname, dtype)
    ref = None
    for c in cs:
        for w in ws:
            h = sp.convert(dA, "csr", vector_width=w, csr_chunk=c)
            y = y0.clone()
            h.run(1.0, x, 1.0, y)
            torch.cuda.synchronize()
            if ref is None:
                ref = y.clone()
            rel = float(((y.double() - ref.double()).abs().max() / ref.double().abs().max()).item())
            t = harness.time_handle(h, x, y0.clone(), reps=30, warmup=3)
            print(json.dumps({"config": config, "dtype": dname, "W": w, "C": c, "ms": round(t["t_mean_ms"], 4),
                              "rel_diff": rel, "env": {k: v for k, v in os.environ.items() if k.startswith("SPMV_")}}),
                  flush=True)
            h.destroy()


if __name__ == "__main__":
    main()
