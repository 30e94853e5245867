"""CSR kernel choices on one matrix: vector_width (A5 rule vs forced) x long-row chunk
length (A25).  usage: python tools/exp_csr.py CONFIG [f64|f32]"""
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
    x = gpu.vector(dA.n_cols, 1, 1, dname, dtype)
    y = gpu.vector(dA.n_rows, 1, 2, dname, dtype)
    ref = None
    for vw in (0, 2, 4, 8, 16, 32):
        for ch in (0, 256, 1024, 4096):
            h = sp.convert(dA, "csr", vector_width=vw, csr_chunk=ch)
            yy = y.clone()
            h.run(1.0, x, 1.0, yy)
            if ref is None:
                ref = yy
            ok = float((yy - ref).abs().max() / (ref.abs().max() + 1))
            t = harness.time_handle(h, x, y.clone(), reps=20, per_call=False)["t_mean_ms"]
            print(json.dumps({"config": config, "vw": vw, "chunk": ch, "W": h.info()["vector_width"],
                              "chunks": h.info()["csr_chunks"], "ms": round(t, 4), "agree": ok}), flush=True)
            h.destroy()


if __name__ == "__main__":
    main()
