"""One spmv_run per format (after warm-up) inside NVTX ranges "spmv_run:<fmt>" (libspmv's own),
for ncu captures whose kernels are attributed to formats by their NVTX range.
usage: python tools/prof_formats.py CONFIG [f64|f32] [formats]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_ipps_nisassvs18_b200 as sp  # noqa: E402
from matgen import gpu  # noqa: E402


def main():
    config = sys.argv[1]
    dname = sys.argv[2] if len(sys.argv) > 2 else "f64"
    dtype = torch.float64 if dname == "f64" else torch.float32
    dA, _ = bench.device_matrix(config, dname, dtype)
    fm = sys.argv[3].split(",") if len(sys.argv) > 3 else bench.RMAT_FORMATS.get(config, ",".join(sp.PAPER_FORMATS)).split(",")
    feats = sp.features(dA)
    handles, _, na = bench.convert_all(sp, dA, fm, feats)
    x = gpu.vector(dA.n_cols, 1, 1, dname, dtype)
    y = gpu.vector(dA.n_rows, 1, 2, dname, dtype)
    for _ in range(3):
        for h in handles.values():
            h.run(1.0, x, 1.0, y)
    torch.cuda.synchronize()
    torch.cuda.cudart().cudaProfilerStart()
    for f, h in handles.items():
        h.run(1.0, x, 1.0, y)
    torch.cuda.synchronize()
    sp.features(dA)
    torch.cuda.synchronize()
    torch.cuda.cudart().cudaProfilerStop()
    print("profiled", list(handles), "N/A", list(na))


if __name__ == "__main__":
    main()
