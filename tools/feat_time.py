"""Warm timing of spmv_features (a2) on LAP4096 / R-MAT24: median wall time of the
blocking call (kernel + 112-byte readback + sync) and the algorithmic bytes
4(n+1)|8(n+1) + 4 nnz over it.  Usage: python tools/feat_time.py [lap4096] [rmat24] ..."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import matgen  # noqa: E402
import paper_conf_ipps_nisassvs18_b200 as sp  # noqa: E402


def build(name):
    if name.startswith("lap"):
        return matgen.laplacian5(int(name[3:]))
    if name.startswith("rmat"):
        return matgen.rmat(int(name[4:]))
    raise SystemExit(name)


def main():
    names = sys.argv[1:] or ["lap4096", "rmat24"]
    for name in names:
        A = build(name)
        dA = sp.CSR.from_host(A)
        f = sp.features(dA)                      # cold: ctx state, module load
        torch.cuda.synchronize()
        ts = []
        for _ in range(30):
            t0 = time.perf_counter()
            g = sp.features(dA)
            ts.append(time.perf_counter() - t0)
            assert g == f
        ts.sort()
        by = (A.n_rows + 1) * dA.row_ptr.element_size() + 4 * A.nnz
        med = ts[len(ts) // 2]
        print(json.dumps({"matrix": name, "n_rows": A.n_rows, "nnz": A.nnz, "ms_median": med * 1e3,
                          "ms_min": ts[0] * 1e3, "bytes": by, "gbs_median": by / med / 1e9,
                          "nnzb_tot": f["nnzb_tot"], "hyb_width_cusp": f["hyb_width_cusp"]}), flush=True)


if __name__ == "__main__":
    main()
