"""Column-stream ceiling of a matrix on this B200 (measurement tool, not the product).

Times tools/gather_probe.cu over the matrix's own col/val arrays -- stream only, and
stream + x[col] gather with three load flavours -- beside the six formats' SpMV, so
"format / probe" shows how much of a format's time the gathers alone impose.

usage: python tools/gather_probe.py [CONFIG ...] [--reps 50] [--out FILE]
"""
import argparse
import ctypes
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import bench  # noqa: E402
import matgen  # noqa: E402
import paper_conf_ipps_nisassvs18_b200 as sp  # noqa: E402
from paper_conf_ipps_nisassvs18_b200 import harness  # noqa: E402

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "gather_probe.cu")
SO = os.path.join(HERE, "gather_probe.so")
MODES = {0: "stream col+val", 1: "+ gather (L1 alloc, L2 evict_last)", 2: "+ gather (L1 no_allocate)",
         3: "+ gather (ld.global)"}


def build():
    if not os.path.exists(SO) or os.path.getmtime(SO) < os.path.getmtime(SRC):
        subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo",
                               "-Xcompiler", "-fPIC", "-shared", SRC, "-o", SO])
    lib = ctypes.CDLL(SO)
    lib.probe_run.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p,
                              ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p]
    return lib


def time_fn(fn, reps, warmup=5):
    s = torch.cuda.current_stream()
    for _ in range(warmup):
        fn()
    s.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(reps):
        fn()
    b.record(s)
    s.synchronize()
    return a.elapsed_time(b) / reps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("configs", nargs="*", default=["lap4096", "rmat24"])
    ap.add_argument("--reps", type=int, default=50)
    ap.add_argument("--out", default="")
    ap.add_argument("--formats", default="")
    ap.add_argument("--modes", default="0,1,2,3")
    a = ap.parse_args()
    lib = build()
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    peak, _ = bench.measured_peak()
    recs = []
    for cfg in a.configs:
        dA, _ = bench.device_matrix(cfg, "f64", torch.float64)     # R-MAT: the GPU generator
        A = dA
        from matgen import gpu
        x = gpu.vector(A.n_cols, 1, 1)
        y = gpu.vector(A.n_rows, 1, 2)
        out = torch.zeros(1, dtype=torch.float64, device="cuda")
        st = torch.cuda.current_stream().cuda_stream
        for m, what in MODES.items():
            if str(m) not in a.modes.split(","):
                continue
            ms = time_fn(lambda: lib.probe_run(m, dA.col.data_ptr(), dA.val.data_ptr(), A.nnz, x.data_ptr(),
                                               out.data_ptr(), sms, st), a.reps)
            byt = 12 * A.nnz
            r = {"config": cfg, "kind": "probe", "mode": m, "what": what, "ms": round(ms, 4),
                 "stream_gbs": round(byt / ms / 1e6, 1), "gathers_per_ns": round(A.nnz / ms / 1e6, 2)}
            recs.append(r)
            print(json.dumps(r), flush=True)
        for fmt in (a.formats.split(",") if a.formats else sp.PAPER_FORMATS):
            if fmt not in sp.FORMATS:
                continue
            try:
                h = sp.convert(dA, fmt)
            except sp.SpmvError:
                continue
            t = harness.time_handle(h, x, y, reps=a.reps, per_call=False)["t_mean_ms"]
            r = {"config": cfg, "kind": "format", "format": fmt, "ms": round(t, 4),
                 "frac_of_peak": round(h.info()["bytes_per_run"] / t / 1e6 / peak, 3)}
            recs.append(r)
            print(json.dumps(r), flush=True)
            h.destroy()
        del dA
        torch.cuda.empty_cache()
    if a.out:
        with open(a.out, "w") as f:
            for r in recs:
                f.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
