"""Experiment (tools/hotset_probe.cu): x gathers of R-MAT with the K hottest columns served
from shared memory vs all through L1/L2.  usage: python tools/hotset_probe.py [scale]"""
import ctypes
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

from matgen import gpu  # noqa: E402

HERE = os.path.dirname(os.path.abspath(__file__))


def main():
    scale = int(sys.argv[1]) if len(sys.argv) > 1 else 24
    so = os.path.join(HERE, "hotset_probe.so")
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-Xcompiler", "-fPIC",
                           "-shared", os.path.join(HERE, "hotset_probe.cu"), "-o", so])
    L = ctypes.CDLL(so)
    L.hp_set_persist.argtypes = [ctypes.c_size_t]
    L.hp_run.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p,
                         ctypes.c_void_p, ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p]
    rp, col, val = gpu.rmat(scale, seed=0x5EED0003)
    n = rp.numel() - 1
    x = gpu.vector(n, 1, 1)
    out = torch.zeros(1, dtype=torch.float64, device="cuda")
    deg = torch.bincount(col.long(), minlength=n)
    order = torch.argsort(deg, descending=True)
    s = torch.cuda.current_stream()

    def t(fn, reps=30):
        for _ in range(5):
            fn()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        for _ in range(reps):
            fn()
        b.record(s)
        torch.cuda.synchronize()
        return a.elapsed_time(b) / reps
    res = {"scale": scale, "nnz": col.numel()}
    for blocks, threads in ((148 * 4, 256),):
        res[f"base_{blocks}x{threads}"] = t(lambda: L.hp_run(0, col.data_ptr(), val.data_ptr(), col.numel(), x.data_ptr(),
                                                              x.data_ptr(), 0, blocks, threads, out.data_ptr(), s.cuda_stream))
    Ks = [int(k) for k in sys.argv[2].split(",")] if len(sys.argv) > 2 else [4096, 12288, 16384, 32768, 65536, 131072, 262144]
    for K in Ks:
        hot = order[:K]
        cover = float(deg[hot].sum().item()) / col.numel()
        slot = torch.full((n,), -1, dtype=torch.int64, device="cuda")
        slot[hot] = torch.arange(K, device="cuda")
        sc = slot[col.long()]
        enc = torch.where(sc >= 0, -(sc + 1), col.long()).to(torch.int32)
        xhot = x[hot].contiguous()
        res[f"glob{K}_592x256"] = t(lambda: L.hp_run(2, enc.data_ptr(), val.data_ptr(), col.numel(), x.data_ptr(),
                                                       xhot.data_ptr(), K, 592, 256, out.data_ptr(), s.cuda_stream))
        L.hp_persist_max.restype = ctypes.c_longlong
        pmax = int(L.hp_persist_max())
        res["persisting_l2_max"] = pmax
        for frac in (0.5, 1.0):
            L.hp_set_persist(ctypes.c_size_t(int(pmax * frac)))
            res[f"persist{K}_{frac}"] = t(lambda: L.hp_run(3, enc.data_ptr(), val.data_ptr(), col.numel(), x.data_ptr(),
                                                             xhot.data_ptr(), K, 592, 256, out.data_ptr(), s.cuda_stream))
        L.hp_set_persist(ctypes.c_size_t(0))
        for blocks, threads in ((148, 1024),):
            if K * 8 * (blocks // 148) > 140 * 1024 or K > 32768:
                continue
            ms = t(lambda: L.hp_run(1, enc.data_ptr(), val.data_ptr(), col.numel(), x.data_ptr(), xhot.data_ptr(), K,
                                    blocks, threads, out.data_ptr(), s.cuda_stream))
            res[f"hot{K}_{blocks}x{threads}"] = ms
        res[f"cover{K}"] = cover
        del enc, sc, slot
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
