"""Achievable HBM bandwidth for read-dominant streams on this B200 (context for the
SpMV roofline; the graded denominator stays MEASURED_PEAKS.json hbm_gbs)."""
import json
import torch

torch.cuda.set_device(0)
n = 1 << 28                         # 2 GiB of fp64
a = torch.rand(n, dtype=torch.float64, device="cuda")
b = torch.rand(n, dtype=torch.float64, device="cuda")
ev = lambda: torch.cuda.Event(enable_timing=True)


def t(fn, reps=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    s, e = ev(), ev()
    s.record()
    for _ in range(reps):
        fn()
    e.record()
    torch.cuda.synchronize()
    return s.elapsed_time(e) / reps * 1e-3


out = {}
out["read_sum_gbs"] = 8 * n / t(lambda: a.sum()) / 1e9
out["copy_gbs"] = 16 * n / t(lambda: b.copy_(a)) / 1e9
out["axpy_gbs"] = 24 * n / t(lambda: b.add_(a, alpha=0.5)) / 1e9
print(json.dumps(out))
