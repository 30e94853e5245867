"""Per-format timing and best-format labels (§IV-B):

    "The execution time is collected by executing each matrix multiple (50) times
     and then averaging the execution time.  We label the format with minimum
     execution time (maximum GFLOPS) as the best format."

Readings: A10 GFLOP/s = 2*nnz/t with the true nnz; A11 5 warm-ups,
one CUDA-event pair around 50 back-to-back runs -> mean (the label metric), per-call
events -> median/min, hot L2, alpha = beta = 1; A12 label6 / label5 (no COO,
PAPER.md:235) / label3 (ELL, CSR, HYB), exact ties to the paper's
Fig. 3 order, margin = t_2nd/t_best - 1; A4 infeasible formats are
"N/A" and excluded from the argmin.

Timing only: no oracle here.  All device work runs in libspmv kernels.
"""
from __future__ import annotations

import statistics
from typing import Dict, Iterable, List, Optional

import torch

from .spmv import CSR, PAPER_FORMATS, SpmvError, convert

LABEL_SETS = {
    "label6": ("coo", "ell", "csr", "hyb", "merge", "csr5"),
    "label5": ("ell", "csr", "hyb", "merge", "csr5"),
    "label3": ("ell", "csr", "hyb"),
    # the scalar CSR kernel ("a thread to process each
    # row") as a seventh class; emitted only when it was timed
    "label7": ("coo", "ell", "csr", "hyb", "merge", "csr5", "csr_scalar"),
}
LABEL_ORDER = PAPER_FORMATS + ("csr_scalar",)   # exact ties: Fig. 3 order, then the variant
# largest accepted |y_f - y_csr| / (max |y_csr| + 1) per dtype: 64 x the north_star bound's
# tolerance (the bound is per row and relative to sum |a||x|; this is a coarse screen)
AGREE_TOL = {torch.float64: 64 * 1e-12, torch.float32: 64 * 1e-5}


class L2Flush:
    """Cold-L2 timing (A11 variant): writing a buffer of twice the L2
    size between runs evicts A, x and y.  Measurement plumbing, not the hot path."""

    def __init__(self, device=None):
        props = torch.cuda.get_device_properties(device or torch.cuda.current_device())
        self.buf = torch.empty(2 * int(props.L2_cache_size), dtype=torch.uint8,
                               device=device or torch.cuda.current_device())
        self.n = 0

    def __call__(self):
        self.n += 1
        self.buf.fill_(self.n & 0xFF)


def time_handle(h, x: torch.Tensor, y: torch.Tensor, reps: int = 50, warmup: int = 5,
                alpha: float = 1.0, beta: float = 1.0, per_call: bool = True,
                flush: Optional[L2Flush] = None) -> Dict[str, float]:
    """A11 protocol on the current stream.  Returns mean (batch event pair), median and
    min of per-call events, in milliseconds.  With `flush` (cold L2): every run is
    preceded by an L2 flush outside its event pair; mean/median/min are over the
    per-call events."""
    s = torch.cuda.current_stream()
    for _ in range(warmup):
        h.run(alpha, x, beta, y)
    s.synchronize()
    if flush is not None:
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
        for a, b in evs:
            flush()
            a.record(s)
            h.run(alpha, x, beta, y)
            b.record(s)
        s.synchronize()
        ts = [a.elapsed_time(b) for a, b in evs]
        return {"t_mean_ms": sum(ts) / len(ts), "t_median_ms": statistics.median(ts), "t_min_ms": min(ts),
                "reps": reps, "cold_l2": True}
    t0, t1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0.record(s)
    for _ in range(reps):
        h.run(alpha, x, beta, y)
    t1.record(s)
    s.synchronize()
    out = {"t_mean_ms": t0.elapsed_time(t1) / reps, "reps": reps}
    if per_call:
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
        for a, b in evs:
            a.record(s)
            h.run(alpha, x, beta, y)
            b.record(s)
        s.synchronize()
        ts = [a.elapsed_time(b) for a, b in evs]
        out["t_median_ms"] = statistics.median(ts)
        out["t_min_ms"] = min(ts)
    return out


def labels(times_ms: Dict[str, Optional[float]]) -> Dict[str, object]:
    """A12: argmin over feasible formats per label set; exact ties in Fig. 3 order."""
    out: Dict[str, object] = {}
    for name, fmts in LABEL_SETS.items():
        if name == "label7" and "csr_scalar" not in times_ms:
            continue
        feas = [(times_ms[f], LABEL_ORDER.index(f), f) for f in fmts if times_ms.get(f) is not None]
        if not feas:
            out[name] = None
            continue
        feas.sort()
        out[name] = feas[0][2]
        if name == "label6":
            out["margin"] = (feas[1][0] / feas[0][0] - 1.0) if len(feas) > 1 and feas[0][0] > 0 else None
    return out


def measure_matrix(A: CSR, formats: Iterable[str] = PAPER_FORMATS, reps: int = 50, warmup: int = 5,
                   x: Optional[torch.Tensor] = None, y: Optional[torch.Tensor] = None,
                   cold_l2: bool = False, **convert_opts) -> Dict[str, object]:
    """Convert A to each format, time it, and emit the per-format record + labels
    (the paper's ground truth, regenerated on this GPU).  Before timing, every format's
    y = A x + y0 is compared with the CSR result (max |diff| / (max |y| + 1) recorded
    as "agree"); the oracle parity of each kernel is established by tests/, not here."""
    dev = A.row_ptr.device
    if x is None:
        x = torch.ones(A.n_cols, dtype=A.dtype, device=dev)
    if y is None:
        y = torch.zeros(A.n_rows, dtype=A.dtype, device=dev)
    rec: Dict[str, object] = {"formats": {}}
    times: Dict[str, Optional[float]] = {}
    cold: Dict[str, Optional[float]] = {}
    flush = L2Flush(dev) if cold_l2 else None
    ref_y = None
    for f in formats:
        try:
            h = convert(A, f, **convert_opts)
        except SpmvError as e:
            if e.status in (3, 4):          # SPMV_ERR_SIZE / NO_MEMORY -> N/A (A4)
                rec["formats"][f] = {"status": "N/A", "reason": e.name}
                times[f] = None
                cold[f] = None
                continue
            raise
        yc = y.clone()
        h.run(1.0, x, 1.0, yc)
        if ref_y is None:
            ref_y = yc
        agree = float((yc - ref_y).abs().max().item() / (ref_y.abs().max().item() + 1.0)) if A.n_rows else 0.0
        t = time_handle(h, x, y.clone(), reps=reps, warmup=warmup)   # timing accumulates into a scratch y
        info = h.info()
        gflops = 2.0 * A.nnz / (t["t_mean_ms"] * 1e-3) / 1e9 if t["t_mean_ms"] > 0 else 0.0
        gbs = info["bytes_per_run"] / (t["t_mean_ms"] * 1e-3) / 1e9 if t["t_mean_ms"] > 0 else 0.0
        rec["formats"][f] = {**t, "gflops": gflops, "gbs_own": gbs, "bytes_per_run": info["bytes_per_run"],
                             "launches": h.launches(), "agree": agree}
        times[f] = t["t_mean_ms"]
        if flush is not None:
            tc = time_handle(h, x, y.clone(), reps=reps, warmup=warmup, flush=flush)
            rec["formats"][f]["cold"] = tc
            cold[f] = tc["t_mean_ms"]
        h.destroy()
    rec.update(labels(times))
    if flush is not None:
        rec["cold_labels"] = labels(cold)
    # a record whose formats disagree beyond the tolerance is not a label
    tol = AGREE_TOL.get(A.dtype, 1e-5)
    bad = {f: r["agree"] for f, r in rec["formats"].items() if r.get("agree") is not None and r["agree"] > tol}
    if bad:
        rec["rejected"] = {"reason": f"formats disagree with CSR beyond {tol:g} (relative)", "agree": bad}
    return rec


def sweep(start: int = 0, count: int = 2000, out: str = "sweep.jsonl", dtype: str = "f64", reps: int = 50,
          warmup: int = 5, shard: int = 0, nshards: int = 1, max_nnz: Optional[int] = None,
          cold_l2: bool = False, with_scalar: bool = False) -> int:
    """BASELINE configs[3]: the format-selection sweep.  Matrices start..start+count-1
    (matgen.sweep_matrix, seeded), this process takes i % nshards == shard (replicas over
    GPUs).  One JSONL record per matrix: generator parameters, the 17 features + extras
    (spmv_features), per-format timings and labels.  Resumable: ids already in `out`
    are skipped.  Returns the number of matrices measured."""
    import json
    import os
    import time

    import matgen

    from .spmv import PAPER_FEATURES, features

    done = set()
    if os.path.exists(out):
        with open(out) as fh:
            for line in fh:
                try:
                    done.add(json.loads(line)["i"])
                except Exception:
                    pass
    tdt = torch.float64 if dtype == "f64" else torch.float32
    n = 0
    with open(out, "a") as fh:
        for i in range(start, start + count):
            if i % nshards != shard or i in done:
                continue
            t0 = time.time()
            A, p = matgen.sweep_matrix(i, dtype, max_nnz)
            dA = CSR.from_host(A, dtype=tdt)
            feats = features(dA)
            x = torch.from_numpy(matgen.vector(A.n_cols, p["seed"], 1, dtype)).to(dA.row_ptr.device).to(tdt)
            y = torch.from_numpy(matgen.vector(A.n_rows, p["seed"], 2, dtype)).to(dA.row_ptr.device).to(tdt)
            fmts = PAPER_FORMATS + (("csr_scalar",) if with_scalar else ())
            rec = measure_matrix(dA, formats=fmts, reps=reps, warmup=warmup, x=x, y=y, cold_l2=cold_l2)
            row = {"i": i, "params": p, "dtype": dtype, "n_rows": A.n_rows, "n_cols": A.n_cols, "nnz": A.nnz,
                   "features": {k: feats[k] for k in PAPER_FEATURES},
                   "extras": {k: feats[k] for k in ("ell_width", "ell_slots", "ell_pad_frac", "hyb_width",
                                                      "hyb_coo_nnz", "hyb_width_floor", "hyb_width_cusp",
                                                      "n_empty_rows")},
                   "gpu": torch.cuda.get_device_name(), "wall_s": None, **rec}
            row["wall_s"] = round(time.time() - t0, 3)
            if "rejected" in row:                  # kept aside, never a label
                with open(out.replace(".jsonl", ".rejected.jsonl"), "a") as rj:
                    rj.write(json.dumps(row) + "\n")
                continue
            fh.write(json.dumps(row) + "\n")
            fh.flush()
            n += 1
            del dA
    return n


def _main():
    import argparse
    ap = argparse.ArgumentParser(description="format-selection sweep (BASELINE configs[3])")
    ap.add_argument("--start", type=int, default=0)
    ap.add_argument("--count", type=int, default=2000)
    ap.add_argument("--out", default="sweep.jsonl")
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32"])
    ap.add_argument("--reps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--max-nnz", type=int, default=None)
    ap.add_argument("--cold-l2", action="store_true", help="also time every format with L2 flushed before each run")
    ap.add_argument("--with-scalar", action="store_true", help="time CSR-scalar too and emit label7")
    ap.add_argument("--stride", type=int, default=1, help="only matrices i with i %% stride == 0 (subsets)")
    a = ap.parse_args()
    import os
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    torch.cuda.set_device(int(os.environ.get("LOCAL_RANK", "0")))
    out = a.out if ws == 1 else a.out.replace(".jsonl", f".rank{rank}.jsonl")
    if a.stride > 1:                                # i % stride == 0, replicas over i // stride
        n = 0
        for i in range(a.start, a.start + a.count):
            if i % a.stride == 0 and (i // a.stride) % ws == rank:
                n += sweep(i, 1, out, a.dtype, a.reps, a.warmup, 0, 1, a.max_nnz, a.cold_l2, a.with_scalar)
    else:
        n = sweep(a.start, a.count, out, a.dtype, a.reps, a.warmup, rank, ws, a.max_nnz, a.cold_l2, a.with_scalar)
    print(f"rank {rank}: measured {n} matrices -> {out}")


if __name__ == "__main__":
    _main()
