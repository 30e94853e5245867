#!/usr/bin/env python
"""bench.py -- SpMV GFLOP/s & HBM GB/s (% of roofline) per format on B200.

One "step" = one pass of the label-collection hot path over the workload matrix:
y_f <- alpha*A_f*x + beta*y_f for every feasible format f of the six (COO, ELL, CSR,
HYB, merge-path CSR, CSR5), alpha = beta = 1 (A11).
Conversions and the feature pass are one-off setup: they are timed and reported
separately, not inside the step.

  value  = sum over formats of 2*nnz / (time of the K timed steps / K)   [GFLOP/s]
  e2e    = the same through the public API with host x in / host y out every step
           (spmv_run_host_multi: x and y_in cross PCIe once, every format's y comes back)

Workload (``--config``): BASELINE configs[1] (lap4096: 5-point Laplacian, 4096^2 grid,
fp64) by default at every N.  At N = 1 the line also carries configs[2] (R-MAT 24,
fp64 and fp32) per-format blocks with their own roofline.  ``--gpus N > 1`` launches N
ranks itself (torch.distributed.run, one per GPU, 127.0.0.1) unless WORLD_SIZE is set:
rows are split at nnz-balanced merge-path diagonals and every format's step packs its x
slice, exchanges it over NCCL and runs its shard -- a point-to-point halo for the
banded Laplacian, the (compressed) all-gather overlapped with the own-column block for
R-MAT (``--config rmat24|rmat27``, built rank-locally by the GPU generator).  All
arrays exceed the 126 MB L2, so no flush is needed between steps.

--impl reference runs the CPU oracle (oracle/, plain C, long double) on rank 0 over
a bounded row sample of the same workload: the baseline arm, not a target.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "SpMV GFLOP/s & HBM GB/s (% of roofline) per format, 1/2/4/8 B200"

CONFIGS = {
    "u2048": dict(desc="BASELINE configs[0]: 2048x2048 uniform random, 16 nnz/row, fp64"),
    "lap4096": dict(desc="BASELINE configs[1]: 2D 5-point Laplacian, 4096x4096 grid (16.8M rows, 83.9M nnz), fp64"),
    "rmat24": dict(desc="BASELINE configs[2]: R-MAT scale 24, edge factor 16, Graph500 (a,b,c)=(.57,.19,.19)"),
    "rmat27": dict(desc="BASELINE configs[4]: R-MAT scale 27, edge factor 16, Graph500 (a,b,c)=(.57,.19,.19), "
                        "int64 row_ptr"),
    "rgg19": dict(desc="synthetic stand-in for rgg_n_2_19_s0 (the matrix PAPER.md:131 quotes): random geometric "
                       "graph, 2^19 points in the unit square, r = 0.55 sqrt(ln n / n), grid-cell numbering "
                       "(matgen.rgg; 524,288 rows, 6.55M nnz vs the file's 6.54M)"),
}
RMAT_FORMATS = {"rmat24": "coo,csr,hyb,merge,csr5", "rmat27": "csr,merge,csr5"}

# R1: the paper's own numbers on its own hardware -- context, not targets
PAPER_CONTEXT = {
    "note": "the paper's published numbers on Kepler/Pascal (context only; BASELINE.json published = {})",
    "hardware": "Tesla K80c (one GK210 die: 13 SMs, 824 MHz, 1.5 MB L2; PAPER.md:199-205, 219) and Tesla P100 "
                "(56 SMs, 1328 MHz, 4 MB L2)",
    "spmv_gflops": [
        {"format": "csr5", "matrix": "rgg_n_2_19_s0", "gflops": 22, "source": "PAPER.md:131"},
        {"format": "csr5", "matrix": "auto", "gflops": 18, "source": "PAPER.md:131"},
        {"format": "merge", "matrix": "rgg_n_2_19_s0", "gflops": 21, "source": "PAPER.md:131"},
        {"format": "merge", "matrix": "auto", "gflops": 15, "source": "PAPER.md:131"},
    ],
    "spmv_precision": "not stated for these values; the surrounding Fig. 3 is single precision on the K80c "
                      "(PAPER.md:139-157)",
    "selection_accuracy": "~88% for six formats (84-88% across K80c/P100 and fp32/fp64), up to 91% for ELL/CSR/HYB "
                          "(XGBoost; PAPER.md:49, 73-75, 257-267)",
    "time_prediction_rme": "~10% (K80c) and 12% (P100) with an MLP ensemble, 7% for CSR5 and merge "
                           "(PAPER.md:49, 295-301)",
    "suitesparse_matrices": "the paper's rgg_n_2_19_s0 / auto are not in this offline image (no network); "
                            "matgen.mtx reads them when staged (bench --config mtx:PATH)",
}


def build_matrix(name, dtype_kind):
    import matgen
    if name == "u2048":
        return matgen.uniform_fixed(2048, 2048, 16, kind=dtype_kind)
    if name == "lap4096":
        return matgen.laplacian5(4096)
    if name.startswith("lap"):
        return matgen.laplacian5(int(name[3:]))
    if name.startswith("rmat"):
        return matgen.rmat(int(name[4:]), seed=matgen.SEEDS.get(name, matgen.SEEDS["rmat24"]), kind=dtype_kind)
    if name.startswith("rgg"):
        return matgen.rgg(int(name[3:]), seed=matgen.SEEDS.get(name, matgen.SEEDS["rgg19"]), kind=dtype_kind)
    if name.startswith("mtx:"):                     # a Matrix Market file
        from matgen.mtx import read_mtx
        A = read_mtx(name[4:])
        if dtype_kind == "f32":
            A.val = A.val.astype("float32").astype("float64")
        return A
    raise SystemExit(f"unknown config {name}")


def measured_peak():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """SM clocks and clock-event (throttle) reasons sampled DURING the timed region: through
    NVML every ~2 ms (a timed region of a few tens of ms gets a dozen samples), else
    nvidia-smi every 200 ms."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, index=0):
        self.index = index
        self.samples = []                  # [sm_mhz, max_mhz, reasons...] (nvidia-smi) or dicts (NVML)
        self.proc = None
        self.nvml = None
        self.stop = threading.Event()
        self.source = None

    def __enter__(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            h = None
            try:                               # the CUDA device's own GPU (CUDA_VISIBLE_DEVICES may remap)
                import torch
                u = str(torch.cuda.get_device_properties(self.index).uuid)
                h = pynvml.nvmlDeviceGetHandleByUUID(u if u.startswith("GPU-") else "GPU-" + u)
            except Exception:
                h = None
            if h is None:
                h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
            mx = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
            bits = [pynvml.nvmlClocksEventReasonHwSlowdown, pynvml.nvmlClocksEventReasonHwThermalSlowdown,
                    pynvml.nvmlClocksEventReasonSwThermalSlowdown, pynvml.nvmlClocksEventReasonSwPowerCap]

            def loop():
                while not self.stop.is_set():
                    try:
                        sm = pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM)
                        rs = pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
                        self.samples.append({"sm": float(sm), "max": float(mx),
                                             "reasons": [n for n, b in zip(self.NAMES, bits) if rs & b]})
                    except Exception:
                        pass
                    self.stop.wait(0.002)

            self.nvml = pynvml
            self.source = "NVML, ~2 ms"
            self.thread = threading.Thread(target=loop, daemon=True)
            self.thread.start()
            return self
        except Exception:
            self.nvml = None
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "200"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.source = "nvidia-smi, 200 ms"
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 7:
                self.samples.append(parts)

    def __exit__(self, *a):
        if self.nvml is not None:
            self.stop.set()
            self.thread.join(timeout=2)
            try:
                self.nvml.nvmlShutdown()
            except Exception:
                pass
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        import statistics
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no clock samples"], "samples": 0}
        if isinstance(self.samples[0], dict):
            sm = [s["sm"] for s in self.samples]
            mx = [s["max"] for s in self.samples]
            reasons = sorted({r for s in self.samples for r in s["reasons"]})
        else:
            sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
            mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
            reasons = sorted({self.NAMES[i] for s in self.samples for i in range(4) if s[3 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "sm_min_mhz": min(sm) if sm else None, "reasons": reasons, "samples": len(self.samples),
                "source": self.source}


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def self_launch(args) -> int:
    """--gpus N > 1 without a launcher: run N ranks under torch.distributed.run (one process
    per GPU of this node, rendezvous on 127.0.0.1) and return their exit status."""
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    return subprocess.call(cmd)


# ---------------------------------------------------------------------- CPU baselines

def host_cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


class OracleRows:
    """The oracle (oracle.spmv_csr, unchanged) over a contiguous row sample [0, m) of about
    `target_nnz` nonzeros, the rows split into `threads` nnz-balanced blocks that host
    threads run at once (the ctypes call releases the GIL; each row is computed exactly as
    in one call over all rows).  One protocol for both the reference arm and cpu_baseline."""

    def __init__(self, A, x, y, target_nnz, threads):
        import numpy as np

        import oracle
        m = int(np.searchsorted(A.row_ptr, min(target_nnz, A.nnz), side="left"))
        self.m = max(1, min(m, A.n_rows))
        self.nnz = int(A.row_ptr[self.m])
        self.threads = max(1, int(threads))
        cuts = np.searchsorted(A.row_ptr[:self.m + 1], np.linspace(0, self.nnz, self.threads + 1), side="left")
        cuts[0], cuts[-1] = 0, self.m
        self.y = y[: self.m].copy()
        self.blocks = []
        for a, b in zip(cuts[:-1], cuts[1:]):
            if b > a:
                self.blocks.append((oracle.CSR(A.row_ptr[a:b + 1], A.col, A.val, (b - a, A.n_cols)), a, b))
        self.x = x
        self.pool = None
        if len(self.blocks) > 1:
            from concurrent.futures import ThreadPoolExecutor
            self.pool = ThreadPoolExecutor(max_workers=len(self.blocks))

    def _one(self, blk, y_out):
        import oracle
        B, a, b = blk
        y_out[a:b] = oracle.spmv_csr(B, self.x, 1.0, 1.0, self.y[a:b])

    def run(self, y_out=None):
        import numpy as np
        y_out = np.empty(self.m) if y_out is None else y_out
        if self.pool is None:
            for blk in self.blocks:
                self._one(blk, y_out)
        else:
            list(self.pool.map(lambda blk: self._one(blk, y_out), self.blocks))
        return y_out

    def close(self):
        if self.pool is not None:
            self.pool.shutdown()


ORACLE_SAMPLE_NNZ = 40_000_000


def oracle_sample_time(A, x, y, threads, budget_s, min_reps=1):
    """Repeat the oracle over the row sample for ~budget_s: (GFLOP/s, reps, seconds, OracleRows, y)."""
    R = OracleRows(A, x, y, ORACLE_SAMPLE_NNZ, threads)
    out = R.run()                                   # untimed warm-up (page-in)
    reps, t0 = 0, time.perf_counter()
    while True:
        R.run(out)
        reps += 1
        if reps >= min_reps and time.perf_counter() - t0 > budget_s:
            break
    dt = time.perf_counter() - t0
    return 2.0 * R.nnz * reps / dt / 1e9, reps, dt, R, out


def cpu_baseline(A, x, y, budget_s=10.0):
    """SURVEY §8(d) d5 on this host (rank 0, N = 1 only), bounded row sample:
    (i) the oracle single-threaded, (ii) the same per-row code on all host cores (verified
    bit-identical to (i)), (iii) a realistic fp64 CSR loop (OpenMP, all cores; not the oracle)."""
    import numpy as np

    import cpubase
    cores = host_cores()
    v_mt, reps_mt, dt_mt, Rmt, y_mt = oracle_sample_time(A, x, y, cores, budget_s / 2)
    v_1t, reps_1t, dt_1t, R1, y_1t = oracle_sample_time(A, x, y, 1, budget_s / 2)
    same = bool(np.array_equal(y_mt, y_1t))
    sample = (f"rows [0,{Rmt.m}) = {Rmt.nnz} of {A.nnz} nonzeros; oracle CSR SpMV (long double, as written), "
              f"{len(Rmt.blocks)} host threads over nnz-balanced row blocks, {reps_mt} reps in {dt_mt:.1f} s")
    m, nnz = Rmt.m, Rmt.nnz
    Rmt.close()
    R1.close()
    # (iii) fp64 all-core loop over the same rows
    yc = y[:m].astype(np.float64).copy()
    cpubase.spmv_f64(m, A.row_ptr[: m + 1], A.col, A.val, x, 1.0, 1.0, yc)
    reps, t0 = 0, time.perf_counter()
    while time.perf_counter() - t0 < min(2.0, budget_s / 4) or reps < 3:
        cpubase.spmv_f64(m, A.row_ptr[: m + 1], A.col, A.val, x, 1.0, 1.0, yc)
        reps += 1
    dt = time.perf_counter() - t0
    return {"value": v_mt, "unit": "GFLOP/s", "cores": len(Rmt.blocks), "kind": "oracle", "sample": sample,
            "cpu_model": cpu_model(), "host_cores": cores,
            "single_thread": {"value": v_1t, "cores": 1, "reps": reps_1t, "seconds": dt_1t},
            "multi_thread_equals_single_thread": same,
            "fp64_allcore": {"value": 2.0 * nnz * reps / dt / 1e9, "unit": "GFLOP/s", "cores": cpubase.threads(),
                             "kind": "fp64 CSR loop, OpenMP over rows (SURVEY d5 iii; not the oracle)",
                             "reps": reps, "seconds": dt}}


def run_reference(args):
    """The CPU oracle on this host (rank 0 only), the same bounded row sample per format
    per step as cpu_baseline (one protocol)."""
    import matgen
    ws, rank, _ = dist_env()
    if rank != 0:
        return
    config = args.config or "lap4096"
    kind = "f64" if args.dtype == "f64" else "f32"
    A = build_matrix(config, kind)
    seed = matgen.SEEDS.get(config, 1)
    x = matgen.vector(A.n_cols, seed, 1, kind)
    y = matgen.vector(A.n_rows, seed, 2, kind)
    fmts = [f for f in (args.formats or RMAT_FORMATS.get(config, "coo,ell,csr,hyb,merge,csr5")).split(",") if f]
    nformats = len(fmts)
    cores = host_cores()
    R = OracleRows(A, x, y, ORACLE_SAMPLE_NNZ, cores)
    out = R.run()

    def step():
        for _ in range(nformats):
            R.run(out)

    for _ in range(args.warmup):
        step()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        step()
    dt = time.perf_counter() - t0
    R.close()
    val = 2.0 * R.nnz * nformats * args.steps / dt / 1e9
    sample = (f"{nformats} oracle CSR SpMVs (long double, {len(R.blocks)} host threads over nnz-balanced row "
              f"blocks) per step over rows [0,{R.m}) = {R.nnz} of {A.nnz} nonzeros of {config} (the cpu_baseline "
              f"sample)")
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "GFLOP/s", "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
            "dtype": args.dtype, "data": "synthetic",
            "config": {"workload": config, "desc": CONFIGS.get(config, {}).get("desc", config)},
            "cpu_baseline": {"value": val, "unit": "GFLOP/s", "cores": len(R.blocks), "kind": "oracle",
                             "sample": sample, "cpu_model": cpu_model()},
            "e2e": {"value": val, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------- our arm: helpers

def ev():
    import torch
    return torch.cuda.Event(enable_timing=True)


def traffic_for(config, fmt, dtype):
    """DRAM bytes per run of this format's kernels (all launches of one spmv_run summed) from
    the committed ncu --set full capture (profiles/ncu_traffic.json), or None."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get(config, {}).get(dtype, {}).get(fmt)
    except Exception:
        return None


def device_matrix(config, kind, dtype):
    """(CSR on the GPU, host accessor) -- R-MAT by the GPU generator (bit-identical to the
    host one), the rest by the host generator."""
    import matgen
    import paper_conf_ipps_nisassvs18_b200 as sp
    if config.startswith("rmat"):
        from matgen import gpu
        seed = matgen.SEEDS.get(config, matgen.SEEDS["rmat24"])
        import torch
        rp, col, val = gpu.rmat(int(config[4:]), seed=seed, kind=kind, dtype=dtype)
        n = rp.numel() - 1
        if config != "rmat27" and col.numel() <= 2 ** 31 - 1:     # configs[4] keeps int64 row_ptr (A17)
            rp = rp.to(torch.int32)
        return sp.CSR(rp, col, val, (n, n)), None
    A = build_matrix(config, kind)
    return sp.CSR.from_host(A, dtype=dtype), A


def host_sample(dA, A_host, target_nnz):
    """A HostCSR with the first rows of the device matrix (about target_nnz nonzeros; the
    oracle's sample) -- the whole host matrix when it already exists."""
    import numpy as np

    import matgen
    if A_host is not None:
        return A_host
    rp = dA.row_ptr.cpu().numpy().astype(np.int64)
    m = int(np.searchsorted(rp, min(target_nnz, dA.nnz), side="left"))
    m = max(1, min(m, dA.n_rows))
    k = int(rp[m])
    rpm = np.concatenate([rp[: m + 1], np.full(dA.n_rows - m, k, np.int64)])
    return matgen.HostCSR(rpm, dA.col[:k].cpu().numpy(), dA.val[:k].cpu().double().numpy(), dA.n_rows, dA.n_cols)


def time_formats(handles, x, y_init, steps, warmup, local, stream, extra_variants=True, flush=None):
    """Per-format CUDA-event timing of `steps` back-to-back steps (one run of every format
    each), with the clocks sampled during the timed region; then the A11 variants
    (beta = 0, and L2 flushed before every run).  Returns (ms per step, per-format times,
    clocks, variants)."""
    import torch
    fmts = list(handles)
    ys = {f: y_init.clone() for f in fmts}

    def step(record=None):
        for f in fmts:
            if record is not None:
                record[f][0].record(stream)
            handles[f].run(1.0, x, 1.0, ys[f])
            if record is not None:
                record[f][1].record(stream)

    for _ in range(warmup):
        step()
    torch.cuda.synchronize()
    evs = {f: [(ev(), ev()) for _ in range(steps)] for f in fmts}
    t0, t1 = ev(), ev()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        t0.record(stream)
        for k in range(steps):
            step({f: evs[f][k] for f in fmts})
        t1.record(stream)
        torch.cuda.synchronize()
    ms_step = t0.elapsed_time(t1) / steps
    per = {f: sorted(a.elapsed_time(b) for a, b in evs[f]) for f in fmts}
    variants = {}
    if extra_variants:
        reps = max(5, min(20, steps))
        for f in fmts:
            yb = torch.empty_like(y_init)
            a, b = ev(), ev()
            handles[f].run(1.0, x, 0.0, yb)
            a.record(stream)
            for _ in range(reps):
                handles[f].run(1.0, x, 0.0, yb)
            b.record(stream)
            torch.cuda.synchronize()
            cold = []
            if flush is not None:
                for _ in range(reps):
                    flush.add_(1)                    # writes 2x L2: nothing of A/x/y survives
                    c0, c1 = ev(), ev()
                    c0.record(stream)
                    handles[f].run(1.0, x, 1.0, ys[f])
                    c1.record(stream)
                    cold.append((c0, c1))
                torch.cuda.synchronize()
            variants[f] = {"ms_beta0": a.elapsed_time(b) / reps,
                           "ms_cold_l2": (sum(c0.elapsed_time(c1) for c0, c1 in cold) / len(cold)) if cold else None}
    return ms_step, per, clk.summary(), variants


def format_block(handles, per, variants, nnz, peak, config, dtype_name, conv_ms):
    """Per-format numbers: mean/median/min ms, GFLOP/s, GB/s of the format's own bytes and
    their fraction of the measured peak and of the 8 TB/s nominal, gbs_csr."""
    infos = {f: handles[f].info() for f in handles}
    csr_by = infos["csr"]["bytes_per_run"] if "csr" in infos else None
    out = {}
    for f in handles:
        ts = per[f]
        mean = sum(ts) / len(ts)
        by = infos[f]["bytes_per_run"]
        tr = traffic_for(config, f, dtype_name)
        out[f] = {"ms_mean": mean, "ms_median": ts[len(ts) // 2], "ms_min": ts[0],
                  "gflops": 2.0 * nnz / (mean * 1e-3) / 1e9,
                  "gbs": by / (mean * 1e-3) / 1e9, "frac_of_peak": by / (mean * 1e-3) / 1e9 / peak,
                  "frac_of_nominal_8tbs": by / (mean * 1e-3) / 1e9 / 8000.0,
                  "gbs_csr": (csr_by / (mean * 1e-3) / 1e9) if csr_by else None,
                  "bytes_per_run": by, "launches": handles[f].launches(), "convert_ms": conv_ms.get(f),
                  "dram_bytes_ncu": tr, "traffic_over_algorithmic": (tr / by) if tr else None}
        if f in variants:
            v = variants[f]
            out[f]["ms_beta0"] = v["ms_beta0"]
            out[f]["gflops_beta0"] = 2.0 * nnz / (v["ms_beta0"] * 1e-3) / 1e9
            out[f]["gbs_beta0"] = infos[f]["bytes_per_run_beta0"] / (v["ms_beta0"] * 1e-3) / 1e9
            if v["ms_cold_l2"]:
                out[f]["ms_cold_l2"] = v["ms_cold_l2"]
                out[f]["gflops_cold_l2"] = 2.0 * nnz / (v["ms_cold_l2"] * 1e-3) / 1e9
    return out


def roofline(pf, f, peak, peak_src):
    p = pf[f]
    return {"bound": "hbm", "achieved": p["gbs"], "peak": peak, "unit": "GB/s", "frac": p["gbs"] / peak,
            "traffic": p.get("dram_bytes_ncu"), "kernel_format": f, "bytes_per_launch": p["bytes_per_run"],
            "avg_launch_ms": p["ms_mean"], "launches_bracketed": p["launches"], "peak_source": peak_src,
            "traffic_source": "profiles/ncu_traffic.json: DRAM bytes of every kernel of one spmv_run of this format "
                              "on this config, from the committed ncu --set full capture (not this run)"}


def convert_all(sp, A, formats, feats=None):
    import torch
    handles, conv_ms, na = {}, {}, {}
    stream = torch.cuda.current_stream()
    for f in formats:
        c0, c1 = ev(), ev()
        c0.record(stream)
        try:
            handles[f] = sp.convert(A, f, features=feats)
        except sp.SpmvError as e:
            if e.status in (3, 4):
                na[f] = e.name
                continue
            raise
        c1.record(stream)
        torch.cuda.synchronize()
        conv_ms[f] = c0.elapsed_time(c1)
    return handles, conv_ms, na


def consistency(handles, x, y_init, dtype):
    """All formats agree (no oracle here: the oracle parity of these exact configurations is
    tests/test_gpu_parity.py)."""
    import torch
    probe = {}
    for f, h in handles.items():
        yp = y_init.clone()
        h.run(1.0, x, 1.0, yp)
        probe[f] = yp
    torch.cuda.synchronize()
    ref = next(iter(probe))
    scale = probe[ref].abs().max().item() + 1.0
    agree = {f: float((probe[f] - probe[ref]).abs().max().item() / scale) for f in probe}
    ok = all(v < (1e-12 if dtype == torch.float64 else 1e-5) * 64 for v in agree.values())
    return ok, agree


def extra_rmat24(sp, args, peak, peak_src, local, config="rmat24", formats=None):
    """configs[2] (R-MAT 24) per-format blocks in fp64 and fp32 beside the headline (and the
    same for the rgg19 stand-in of the paper's rgg_n_2_19_s0)."""
    import torch

    from matgen import gpu
    out = {}
    stream = torch.cuda.current_stream()
    for dname, dtype, kind in (("f64", torch.float64, "f64"), ("f32", torch.float32, "f32")):
        dA, _ = device_matrix(config, kind, dtype)
        feats = sp.features(dA)
        torch.cuda.synchronize()
        ft = []
        for _ in range(max(3, args.feat_reps // 2)):
            t0 = time.perf_counter()
            sp.features(dA)
            ft.append(time.perf_counter() - t0)
        ft.sort()
        fbytes = (dA.n_rows + 1) * dA.row_ptr.element_size() + 4 * dA.nnz
        handles, conv_ms, na = convert_all(sp, dA, (formats or RMAT_FORMATS["rmat24"]).split(","), feats)
        x = gpu.vector(dA.n_cols, 0x5EED0003, 1, kind, dtype)
        y0 = gpu.vector(dA.n_rows, 0x5EED0003, 2, kind, dtype)
        ok, agree = consistency(handles, x, y0, dtype)
        if not ok:
            raise SystemExit(f"{config} {dname}: formats disagree {agree}")
        steps = max(5, min(args.steps, args.extra_steps))
        # A11 variants (beta = 0, cold L2) for configs[2] too; the rgg19 stand-in fits the L2
        # and keeps the plain timing
        var = config.startswith("rmat") and not args.no_variants
        l2 = sp.context().l2_bytes
        flush = torch.zeros(max(2 * l2, 1 << 20) // 4, dtype=torch.float32, device="cuda") if var else None
        ms_step, per, clocks, variants = time_formats(handles, x, y0, steps, args.warmup, local, stream,
                                                      extra_variants=var, flush=flush)
        del flush
        pf = format_block(handles, per, variants, dA.nnz, peak, config, dname, conv_ms)
        for f, why in na.items():
            pf[f] = {"status": "N/A", "reason": why}
        fm = [f for f in handles]
        best = min(fm, key=lambda f: pf[f]["ms_mean"])
        dom = max(fm, key=lambda f: pf[f]["ms_mean"])
        out[dname] = {"n_rows": dA.n_rows, "nnz": dA.nnz, "steps": steps, "ms_per_step": ms_step,
                      "gflops_step": 2.0 * dA.nnz * len(fm) / (ms_step * 1e-3) / 1e9,
                      "per_format": pf, "best_format": best, "roofline": roofline(pf, dom, peak, peak_src),
                      "roofline_best": roofline(pf, best, peak, peak_src), "clocks": clocks,
                      "formats_agree": agree,
                      "features": {"ms": ft[len(ft) // 2] * 1e3, "bytes": fbytes,
                                   "gbs": fbytes / ft[len(ft) // 2] / 1e9,
                                   "frac_of_peak": fbytes / ft[len(ft) // 2] / 1e9 / peak}}
        for h in handles.values():
            h.destroy()
        del handles, dA
        torch.cuda.empty_cache()
    return out


# ---------------------------------------------------------------------- our arm: 1 GPU

def run_single(args):
    import numpy as np
    import torch

    import matgen
    import paper_conf_ipps_nisassvs18_b200 as sp

    torch.cuda.set_device(0)
    config = args.config or "lap4096"
    dtype = torch.float64 if args.dtype == "f64" else torch.float32
    kind = "f64" if args.dtype == "f64" else "f32"
    t_gen = time.perf_counter()
    dA, A_host = device_matrix(config, kind, dtype)
    torch.cuda.synchronize()
    t_gen = time.perf_counter() - t_gen
    seed = matgen.SEEDS.get(config, 1)
    from matgen import gpu
    x = gpu.vector(dA.n_cols, seed, 1, kind, dtype)
    y0 = gpu.vector(dA.n_rows, seed, 2, kind, dtype)
    stream = torch.cuda.current_stream()
    default_formats = RMAT_FORMATS.get(config, ",".join(sp.PAPER_FORMATS))
    formats = [f for f in (args.formats or default_formats).split(",") if f]

    # ---- features (a2): one untimed call (ctx state, module load), then the warm median
    feats = sp.features(dA)
    torch.cuda.synchronize()
    feat_t = []
    for _ in range(args.feat_reps):
        t0 = time.perf_counter()
        sp.features(dA)
        feat_t.append(time.perf_counter() - t0)
    feat_t.sort()
    feat_ms = feat_t[len(feat_t) // 2] * 1e3
    feat_bytes = (dA.n_rows + 1) * dA.row_ptr.element_size() + 4 * dA.nnz

    # ---- conversions (a3-a7), reusing the feature pass
    handles, conv_ms, na = convert_all(sp, dA, formats, feats)
    fmts = list(handles)
    ok, agree = consistency(handles, x, y0, dtype)
    closed_form = None
    if config.startswith("lap"):
        g = int(round(dA.n_rows ** 0.5))
        ones = torch.ones(dA.n_cols, dtype=dtype, device="cuda")
        exp = torch.zeros((g, g), dtype=dtype, device="cuda")
        exp[0, :] += 1; exp[-1, :] += 1; exp[:, 0] += 1; exp[:, -1] += 1
        closed_form = True
        for f in fmts:
            yc = torch.empty(dA.n_rows, dtype=dtype, device="cuda")
            handles[f].run(1.0, ones, 0.0, yc)
            closed_form = closed_form and bool(torch.equal(yc.view(g, g), exp))
    if not ok or closed_form is False:
        raise SystemExit(f"consistency check failed: agree={agree} closed_form={closed_form}")

    # ---- timed steps (+ beta = 0 and cold-L2 variants, A11)
    l2 = sp.context().l2_bytes
    flush = torch.zeros(max(2 * l2, 1 << 20) // 4, dtype=torch.float32, device="cuda")
    ms_step, per, clocks, variants = time_formats(handles, x, y0, args.steps, args.warmup, 0, stream,
                                                  extra_variants=not args.no_variants, flush=flush)
    del flush
    value = 2.0 * dA.nnz * len(fmts) / (ms_step * 1e-3) / 1e9
    peak, peak_src = measured_peak()
    pf = format_block(handles, per, variants, dA.nnz, peak, config, args.dtype, conv_ms)
    for f, why in na.items():
        pf[f] = {"status": "N/A", "reason": why}
    best = min(fmts, key=lambda f: pf[f]["ms_mean"])
    dom = max(fmts, key=lambda f: pf[f]["ms_mean"])
    launches_per_step = sum(handles[f].launches() for f in fmts)

    # ---- end to end through the C ABI with pinned host buffers
    e2e = None
    if not args.no_e2e and not (args.e2e_per_call or args.e2e_serial):
        # the label-collection call: x and y_in cross PCIe once per step for all formats,
        # each format's result comes back (spmv_run_host_multi)
        xnp = x.cpu().pin_memory().numpy()
        yin = y0.cpu().pin_memory().numpy()
        outs = [y0.cpu().pin_memory().numpy() for _ in fmts]
        hl = [handles[f] for f in fmts]
        e2e_steps = max(3, min(args.steps, args.e2e_steps))
        sp.run_host_multi(hl, 1.0, xnp, 1.0, yin, outs)          # first call allocates the io buffers
        sp.run_host_multi(hl, 1.0, xnp, 1.0, yin, outs)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(e2e_steps):
            sp.run_host_multi(hl, 1.0, xnp, 1.0, yin, outs)
        dt = time.perf_counter() - t0
        V = 8 if dtype == torch.float64 else 4
        e2e = {"value": 2.0 * dA.nnz * len(fmts) / (dt / e2e_steps) / 1e9, "unit": "GFLOP/s",
               "h2d_bytes_per_step": (dA.n_cols + dA.n_rows) * V,
               "d2h_bytes_per_step": len(fmts) * dA.n_rows * V, "steps": e2e_steps,
               "api": "spmv_run_host_multi (pinned host x and y_in -> device once, every format run from a "
                      "device copy of y_in, each result -> host while the next format runs, sync)"}
    elif not args.no_e2e:
        xnp = x.cpu().pin_memory().numpy()
        ynps = {f: y0.cpu().pin_memory().numpy() for f in fmts}
        e2e_steps = max(3, min(args.steps, args.e2e_steps))
        for f in fmts:                             # first calls allocate the handles' io buffers
            handles[f].run_host(1.0, xnp, 1.0, ynps[f])
        torch.cuda.synchronize()
        # one host thread and one CUDA stream per format: H2D copies, runs and D2H copies of
        # the formats overlap; the step ends when every format's y is back on the host
        streams = {f: torch.cuda.Stream() for f in fmts}
        pool = None
        if not args.e2e_serial and len(fmts) > 1:
            from concurrent.futures import ThreadPoolExecutor
            pool = ThreadPoolExecutor(max_workers=len(fmts))

        def e2e_step():
            if pool is None:
                for f in fmts:
                    handles[f].run_host(1.0, xnp, 1.0, ynps[f], stream=streams[f])
            else:
                list(pool.map(lambda f: handles[f].run_host(1.0, xnp, 1.0, ynps[f], stream=streams[f]), fmts))
        e2e_step()
        t0 = time.perf_counter()
        for _ in range(e2e_steps):
            e2e_step()
        dt = time.perf_counter() - t0
        if pool is not None:
            pool.shutdown()
        V = 8 if dtype == torch.float64 else 4
        e2e = {"value": 2.0 * dA.nnz * len(fmts) / (dt / e2e_steps) / 1e9, "unit": "GFLOP/s",
               "h2d_bytes_per_step": len(fmts) * (dA.n_cols + dA.n_rows) * V,
               "d2h_bytes_per_step": len(fmts) * dA.n_rows * V, "steps": e2e_steps,
               "api": ("spmv_run_host (pinned host x,y -> device, run, y -> host, sync)"
                       + (", one host thread + CUDA stream per format" if pool is not None else ", formats in turn"))}

    cpu = None
    if not args.no_cpu:
        Ah = host_sample(dA, A_host, ORACLE_SAMPLE_NNZ)
        cpu = cpu_baseline(Ah, x.cpu().double().numpy(), y0.cpu().double().numpy(), budget_s=args.cpu_budget)

    # ---- configs[2] beside the headline (default run)
    extra = None
    if config == "lap4096" and not args.no_extra:
        for h in handles.values():
            h.destroy()
        handles = None
        torch.cuda.empty_cache()
        extra = {"rmat24": extra_rmat24(sp, args, peak, peak_src, 0)}
        rg = extra_rmat24(sp, args, peak, peak_src, 0, config="rgg19", formats=",".join(sp.PAPER_FORMATS))
        # R1: the paper's own numbers for this matrix (K80c, single precision, the real file)
        # beside ours (B200, the synthetic stand-in, fp32 storage with fp64 accumulation)
        rg["vs_paper"] = {f: {"paper_k80c_gflops": g, "b200_gflops_f32": rg["f32"]["per_format"][f]["gflops"]}
                          for f, g in (("csr5", 22), ("merge", 21)) if "gflops" in rg["f32"]["per_format"].get(f, {})}
        rg["vs_paper"]["source"] = "PAPER.md:131 (rgg_n_2_19_s0 on a Tesla K80c)"
        rg["l2"] = ("the matrix (~80 MB in fp64) fits the 126 MB L2: back-to-back runs are L2-warm, as in the "
                    "paper's timing loop (A11); frac_of_peak is against HBM and can overstate")
        extra["rgg19"] = rg

    line = {
        "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": 1, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
        # the same fixed matrix at every N (N > 1 splits its rows): strong scaling
        "scaling": "strong",
        "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
        "config": {"workload": config, "desc": CONFIGS.get(config, {}).get("desc", config),
                   "n_rows": dA.n_rows, "n_cols": dA.n_cols, "nnz": dA.nnz, "formats": fmts,
                   "step": "one SpMV (alpha=1, beta=1) in each feasible format",
                   "l2": "no flush: every format's arrays exceed the 126 MB L2 (cold-L2 variant per format: "
                         "ms_cold_l2, a 2x L2 write before each run)",
                   "parallelism": "1 GPU"},
        "per_format": pf, "best_format": best,
        "roofline": roofline(pf, dom, peak, peak_src), "roofline_best": roofline(pf, best, peak, peak_src),
        "features": {"ms": feat_ms, "ms_min": feat_t[0] * 1e3, "bytes": feat_bytes,
                     "gbs": feat_bytes / (feat_ms * 1e-3) / 1e9,
                     "frac_of_peak": feat_bytes / (feat_ms * 1e-3) / 1e9 / peak,
                     "timing": f"warm median of {len(feat_t)} blocking spmv_features calls (wall clock: one kernel "
                               "launch + one 112-byte readback each)",
                     "values": {k: feats[k] for k in sp.PAPER_FEATURES}},
        "label6": best, "gpu_launches": launches_per_step * args.steps,
        "clocks": clocks, "e2e": e2e, "cpu_baseline": cpu,
        "checks": {"formats_agree": agree, "laplacian_closed_form": closed_form},
        "extra_configs": extra, "paper_context": PAPER_CONTEXT, "gen_s": t_gen,
    }
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------- our arm: N GPUs

def run_multi(args):
    """N ranks, one GPU each: every format's step = pack x -> exchange (NCCL) -> shard SpMV,
    timed per format with CUDA events, max over ranks."""
    import numpy as np
    import torch
    import torch.distributed as dist

    import matgen
    import paper_conf_ipps_nisassvs18_b200 as sp
    from matgen import gpu
    from paper_conf_ipps_nisassvs18_b200.dist import DistSpMV, HaloSpMV, RowRangeCSR, time_exchange

    ws, rank, local = dist_env()
    if args.dist_backend == "gloo":
        # functional check of the N-rank step on fewer GPUs (ranks may share a device;
        # collectives staged through host memory): not a performance number
        local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    if args.nccl_algo != "default":
        os.environ["NCCL_ALGO"] = args.nccl_algo
    if args.dist_backend == "gloo":
        dist.init_process_group("gloo")
    else:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    config = args.config or "lap4096"
    dtype = torch.float64 if args.dtype == "f64" else torch.float32
    kind = "f64" if args.dtype == "f64" else "f32"
    seed = matgen.SEEDS.get(config, matgen.SEEDS["rmat24"])
    t_gen = time.perf_counter()
    rmat = config.startswith("rmat")
    if rmat:
        # rank-local construction: GPU generator, row_ptr/col on this device, values for this
        # rank's rows only (DistSpMV.from_rmat's recipe, shared by every format)
        from matgen.gpu import DeviceRMAT
        from paper_conf_ipps_nisassvs18_b200.spmv import partition
        g = DeviceRMAT(int(config[4:]), 16, seed)
        col = g.col()
        probe = RowRangeCSR(g.row_ptr, col, torch.empty(0, dtype=dtype, device="cuda"), g.n, 0)
        splits = partition(probe, ws)
        r0, r1 = int(splits[rank]), int(splits[rank + 1])
        k0, k1 = (int(v) for v in g.row_ptr[[r0, r1]].tolist())
        A = RowRangeCSR(g.row_ptr, col, g.values(k0, k1, kind=kind, dtype=dtype), g.n, k0)
        nnz_total = g.nnz
        g.release()
        formats = [f for f in (args.formats or RMAT_FORMATS[config]).split(",") if f]
        ops = {f: DistSpMV(A, f, compress=not args.dense, overlap=not args.no_overlap) for f in formats}
        exchange = ("compressed " if not args.dense else "") + "all-gather (NCCL all_gather_into_tensor)" + \
            (" overlapped with the own-column block" if not args.no_overlap else "")
    else:
        A_host = build_matrix(config, kind)
        dA = sp.CSR.from_host(A_host, dtype=dtype)
        nnz_total = dA.nnz
        formats = [f for f in (args.formats or ",".join(sp.PAPER_FORMATS)).split(",") if f]
        ops = {}
        for f in formats:
            try:
                ops[f] = HaloSpMV(dA, f)
            except sp.SpmvError as e:
                if e.status not in (3, 4):
                    raise
        exchange = "point-to-point halo (NCCL all_to_all_single) overlapped with the own-column block"
        A = dA
    torch.cuda.synchronize()
    t_gen = time.perf_counter() - t_gen
    fmts = list(ops)
    lay = ops[fmts[0]].layout
    x_local = gpu.vector(lay.rows, seed, 1, kind, dtype, i0=lay.r0)
    y_init = gpu.vector(lay.rows, seed, 2, kind, dtype, i0=lay.r0)
    del A
    torch.cuda.empty_cache()
    stream = torch.cuda.current_stream()

    # ---- consistency: every format's distributed product agrees (max over ranks)
    probe = {}
    for f in fmts:
        yp = y_init.clone()
        ops[f].run(1.0, 1.0, yp, x_local=x_local)
        probe[f] = yp
    torch.cuda.synchronize()
    scale = max(p.abs().max().item() for p in probe.values()) + 1.0
    dev_max = torch.tensor([max((probe[f] - probe[fmts[0]]).abs().max().item() / scale for f in fmts)],
                           dtype=torch.float64, device="cuda")
    dist.all_reduce(dev_max, op=dist.ReduceOp.MAX)
    if dev_max.item() > (1e-12 if dtype == torch.float64 else 1e-5) * 64:
        raise SystemExit(f"formats disagree across ranks: {dev_max.item()}")

    # ---- timed steps: per format pack + exchange + SpMV
    ys = {f: y_init.clone() for f in fmts}

    def step(record=None):
        for f in fmts:
            if record is not None:
                record[f][0].record(stream)
            ops[f].run(1.0, 1.0, ys[f], x_local=x_local)
            if record is not None:
                record[f][1].record(stream)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    evs = {f: [(ev(), ev()) for _ in range(args.steps)] for f in fmts}
    t0, t1 = ev(), ev()
    dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        t0.record(stream)
        for k in range(args.steps):
            step({f: evs[f][k] for f in fmts})
        t1.record(stream)
        torch.cuda.synchronize()
    dist.barrier()
    ms = torch.tensor([t0.elapsed_time(t1)] + [sum(a.elapsed_time(b) for a, b in evs[f]) / args.steps for f in fmts],
                      dtype=torch.float64, device="cuda")
    dist.all_reduce(ms, op=dist.ReduceOp.MAX)
    ms_step = float(ms[0].item()) / args.steps
    ms_fmt = {f: float(ms[1 + i].item()) for i, f in enumerate(fmts)}
    value = 2.0 * nnz_total * len(fmts) / (ms_step * 1e-3) / 1e9

    # ---- exchange alone, compute alone, overlap, per-rank HBM and NVLink rates
    peak, peak_src = measured_peak()
    d7 = {}
    for f in fmts:
        op = ops[f]
        t_ex = time_exchange(op, iters=max(5, min(args.steps, 30)))
        yl = y_init.clone()
        for _ in range(3):
            op.run_local(1.0, 1.0, yl)
        a, b = ev(), ev()
        reps = max(5, min(args.steps, 30))
        a.record(stream)
        for _ in range(reps):
            op.run_local(1.0, 1.0, yl)
        b.record(stream)
        torch.cuda.synchronize()
        t_loc = a.elapsed_time(b) / reps
        vals = torch.tensor([t_ex, t_loc], dtype=torch.float64, device="cuda")
        dist.all_reduce(vals, op=dist.ReduceOp.MAX)
        t_ex, t_loc = (float(v) for v in vals.tolist())
        lb = op.local_bytes()
        recv = op.exchange_bytes()
        hidden = max(0.0, min(1.0, (t_ex + t_loc - ms_fmt[f]) / t_ex)) if t_ex > 0 else None
        d7[f] = {"ms_step": ms_fmt[f], "ms_exchange_alone": t_ex, "ms_local_alone": t_loc,
                 "gflops": 2.0 * nnz_total / (ms_fmt[f] * 1e-3) / 1e9,
                 "per_rank_hbm_gbs": lb / (t_loc * 1e-3) / 1e9, "per_rank_frac_of_peak": lb / (t_loc * 1e-3) / 1e9 / peak,
                 "local_bytes_rank": lb, "exchange_bytes_per_rank": recv,
                 "nvlink_gbs": recv / (t_ex * 1e-3) / 1e9 if t_ex > 0 else None,
                 "comm_hidden_fraction": hidden, "launches": op.launches()}
    dom = max(fmts, key=lambda f: d7[f]["ms_local_alone"])
    launches_per_step = sum(ops[f].launches() for f in fmts)

    # ---- e2e: host x slice in (pinned), distributed step, host y slice out, every step
    e2e = None
    if not args.no_e2e:
        xh = x_local.cpu().pin_memory()
        yh = {f: y_init.cpu().pin_memory() for f in fmts}
        xd = torch.empty_like(x_local)
        e2e_steps = max(3, min(args.steps, args.e2e_steps))

        def e2e_step():
            xd.copy_(xh, non_blocking=True)
            for f in fmts:
                ops[f].run(1.0, 1.0, ys[f], x_local=xd)
                yh[f].copy_(ys[f], non_blocking=True)
            torch.cuda.synchronize()
        e2e_step()
        dist.barrier()
        tt = time.perf_counter()
        for _ in range(e2e_steps):
            e2e_step()
        dist.barrier()
        dt = torch.tensor([time.perf_counter() - tt], dtype=torch.float64, device="cuda")
        dist.all_reduce(dt, op=dist.ReduceOp.MAX)
        V = 8 if dtype == torch.float64 else 4
        e2e = {"value": 2.0 * nnz_total * len(fmts) / (float(dt.item()) / e2e_steps) / 1e9, "unit": "GFLOP/s",
               "h2d_bytes_per_step": ws * lay.rows * V, "d2h_bytes_per_step": ws * len(fmts) * lay.rows * V,
               "steps": e2e_steps, "api": "DistSpMV/HaloSpMV.run with the x slice copied from pinned host memory "
                                          "and every format's y slice copied back, every step (max over ranks)"}

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": args.dtype, "data": "synthetic",
            "config": {"workload": config, "desc": CONFIGS.get(config, {}).get("desc", config),
                       "n_rows": int(lay.splits[-1]),
                       "nnz": nnz_total, "formats": fmts,
                       "step": "per format: pack x slice -> exchange -> shard SpMV (alpha=1, beta=1)",
                       "l2": "no flush: every rank's shard and x exceed the 126 MB L2" if nnz_total > 5e8 else
                             "no flush (back-to-back steps, A11 hot-L2 protocol)",
                       "parallelism": f"row-partitioned x{ws} (nnz-balanced merge-path splits), {exchange}",
                       "nccl_algo": os.environ.get("NCCL_ALGO", "default (NCCL's choice; NVLS on NVSwitch when "
                                                               "available)"),
                       "backend": args.dist_backend + ("" if args.dist_backend == "nccl" else
                                                       " (functional check: ranks may share a GPU, host-staged "
                                                       "collectives -- not a performance number)"),
                       "construction": ("rank-local: GPU R-MAT generator, values of the rank's rows only"
                                        if rmat else "every rank builds the matrix, keeps its shard")},
            "per_format": d7, "best_format": min(fmts, key=lambda f: ms_fmt[f]),
            "roofline": {"bound": "hbm", "achieved": d7[dom]["per_rank_hbm_gbs"], "peak": peak, "unit": "GB/s",
                         "frac": d7[dom]["per_rank_hbm_gbs"] / peak, "traffic": None, "kernel_format": dom,
                         "bytes_per_launch": d7[dom]["local_bytes_rank"], "avg_launch_ms": d7[dom]["ms_local_alone"],
                         "peak_source": peak_src, "scope": "one rank's shard kernels (max over ranks)"},
            "gpu_launches": launches_per_step * args.steps, "clocks": clk.summary(), "e2e": e2e,
            "cpu_baseline": None, "paper_context": PAPER_CONTEXT, "gen_s": t_gen,
        }
        print(json.dumps(line), flush=True)
    dist.barrier()
    dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=300)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="", help="lap4096 (default), rmat24, rmat27, u2048, lapG, rmatS, mtx:PATH")
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32"])
    ap.add_argument("--formats", default="")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-variants", action="store_true", help="skip the beta=0 / cold-L2 per-format variants")
    ap.add_argument("--no-extra", action="store_true", help="skip the R-MAT 24 blocks of the default line")
    ap.add_argument("--extra-steps", type=int, default=50)
    ap.add_argument("--dense", action="store_true", help="N > 1 R-MAT: exchange the whole x (no compression)")
    ap.add_argument("--no-overlap", action="store_true", help="N > 1 R-MAT: no own-column overlap")
    ap.add_argument("--nccl-algo", default="default", choices=["default", "Ring", "NVLS", "Tree", "NVLSTree"])
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="gloo: functional check of N ranks on fewer GPUs (not a performance number)")
    ap.add_argument("--e2e-steps", type=int, default=10)
    ap.add_argument("--e2e-serial", action="store_true", help="e2e: per-format spmv_run_host calls in turn")
    ap.add_argument("--e2e-per-call", action="store_true",
                    help="e2e: per-format spmv_run_host calls (x/y copied per format), one host thread each")
    ap.add_argument("--feat-reps", type=int, default=20, help="warm spmv_features calls timed")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=10.0)
    args = ap.parse_args()
    if args.warmup < 3:
        print("warning: --warmup < 3 gives no valid bench number", file=sys.stderr)
    ws, _, _ = dist_env()
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(self_launch(args))
    if args.impl == "reference":
        run_reference(args)
    elif ws > 1:
        run_multi(args)
    else:
        run_single(args)


if __name__ == "__main__":
    main()
