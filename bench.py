#!/usr/bin/env python
"""bench.py -- SpMV GFLOP/s & HBM GB/s (% of roofline) per format on B200.

One "step" = one pass of the label-collection hot path over the workload matrix:
y_f <- alpha*A_f*x + beta*y_f for every feasible format f of the six (COO, ELL, CSR,
HYB, merge-path CSR, CSR5), alpha = beta = 1 (A11).
Conversions and the feature pass are one-off setup: they are timed and reported
separately, not inside the step.

  value  = sum over formats of 2*nnz / (time of the K timed steps / K)   [GFLOP/s]
  e2e    = the same through spmv_run_host (pinned host x/y in, y out, every step)

Default workload: BASELINE configs[1] (5-point Laplacian, 4096^2 grid, fp64), which
fits one GPU; its arrays (>= 1.4 GB per format) exceed the 126 MB L2, so no flush
is needed between steps.  Under torchrun (N > 1) the matrix is row-partitioned by
nnz-balanced merge-path splits, x is all-gathered with NCCL every step and each
rank runs its shard (strong scaling).

--impl reference runs the CPU oracle (oracle/, plain C, long double) on rank 0 over
a bounded row sample of the same workload: the baseline arm, not a target.
"""
from __future__ import annotations

import argparse
import json
import os
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
}


def build_matrix(name, dtype_kind):
    import matgen
    if name == "u2048":
        return matgen.uniform_fixed(2048, 2048, 16, kind=dtype_kind)
    if name == "lap4096":
        return matgen.laplacian5(4096)
    if name == "rmat24":
        return matgen.rmat(24, kind=dtype_kind)
    if name.startswith("lap"):
        return matgen.laplacian5(int(name[3:]))
    if name.startswith("rmat"):
        return matgen.rmat(int(name[4:]), kind=dtype_kind)
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
    """nvidia-smi clocks / throttle reasons sampled every 200 ms during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, index=0):
        self.index = index
        self.samples = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.index), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "200"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
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
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        import statistics
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no nvidia-smi samples"], "samples": 0}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4) if s[3 + i].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.samples)}


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


# ---------------------------------------------------------------------- reference arm

def host_cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


class OracleRows:
    """The oracle (oracle.spmv_csr, unchanged) over a contiguous row sample, the rows split
    into `threads` nnz-balanced blocks that host threads run at once (the ctypes call
    releases the GIL; each row is computed exactly as in one call over all rows)."""

    def __init__(self, A, x, y, target_nnz, threads):
        import numpy as np

        import oracle
        m = int(np.searchsorted(A.row_ptr, min(target_nnz, A.nnz), side="left"))
        self.m = max(1, min(m, A.n_rows))
        self.nnz = int(A.row_ptr[self.m])
        self.threads = max(1, int(threads))
        cuts = np.searchsorted(A.row_ptr[:self.m + 1], np.linspace(0, self.nnz, self.threads + 1), side="left")
        cuts[0], cuts[-1] = 0, self.m
        self.blocks = []
        for a, b in zip(cuts[:-1], cuts[1:]):
            if b > a:
                self.blocks.append((oracle.CSR(A.row_ptr[a:b + 1], A.col, A.val, (b - a, A.n_cols)), y[a:b]))
        self.x = x
        self.pool = None
        if len(self.blocks) > 1:
            from concurrent.futures import ThreadPoolExecutor
            self.pool = ThreadPoolExecutor(max_workers=len(self.blocks))

    def run(self):
        import oracle
        if self.pool is None:
            for B, yb in self.blocks:
                oracle.spmv_csr(B, self.x, 1.0, 1.0, yb)
            return
        list(self.pool.map(lambda b: oracle.spmv_csr(b[0], self.x, 1.0, 1.0, b[1]), self.blocks))

    def close(self):
        if self.pool is not None:
            self.pool.shutdown()


def run_reference(args):
    """The CPU oracle on this host (rank 0 only), bounded row sample per step."""
    import numpy as np

    import matgen
    import oracle
    ws, rank, _ = dist_env()
    if rank != 0:
        return
    kind = "f64" if args.dtype == "f64" else "f32"
    A = build_matrix(args.config, kind)
    x = matgen.vector(A.n_cols, 1, 1, kind)
    y = matgen.vector(A.n_rows, 1, 2, kind)
    # each step: the oracle computes, for every format of the step, the same rows' y on a
    # contiguous row sample (~target nonzeros per host core), long double, all host cores
    nformats = 6 if args.config != "rmat24" else 5
    cores = host_cores()
    R = OracleRows(A, x, y, max(1, int(args.ref_sample_nnz)) * cores, cores)

    def step():
        for _ in range(nformats):
            R.run()

    for _ in range(args.warmup):
        step()
    t0 = time.perf_counter()
    for _ in range(args.steps):
        step()
    dt = time.perf_counter() - t0
    R.close()
    nnz_s, m = R.nnz, R.m
    flops = 2.0 * nnz_s * nformats * args.steps
    val = flops / dt / 1e9
    sample = (f"{nformats} oracle CSR SpMVs (long double, {len(R.blocks)} host threads over nnz-balanced row "
              f"blocks) per step over rows [0,{m}) = {nnz_s} of {A.nnz} nonzeros of {args.config}")
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "GFLOP/s", "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt / args.steps * 1e3,
            "higher_is_better": True, "scaling": "strong" if ws > 1 else "weak", "vs_baseline": None,
            "dtype": args.dtype, "data": "synthetic",
            "config": {"workload": args.config, "desc": CONFIGS.get(args.config, {}).get("desc", args.config)},
            "cpu_baseline": {"value": val, "unit": "GFLOP/s", "cores": len(R.blocks), "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": val, "unit": "GFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------- our arm

def cpu_baseline(A, x, y, budget_s=10.0):
    """The oracle as it stands, timed on this host (rank 0, N = 1 only), bounded sample:
    all host cores (nnz-balanced row blocks, one thread each), and one thread beside it."""
    out = None
    for threads in (host_cores(), 1):
        R = OracleRows(A, x, y, 40_000_000, threads)
        reps, t0 = 0, time.perf_counter()
        while True:
            R.run()
            reps += 1
            if time.perf_counter() - t0 > budget_s / 2:
                break
        dt = time.perf_counter() - t0
        R.close()
        rec = {"value": 2.0 * R.nnz * reps / dt / 1e9, "unit": "GFLOP/s", "cores": len(R.blocks), "kind": "oracle",
               "sample": f"{reps} oracle CSR SpMV(s) (long double, {len(R.blocks)} host thread(s) over nnz-balanced "
                         f"row blocks) over rows [0,{R.m}) = {R.nnz} nonzeros of the workload, {dt:.1f} s"}
        if out is None:
            out = rec
        else:
            out["single_thread"] = {k: rec[k] for k in ("value", "cores", "sample")}
    return out


def run_ours(args):
    import numpy as np
    import torch

    import matgen
    import paper_conf_ipps_nisassvs18_b200 as sp

    ws, rank, local = dist_env()
    torch.cuda.set_device(local)
    dist = None
    if ws > 1:
        import torch.distributed as dist
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dtype = torch.float64 if args.dtype == "f64" else torch.float32
    kind = "f64" if args.dtype == "f64" else "f32"
    t_gen = time.perf_counter()
    A = build_matrix(args.config, kind)
    t_gen = time.perf_counter() - t_gen
    seed = matgen.SEEDS.get(args.config, 1)
    x_h = matgen.vector(A.n_cols, seed, 1, kind)
    y_h = matgen.vector(A.n_rows, seed, 2, kind)
    dA = sp.CSR.from_host(A, dtype=dtype)
    stream = torch.cuda.current_stream()
    ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731

    formats = [f for f in args.formats.split(",") if f] if args.formats else list(sp.PAPER_FORMATS)

    # ---- features (a2): one untimed call (ctx state, module load), then the warm median of
    # `feat_reps` blocking calls (one kernel + one 112-byte readback each)
    feats = sp.features(dA)
    torch.cuda.synchronize()
    feat_t = []
    for _ in range(args.feat_reps):
        t0 = time.perf_counter()
        sp.features(dA)
        feat_t.append(time.perf_counter() - t0)
    feat_t.sort()
    feat_ms = feat_t[len(feat_t) // 2] * 1e3
    feat_bytes = (A.n_rows + 1) * dA.row_ptr.element_size() + 4 * A.nnz

    # ---- partition (a14) for N > 1: this rank's rows, columns remapped to gathered-x slots
    # (DistSpMV: merge-path row splits, shard, optional compressed exchange)
    dsp = None
    if ws > 1:
        from paper_conf_ipps_nisassvs18_b200.dist import DistSpMV
        dsp = DistSpMV(dA, formats[0] if args.formats else "csr5", compress=args.compress)
        lay = dsp.layout
        local_A = dsp.shard
        dsp.set_x(torch.from_numpy(x_h[lay.r0:lay.r1].copy()).cuda().to(dtype))
        x_run = dsp.x_gathered
        y_init = torch.from_numpy(y_h[lay.r0:lay.r1].copy()).cuda().to(dtype)
        S = dsp.slot
    else:
        local_A = dA
        x_run = torch.from_numpy(x_h).cuda().to(dtype)
        y_init = torch.from_numpy(y_h).cuda().to(dtype)
        S = A.n_rows

    # ---- conversions (a3-a7), timed once each
    handles, conv_ms, na = {}, {}, {}
    for f in formats:
        c0, c1 = ev(), ev()
        c0.record(stream)
        try:
            handles[f] = sp.convert(local_A, f, features=feats if local_A is dA else None)
        except sp.SpmvError as e:
            if e.status in (3, 4):
                na[f] = e.name
                continue
            raise
        c1.record(stream)
        torch.cuda.synchronize()
        conv_ms[f] = c0.elapsed_time(c1)
    fmts = [f for f in formats if f in handles]
    ys = {f: y_init.clone() for f in fmts}
    split = {}
    halo = None
    if ws > 1 and args.halo:
        # halo exchange: each rank receives only the x entries its rows
        # reference, point to point (all_to_all_single), own-column blocks overlap it
        from paper_conf_ipps_nisassvs18_b200.dist import HaloPlan
        from paper_conf_ipps_nisassvs18_b200.spmv import spmv_slice_split
        lay = dsp.layout
        halo = HaloPlan(dA.row_ptr, dA.col, A.n_cols, lay.splits, lay.rank)
        split = {f: (sp.convert(spmv_slice_split(dA, lay.splits, lay.rank, 0), f),
                     sp.convert(spmv_slice_split(dA, lay.splits, lay.rank, 1, halo.colmap, halo.S), f)) for f in fmts}
        x_own = torch.from_numpy(x_h[lay.r0:lay.r1].copy()).cuda().to(dtype)
        halo_send = torch.zeros(halo.send_index.numel(), dtype=dtype, device="cuda")
        halo_recv = torch.zeros(halo.recv_len, dtype=dtype, device="cuda")
    elif ws > 1 and args.overlap:
        split = {f: dsp.split_handles(f) for f in fmts}
        x_own = torch.from_numpy(x_h[dsp.layout.r0:dsp.layout.r1].copy()).cuda().to(dtype)

    # ---- consistency before timing (no oracle here: the oracle parity of this exact
    # configuration is tests/test_gpu_parity.py::test_full_size_lap4096): all formats
    # agree, and for the Laplacian the closed form A*1 = {0 interior, 1 edge, 2 corner}
    if ws > 1:
        dsp.exchange()
    probe = {}
    for f in fmts:
        yp = y_init.clone()
        handles[f].run(1.0, x_run, 1.0, yp)
        probe[f] = yp
    torch.cuda.synchronize()
    ref_f = fmts[0]
    scale = probe[ref_f].abs().max().item() + 1.0
    agree = {f: float((probe[f] - probe[ref_f]).abs().max().item() / scale) for f in fmts}
    consistent = all(v < (1e-12 if dtype == torch.float64 else 1e-5) * 64 for v in agree.values())
    closed_form = None
    if args.config.startswith("lap") and ws == 1:
        g = int(round(A.n_rows ** 0.5))
        ones = torch.ones(A.n_cols, dtype=dtype, device="cuda")
        exp = torch.zeros((g, g), dtype=dtype, device="cuda")
        exp[0, :] += 1; exp[-1, :] += 1; exp[:, 0] += 1; exp[:, -1] += 1
        closed_form = True
        for f in fmts:
            yc = torch.empty(A.n_rows, dtype=dtype, device="cuda")
            handles[f].run(1.0, ones, 0.0, yc)
            closed_form = closed_form and bool(torch.equal(yc.view(g, g), exp))
    if not consistent or closed_form is False:
        raise SystemExit(f"consistency check failed: agree={agree} closed_form={closed_form}")

    # ---- timed steps
    nnz_local = local_A.nnz
    infos = {f: handles[f].info() for f in fmts}
    launches_per_step = sum(handles[f].launches() for f in fmts)
    if ws > 1:
        dist.barrier()

    def step(record=None):
        if halo is not None:
            from paper_conf_ipps_nisassvs18_b200.spmv import spmv_gather
            spmv_gather(x_own, halo.send_index, halo_send)
            work = halo.exchange(halo_send, halo_recv, async_op=True)
            for f in fmts:
                split[f][0].run(1.0, x_own, 1.0, ys[f])
            work.wait()
            for f in fmts:
                split[f][1].run(1.0, halo_recv, 1.0, ys[f])
            return
        if split:
            # overlap: own-column blocks while the all-gather is in flight
            work = dsp.exchange_async()
            for f in fmts:
                split[f][0].run(1.0, x_own, 1.0, ys[f])
            if work is not None:
                work.wait()
            for f in fmts:
                split[f][1].run(1.0, x_run, 1.0, ys[f])
            return
        if ws > 1:
            dsp.exchange()                         # the step's x all-gather (NCCL)
        for f in fmts:
            if record is not None:
                record[f][0].record(stream)
            handles[f].run(1.0, x_run, 1.0, ys[f])
            if record is not None:
                record[f][1].record(stream)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    evs = {f: [(ev(), ev()) for _ in range(args.steps)] for f in fmts}
    t_start, t_stop = ev(), ev()
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        t_start.record(stream)
        for k in range(args.steps):
            step({f: evs[f][k] for f in fmts})
        t_stop.record(stream)
        torch.cuda.synchronize()
    if ws > 1:
        dist.barrier()
    ms_total = t_start.elapsed_time(t_stop)
    if ws > 1:
        tt = torch.tensor([ms_total], dtype=torch.float64, device="cuda")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        ms_total = float(tt.item())
    ms_step = ms_total / args.steps
    total_flops = 2.0 * A.nnz * len(fmts)
    value = total_flops / (ms_step * 1e-3) / 1e9

    peak, peak_src = measured_peak()
    per_format = {}
    # format-neutral effective bandwidth: the canonical CSR bytes over each
    # format's time, and every fraction also against the 8 TB/s nominal
    csr_by = infos["csr"]["bytes_per_run"] if "csr" in infos else None
    for f in fmts:
        if split:                                  # overlap: formats interleave, no per-format events
            evs[f] = [(t_start, t_stop)]
        ts = sorted(a.elapsed_time(b) / (args.steps * len(fmts) if split else 1) for a, b in evs[f])
        mean = sum(ts) / len(ts)
        by = infos[f]["bytes_per_run"]
        per_format[f] = {"ms_mean": mean, "ms_median": ts[len(ts) // 2], "ms_min": ts[0],
                         "gflops": 2.0 * nnz_local / (mean * 1e-3) / 1e9,
                         "gbs": by / (mean * 1e-3) / 1e9, "frac_of_peak": by / (mean * 1e-3) / 1e9 / peak,
                         "frac_of_nominal_8tbs": by / (mean * 1e-3) / 1e9 / 8000.0,
                         "gbs_csr": (csr_by / (mean * 1e-3) / 1e9) if csr_by else None,
                         "bytes_per_run": by, "launches": handles[f].launches(), "convert_ms": conv_ms[f]}
    for f, why in na.items():
        per_format[f] = {"status": "N/A", "reason": why}
    best = min(fmts, key=lambda f: per_format[f]["ms_mean"])
    dom = max(fmts, key=lambda f: per_format[f]["ms_mean"])

    def roof(f):
        p = per_format[f]
        return {"bound": "hbm", "achieved": p["gbs"], "peak": peak, "unit": "GB/s", "frac": p["gbs"] / peak,
                "traffic": traffic_for(args.config, f, args.dtype), "kernel_format": f,
                "bytes_per_launch": p["bytes_per_run"], "avg_launch_ms": p["ms_mean"],
                "launches_bracketed": p["launches"], "peak_source": peak_src}

    # ---- end to end through the C ABI with pinned host buffers (N = 1 only)
    e2e = None
    if ws == 1 and not args.no_e2e:
        xp = torch.from_numpy(x_h).to(dtype).pin_memory()
        yps = {f: torch.from_numpy(y_h).to(dtype).pin_memory() for f in fmts}
        xnp = xp.numpy()
        ynps = {f: yps[f].numpy() for f in fmts}
        e2e_steps = max(3, min(args.steps, args.e2e_steps))
        for f in fmts:                             # first calls allocate the handles' io buffers
            handles[f].run_host(1.0, xnp, 1.0, ynps[f])
        torch.cuda.synchronize()
        # one host thread and one CUDA stream per format: the formats' H2D copies, runs and
        # D2H copies overlap (copy engines both ways + SMs); the step ends when every
        # format's y is back on the host (spmv_run_host synchronizes its stream)
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
        e2e = {"value": total_flops / (dt / e2e_steps) / 1e9, "unit": "GFLOP/s",
               "h2d_bytes_per_step": len(fmts) * (A.n_cols + A.n_rows) * V,
               "d2h_bytes_per_step": len(fmts) * A.n_rows * V, "steps": e2e_steps,
               "api": ("spmv_run_host (pinned host x,y -> device, run, y -> host, sync)"
                       + (", one host thread + CUDA stream per format" if pool is not None else ", formats in turn"))}

    cpu = None
    if ws == 1 and rank == 0 and not args.no_cpu:
        cpu = cpu_baseline(A, x_h, y_h, budget_s=args.cpu_budget)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "GFLOP/s", "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
            "scaling": "strong" if ws > 1 else "weak", "vs_baseline": None, "dtype": args.dtype,
            "data": "synthetic",
            "config": {"workload": args.config, "desc": CONFIGS.get(args.config, {}).get("desc", args.config),
                       "n_rows": A.n_rows, "n_cols": A.n_cols, "nnz": A.nnz, "formats": fmts,
                       "step": "one SpMV (alpha=1, beta=1) in each feasible format",
                       "l2": "no flush: every format's arrays exceed the 126 MB L2",
                       "parallelism": ((f"row-partitioned x{ws}, NCCL all_to_all halo exchange of x overlapped "
                                        "with own-column blocks") if halo is not None else
                                       (f"row-partitioned x{ws}, NCCL all-gather of x"
                                        + (" (compressed)" if args.compress else "")
                                        + (" overlapped with own-column blocks" if args.overlap else "")))
                                      if ws > 1 else "1 GPU",
                       "exchange_bytes_per_rank": (halo.exchange_bytes(ys[fmts[0]].element_size()) if halo is not None
                                                   else dsp.exchange_bytes() if dsp is not None else 0)},
            "per_format": per_format, "best_format": best,
            "roofline": roof(dom), "roofline_best": roof(best),
            "features": {"ms": feat_ms, "ms_min": feat_t[0] * 1e3, "bytes": feat_bytes,
                         "gbs": feat_bytes / (feat_ms * 1e-3) / 1e9,
                         "frac_of_peak": feat_bytes / (feat_ms * 1e-3) / 1e9 / peak,
                         "timing": f"warm median of {len(feat_t)} blocking spmv_features calls (wall clock: "
                                   "one kernel launch + one 112-byte readback each)",
                         "values": {k: feats[k] for k in sp.PAPER_FEATURES}},
            "label6": best, "gpu_launches": launches_per_step * args.steps,
            "clocks": clk.summary(), "e2e": e2e, "cpu_baseline": cpu,
            "checks": {"formats_agree": agree, "laplacian_closed_form": closed_form},
            "gen_s": t_gen,
        }
        print(json.dumps(line), flush=True)
    if ws > 1:
        dist.destroy_process_group()


def traffic_for(config, fmt, dtype):
    """DRAM bytes per launch of this format's main kernel from the committed ncu
    --set full capture (profiles/ncu_traffic.json), or None."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    try:
        with open(p) as f:
            d = json.load(f)
        return d.get(config, {}).get(dtype, {}).get(fmt)
    except Exception:
        return None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=300)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="lap4096")
    ap.add_argument("--dtype", default="f64", choices=["f64", "f32"])
    ap.add_argument("--formats", default="")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--compress", action="store_true", help="N > 1: exchange only referenced columns")
    ap.add_argument("--halo", action="store_true",
                    help="N > 1: point-to-point halo exchange of the referenced x entries (all_to_all_single)")
    ap.add_argument("--overlap", action="store_true",
                    help="N > 1: own-column blocks run while the x all-gather is in flight")
    ap.add_argument("--e2e-steps", type=int, default=10)
    ap.add_argument("--feat-reps", type=int, default=20, help="warm spmv_features calls timed")
    ap.add_argument("--e2e-serial", action="store_true", help="e2e: run the formats' host calls in turn")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=10.0)
    ap.add_argument("--ref-sample-nnz", type=float, default=400_000)
    args = ap.parse_args()
    if args.warmup < 3:
        print("warning: --warmup < 3 gives no valid bench number", file=sys.stderr)
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
