"""bench.py host-side pieces (no GPU): the oracle's all-cores row split is exact, the CPU
baselines agree, --impl reference prints the contract's JSON line, and --gpus N launches
N ranks by itself (the reference arm's rank 0 alone prints)."""
import json
import os
import subprocess
import sys

import numpy as np

import matgen
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402


def test_oracle_rows_split_is_the_single_call():
    """Each row is computed by the same oracle call code whichever block holds it, so the
    threaded row split reproduces one call over all sampled rows bit for bit."""
    A = matgen.rmat(12, seed=3)
    x = matgen.vector(A.n_cols, 3, 1)
    y = matgen.vector(A.n_rows, 3, 2)
    R = bench.OracleRows(A, x, y, A.nnz, 5)
    assert R.nnz == A.nnz and int(A.row_ptr[R.m]) == A.nnz and len(R.blocks) == 5   # trailing empty rows dropped
    got = R.run()
    R1 = bench.OracleRows(A, x, y, A.nnz, 1)
    one = R1.run()
    R.close()
    R1.close()
    ref = oracle.spmv_csr(A, x, 1.0, 1.0, y)[:R.m]
    assert np.array_equal(got, ref) and np.array_equal(one, ref)


def test_cpu_baseline_protocol():
    """oracle all-cores == oracle 1 thread bit for bit; the fp64 all-core loop
    (not the oracle) is within fp64 rounding of the oracle."""
    import cpubase
    A = matgen.rmat(13, seed=4)
    x = matgen.vector(A.n_cols, 4, 1)
    y = matgen.vector(A.n_rows, 4, 2)
    cb = bench.cpu_baseline(A, x, y, budget_s=0.4)
    assert cb["kind"] == "oracle" and cb["multi_thread_equals_single_thread"] is True
    assert cb["value"] > 0 and cb["single_thread"]["value"] > 0 and cb["fp64_allcore"]["value"] > 0
    ref, bound = oracle.spmv_csr(A, x, 1.0, 1.0, y, with_bound=True)
    yc = y.copy()
    cpubase.spmv_f64(A.n_rows, A.row_ptr, A.col, A.val, x, 1.0, 1.0, yc)
    assert oracle.check_tolerance(yc, ref, bound, 1e-12)[0]


def _last_json(out):
    return json.loads([ln for ln in out.stdout.strip().splitlines() if ln.startswith("{")][-1])


def test_reference_arm_json_line():
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config",
                          "u2048", "--steps", "3", "--warmup", "3"], capture_output=True, text=True, timeout=600,
                         cwd=ROOT)
    assert out.returncode == 0, out.stderr
    line = _last_json(out)
    assert line["impl"] == "reference" and line["unit"] == "GFLOP/s" and line["value"] > 0
    assert line["cpu_baseline"]["kind"] == "oracle" and line["cpu_baseline"]["cores"] >= 1
    assert line["e2e"]["h2d_bytes_per_step"] == 0 and line["e2e"]["value"] == line["value"]
    assert line["config"]["workload"] == "u2048" and line["n_gpus"] == 1


def test_gpus_flag_self_launches_ranks():
    """--gpus 2 without WORLD_SIZE: bench.py runs 2 ranks under torch.distributed.run on
    127.0.0.1; the reference arm's rank 0 prints one line with n_gpus 2, rank 1 exits 0."""
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--gpus", "2",
                          "--config", "u2048", "--steps", "3", "--warmup", "3"], capture_output=True, text=True,
                         timeout=600, cwd=ROOT, env=env)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [ln for ln in out.stdout.strip().splitlines() if ln.startswith("{")]
    assert len(lines) == 1
    line = json.loads(lines[0])
    assert line["impl"] == "reference" and line["n_gpus"] == 2 and line["scaling"] == "strong"
