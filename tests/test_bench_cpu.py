"""bench.py host-side pieces (no GPU): the oracle's all-cores row split is exact, and
the --impl reference arm prints the contract's JSON line."""
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
    outs = [oracle.spmv_csr(B, x, 1.0, 1.0, yb) for B, yb in R.blocks]
    R.run()
    R.close()
    ref = oracle.spmv_csr(A, x, 1.0, 1.0, y)[:R.m]
    assert np.array_equal(np.concatenate(outs), ref)


def test_reference_arm_json_line():
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config",
                          "u2048", "--steps", "3", "--warmup", "3"], capture_output=True, text=True, timeout=600,
                         cwd=ROOT)
    assert out.returncode == 0, out.stderr
    line = json.loads(out.stdout.strip().splitlines()[-1])
    assert line["impl"] == "reference" and line["unit"] == "GFLOP/s" and line["value"] > 0
    assert line["cpu_baseline"]["kind"] == "oracle" and line["cpu_baseline"]["cores"] >= 1
    assert line["e2e"]["h2d_bytes_per_step"] == 0 and line["e2e"]["value"] == line["value"]
    assert line["config"]["workload"] == "u2048"
