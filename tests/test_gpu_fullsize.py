"""BASELINE configs at full size in bench.py's launch configuration (SURVEY §8(c) bar):
configs[2] (R-MAT 24) in fp32 with general values against the 1e-5 bound on every row,
and configs[4] (R-MAT 27, 2.1e9 nonzeros, int64 row_ptr, built by the GPU generator as in
bench.py) on sampled rows the oracle computes one by one -- general fp64 values within
the 1e-12 bound and the integer regime bit-exact -- for CSR, merge and CSR5.  The GPU
generator equals the host one (tests/test_gpu_matgen.py), so the sampled rows are the
rows of matgen.rmat(27)."""
import numpy as np
import pytest
import torch

import matgen
import oracle

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sp():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_nisassvs18_b200 as pkg
    return pkg


def _run(sp, dA, fmt, alpha, x, beta, y):
    h = sp.convert(dA, fmt)
    yd = y.clone()
    h.run(alpha, x, beta, yd)
    torch.cuda.synchronize()
    h.destroy()
    return yd


def test_full_size_rmat24_fp32_general(sp):
    """fp32 storage, general values (2^-23 grid), alpha = 1.5, beta = -0.5: every row of
    every feasible format within 1e-5 of the bound (A13: fp32 accumulates in fp64)."""
    from matgen import gpu
    seed = matgen.SEEDS["rmat24"]
    rp, col, val = gpu.rmat(24, seed=seed, kind="f32", dtype=torch.float32)
    n = rp.numel() - 1
    dA = sp.CSR(rp.to(torch.int32), col, val, (n, n))
    A = matgen.HostCSR(rp.cpu().numpy(), col.cpu().numpy(), val.cpu().double().numpy(), n, n)
    x = gpu.vector(n, seed, 1, "f32", torch.float32)
    y = gpu.vector(n, seed, 2, "f32", torch.float32)
    ref, bound = oracle.spmv_csr(A, x.cpu().double().numpy(), 1.5, -0.5, y.cpu().double().numpy(), with_bound=True)
    for fmt in ("coo", "csr", "hyb", "merge", "csr5"):
        out = _run(sp, dA, fmt, 1.5, x, -0.5, y).cpu().double().numpy()
        ok, ratio, nbad = oracle.check_tolerance(out, ref, bound, 1e-5)
        assert ok, (fmt, nbad, ratio)


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32], ids=["f64", "f32"])
@pytest.mark.parametrize("beta", [0.0, 1.0, -0.5], ids=["beta0", "beta1", "beta"])
def test_dynamic_csr_rows_every_row(sp, dtype, beta):
    """The CSR-vector kernel's dynamically scheduled paths (>= 1.82M rows: fp64 contiguous
    32-row batches, fp32 compacted 64-row windows; long rows chunked, A25) on R-MAT 21
    (2.1M rows, 58% empty, rows up to 10^4): every row within the bound against the oracle,
    for beta = 0 (y write-only, NaN on entry: empty and chunked rows must become 0), 1
    (nothing written for rows without work) and -0.5 (beta*y for them)."""
    from matgen import gpu
    kind = "f64" if dtype == torch.float64 else "f32"
    rp, col, val = gpu.rmat(21, seed=21, kind=kind, dtype=dtype)
    n = rp.numel() - 1
    assert n >= 1_820_000 and int((rp[1:] - rp[:-1]).max()) > 1024
    dA = sp.CSR(rp.to(torch.int32), col, val, (n, n))
    A = matgen.HostCSR(rp.cpu().numpy(), col.cpu().numpy(), val.cpu().double().numpy(), n, n)
    x = gpu.vector(n, 21, 1, kind, dtype)
    y = gpu.vector(n, 21, 2, kind, dtype)
    ref, bound = oracle.spmv_csr(A, x.cpu().double().numpy(), 1.5, beta, y.cpu().double().numpy(), with_bound=True)
    h = sp.convert(dA, "csr")
    assert h.info()["csr_chunks"] > 0
    yd = torch.full_like(y, float("nan")) if beta == 0.0 else y.clone()
    h.run(1.5, x, beta, yd)
    torch.cuda.synchronize()
    out = yd.cpu().double().numpy()
    assert np.isfinite(out).all()
    ok, ratio, nbad = oracle.check_tolerance(out, ref, bound, 1e-12 if dtype == torch.float64 else 1e-5)
    assert ok, (nbad, ratio)


def _sample_rows(rp_host, n, k, seed):
    """k random rows, the 64 longest rows and the last rows (empty-row stretches)."""
    rng = np.random.default_rng(seed)
    lens = np.diff(rp_host)
    hub = np.argsort(lens)[-64:]
    return np.unique(np.concatenate([rng.integers(0, n, k), hub, np.arange(n - 64, n), np.arange(64)]))


def _rows_ref(rp_host, col, val, rows, x, alpha, beta, y_rows):
    """The oracle over the sampled rows only: a CSR of those rows (copied from the device)."""
    starts, ends = rp_host[rows], rp_host[rows + 1]
    srp = np.zeros(rows.size + 1, np.int64)
    np.cumsum(ends - starts, out=srp[1:])
    idx = np.concatenate([np.arange(a, b) for a, b in zip(starts, ends)]) if srp[-1] else np.zeros(0, np.int64)
    it = torch.from_numpy(idx).cuda()
    S = matgen.HostCSR(srp, col[it].cpu().numpy(), val[it].cpu().double().numpy(), rows.size, x.size)
    return oracle.spmv_csr(S, x, alpha, beta, y_rows, with_bound=True)


def test_full_size_rmat27_sampled(sp):
    """configs[4]: R-MAT scale 27 on one GPU (int64 row_ptr), CSR / merge / CSR5; the
    oracle on ~20K sampled rows (random, hubs, the head and the empty tail)."""
    from matgen import gpu
    free, total = torch.cuda.mem_get_info()
    if free < 120e9:
        pytest.skip(f"needs ~120 GB of device memory, {free / 1e9:.0f} GB free")
    seed = matgen.SEEDS["rmat27"]
    g = gpu.DeviceRMAT(27, 16, seed)
    n = g.n
    col = g.col()
    for kind, exact in (("f64", False), ("int", True)):
        val = g.values(kind=kind, dtype=torch.float64)
        dA = sp.CSR(g.row_ptr, col, val, (n, n))
        assert dA.row_ptr.dtype == torch.int64 and dA.nnz > 2e9
        rp_host = g.row_ptr.cpu().numpy()
        rows = _sample_rows(rp_host, n, 20000, 27)
        x = gpu.vector(n, seed, 1, kind)
        y = gpu.vector(n, seed, 2, kind)
        xh = x.cpu().numpy()
        ref, bound = _rows_ref(rp_host, col, val, rows, xh, 1.0, 1.0, y.cpu().numpy()[rows])
        rows_t = torch.from_numpy(rows).cuda()
        for fmt in ("csr", "merge", "csr5"):
            out = _run(sp, dA, fmt, 1.0, x, 1.0, y)[rows_t].cpu().numpy()
            if exact:
                assert np.array_equal(out, ref), fmt
            else:
                ok, ratio, nbad = oracle.check_tolerance(out, ref, bound, 1e-12)
                assert ok, (fmt, nbad, ratio)
        del dA, val
        torch.cuda.empty_cache()
    g.release()


@pytest.mark.parametrize("seed", [101, 202, 303])
@pytest.mark.parametrize("dtype", [torch.float64, torch.float32], ids=["f64", "f32"])
def test_dynamic_csr_random_shapes(sp, seed, dtype):
    """Randomized shapes at the CSR-vector dynamic-scheduling size (2M rows): a mix of empty
    runs, short rows, rows just over the group width, 40..300-long rows and rows past the
    chunk threshold (A25), in random order -- CSR (and CSR5 / merge on the same matrix)
    within the bound on every row, beta = 0.75."""
    rng = np.random.default_rng(seed)
    n = 2_000_000
    kind = rng.choice(5, size=n, p=[0.45, 0.35, 0.12, 0.0795, 0.0005])
    lens = np.select([kind == 0, kind == 1, kind == 2, kind == 3, kind == 4],
                     [0, rng.integers(1, 17, n), rng.integers(17, 40, n), rng.integers(40, 301, n),
                      rng.integers(1025, 20000, n)])
    k = "f64" if dtype == torch.float64 else "f32"
    A = matgen.from_lengths(lens, 3_000_000, seed=seed, kind=k)
    dA = sp.CSR.from_host(A, dtype=dtype)
    x = matgen.vector(A.n_cols, seed, 1, k)
    y = matgen.vector(A.n_rows, seed, 2, k)
    ref, bound = oracle.spmv_csr(A, x, 1.25, 0.75, y, with_bound=True)
    xd = torch.from_numpy(x).cuda().to(dtype)
    yd0 = torch.from_numpy(y).cuda().to(dtype)
    for fmt in ("csr", "csr5", "merge"):
        out = _run(sp, dA, fmt, 1.25, xd, 0.75, yd0).cpu().double().numpy()
        ok, ratio, nbad = oracle.check_tolerance(out, ref, bound, 1e-12 if dtype == torch.float64 else 1e-5)
        assert ok, (fmt, nbad, ratio)
