"""A30 hot x columns through the real kernels: a handle that packs its hot columns'
x entries densely (forced with hot_x = K, any matrix) must (1) choose exactly the
oracle's hot set, (2) export the same column arrays as a plain handle (decoded), and
(3) produce the same SpMV: within the bound against the oracle, bit-exact in the
integer regime, and bit-identical to the plain handle (same values, same order)."""
import numpy as np
import pytest
import torch

import matgen
import oracle

pytestmark = pytest.mark.gpu

FORMATS = ("coo", "ell", "csr", "hyb", "merge", "csr5")
COL_ARRAYS = ("col", "ell_col", "hyb_coo_col")


@pytest.fixture(scope="module")
def sp():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_nisassvs18_b200 as pkg
    return pkg


def _case(name, kind="f64"):
    rng = np.random.default_rng(30)
    if name == "rmat12":
        return matgen.rmat(12, seed=31, kind=kind)
    if name == "rmat15":
        return matgen.rmat(15, seed=32, kind=kind)
    if name == "lap64":
        return matgen.laplacian5(64, kind=kind)
    if name == "long_row":
        lens = rng.integers(1, 6, 20000)
        lens[7777] = 15000
        return matgen.from_lengths(lens, 20000, seed=33, kind=kind)
    lens = np.where(rng.random(30000) < 0.02, rng.integers(1, 9, 30000), 0)
    return matgen.from_lengths(lens, 30000, seed=34, kind=kind)


def _export_cols(h, sp):
    out = {}
    for a in COL_ARRAYS:
        try:
            out[a] = h.export(a)
        except sp.SpmvError:
            pass
    return out


@pytest.mark.parametrize("K", [1, 64, 3000, 10 ** 9])
@pytest.mark.parametrize("name", ["rmat12", "rmat15", "lap64", "long_row", "sparse"])
@pytest.mark.parametrize("fmt", FORMATS)
def test_hot_columns_parity(sp, fmt, name, K):
    A = _case(name)
    dA = sp.CSR.from_host(A)
    try:
        plain = sp.convert(dA, fmt, hot_x=-1)
    except sp.SpmvError as e:
        assert fmt in ("ell", "hyb") and e.status == 3
        pytest.skip("ELL/HYB infeasible (A4)")
    h = sp.convert(dA, fmt, hot_x=K)
    hot = oracle.hot_columns(A, K)
    assert h.info()["hot_cols"] == hot.size and plain.info()["hot_cols"] == 0
    assert np.array_equal(h.export("hot_cols"), hot)
    pe, he = _export_cols(plain, sp), _export_cols(h, sp)
    assert pe.keys() == he.keys() and all(np.array_equal(pe[k], he[k]) for k in pe)
    x = matgen.vector(A.n_cols, 35, 1)
    y0 = matgen.vector(A.n_rows, 35, 2)
    ref, bound = oracle.spmv_csr(A, x, 1.5, -0.5, y0, with_bound=True)
    xd = torch.from_numpy(x).cuda()
    y1, y2 = torch.from_numpy(y0).cuda(), torch.from_numpy(y0).cuda()
    plain.run(1.5, xd, -0.5, y1)
    h.run(1.5, xd, -0.5, y2)
    torch.cuda.synchronize()
    assert torch.equal(y1, y2)
    assert oracle.check_tolerance(y2.cpu().numpy(), ref, bound, 1e-12)[0]


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32], ids=["f64", "f32"])
@pytest.mark.parametrize("fmt", FORMATS)
def test_hot_columns_integer_regime(sp, fmt, dtype):
    A = _case("rmat15", "int")
    dA = sp.CSR.from_host(A, dtype=dtype)
    try:
        h = sp.convert(dA, fmt, hot_x=500)
    except sp.SpmvError as e:
        assert fmt in ("ell", "hyb") and e.status == 3
        pytest.skip("ELL/HYB infeasible (A4)")
    assert h.info()["hot_cols"] > 0
    x = matgen.vector(A.n_cols, 36, 1, "int")
    y0 = matgen.vector(A.n_rows, 36, 2, "int")
    ref = oracle.spmv_csr(A, x, 2.0, -1.0, y0)
    yd = torch.from_numpy(y0).cuda().to(dtype)
    h.run(2.0, torch.from_numpy(x).cuda().to(dtype), -1.0, yd)
    torch.cuda.synchronize()
    assert np.array_equal(yd.cpu().double().numpy(), ref)


def test_hot_columns_alias_and_graph(sp):
    """No hot columns when the handle aliases the caller's column array; the per-run pack
    is captured in a CUDA graph and replays bit-identically."""
    A = _case("rmat15")
    dA = sp.CSR.from_host(A)
    assert sp.convert(dA, "csr", alias_input=1, hot_x=100).info()["hot_cols"] == 0
    h = sp.convert(dA, "csr5", hot_x=100)
    x = torch.from_numpy(matgen.vector(A.n_cols, 37, 1)).cuda()
    y = torch.zeros(A.n_rows, dtype=torch.float64, device="cuda")
    h.run(1.0, x, 0.0, y)
    ref = y.clone()
    g = torch.cuda.CUDAGraph()
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        with torch.cuda.graph(g):
            h.run(1.0, x, 0.0, y)
    y.zero_()
    g.replay()
    torch.cuda.synchronize()
    assert torch.equal(y, ref)


def test_hot_columns_auto(sp):
    """Auto mode: R-MAT 25 (x = 268 MB > 2 x L2) gets hot columns and the same SpMV bits as
    without; R-MAT 24 (x ~ L2) and the Laplacian (no hot columns) do not."""
    from matgen import gpu
    for scale, want in ((24, False), (25, True)):
        rp, col, val = gpu.rmat(scale, seed=matgen.SEEDS["rmat24"])
        n = rp.numel() - 1
        dA = sp.CSR(rp.to(torch.int32), col, val, (n, n))
        h = sp.convert(dA, "csr5")
        assert (h.info()["hot_cols"] > 10 ** 6) == want, scale
        if want:
            plain = sp.convert(dA, "csr5", hot_x=-1)
            x = gpu.vector(n, 38, 1)
            y1, y2 = gpu.vector(n, 38, 2), gpu.vector(n, 38, 2)
            h.run(1.0, x, 1.0, y1)
            plain.run(1.0, x, 1.0, y2)
            torch.cuda.synchronize()
            assert torch.equal(y1, y2)
        del h, dA, rp, col, val
        torch.cuda.empty_cache()
    L = sp.CSR.from_host(matgen.laplacian5(4096))
    assert sp.convert(L, "csr5").info()["hot_cols"] == 0
