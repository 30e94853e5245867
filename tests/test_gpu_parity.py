"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Bars (north_star): conversions, partitions and integer features
bit-exact; fp64 |y - y_ref| <= 1e-12 * bound, fp32 1e-5 * bound, with
bound_i = |alpha| sum_j |a_ij||x_j| + |beta||y_i|; the integer-exact regime (P5)
bit-exact in every format.
"""
import numpy as np
import pytest
import torch

import matgen
import oracle

pytestmark = pytest.mark.gpu

ALPHA_BETA = [(1.0, 0.0), (1.5, -0.5), (0.0, 2.0), (-1.0, 1.0)]
ALL_FORMATS = ("coo", "ell", "csr", "hyb", "merge", "csr5", "csr_scalar")
TOL = {torch.float64: 1e-12, torch.float32: 1e-5}
KIND = {torch.float64: "f64", torch.float32: "f32"}


@pytest.fixture(scope="module")
def sp():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_nisassvs18_b200 as pkg
    return pkg


def _lens_matrix(lens, n_cols, seed, kind="f64"):
    return matgen.from_lengths(np.asarray(lens, np.int64), n_cols, seed=seed, kind=kind)


def edge_cases(kind="f64"):
    """Edge suite of SURVEY §4 T2 (shapes, empty rows, long rows, tile boundaries)."""
    rng = np.random.default_rng(1234)
    cases = {}
    cases["empty0x0"] = matgen.HostCSR(np.zeros(1, np.int64), np.zeros(0, np.int32), np.zeros(0), 0, 0)
    cases["1x1"] = _lens_matrix([1], 1, 1, kind)
    cases["dense_row_1x5000"] = _lens_matrix([5000], 5000, 2, kind)
    cases["col_n_x_1"] = _lens_matrix(np.ones(3000, np.int64), 1, 3, kind)
    cases["rect_3x7"] = _lens_matrix([2, 7, 0], 7, 4, kind)
    cases["rect_7x3"] = _lens_matrix([1, 0, 3, 2, 0, 0, 1], 3, 5, kind)
    cases["nnz0_rows5"] = matgen.HostCSR(np.zeros(6, np.int64), np.zeros(0, np.int32), np.zeros(0), 5, 9)
    lens = rng.integers(0, 12, 5000)
    lens[:37] = 0                      # leading empty rows
    lens[-53:] = 0                     # trailing empty rows
    lens[1000:1400] = 0                # a run of empty rows
    cases["empty_runs"] = _lens_matrix(lens, 4000, 6, kind)
    lens = rng.integers(1, 6, 20000)
    lens[7777] = 100000                # one long row amid short ones
    cases["long_row"] = _lens_matrix(lens, 200000, 7, kind)
    # rows exactly at / around CSR5 tile (32*sigma) and merge/COO CTA (2048) boundaries
    cases["tile_bounds"] = _lens_matrix([511, 512, 513, 2047, 2048, 2049, 1, 0, 4095, 4096, 4097] * 7, 9000, 8, kind)
    cases["u2048"] = matgen.uniform_fixed(2048, 2048, 16, kind=kind)          # configs[0]
    cases["lap37"] = matgen.laplacian5(37, kind=kind)
    cases["lap64"] = matgen.laplacian5(64, kind=kind)
    cases["rmat12"] = matgen.rmat(12, seed=12, kind=kind)
    cases["rmat15"] = matgen.rmat(15, seed=15, kind=kind)
    cases["rgg12"] = matgen.rgg(12, seed=12, kind=kind)      # the paper's rgg_n_2_k_s0 recipe
    cases["banded"] = matgen.window(3000, 3000, 9, 0.6, seed=9, mode=0, kind=kind)
    cases["blockdiag"] = matgen.window(2500, 4000, 64, 0.8, seed=10, mode=1, kind=kind)
    cases["poisson_rect"] = _lens_matrix(rng.poisson(20, 4000), 1500, 11, kind)
    # mostly empty rows: COO / CSR5 / merge tiles spanning thousands of rows, with rows
    # that have nonzeros past the tiles' 128-row output windows
    lens = np.where(rng.random(60000) < 0.01, rng.integers(1, 9, 60000), 0)
    cases["sparse_rows"] = _lens_matrix(lens, 60000, 13, kind)
    # the same stretches between dense blocks (mean ~15: CSR5 sigma = 16, CSR W = 16)
    lens = np.where(rng.random(60000) < 0.01, rng.integers(1, 9, 60000), 0)
    lens[:20000] = 30
    lens[40000:50000] = 30
    cases["mixed_sparse"] = _lens_matrix(lens, 60000, 14, kind)
    zero = _lens_matrix(rng.integers(0, 9, 700), 700, 12, kind)
    cases["all_zero_vals"] = matgen.HostCSR(zero.row_ptr, zero.col, np.zeros(zero.nnz), zero.n_rows, zero.n_cols)
    return cases


_CASES = {}


def case(name, kind):
    if kind not in _CASES:
        _CASES[kind] = edge_cases(kind)
    return _CASES[kind][name]


CASE_NAMES = ["empty0x0", "1x1", "dense_row_1x5000", "col_n_x_1", "rect_3x7", "rect_7x3", "nnz0_rows5",
              "empty_runs", "long_row", "tile_bounds", "u2048", "lap37", "lap64", "rmat12", "rmat15", "rgg12",
              "banded", "blockdiag", "poisson_rect", "all_zero_vals", "sparse_rows", "mixed_sparse"]


def _guard(A, V):
    """spmv.h: default guard max(8x the CSR bytes, 64 MiB) (free memory is not binding here)."""
    return max(8 * (A.nnz * (4 + V) + (A.n_rows + 1) * 4), 64 << 20)


def ell_expected_infeasible(A, dtype):
    K, ld = oracle.ell_dims(A)
    V = 8 if dtype == torch.float64 else 4
    return K * ld * (4 + V) > _guard(A, V)


def hyb_expected_infeasible(A, dtype, rule="ceil"):
    Kh = oracle.hyb_width(A, rule)
    ld = oracle.ell_dims(A)[1]
    V = 8 if dtype == torch.float64 else 4
    ncoo = oracle.lib().ora_hyb_coo_nnz(A.n_rows, A.row_ptr.ctypes.data, Kh)
    return Kh * ld * (4 + V) + ncoo * (8 + V) > _guard(A, V)


def expected_infeasible(A, fmt, dtype):
    return ((fmt == "ell" and ell_expected_infeasible(A, dtype)) or
            (fmt == "hyb" and hyb_expected_infeasible(A, dtype)))


def to_dev(sp, A, dtype):
    return sp.CSR.from_host(A, dtype=dtype)


def run_format(sp, A, dA, fmt, dtype, alpha, beta, x, y0, **opts):
    h = sp.convert(dA, fmt, **opts)
    xd = torch.from_numpy(x).cuda().to(dtype)
    if beta == 0.0:
        yd = torch.full((A.n_rows,), float("nan"), dtype=dtype, device="cuda")   # must not be read
    else:
        yd = torch.from_numpy(y0).cuda().to(dtype)
    h.run(alpha, xd, beta, yd)
    torch.cuda.synchronize()
    out = yd.cpu().double().numpy()
    return h, out


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32], ids=["f64", "f32"])
@pytest.mark.parametrize("fmt", ALL_FORMATS)
@pytest.mark.parametrize("name", CASE_NAMES)
def test_spmv_parity(sp, name, fmt, dtype):
    A = case(name, KIND[dtype])
    dA = to_dev(sp, A, dtype)
    x = matgen.vector(A.n_cols, 77, 1, KIND[dtype])
    y0 = matgen.vector(A.n_rows, 77, 2, KIND[dtype])
    if expected_infeasible(A, fmt, dtype):
        with pytest.raises(sp.SpmvError) as e:
            sp.convert(dA, fmt)
        assert e.value.status == 3
        return
    for alpha, beta in ALPHA_BETA:
        ref, bound = oracle.spmv_csr(A, x, alpha, beta, y0, with_bound=True)
        h, out = run_format(sp, A, dA, fmt, dtype, alpha, beta, x, y0)
        ok, ratio, nbad = oracle.check_tolerance(out, ref, bound, TOL[dtype])
        assert ok, f"{name}/{fmt}/{dtype} a={alpha} b={beta}: {nbad} bad rows, max ratio {ratio}"
        h.destroy()


INT_CASES = ["rmat15", "lap64", "long_row", "tile_bounds", "empty_runs", "u2048", "poisson_rect", "dense_row_1x5000",
             "sparse_rows", "mixed_sparse"]


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32], ids=["f64", "f32"])
@pytest.mark.parametrize("fmt", ALL_FORMATS)
@pytest.mark.parametrize("name", INT_CASES)
def test_integer_regime_bit_exact(sp, name, fmt, dtype):
    """P5: a, x in {+-1, +-2}, small integer y, integer alpha/beta: any summation order gives
    the same bits, so every format must match the oracle exactly."""
    base = case(name, "f64")
    A = matgen.set_values(base, 991, "int")
    dA = to_dev(sp, A, dtype)
    if expected_infeasible(A, fmt, dtype):
        pytest.skip("infeasible (A4)")
    x = matgen.vector(A.n_cols, 5, 1, "int")
    y0 = np.round(matgen.vector(A.n_rows, 5, 2, "f64") * 8)
    for alpha, beta in [(1.0, 0.0), (2.0, -1.0), (-1.0, 2.0), (0.0, -2.0)]:
        ref = oracle.spmv_csr(A, x, alpha, beta, y0)
        h, out = run_format(sp, A, dA, fmt, dtype, alpha, beta, x, y0)
        assert np.array_equal(out, ref), f"{name}/{fmt}: not bit-exact (alpha={alpha}, beta={beta})"
        h.destroy()


# ------------------------------------------------------------------ conversions

CONV_CASES = ["u2048", "rmat12", "rmat15", "empty_runs", "tile_bounds", "lap64", "rect_7x3", "nnz0_rows5",
              "long_row", "banded"]


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32], ids=["f64", "f32"])
@pytest.mark.parametrize("name", CONV_CASES)
def test_conversions_bit_exact(sp, name, dtype):
    A = case(name, KIND[dtype])
    dA = to_dev(sp, A, dtype)
    npv = np.float64 if dtype == torch.float64 else np.float32
    vb = 8 if dtype == torch.float64 else 4
    # CSR copies the input
    h = sp.convert(dA, "csr")
    assert np.array_equal(h.export("row_ptr").astype(np.int64), A.row_ptr)
    assert np.array_equal(h.export("col"), A.col)
    assert np.array_equal(h.export("val"), A.val.astype(npv))
    # COO
    h = sp.convert(dA, "coo")
    assert np.array_equal(h.export("coo_row"), oracle.csr2coo(A))
    # ELL (A3)
    if not ell_expected_infeasible(A, dtype):
        h = sp.convert(dA, "ell")
        e = oracle.csr2ell(A)
        assert h.info()["ell_width"] == e["K"] and h.info()["ell_ld"] == e["ld"]
        assert np.array_equal(h.export("ell_col"), e["col"])
        assert np.array_equal(h.export("ell_val"), e["val"].astype(npv))
    # HYB (A1/A2) with each width rule
    for rule in ("ceil", "floor", "cusp"):
        if hyb_expected_infeasible(A, dtype, rule):
            continue
        h = sp.convert(dA, "hyb", hyb_rule=rule)
        e = oracle.csr2hyb(A, rule)
        assert h.info()["ell_width"] == e["K"], rule
        assert np.array_equal(h.export("ell_col"), e["ell_col"])
        assert np.array_equal(h.export("ell_val"), e["ell_val"].astype(npv))
        assert np.array_equal(h.export("coo_row"), e["coo_row"])
        assert np.array_equal(h.export("hyb_coo_col"), e["coo_col"])
        assert np.array_equal(h.export("hyb_coo_val"), e["coo_val"].astype(npv))
    # merge-path coordinates (A7)
    h = sp.convert(dA, "merge")
    T = h.info()["merge_items"]
    cr, cn = oracle.merge_coords(A, T)
    assert np.array_equal(h.export("merge_coord_row"), cr)
    assert np.array_equal(h.export("merge_coord_nz"), cn)
    cls = oracle.merge_class(A, T)
    assert np.array_equal(h.export("merge_tile_class"), cls)
    assert np.array_equal(h.export("merge_tile_order"), np.argsort(1 - cls.astype(np.int64), kind="stable"))
    # CSR5 (A6), default sigma and each legal sigma
    for sigma in (None, 4, 8, 12, 16):
        h = sp.convert(dA, "csr5", csr5_sigma=sigma or 0)
        e = oracle.csr5_encode(A, val_bytes=vb, sigma=sigma)
        assert h.info()["csr5_sigma"] == e["sigma"]
        assert np.array_equal(h.export("csr5_tile_ptr"), e["tile_ptr"])
        assert np.array_equal(h.export("csr5_row_lo"), e["row_lo"])
        assert np.array_equal(h.export("csr5_tile_desc"), e["tile_desc"])
        assert np.array_equal(h.export("csr5_map_off"), e["map_off"])
        assert np.array_equal(h.export("csr5_seg_map"), e["seg_map"])
        assert np.array_equal(h.export("col"), e["col_perm"])
        assert np.array_equal(h.export("val"), e["val_perm"].astype(npv))


# ------------------------------------------------------------------ features

@pytest.mark.parametrize("name", CASE_NAMES)
def test_features_bit_exact(sp, name):
    A = case(name, "f64")
    f = sp.features(to_dev(sp, A, torch.float64))
    fo = oracle.features(A)
    for k, v in fo.items():
        assert f[k] == v, (name, k, f[k], v)


def test_features_lap4096_full_size(sp):
    """configs[1] at full size: features equal the App. B closed forms via the oracle."""
    A = matgen.laplacian5(4096)
    f = sp.features(to_dev(sp, A, torch.float64))
    fo = oracle.features(A)
    for k, v in fo.items():
        assert f[k] == v, k


def test_int64_row_ptr_input(sp):
    A = case("rmat12", "f64")
    dA = sp.CSR.from_host(A, dtype=torch.float64, ptr_dtype=torch.int64)
    f = sp.features(dA)
    assert f["nnzb_tot"] == oracle.features(A)["nnzb_tot"]
    x = matgen.vector(A.n_cols, 3, 1)
    ref, bound = oracle.spmv_csr(A, x, 1.0, 0.0, None, with_bound=True)
    for fmt in ("csr", "merge", "csr5", "coo"):
        h, out = run_format(sp, A, dA, fmt, torch.float64, 1.0, 0.0, x, None)
        assert oracle.check_tolerance(out, ref, bound, 1e-12)[0], fmt


# ------------------------------------------------------------------ partition

def square_cases():
    rng = np.random.default_rng(99)
    lens = rng.integers(0, 12, 5000)
    lens[:37] = 0
    lens[1000:1400] = 0
    lens[-53:] = 0
    out = {"empty_runs_sq": _lens_matrix(lens, 5000, 21)}
    lens = rng.integers(1, 6, 20000)
    lens[7777] = 15000
    out["long_row_sq"] = _lens_matrix(lens, 20000, 22)
    return out


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("name", ["rmat15", "empty_runs_sq", "lap64", "long_row_sq", "u2048", "banded"])
def test_partition_and_remap_bit_exact(sp, name, P):
    """Remap needs a square matrix (x is owned in the row ranges of y)."""
    A = square_cases()[name] if name.endswith("_sq") else case(name, "f64")
    dA = to_dev(sp, A, torch.float64)
    splits = sp.partition(dA, P)
    assert np.array_equal(splits, oracle.partition(A, P))
    for part in range(P):
        shard, S = sp.slice_remap(dA, splits, part)
        assert S == oracle.partition_slot(splits)
        rp, col, val = oracle.slice_remap(A, splits, part)
        assert np.array_equal(shard.row_ptr.cpu().numpy().astype(np.int64), rp)
        assert np.array_equal(shard.col.cpu().numpy(), col)
        assert np.array_equal(shard.val.cpu().numpy(), val)


# ------------------------------------------------------------------ errors, semantics

def test_not_canonical_rejected(sp):
    A = case("u2048", "f64")
    bad_cols = [A.col.copy() for _ in range(3)]
    bad_cols[0][[3, 4]] = bad_cols[0][[4, 3]]              # unsorted within a row
    bad_cols[1][5] = bad_cols[1][4]                         # duplicate
    bad_cols[2][9] = A.n_cols                               # out of range
    for c in bad_cols:
        B = matgen.HostCSR(A.row_ptr, c, A.val, A.n_rows, A.n_cols)
        dB = to_dev(sp, B, torch.float64)
        with pytest.raises(sp.SpmvError) as e:
            sp.features(dB)
        assert e.value.status == 2
        for fmt in ALL_FORMATS:
            with pytest.raises(sp.SpmvError) as e:
                sp.convert(dB, fmt)
            assert e.value.status == 2
    rp = A.row_ptr.copy()
    rp[10], rp[11] = rp[11], rp[10]                         # non-monotone row_ptr
    dB = to_dev(sp, matgen.HostCSR(rp, A.col, A.val, A.n_rows, A.n_cols), torch.float64)
    with pytest.raises(sp.SpmvError) as e:
        sp.convert(dB, "csr")
    assert e.value.status == 2


def test_ell_size_guard(sp):
    A = case("rmat15", "f64")
    with pytest.raises(sp.SpmvError) as e:
        sp.convert(to_dev(sp, A, torch.float64), "ell")
    assert e.value.status == 3
    with pytest.raises(sp.SpmvError) as e:
        sp.convert(to_dev(sp, case("u2048", "f64"), torch.float64), "ell", max_bytes=1000)
    assert e.value.status == 3


def test_x_y_overlap_rejected(sp):
    A = matgen.uniform_fixed(64, 64, 4)
    h = sp.convert(to_dev(sp, A, torch.float64), "csr")
    buf = torch.zeros(64, dtype=torch.float64, device="cuda")
    with pytest.raises(sp.SpmvError) as e:
        h.run(1.0, buf, 0.0, buf)
    assert e.value.status == 1


@pytest.mark.parametrize("fmt", ALL_FORMATS)
def test_deterministic_bits(sp, fmt):
    A = case("rmat15", "f64")
    dA = to_dev(sp, A, torch.float64)
    if fmt == "ell":
        pytest.skip("ELL infeasible on R-MAT")
    x = matgen.vector(A.n_cols, 1, 1)
    outs = []
    for _ in range(3):
        h, out = run_format(sp, A, dA, fmt, torch.float64, 1.0, 0.0, x, None)
        outs.append(out)
    assert all(np.array_equal(outs[0], o) for o in outs[1:])


@pytest.mark.parametrize("fmt", ("csr", "merge", "csr5", "coo", "hyb"))
def test_run_host_end_to_end(sp, fmt):
    A = case("rmat12", "f64")
    h = sp.convert(to_dev(sp, A, torch.float64), fmt)
    x = matgen.vector(A.n_cols, 4, 1)
    y = matgen.vector(A.n_rows, 4, 2)
    ref, bound = oracle.spmv_csr(A, x, 2.0, 0.5, y, with_bound=True)
    out = y.copy()
    h.run_host(2.0, x, 0.5, out)
    assert oracle.check_tolerance(out, ref, bound, 1e-12)[0]


@pytest.mark.parametrize("beta", [0.5, 0.0], ids=["beta", "beta0"])
@pytest.mark.parametrize("dtype", [torch.float64, torch.float32], ids=["f64", "f32"])
@pytest.mark.parametrize("name", ["rmat12", "lap37", "sparse_rows", "nnz0_rows5"])
def test_run_host_multi(sp, name, dtype, beta):
    """spmv_run_host_multi (x and y_in cross PCIe once for all formats): every result
    is bit-identical to the handle's own spmv_run on device buffers and within the bound
    of the oracle; y_in is left untouched (and not read when beta == 0)."""
    kind = "f64" if dtype == torch.float64 else "f32"
    A = case(name, kind)
    dA = to_dev(sp, A, dtype)
    hs, fmts = [], []
    for f in sp.PAPER_FORMATS:
        try:
            hs.append(sp.convert(dA, f))
            fmts.append(f)
        except sp.SpmvError as e:
            assert e.status == 3
    npd = np.float64 if dtype == torch.float64 else np.float32
    x = matgen.vector(A.n_cols, 6, 1).astype(npd)
    y0 = matgen.vector(A.n_rows, 6, 2).astype(npd)
    y_in = None if beta == 0.0 else y0.copy()
    outs = [np.full(A.n_rows, np.nan, npd) for _ in hs]
    sp.run_host_multi(hs, 1.5, x, beta, y_in, outs)
    if y_in is not None:
        assert np.array_equal(y_in, y0)
    ref, bound = oracle.spmv_csr(A, x.astype(np.float64), 1.5, beta, y0.astype(np.float64), with_bound=True)
    tol = 1e-12 if dtype == torch.float64 else 1e-5
    xd = torch.from_numpy(x).cuda()
    for f, h, out in zip(fmts, hs, outs):
        yd = torch.from_numpy(y0).cuda() if beta != 0.0 else torch.full((A.n_rows,), float("nan"), dtype=dtype, device="cuda")
        h.run(1.5, xd, beta, yd)
        torch.cuda.synchronize()
        assert np.array_equal(yd.cpu().numpy(), out), f
        assert oracle.check_tolerance(out.astype(np.float64), ref, bound, tol)[0], f


def test_run_host_multi_errors(sp):
    A, B = case("rmat12", "f64"), case("lap37", "f64")
    hA = sp.convert(to_dev(sp, A, torch.float64), "csr")
    hB = sp.convert(to_dev(sp, B, torch.float64), "csr")
    x = matgen.vector(A.n_cols, 1, 1)
    y = matgen.vector(A.n_rows, 1, 2)
    out = [np.zeros(A.n_rows), np.zeros(A.n_rows)]
    for hs in ([hA, hB], [hA, hA]):
        with pytest.raises(sp.SpmvError) as e:
            sp.run_host_multi(hs, 1.0, x, 1.0, y, out)
        assert e.value.status == 1
    with pytest.raises(sp.SpmvError) as e:                 # beta != 0 needs y_in
        sp.run_host_multi([hA], 1.0, x, 1.0, None, out[:1])
    assert e.value.status == 1


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32], ids=["f64", "f32"])
@pytest.mark.parametrize("fmt", ("csr", "merge", "csr5", "coo", "hyb", "ell"))
def test_long_sequential_stress(sp, fmt, dtype):
    """P9: positive non-dyadic values (0.1), x = 1, rows up to 1e6: the bound must hold
    (catches long sequential fp32/fp64 accumulation chains, A13).  CSR-scalar is exempt:
    one thread per row is the variant the paper describes, not a label."""
    lens = np.array([1_000_000, 3, 30_000, 1, 250_000], np.int64)
    n_cols = 1_000_000
    rp = np.zeros(lens.size + 1, np.int64)
    np.cumsum(lens, out=rp[1:])
    col = np.concatenate([np.arange(l, dtype=np.int32) for l in lens])
    A = matgen.HostCSR(rp, col, np.full(col.size, 0.1), lens.size, n_cols)
    if dtype == torch.float32:
        A = matgen.HostCSR(rp, col, np.full(col.size, float(np.float32(0.1))), lens.size, n_cols)
    x = np.ones(n_cols)
    ref, bound = oracle.spmv_csr(A, x, 1.0, 0.0, None, with_bound=True)
    opts = {"max_bytes": 1 << 31} if fmt == "ell" else {}
    h, out = run_format(sp, A, to_dev(sp, A, dtype), fmt, dtype, 1.0, 0.0, x, None, **opts)
    ok, ratio, _ = oracle.check_tolerance(out, ref, bound, TOL[dtype])
    assert ok, ratio


# ------------------------------------------------------------------ full-size configs

@pytest.mark.parametrize("fmt", ("coo", "ell", "csr", "hyb", "merge", "csr5"))
def test_full_size_lap4096(sp, fmt):
    """BASELINE configs[1] at full size, in the launch configuration bench.py times:
    every row against the oracle (fp64, alpha=1, beta=1 with uniform x, y)."""
    A = _lap4096()
    x = matgen.vector(A.n_cols, matgen.SEEDS["lap4096"], 1)
    y0 = matgen.vector(A.n_rows, matgen.SEEDS["lap4096"], 2)
    ref, bound = _lap_ref(A, x, y0)
    dA = _lap4096_dev(sp)
    h, out = run_format(sp, A, dA, fmt, torch.float64, 1.0, 1.0, x, y0)
    ok, ratio, nbad = oracle.check_tolerance(out, ref, bound, 1e-12)
    assert ok, (fmt, nbad, ratio)


_BIG = {}


def _lap4096():
    if "lap" not in _BIG:
        _BIG["lap"] = matgen.laplacian5(4096)
    return _BIG["lap"]


def _lap4096_dev(sp):
    if "lapd" not in _BIG:
        _BIG["lapd"] = sp.CSR.from_host(_lap4096(), dtype=torch.float64)
    return _BIG["lapd"]


def _lap_ref(A, x, y0):
    if "lapref" not in _BIG:
        _BIG["lapref"] = oracle.spmv_csr(A, x, 1.0, 1.0, y0, with_bound=True)
    return _BIG["lapref"]


I64_CASES = ["rmat15", "empty_runs", "long_row", "tile_bounds", "u2048", "nnz0_rows5", "rect_7x3"]


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32], ids=["f64", "f32"])
@pytest.mark.parametrize("fmt", ALL_FORMATS)
@pytest.mark.parametrize("name", I64_CASES)
def test_index64_path(sp, name, fmt, dtype):
    """A17: handles with int64 row pointers/offsets (the > 2^31-nonzero path of configs[4]),
    forced on small matrices with convert option index64=1."""
    A = case(name, KIND[dtype])
    dA = to_dev(sp, A, dtype)
    if expected_infeasible(A, fmt, dtype):
        pytest.skip("infeasible (A4)")
    x = matgen.vector(A.n_cols, 88, 1, KIND[dtype])
    y0 = matgen.vector(A.n_rows, 88, 2, KIND[dtype])
    ref, bound = oracle.spmv_csr(A, x, 1.5, -0.5, y0, with_bound=True)
    h, out = run_format(sp, A, dA, fmt, dtype, 1.5, -0.5, x, y0, index64=1)
    if fmt in ("csr", "csr_scalar", "merge", "csr5"):
        assert h.info()["ptr_type"] == 1
    ok, ratio, nbad = oracle.check_tolerance(out, ref, bound, TOL[dtype])
    assert ok, (nbad, ratio)
    if fmt == "merge":
        cr, cn = oracle.merge_coords(A, h.info()["merge_items"])
        assert np.array_equal(h.export("merge_coord_nz"), cn)
        assert np.array_equal(h.export("merge_tile_class"), oracle.merge_class(A, h.info()["merge_items"]))
    if fmt == "csr5":
        e = oracle.csr5_encode(A, val_bytes=8 if dtype == torch.float64 else 4)
        assert np.array_equal(h.export("csr5_tile_desc"), e["tile_desc"])
        assert np.array_equal(h.export("row_ptr"), A.row_ptr)


@pytest.mark.parametrize("name", ["rmat15", "empty_runs"])
@pytest.mark.parametrize("offset", [0, 1, 3])
@pytest.mark.parametrize("fmt", ("coo", "csr", "merge", "csr5"))
def test_alias_input_any_alignment(sp, fmt, offset, name):
    """alias_input with col/val slices starting `offset` elements into their buffers: a
    handle that references them must not assume vector alignment (COO copies unless both
    are 32-byte aligned, include/spmv.h; the short-row CSR batch kernel (A29) runs only
    on 32-byte aligned arrays), and results stay within tolerance."""
    A = case(name, "f64")
    dA = to_dev(sp, A, torch.float64)
    cb = torch.zeros(A.nnz + 8, dtype=torch.int32, device="cuda")
    vb = torch.zeros(A.nnz + 8, dtype=torch.float64, device="cuda")
    cb[offset: offset + A.nnz] = dA.col
    vb[offset: offset + A.nnz] = dA.val
    dS = sp.CSR(dA.row_ptr, cb[offset: offset + A.nnz], vb[offset: offset + A.nnz], (A.n_rows, A.n_cols))
    x = matgen.vector(A.n_cols, 78, 1)
    y0 = matgen.vector(A.n_rows, 78, 2)
    ref, bound = oracle.spmv_csr(A, x, 1.5, -0.5, y0, with_bound=True)
    h, out = run_format(sp, A, dS, fmt, torch.float64, 1.5, -0.5, x, y0, alias_input=1)
    ok, ratio, nbad = oracle.check_tolerance(out, ref, bound, TOL[torch.float64])
    assert ok, f"{fmt} offset {offset}: {nbad} bad rows, max ratio {ratio}"
    h.destroy()


# ------------------------------------------------------------------ CSR long-row chunks (A25)

@pytest.mark.parametrize("chunk", [1, 7, 32, 300])
@pytest.mark.parametrize("name", ["dense_row_1x5000", "long_row", "rmat15", "empty_runs", "tile_bounds", "u2048"])
def test_csr_long_row_chunks(sp, name, chunk):
    """CSR with rows longer than 2*chunk split into chunks (one warp each, carries + fix-up):
    chunk arrays equal the oracle's bit for bit, results within tolerance for every
    (alpha, beta), bit-exact in the integer regime."""
    A = case(name, "f64")
    dA = to_dev(sp, A, torch.float64)
    h = sp.convert(dA, "csr", csr_chunk=chunk)
    cr, cl = oracle.csr_chunks(A, chunk)
    assert h.info()["csr_chunks"] == cr.size
    assert np.array_equal(h.export("csr_chunk_row"), cr)
    assert np.array_equal(h.export("csr_chunk_lo"), cl)
    assert h.launches() == (1 + (2 if cr.size else 0) if A.n_rows else 0)
    h.destroy()
    x = matgen.vector(A.n_cols, 79, 1)
    y0 = matgen.vector(A.n_rows, 79, 2)
    for alpha, beta in ALPHA_BETA:
        ref, bound = oracle.spmv_csr(A, x, alpha, beta, y0, with_bound=True)
        h, out = run_format(sp, A, dA, "csr", torch.float64, alpha, beta, x, y0, csr_chunk=chunk)
        ok, ratio, nbad = oracle.check_tolerance(out, ref, bound, TOL[torch.float64])
        assert ok, f"{name} chunk={chunk} a={alpha} b={beta}: {nbad} bad rows, max ratio {ratio}"
        h.destroy()
    Ai = matgen.set_values(A, 991, "int")
    dAi = to_dev(sp, Ai, torch.float32)
    xi = matgen.vector(A.n_cols, 5, 1, "int")
    yi = np.round(matgen.vector(A.n_rows, 5, 2, "f64") * 8)
    ref = oracle.spmv_csr(Ai, xi, 2.0, -1.0, yi)
    h, out = run_format(sp, Ai, dAi, "csr", torch.float32, 2.0, -1.0, xi, yi, csr_chunk=chunk)
    assert np.array_equal(out, ref)
    h.destroy()


def test_csr_chunks_disabled_and_default(sp):
    A = case("dense_row_1x5000", "f64")
    dA = to_dev(sp, A, torch.float64)
    assert sp.convert(dA, "csr", csr_chunk=-1).info()["csr_chunks"] == 0
    assert sp.convert(dA, "csr").info()["csr_chunks"] == oracle.csr_chunks(A, 512)[0].size == 10   # default C = 512
    assert sp.convert(dA, "csr_scalar", csr_chunk=7).info()["csr_chunks"] == 0


# ------------------------------------------------------------------ configs[2] at full size

def _rmat24():
    if "rmat" not in _BIG:
        _BIG["rmat"] = matgen.rmat(24)
    return _BIG["rmat"]


RMAT_FORMATS = ("coo", "csr", "hyb", "merge", "csr5")   # ELL is infeasible (A4)


def test_full_size_rmat24(sp):
    """BASELINE configs[2] (R-MAT scale 24, 2.6e8 nonzeros, 56% empty rows, a 190K-nonzero
    hub row) at full size in bench.py's launch configuration: features bit-exact; fp64
    alpha = beta = 1 within the A16 bound on every row; the integer regime (fp32 storage,
    alpha = 2, beta = -1) bit-exact on every row, for every feasible format."""
    A = _rmat24()
    dA = sp.CSR.from_host(A, dtype=torch.float64)
    f, fo = sp.features(dA), oracle.features(A)
    assert all(f[k] == fo[k] for k in sp.PAPER_FEATURES)
    with pytest.raises(sp.SpmvError) as e:
        sp.convert(dA, "ell")
    assert e.value.status == 3
    x = matgen.vector(A.n_cols, matgen.SEEDS["rmat24"], 1)
    y0 = matgen.vector(A.n_rows, matgen.SEEDS["rmat24"], 2)
    ref, bound = oracle.spmv_csr(A, x, 1.0, 1.0, y0, with_bound=True)
    for fmt in RMAT_FORMATS:
        h, out = run_format(sp, A, dA, fmt, torch.float64, 1.0, 1.0, x, y0)
        ok, ratio, nbad = oracle.check_tolerance(out, ref, bound, 1e-12)
        h.destroy()
        assert ok, (fmt, nbad, ratio)
    del dA, ref, bound
    Ai = matgen.set_values(A, 991, "int")
    dAi = sp.CSR.from_host(Ai, dtype=torch.float32)
    xi = matgen.vector(A.n_cols, 5, 1, "int")
    yi = np.round(matgen.vector(A.n_rows, 5, 2, "f64") * 8)
    refi = oracle.spmv_csr(Ai, xi, 2.0, -1.0, yi)
    for fmt in RMAT_FORMATS:
        h, out = run_format(sp, Ai, dAi, fmt, torch.float32, 2.0, -1.0, xi, yi)
        h.destroy()
        assert np.array_equal(out, refi), fmt


# merge tile classes (A28): the three schedules -- all tiles row-sum (short rows), most
# row-sum with some segmented-sum tiles (short rows + a few long rows), few row-sum tiles
def _merge_class_cases():
    rng = np.random.default_rng(28)
    short = rng.integers(3, 8, 20000)
    mixed = short.copy()
    mixed[[500, 7000, 15000]] = [900, 2500, 300]
    mostly_long = rng.integers(30, 200, 3000)
    return {"all_rowsum": short, "mixed": mixed, "few_rowsum": mostly_long}


@pytest.mark.parametrize("dtype", [torch.float64, torch.float32], ids=["f64", "f32"])
@pytest.mark.parametrize("which", ["all_rowsum", "mixed", "few_rowsum"])
def test_merge_tile_schedules(sp, which, dtype):
    lens = _merge_class_cases()[which]
    A = _lens_matrix(lens, 30000, 2801, KIND[dtype])
    cls = oracle.merge_class(A, 256)
    nl, nt = int(cls.sum()), cls.size
    expect = {"all_rowsum": nl == nt, "mixed": nt > nl and 2 * nl >= nt, "few_rowsum": 2 * nl < nt}[which]
    assert expect, (which, nl, nt)
    dA = to_dev(sp, A, dtype)
    x = matgen.vector(A.n_cols, 28, 1, KIND[dtype])
    y0 = matgen.vector(A.n_rows, 28, 2, KIND[dtype])
    for alpha, beta in ALPHA_BETA:
        ref, bound = oracle.spmv_csr(A, x, alpha, beta, y0, with_bound=True)
        h, out = run_format(sp, A, dA, "merge", dtype, alpha, beta, x, y0)
        assert np.array_equal(h.export("merge_tile_class"), cls)
        ok, ratio, nbad = oracle.check_tolerance(out, ref, bound, TOL[dtype])
        assert ok, (alpha, beta, nbad, ratio)
        h.destroy()


def test_harness_record_cold_l2_and_scalar(sp):
    """The timing/label harness (a16) on one matrix: every format timed hot and cold
    (L2 flushed before each run), labels over six and seven classes,
    each format's y agreeing with CSR's."""
    from paper_conf_ipps_nisassvs18_b200 import harness
    A = _lens_matrix(np.random.default_rng(5).integers(0, 20, 3000), 3000, 55)
    dA = to_dev(sp, A, torch.float64)
    rec = harness.measure_matrix(dA, formats=sp.PAPER_FORMATS + ("csr_scalar",), reps=5, warmup=2, cold_l2=True)
    assert rec["label6"] in sp.PAPER_FORMATS and rec["label7"] in sp.PAPER_FORMATS + ("csr_scalar",)
    assert rec["cold_labels"]["label6"] in sp.PAPER_FORMATS
    for f, r in rec["formats"].items():
        if r.get("status") == "N/A":
            continue
        assert r["agree"] < 1e-12, f
        assert r["cold"]["cold_l2"] and r["cold"]["t_mean_ms"] > 0 and r["t_mean_ms"] > 0


@pytest.mark.parametrize("name", ["lap64", "rmat12", "empty_runs", "big_skewed"])
def test_cuda_graph_capture(sp, name):
    """spmv_run is fully asynchronous and CUDA-graph capturable (include/spmv.h): every
    format captured into a graph (beta = 0) replays bit-identically to the eager run --
    including the CSR dynamic batch scheduler's counter reset (a >= 1.8M-row skewed
    matrix) and the fix-up launches."""
    A = matgen.rmat(21, seed=21) if name == "big_skewed" else case(name, "f64")
    dA = to_dev(sp, A, torch.float64)
    x = torch.from_numpy(matgen.vector(A.n_cols, 91, 1)).cuda()
    fmts = ("csr", "merge", "csr5") if name == "big_skewed" else ("coo", "ell", "csr", "hyb", "merge", "csr5")
    for fmt in fmts:
        try:
            h = sp.convert(dA, fmt)
        except sp.SpmvError as e:
            assert e.status == 3
            continue
        y_eager = torch.full((A.n_rows,), float("nan"), dtype=torch.float64, device="cuda")
        h.run(1.25, x, 0.0, y_eager)
        y_graph = torch.full((A.n_rows,), float("nan"), dtype=torch.float64, device="cuda")
        s = torch.cuda.Stream()
        s.wait_stream(torch.cuda.current_stream())
        with torch.cuda.stream(s):
            h.run(1.25, x, 0.0, y_graph)                       # warm-up on the capture stream
        torch.cuda.current_stream().wait_stream(s)
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            h.run(1.25, x, 0.0, y_graph)
        y_graph.fill_(float("nan"))
        for _ in range(2):
            g.replay()
        torch.cuda.synchronize()
        assert torch.equal(y_graph, y_eager), fmt
        del g
        h.destroy()


_PDL_SCRIPT = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import matgen
import paper_conf_ipps_nisassvs18_b200 as sp
outs = []
for A in (matgen.rmat(21, seed=21), matgen.from_lengths(np.r_[np.ones(3000, np.int64), [40000], np.ones(3000, np.int64)], 50000, seed=3)):
    dA = sp.CSR.from_host(A, dtype=torch.float64)
    h = sp.convert(dA, "csr")
    x = torch.from_numpy(matgen.vector(A.n_cols, 17, 1)).cuda()
    y = torch.from_numpy(matgen.vector(A.n_rows, 17, 2)).cuda()
    h.run(1.5, x, -0.5, y)
    torch.cuda.synchronize()
    outs.append(y.cpu().numpy())
    h.destroy()
np.save(sys.argv[2], np.concatenate(outs))
"""


def test_csr_pdl_matches_serial(sp, tmp_path):
    """A25's launch order -- long-row chunk kernel first, the row kernel a programmatic
    dependent launch beside it -- changes no arithmetic: y is bit-identical to the serial
    order (SPMV_CSR_PDL=0, row kernel then chunks), on R-MAT 21 (dynamic batch scheduler
    + chunks) and a short-row matrix with one 40,000-nonzero row; both within the bound."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    res = {}
    for pdl in ("1", "0"):
        out = tmp_path / f"y_pdl{pdl}.npy"
        env = dict(os.environ, SPMV_CSR_PDL=pdl)
        subprocess.run([sys.executable, "-c", _PDL_SCRIPT, root, str(out)], env=env, check=True, timeout=600)
        res[pdl] = np.load(out)
    assert np.array_equal(res["1"].view(np.uint64), res["0"].view(np.uint64))
    A = matgen.rmat(21, seed=21)
    x, y0 = matgen.vector(A.n_cols, 17, 1), matgen.vector(A.n_rows, 17, 2)
    ref, bound = oracle.spmv_csr(A, x, 1.5, -0.5, y0, with_bound=True)
    ok, ratio, nbad = oracle.check_tolerance(res["1"][:A.n_rows], ref, bound, TOL[torch.float64])
    assert ok, f"R-MAT 21 CSR (PDL): {nbad} bad rows, max ratio {ratio}"
