"""Pins for the oracle's converters, merge-path coordinates, CSR5 encoding,
features and partition, CPU only."""
import json
import os

import numpy as np
import pytest

import matgen
import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def load(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def csr_of(g):
    return matgen.HostCSR(np.array(g["row_ptr"], np.int64), np.array(g["col"], np.int32),
                          np.array(g["val"], np.float64), g["n_rows"], g["n_cols"])


def structured_cases():
    """Small matrices with empty rows (leading/trailing/runs), long rows, runs of
    consecutive columns, rectangular shapes."""
    out = [csr_of(load("app_a_4x4.json")), csr_of(load("app_a_5x5.json"))]
    out.append(matgen.window(300, 300, 6, 0.7, seed=5, mode=0))
    out.append(matgen.window(257, 500, 16, 0.9, seed=6, mode=1))
    lens = np.zeros(400, np.int64)
    lens[[3, 4, 200, 201, 202, 350]] = [1, 700, 5, 64, 1, 2000]
    out.append(matgen.from_lengths(lens, 3000, seed=7))
    out.append(matgen.rmat(9, seed=8))
    out.append(matgen.from_lengths(np.random.default_rng(9).integers(0, 30, 123), 41, seed=9))
    out.append(matgen.HostCSR(np.zeros(6, np.int64), np.zeros(0, np.int32), np.zeros(0), 5, 7))
    out.append(matgen.from_lengths([1500], 1500, seed=10))              # one dense row
    out.append(matgen.from_lengths(np.ones(700, np.int64), 1, seed=11))  # n x 1
    return out


N_CASES = 10


# ------------------------------------------------------------------ COO / ELL / HYB

def test_golden_coo_ell_hyb():
    g = load("app_a_4x4.json")
    A = csr_of(g)
    assert oracle.csr2coo(A).tolist() == g["coo_row"]
    e = oracle.csr2ell(A)
    assert e["K"] == g["ell_K"] and e["ld"] == 32
    for j in range(e["K"]):
        assert e["col"][j * 32:j * 32 + 4].tolist() == g["ell_first4_by_slice"]["col"][j]
        assert e["val"][j * 32:j * 32 + 4].tolist() == g["ell_first4_by_slice"]["val"][j]
        assert np.all(e["col"][j * 32 + 4:(j + 1) * 32] == -1)
    h = oracle.csr2hyb(A)
    assert h["K"] == g["hyb"]["K"]
    assert h["coo_row"].tolist() == g["hyb"]["coo_row"]
    assert h["coo_col"].tolist() == g["hyb"]["coo_col"]
    assert h["coo_val"].tolist() == g["hyb"]["coo_val"]
    assert oracle.hyb_width(A, "floor") == g["hyb"]["K_floor"]
    assert oracle.hyb_width(A, "cusp") == g["hyb"]["K_cusp"]


@pytest.mark.parametrize("i", range(N_CASES))
def test_ell_hyb_coo_round_trip(i):
    """Decoding each format back to CSR gives the input (numpy decoders)."""
    A = structured_cases()[i]
    n = A.n_rows
    lens = np.diff(A.row_ptr)
    # COO
    row = oracle.csr2coo(A)
    assert np.array_equal(row, np.repeat(np.arange(n), lens))
    # ELL: column-major slices; per-row the first len entries, then sentinels
    e = oracle.csr2ell(A)
    K, ld = e["K"], e["ld"]
    assert K == (lens.max() if n else 0) and ld % 32 == 0 and ld >= n
    C = e["col"].reshape(K, ld).T if K else np.zeros((ld, 0), np.int32)
    V = e["val"].reshape(K, ld).T if K else np.zeros((ld, 0))
    for r in range(n):
        s, t = A.row_ptr[r], A.row_ptr[r + 1]
        assert np.array_equal(C[r, :t - s], A.col[s:t]) and np.array_equal(V[r, :t - s], A.val[s:t])
        assert np.all(C[r, t - s:] == -1) and np.all(V[r, t - s:] == 0)
    assert np.all(C[n:] == -1)
    # HYB
    for rule in ("ceil", "floor", "cusp"):
        h = oracle.csr2hyb(A, rule)
        Kh = h["K"]
        HC = h["ell_col"].reshape(Kh, ld).T if Kh else np.zeros((ld, 0), np.int32)
        rows_c, cols_c, vals_c = [], [], []
        for r in range(n):
            s, t = A.row_ptr[r], A.row_ptr[r + 1]
            m = min(t - s, Kh)
            assert np.array_equal(HC[r, :m], A.col[s:s + m]) and np.all(HC[r, m:] == -1)
            rows_c += [r] * (t - s - m)
            cols_c += A.col[s + m:t].tolist()
            vals_c += A.val[s + m:t].tolist()
        assert h["coo_row"].tolist() == rows_c and h["coo_col"].tolist() == cols_c
        assert h["coo_val"].tolist() == vals_c


def test_hyb_width_rules_definitions():
    """A2: ceil/floor of nnz_mu; the [2]-style rule by brute definition over k."""
    for A in structured_cases():
        n = A.n_rows
        lens = np.diff(A.row_ptr)
        nnz = A.nnz
        assert oracle.hyb_width(A, "ceil") == (-(-nnz // n) if n else 0)
        assert oracle.hyb_width(A, "floor") == (nnz // n if n else 0)
        K = int(lens.max()) if n else 0
        exp = K
        for k in range(K):
            longer = int((lens > k).sum())
            if 3 * longer < n or longer < 4096:
                exp = k
                break
        assert oracle.hyb_width(A, "cusp") == (exp if n else 0)


# ------------------------------------------------------------------ merge path

def merge_coord_formula(row_ptr, d):
    """A7 closed form: i = largest i in [0, min(d, n)] with row_ptr[i] + i <= d."""
    n = row_ptr.size - 1
    key = row_ptr + np.arange(n + 1)
    i = int(np.searchsorted(key, d, side="right")) - 1
    i = min(i, min(d, n))
    return i, d - i


@pytest.mark.parametrize("name", ["app_a_4x4.json", "app_a_5x5.json"])
def test_golden_merge_coords(name):
    g = load(name)
    A = csr_of(g)
    cr, cn = oracle.merge_coords(A, 1)
    assert [[int(a), int(b)] for a, b in zip(cr, cn)] == g["merge_coords_T1"]


@pytest.mark.parametrize("T", [1, 3, 7, 64, 1000])
def test_merge_walk_equals_binary_search(T):
    for A in structured_cases():
        cr, cn = oracle.merge_coords(A, T)
        total = A.n_rows + A.nnz
        nt = -(-total // T)
        assert cr.size == nt + 1
        for t in range(nt + 1):
            d = min(t * T, total)
            assert (cr[t], cn[t]) == merge_coord_formula(A.row_ptr, d)
        assert cr[-1] == A.n_rows and cn[-1] == A.nnz
        assert np.all(np.diff(cr) >= 0) and np.all(np.diff(cn) >= 0)


# merge tile class (A28): 1 iff the tile consumes < max_rows row ends and no row gets
# more than max_len of its nonzeros.  Pinned by closed forms and by the coordinate
# formula (binary search, not a walk) applied to the definition.

def merge_class_formula(A, T, max_rows=64, max_len=32):
    total = A.n_rows + A.nnz
    nt = -(-total // T)
    out = []
    for t in range(nt):
        r0, k0 = merge_coord_formula(A.row_ptr, min(t * T, total))
        r1, k1 = merge_coord_formula(A.row_ptr, min((t + 1) * T, total))
        rp = np.clip(np.asarray(A.row_ptr[r0:min(r1 + 2, A.n_rows + 1)], np.int64), k0, k1)
        parts = np.diff(np.concatenate([[k0], rp[1:], [k1]]))
        out.append(int(r1 - r0 < max_rows and parts.max(initial=0) <= max_len))
    return np.array(out, np.uint8)


@pytest.mark.parametrize("T", [7, 64, 128, 256])
def test_merge_class_definition(T):
    for A in structured_cases():
        assert np.array_equal(oracle.merge_class(A, T), merge_class_formula(A, T))


def test_merge_class_closed_forms():
    # 5-point Laplacian (App. B): rows <= 5 nonzeros, ~43 row ends per 256 items -> all 1
    A = matgen.laplacian5(16)
    assert oracle.merge_class(A, 256).all()
    # a row of exactly 32 / 33 nonzeros alone in a tile: 32 is a row-sum tile, 33 is not
    for L, exp in ((32, 1), (33, 0)):
        A = matgen.from_lengths([L], 40, seed=1)
        assert oracle.merge_class(A, 256).tolist() == [exp]
    # 63 / 64 empty rows then nothing: 63 row ends -> 1, 64 -> 0 (T = 256 holds them all)
    for n, exp in ((63, 1), (64, 0)):
        A = matgen.HostCSR(np.zeros(n + 1, np.int64), np.zeros(0, np.int32), np.zeros(0), n, 4)
        assert oracle.merge_class(A, 256).tolist() == [exp]
    # one 1500-nonzero row split over 6 tiles of 256 items: every tile has a part > 32
    A = matgen.from_lengths([1500], 1500, seed=10)
    assert not oracle.merge_class(A, 256).any()
    # the same test with the limits opened up: every tile qualifies
    assert oracle.merge_class(A, 256, max_rows=300, max_len=256).all()


# ------------------------------------------------------------------ partition

@pytest.mark.parametrize("name", ["app_a_4x4.json", "app_a_5x5.json"])
def test_golden_partition(name):
    g = load(name)
    A = csr_of(g)
    for P, exp in g["partition"].items():
        assert oracle.partition(A, int(P)).tolist() == exp


@pytest.mark.parametrize("P", [1, 2, 3, 4, 8])
def test_partition_invariants(P):
    for A in structured_cases():
        s = oracle.partition(A, P)
        total = A.n_rows + A.nnz
        assert s[0] == 0 and s[-1] == A.n_rows and np.all(np.diff(s) >= 0)
        lens = np.diff(A.row_ptr)
        longest = int(lens.max()) if A.n_rows else 0
        for k in range(P):
            assert s[k] == merge_coord_formula(A.row_ptr, (k * total) // P)[0]
            items = (s[k + 1] - s[k]) + (A.row_ptr[s[k + 1]] - A.row_ptr[s[k]])
            assert items <= -(-total // P) + longest + 1


@pytest.mark.parametrize("P", [1, 2, 3, 5])
def test_slice_remap_reassembles_spmv(P):
    """Shard SpMV with the gathered (padded) x equals the unpartitioned oracle bit-exactly."""
    A = matgen.rmat(10, seed=21)
    x = matgen.vector(A.n_cols, 21, 1)
    y = matgen.vector(A.n_rows, 21, 2)
    s = oracle.partition(A, P)
    S = oracle.partition_slot(s)
    xg = np.zeros(P * S)
    for k in range(P):
        xg[k * S:k * S + s[k + 1] - s[k]] = x[s[k]:s[k + 1]]
    full = oracle.spmv_csr(A, x, 1.5, -0.5, y)
    for k in range(P):
        rp, col, val = oracle.slice_remap(A, s, k)
        shard = matgen.HostCSR(rp, col, val, int(s[k + 1] - s[k]), P * S)
        part = oracle.spmv_csr(shard, xg, 1.5, -0.5, y[s[k]:s[k + 1]])
        assert np.array_equal(part, full[s[k]:s[k + 1]])


# ------------------------------------------------------------------ CSR5

def test_csr5_sigma_rule():
    """A6 (B200 rule, tools/csr5_sigma_sweep.py): sigma = 4 for ceil(nnz_mu) <= 3, 8 for
    ceil(nnz_mu) = 4, 12 above."""
    assert oracle.csr5_sigma(matgen.laplacian5(16)) == 12         # mu ~ 4.7 -> 5 -> 12
    assert oracle.csr5_sigma(matgen.uniform_fixed(64, 64, 16)) == 12
    assert oracle.csr5_sigma(matgen.uniform_fixed(64, 64, 1)) == 4
    assert oracle.csr5_sigma(matgen.uniform_fixed(64, 64, 3)) == 4
    assert oracle.csr5_sigma(matgen.uniform_fixed(64, 64, 4)) == 8
    assert oracle.csr5_sigma(matgen.uniform_fixed(64, 64, 40)) == 12


@pytest.mark.parametrize("i", range(N_CASES))
@pytest.mark.parametrize("val_bytes", [4, 8])
@pytest.mark.parametrize("sigma", [None, 4, 16])
def test_csr5_round_trip_and_invariants(i, val_bytes, sigma):
    A = structured_cases()[i]
    e = oracle.csr5_encode(A, val_bytes=val_bytes, sigma=sigma)
    sg = e["sigma"]
    W = 32 * sg
    nt = e["n_tiles"]
    assert nt == A.nnz // W
    rc, rp, col, val = oracle.csr5_decode((A.n_rows, A.nnz), e, A.row_ptr, val_bytes)
    assert rc == 0
    assert np.array_equal(rp, A.row_ptr) and np.array_equal(col, A.col) and np.array_equal(val, A.val)
    # invariants: popcounts = non-empty rows starting inside full tiles
    desc = e["tile_desc"].reshape(nt, 32) if nt else np.zeros((0, 32), np.uint32)
    flags = desc & 0xFFFF
    starts = A.row_ptr[:-1][np.diff(A.row_ptr) > 0]
    assert sum(bin(int(f)).count("1") for f in flags.ravel()) == int((starts < nt * W).sum())
    for t in range(nt):
        yoff = (desc[t] >> 16) & 0x1FF
        pc = np.array([bin(int(f)).count("1") for f in flags[t]])
        assert np.array_equal(yoff, np.concatenate([[0], np.cumsum(pc)[:-1]]))
        for l in range(32):
            m = 0
            while l + m + 1 < 32 and flags[t, l + m + 1] == 0:
                m += 1
            assert (desc[t, l] >> 25) & 0x1F == m
    assert np.all(np.diff(e["row_lo"]) >= 0)
    # row_lo[t] = first row whose start >= t*W (A6)
    for t in range(nt + 1):
        exp = int(np.searchsorted(A.row_ptr[:-1], t * W, side="left"))
        assert e["row_lo"][t] == exp


def test_csr5_decode_detects_corruption():
    A = matgen.rmat(9, seed=8)
    e = oracle.csr5_encode(A)
    assert e["n_tiles"] > 2
    bad = dict(e)
    bad["tile_desc"] = e["tile_desc"].copy()
    bad["tile_desc"][33] ^= (1 << 16)          # y_offset off by one
    assert oracle.csr5_decode((A.n_rows, A.nnz), bad, A.row_ptr)[0] != 0
    bad2 = dict(e)
    bad2["tile_ptr"] = e["tile_ptr"].copy()
    bad2["tile_ptr"][1] += 1
    assert oracle.csr5_decode((A.n_rows, A.nnz), bad2, A.row_ptr)[0] != 0


def test_csr5_layout_is_lane_interleaved():
    """A6 layout: element e = t*W + l*sigma + s at t*W + (s//v)*32*v + l*v + s%v."""
    A = matgen.uniform_fixed(256, 4096, 16, seed=3)
    for sigma, pts in ((16, [(0, 0, 0), (0, 5, 3), (1, 31, 15), (2, 7, 9)]),
                       (12, [(0, 0, 0), (0, 5, 3), (1, 31, 11), (2, 7, 9)])):
        e = oracle.csr5_encode(A, val_bytes=8, sigma=sigma)
        sg, W = e["sigma"], 32 * e["sigma"]
        assert sg == sigma
        for (t, l, s) in pts:
            src = t * W + l * sg + s
            assert e["col_perm"][t * W + (s // 4) * 128 + l * 4 + s % 4] == A.col[src]
            assert e["val_perm"][t * W + (s // 2) * 64 + l * 2 + s % 2] == A.val[src]


# ------------------------------------------------------------------ features

def features_brute(A):
    """numpy/python brute force of Table II per A8/A9 (independent of oracle.c)."""
    n, m = A.n_rows, A.n_cols
    lens = np.diff(A.row_ptr).astype(np.int64)
    blocks, bsizes = [], []
    for r in range(n):
        c = A.col[A.row_ptr[r]:A.row_ptr[r + 1]].astype(np.int64)
        if c.size == 0:
            blocks.append(0)
            continue
        cuts = np.nonzero(np.diff(c) != 1)[0]
        edges = np.concatenate([[0], cuts + 1, [c.size]])
        sizes = np.diff(edges)
        blocks.append(sizes.size)
        bsizes += sizes.tolist()
    blocks = np.array(blocks, np.int64)
    bs = np.array(bsizes, np.int64)
    nnz = int(lens.sum())

    def sig(vals, cnt):
        S1, S2 = int(vals.sum()), int((vals.astype(object) ** 2).sum()) if vals.size else 0
        return float(np.sqrt(float(cnt * S2 - S1 * S1))) / cnt if cnt else 0.0

    f = dict(n_rows=n, n_cols=m, nnz_tot=nnz,
             nnz_mu=nnz / n if n else 0.0,
             nnz_frac=float(100 * nnz) / float(n * m) if n and m else 0.0,
             nnz_max=int(lens.max()) if n else 0, nnz_min=int(lens.min()) if n else 0,
             nnz_sigma=sig(lens, n),
             nnzb_tot=int(blocks.sum()), nnzb_mu=float(blocks.sum()) / n if n else 0.0,
             nnzb_sigma=sig(blocks, n),
             nnzb_min=int(blocks.min()) if n else 0, nnzb_max=int(blocks.max()) if n else 0,
             snzb_mu=nnz / bs.size if bs.size else 0.0, snzb_sigma=sig(bs, bs.size),
             snzb_min=int(bs.min()) if bs.size else 0, snzb_max=int(bs.max()) if bs.size else 0,
             n_empty_rows=int((lens == 0).sum()))
    f["ell_width"] = f["nnz_max"]
    f["ell_slots"] = f["nnz_max"] * n
    f["ell_pad_frac"] = (f["ell_slots"] - nnz) / f["ell_slots"] if f["ell_slots"] else 0.0
    return f


@pytest.mark.parametrize("name", ["app_a_4x4.json", "app_a_5x5.json"])
def test_golden_features(name):
    g = load(name)
    f = oracle.features(csr_of(g))
    for k, v in g["features"].items():
        assert f[k] == v, k


@pytest.mark.parametrize("i", range(N_CASES))
def test_features_vs_brute_force(i):
    A = structured_cases()[i]
    f = oracle.features(A)
    for k, v in features_brute(A).items():
        assert f[k] == v, (k, f[k], v)


def test_features_lap4096_closed_forms():
    """App. B closed forms with m = g - 2, evaluated here from the formulas."""
    g = load("app_b_lap4096.json")
    G = g["g"]
    m = G - 2
    A = matgen.laplacian5(G)
    f = oracle.features(A)
    assert f["nnz_tot"] == 5 * G * G - 4 * G
    assert f["sum_len2"] == 25 * m * m + 64 * m + 36
    assert f["nnzb_tot"] == 3 * m * m + 10 * m + 8
    assert f["sum_nnzb2"] == 9 * m * m + 26 * m + 16
    assert f["sum_snzb2"] == 11 * m * m + 32 * m + 20
    for k, v in g["features"].items():
        assert f[k] == v, k
    assert f["ell_pad_frac"] == 1 / 5120


@pytest.mark.parametrize("G", [3, 4, 5, 8])
def test_features_laplacian_small_brute(G):
    A = matgen.laplacian5(G)
    f = oracle.features(A)
    for k, v in features_brute(A).items():
        assert f[k] == v, k


def test_features_u2048():
    """cfg1 closed forms: 16 per row, nnz_frac 0.78125, pad 0, K_h 16, K_cusp 0."""
    A = matgen.uniform_fixed(2048, 2048, 16)
    f = oracle.features(A)
    assert f["nnz_max"] == f["nnz_min"] == 16 and f["nnz_sigma"] == 0.0
    assert f["nnz_frac"] == 0.78125 and f["ell_pad_frac"] == 0.0
    assert f["hyb_width"] == 16 and f["hyb_width_cusp"] == 0


@pytest.mark.parametrize("P", [1, 2, 3, 5])
def test_compressed_exchange_reassembles_spmv(P):
    """only referenced columns are exchanged; the shard SpMV against the
    compressed gathered x equals the unpartitioned oracle bit-exactly, and the slots are
    dense (referenced columns of each owner numbered 0..count-1 in column order)."""
    A = matgen.rmat(10, seed=23)
    x = matgen.vector(A.n_cols, 23, 1)
    y = matgen.vector(A.n_rows, 23, 2)
    s = oracle.partition(A, P)
    cm, S = oracle.partition_colmap(A, s)
    used = np.zeros(A.n_cols, bool)
    used[A.col] = True
    assert np.array_equal(cm >= 0, used)
    xg = np.zeros(P * S)
    for k in range(P):
        js = np.nonzero(used[s[k]:s[k + 1]])[0] + s[k]
        assert np.array_equal(cm[js], k * S + np.arange(js.size))
        assert js.size <= S
        xg[k * S:k * S + js.size] = x[js]
    full = oracle.spmv_csr(A, x, 0.5, 2.0, y)
    for k in range(P):
        rp, col, val = oracle.slice_remap_colmap(A, s, k, cm)
        shard = matgen.HostCSR(rp, col, val, int(s[k + 1] - s[k]), P * S)
        assert np.array_equal(oracle.spmv_csr(shard, xg, 0.5, 2.0, y[s[k]:s[k + 1]]), full[s[k]:s[k + 1]])


@pytest.mark.parametrize("compress", [False, True])
@pytest.mark.parametrize("P", [1, 2, 4])
def test_own_foreign_split_reassembles(P, compress):
    """own block (x slice) + foreign block (gathered x) = the shard's product;
    the two blocks partition the shard's nonzeros."""
    A = matgen.rmat(10, seed=29)
    x = matgen.vector(A.n_cols, 29, 1)
    y = matgen.vector(A.n_rows, 29, 2)
    s = oracle.partition(A, P)
    ref, bound = oracle.spmv_csr(A, x, 1.5, -0.5, y, with_bound=True)
    if compress:
        cm, S = oracle.partition_colmap(A, s)
    else:
        cm, S = None, oracle.partition_slot(s)
    xg = np.zeros(P * S)
    for k in range(P):
        if compress:
            js = np.nonzero(cm[s[k]:s[k + 1]] >= 0)[0] + s[k]
            xg[k * S:k * S + js.size] = x[js]
        else:
            xg[k * S:k * S + s[k + 1] - s[k]] = x[s[k]:s[k + 1]]
    for k in range(P):
        r0, r1 = int(s[k]), int(s[k + 1])
        rpo, co, vo = oracle.slice_split(A, s, k, 0, cm)
        rpf, cf, vf = oracle.slice_split(A, s, k, 1, cm)
        assert co.size + cf.size == A.row_ptr[r1] - A.row_ptr[r0]
        assert np.all((co >= 0) & (co < r1 - r0))
        own = matgen.HostCSR(rpo, co, vo, r1 - r0, r1 - r0)
        foreign = matgen.HostCSR(rpf, cf, vf, r1 - r0, P * S)
        part = oracle.spmv_csr(own, x[r0:r1], 1.5, -0.5, y[r0:r1])
        part = oracle.spmv_csr(foreign, xg, 1.5, 1.0, part)
        ok, ratio, _ = oracle.check_tolerance(part, ref[r0:r1], bound[r0:r1], 1e-13)
        assert ok, ratio


# ------------------------------------------------------------------ CSR long-row chunks (A25)

def test_csr_chunks_hand_example():
    # row lengths 0, 5, 10, 3 with C = 2: rows longer than 4 are split into 2-nonzero chunks
    A = matgen.from_lengths(np.array([0, 5, 10, 3]), 20, seed=3)
    cr, cl = oracle.csr_chunks(A, 2)
    assert cr.tolist() == [1, 1, 1, 2, 2, 2, 2, 2]
    assert cl.tolist() == [0, 2, 4, 5, 7, 9, 11, 13]


@pytest.mark.parametrize("C", [1, 2, 7, 64, 5000])
def test_csr_chunks_tile_long_rows(C):
    """Each long row's chunks tile [row_ptr[r], row_ptr[r+1]) in steps of C (last one
    shorter), short rows have none, and summing the chunk partials reproduces the row."""
    rng = np.random.default_rng(C)
    for A in structured_cases():
        cr, cl = oracle.csr_chunks(A, C)
        lens = np.diff(A.row_ptr)
        long_rows = np.nonzero(lens > 2 * C)[0]
        assert cr.size == int(sum(-(-int(lens[r]) // C) for r in long_rows))
        assert np.all(np.diff(cr) >= 0)
        assert set(cr.tolist()) == set(long_rows.tolist())
        x = rng.standard_normal(A.n_cols)
        for r in long_rows:
            sel = cr == r
            lo = cl[sel]
            a, b = int(A.row_ptr[r]), int(A.row_ptr[r + 1])
            assert lo.tolist() == list(range(a, b, C))
            parts = [np.sum(A.val[k:min(k + C, b)] * x[A.col[k:min(k + C, b)]]) for k in lo]
            assert abs(sum(parts) - np.sum(A.val[a:b] * x[A.col[a:b]])) <= 1e-12 * np.sum(np.abs(A.val[a:b] * x[A.col[a:b]])) + 1e-300


def _halo_brute(A, splits, k):
    """Receiver k's halo by sets: foreign columns referenced by k's rows, per owner sorted."""
    s = np.asarray(splits, np.int64)
    P = s.size - 1
    a, b = int(A.row_ptr[s[k]]), int(A.row_ptr[s[k + 1]])
    cols = np.unique(A.col[a:b].astype(np.int64))
    owner = np.searchsorted(s, cols, side="right") - 1
    cols, owner = cols[owner != k], owner[owner != k]
    counts = np.bincount(owner, minlength=P).astype(np.int64)
    S = max(1, int(counts.max()) if counts.size else 1)
    cm = np.full(A.n_cols, -1, np.int32)
    for o in range(P):
        mine = cols[owner == o]
        cm[mine] = o * S + np.arange(mine.size)
    return cm, counts, S


@pytest.mark.parametrize("P", [1, 2, 3, 4, 7])
@pytest.mark.parametrize("case", ["lap30", "rmat10", "band", "ragged"])
def test_oracle_halo_colmap_brute_force(case, P):
    """ora_halo_colmap == a set-based brute force; every referenced
    foreign column lands in its owner's slot range, distinct and in column order."""
    if case == "lap30":
        A = matgen.laplacian5(30)
    elif case == "rmat10":
        A = matgen.rmat(10, seed=3)
    elif case == "band":
        A = matgen.window(700, 700, 6, 0.7, seed=5, mode=0)
    else:
        lens = np.random.default_rng(8).integers(0, 9, 900)
        lens[50:300] = 0
        lens[600] = 800
        A = matgen.from_lengths(lens, 900, seed=8)
    splits = oracle.partition(A, P)
    for k in range(P):
        cm, cnt, S = oracle.halo_colmap(A, splits, k)
        cmb, cntb, Sb = _halo_brute(A, splits, k)
        assert S == Sb and np.array_equal(cnt, cntb) and np.array_equal(cm, cmb), (case, P, k)
        for snd in range(P):
            idx = oracle.halo_pack_index(cm, splits, snd, S)
            assert idx.size == cnt[snd]
            js = idx.astype(np.int64) + int(splits[snd])
            assert np.all(np.diff(js) > 0)
            assert np.array_equal(cm[js], snd * S + np.arange(idx.size))
    if case == "lap30" and P > 1:
        assert max(oracle.halo_colmap(A, splits, k)[2] for k in range(P)) <= 30   # one grid line


@pytest.mark.parametrize("kmax", [1, 7, 100, 5000, 10 ** 9])
@pytest.mark.parametrize("case", ["rmat10", "lap30", "ragged", "u2048"])
def test_oracle_hot_columns_brute_force(case, kmax):
    """A30: ora_hot_columns == the (kmax+1)-th largest degree rule by sorting; the hot set
    holds at most kmax columns, every hot column outranks every other referenced column,
    and the threshold is the smallest that fits."""
    if case == "rmat10":
        A = matgen.rmat(10, seed=9)
    elif case == "lap30":
        A = matgen.laplacian5(30)
    elif case == "u2048":
        A = matgen.uniform_fixed(2048, 2048, 16)
    else:
        lens = np.random.default_rng(10).integers(0, 9, 900)
        lens[600] = 850
        A = matgen.from_lengths(lens, 900, seed=10)
    hot = oracle.hot_columns(A, kmax)
    deg = np.bincount(A.col, minlength=A.n_cols)
    ref = np.sort(deg)[::-1]
    if (deg > 0).sum() <= kmax:
        t = 1
    else:
        t = int(ref[kmax]) + 1
    assert np.array_equal(hot, np.nonzero(deg >= t)[0].astype(np.int32))
    assert hot.size <= kmax
    if t > 1:                                   # one lower threshold would exceed the budget
        assert (deg >= t - 1).sum() > kmax
    if hot.size:
        rest = deg[(deg > 0) & (deg < t)]
        assert rest.size == 0 or rest.max() < deg[hot].min()


# ---- A33: compressed rows (the foreign-column block of a halo step)

def test_compress_rows_hand_example():
    # rows 0..4 of lengths 0, 2, 0, 1, 0: the non-empty rows are 1 and 3
    A = matgen.HostCSR(np.array([0, 0, 2, 2, 3, 3], np.int64), np.array([1, 4, 0], np.int32), np.ones(3), 5, 5)
    rows, rp = oracle.compress_rows(A)
    assert rows.tolist() == [1, 3] and rp.tolist() == [0, 2, 3]


@pytest.mark.parametrize("case", ["no_empty", "all_empty", "zero_rows", "sparse_rows"])
def test_compress_rows_special_cases_and_round_trip(case):
    """No empty row: the identity (rows = 0..n-1, rp unchanged); all rows empty: nothing
    and rp = [0]; n = 0: nothing; otherwise expanding (rows, rp) back over all rows
    reproduces row_ptr, so the compressed CSR holds exactly A's nonzeros, row by row."""
    rng = np.random.default_rng(33)
    lens = {"no_empty": rng.integers(1, 9, 500), "all_empty": np.zeros(300, np.int64),
            "zero_rows": np.zeros(0, np.int64),
            "sparse_rows": np.where(rng.random(5000) < 0.02, rng.integers(1, 7, 5000), 0)}[case]
    A = matgen.from_lengths(lens, 1000, seed=5)
    rows, rp = oracle.compress_rows(A)
    n = A.n_rows
    if case == "no_empty":
        assert np.array_equal(rows, np.arange(n)) and np.array_equal(rp, A.row_ptr)
    if case in ("all_empty", "zero_rows"):
        assert rows.size == 0 and rp.tolist() == [0]
    assert np.all(np.diff(rows) > 0) and np.all(np.diff(rp) > 0)
    back = np.zeros(n + 1, np.int64)                  # expand: row r ends where its successor starts
    full = np.zeros(n, np.int64)
    full[rows] = np.diff(rp)
    np.cumsum(full, out=back[1:])
    assert np.array_equal(back, A.row_ptr)
