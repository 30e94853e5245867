"""GPU side of the row-partitioned SpMV: shards built by
spmv_partition + spmv_slice_remap on the GPU, run in any format against the gathered x
(assembled on one GPU -- the virtual partition), compared with the oracle; and the
DistSpMV class end to end over a world-size-1 NCCL process group."""
import os
import socket

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


@pytest.mark.parametrize("P", [2, 3, 4, 8])
@pytest.mark.parametrize("fmt", ["csr", "merge", "csr5", "coo", "hyb"])
@pytest.mark.parametrize("case", ["rmat13", "lap96"])
def test_virtual_partition(sp, case, fmt, P):
    from paper_conf_ipps_nisassvs18_b200.dist import ShardLayout
    A = matgen.rmat(13, seed=41) if case == "rmat13" else matgen.laplacian5(96)
    x = matgen.vector(A.n_cols, 41, 1)
    y = matgen.vector(A.n_rows, 41, 2)
    ref, bound = oracle.spmv_csr(A, x, 1.5, 0.75, y, with_bound=True)
    dA = sp.CSR.from_host(A)
    splits = sp.partition(dA, P)
    assert np.array_equal(splits, oracle.partition(A, P))
    lays = [ShardLayout(splits, k) for k in range(P)]
    S = lays[0].S
    xd = torch.from_numpy(x).cuda()
    gathered = torch.cat([lay.pack_x(lay.local_slice(xd)) for lay in lays])
    out = np.empty(A.n_rows)
    for k, lay in enumerate(lays):
        shard, S2 = sp.slice_remap(dA, splits, k)
        assert S2 == S
        h = sp.convert(shard, fmt)
        yl = torch.from_numpy(y[lay.r0:lay.r1].copy()).cuda()
        h.run(1.5, gathered, 0.75, yl)
        out[lay.r0:lay.r1] = yl.cpu().numpy()
    ok, ratio, nbad = oracle.check_tolerance(out, ref, bound, 1e-12)
    assert ok, (nbad, ratio)


def test_distspmv_nccl_world1(sp):
    import torch.distributed as dist
    from paper_conf_ipps_nisassvs18_b200.dist import DistSpMV
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK="0", WORLD_SIZE="1")
    dist.init_process_group("nccl", device_id=torch.device("cuda", 0))
    try:
        A = matgen.rmat(12, seed=43)
        x = matgen.vector(A.n_cols, 43, 1)
        y = matgen.vector(A.n_rows, 43, 2)
        ref, bound = oracle.spmv_csr(A, x, 2.0, -1.0, y, with_bound=True)
        D = DistSpMV(sp.CSR.from_host(A), "merge")
        yl = torch.from_numpy(y[D.layout.r0:D.layout.r1].copy()).cuda()
        D.run(2.0, -1.0, yl, x_local=torch.from_numpy(x[D.layout.r0:D.layout.r1].copy()).cuda())
        full = D.gather_y(yl).cpu().numpy()
        assert oracle.check_tolerance(full, ref, bound, 1e-12)[0]
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("P", [1, 2, 4, 8])
@pytest.mark.parametrize("case", ["rmat13", "empty_cols"])
def test_compressed_exchange(sp, case, P):
    """colmap / compressed remap / pack index bit-exact against the oracle, and the
    compressed virtual partition reproduces the product."""
    from paper_conf_ipps_nisassvs18_b200.spmv import (spmv_colmap_pack_index, spmv_gather,
                                                       spmv_partition_colmap, spmv_slice_remap_colmap)
    if case == "rmat13":
        A = matgen.rmat(13, seed=47)
    else:
        lens = np.random.default_rng(3).integers(0, 6, 4000)
        A = matgen.from_lengths(lens, 4000, seed=48)
        keep = A.col % 3 != 0                                  # a third of the columns never used
        rows = np.repeat(np.arange(A.n_rows), np.diff(A.row_ptr))[keep]
        rp = np.zeros(A.n_rows + 1, np.int64)
        np.add.at(rp, rows + 1, 1)
        A = matgen.HostCSR(np.cumsum(rp), A.col[keep].copy(), A.val[keep].copy(), A.n_rows, A.n_cols)
    x = matgen.vector(A.n_cols, 47, 1)
    y = matgen.vector(A.n_rows, 47, 2)
    ref, bound = oracle.spmv_csr(A, x, 1.0, -1.0, y, with_bound=True)
    dA = sp.CSR.from_host(A)
    splits = sp.partition(dA, P)
    cm_o, S_o = oracle.partition_colmap(A, splits)
    cm, S = spmv_partition_colmap(dA, splits)
    assert S == S_o and np.array_equal(cm.cpu().numpy(), cm_o)
    xd = torch.from_numpy(x).cuda()
    xg = torch.zeros(P * S, dtype=torch.float64, device="cuda")
    for k in range(P):
        idx = spmv_colmap_pack_index(cm, splits, k, S)
        exp_idx = np.nonzero(cm_o[splits[k]:splits[k + 1]] >= 0)[0]
        assert np.array_equal(idx.cpu().numpy(), exp_idx)
        spmv_gather(xd[int(splits[k]):int(splits[k + 1])], idx, xg[k * S:(k + 1) * S])
    out = np.empty(A.n_rows)
    for k in range(P):
        shard = spmv_slice_remap_colmap(dA, splits, k, cm, S)
        rp, col, val = oracle.slice_remap_colmap(A, splits, k, cm_o)
        assert np.array_equal(shard.col.cpu().numpy(), col)
        assert np.array_equal(shard.row_ptr.cpu().numpy().astype(np.int64), rp)
        h = sp.convert(shard, "csr5")
        yl = torch.from_numpy(y[splits[k]:splits[k + 1]].copy()).cuda()
        h.run(1.0, xg, -1.0, yl)
        out[splits[k]:splits[k + 1]] = yl.cpu().numpy()
    assert oracle.check_tolerance(out, ref, bound, 1e-12)[0]


def test_distspmv_nccl_world1_compressed(sp):
    import torch.distributed as dist
    from paper_conf_ipps_nisassvs18_b200.dist import DistSpMV
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK="0", WORLD_SIZE="1")
    dist.init_process_group("nccl", device_id=torch.device("cuda", 0))
    try:
        A = matgen.rmat(12, seed=44)
        x = matgen.vector(A.n_cols, 44, 1)
        y = matgen.vector(A.n_rows, 44, 2)
        ref, bound = oracle.spmv_csr(A, x, 1.0, 1.0, y, with_bound=True)
        D = DistSpMV(sp.CSR.from_host(A), "merge", compress=True)
        assert D.slot < A.n_cols                               # R-MAT has empty columns
        yl = torch.from_numpy(y.copy()).cuda()
        D.run(1.0, 1.0, yl, x_local=torch.from_numpy(x).cuda())
        assert oracle.check_tolerance(yl.cpu().numpy(), ref, bound, 1e-12)[0]
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("compress", [False, True])
@pytest.mark.parametrize("P", [2, 4])
def test_own_foreign_split_bit_exact(sp, P, compress):
    from paper_conf_ipps_nisassvs18_b200.spmv import spmv_partition_colmap, spmv_slice_split
    A = matgen.rmat(13, seed=51)
    dA = sp.CSR.from_host(A)
    splits = sp.partition(dA, P)
    if compress:
        cm, S = spmv_partition_colmap(dA, splits)
        cm_o, _ = oracle.partition_colmap(A, splits)
    else:
        cm, S, cm_o = None, None, None
    for k in range(P):
        for which in (0, 1):
            blk = spmv_slice_split(dA, splits, k, which, cm, S)
            rp, col, val = oracle.slice_split(A, splits, k, which, cm_o)
            assert np.array_equal(blk.row_ptr.cpu().numpy().astype(np.int64), rp)
            assert np.array_equal(blk.col.cpu().numpy(), col)
            assert np.array_equal(blk.val.cpu().numpy(), val)


@pytest.mark.parametrize("compress", [False, True])
def test_distspmv_nccl_world1_overlap(sp, compress):
    import torch.distributed as dist
    from paper_conf_ipps_nisassvs18_b200.dist import DistSpMV
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK="0", WORLD_SIZE="1")
    dist.init_process_group("nccl", device_id=torch.device("cuda", 0))
    try:
        A = matgen.rmat(12, seed=45)
        x = matgen.vector(A.n_cols, 45, 1)
        y = matgen.vector(A.n_rows, 45, 2)
        ref, bound = oracle.spmv_csr(A, x, 2.0, 0.5, y, with_bound=True)
        D = DistSpMV(sp.CSR.from_host(A), "csr5", compress=compress, overlap=True)
        yl = torch.from_numpy(y.copy()).cuda()
        D.run(2.0, 0.5, yl, x_local=torch.from_numpy(x).cuda())
        assert oracle.check_tolerance(yl.cpu().numpy(), ref, bound, 1e-12)[0]
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("P", [2, 3, 5])
@pytest.mark.parametrize("case", ["lap96", "rmat12"])
@pytest.mark.parametrize("fmt", ["csr", "merge", "csr5", "ell"])
def test_halo_virtual(sp, case, fmt, P):
    """Halo exchange of P virtual ranks on one GPU: each rank's own
    block (spmv_slice_split which=0) and foreign block remapped through its HaloPlan
    colmap, halos packed by spmv_gather and moved by device copies standing in for the
    all_to_all; integer regime, so bit-exact against the oracle."""
    from paper_conf_ipps_nisassvs18_b200.dist import HaloPlan, ShardLayout
    from paper_conf_ipps_nisassvs18_b200.spmv import spmv_gather, spmv_slice_split
    A = matgen.rmat(12, seed=44, kind="int") if case == "rmat12" else matgen.laplacian5(96)
    x = matgen.vector(A.n_cols, 44, 1, "int")
    y = matgen.vector(A.n_rows, 44, 2, "int")
    ref = oracle.spmv_csr(A, x, 2.0, -1.0, y)
    dA = sp.CSR.from_host(A)
    splits = sp.partition(dA, P)
    lays = [ShardLayout(splits, k) for k in range(P)]
    plans = [HaloPlan(dA, splits, k) for k in range(P)]
    xd = torch.from_numpy(x).cuda()
    sends = []
    for k, lay in enumerate(lays):
        buf = torch.empty(plans[k].send_index.numel(), dtype=torch.float64, device="cuda")
        spmv_gather(lay.local_slice(xd).contiguous(), plans[k].send_index, buf)
        sends.append(buf)
    out = np.empty(A.n_rows)
    for k, lay in enumerate(lays):
        S = plans[k].S
        recv = torch.zeros(P * S, dtype=torch.float64, device="cuda")
        for o in range(P):                       # what all_to_all_single delivers
            off = sum(plans[o].slots[:k])
            recv[o * S: o * S + plans[o].slots[k]] = sends[o][off: off + plans[o].slots[k]]
        try:
            own = sp.convert(spmv_slice_split(dA, splits, k, 0), fmt)
            foreign = sp.convert(spmv_slice_split(dA, splits, k, 1, plans[k].colmap, S), fmt)
        except sp.SpmvError as e:
            assert fmt == "ell" and e.status == 3
            pytest.skip("ELL infeasible (A4)")
        yl = torch.from_numpy(y[lay.r0:lay.r1].copy()).cuda()
        own.run(2.0, lay.local_slice(xd).contiguous(), -1.0, yl)
        foreign.run(2.0, recv, 1.0, yl)
        out[lay.r0:lay.r1] = yl.cpu().numpy()
    assert np.array_equal(out, ref)
    if case == "lap96":
        assert max(p.S for p in plans) <= 96        # one grid line per neighbour


def test_halospmv_nccl_world1(sp):
    import torch.distributed as dist
    from paper_conf_ipps_nisassvs18_b200.dist import HaloSpMV
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK="0", WORLD_SIZE="1")
    dist.init_process_group("nccl", device_id=torch.device("cuda", 0))
    try:
        A = matgen.laplacian5(80)
        x = matgen.vector(A.n_cols, 45, 1)
        y = matgen.vector(A.n_rows, 45, 2)
        ref, bound = oracle.spmv_csr(A, x, 2.0, -1.0, y, with_bound=True)
        H = HaloSpMV(sp.CSR.from_host(A), "csr")
        yl = torch.from_numpy(y.copy()).cuda()
        H.run(2.0, -1.0, yl, torch.from_numpy(x).cuda())
        torch.cuda.synchronize()
        ok, ratio, nbad = oracle.check_tolerance(yl.cpu().numpy(), ref, bound, 1e-12)
        assert ok, (nbad, ratio)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("P", [1, 2, 3, 5, 8])
@pytest.mark.parametrize("case", ["lap96", "rmat12", "empty_runs"])
def test_halo_colmap_bit_exact(sp, case, P):
    """spmv_halo_colmap + spmv_colmap_pack_index (the halo plan's index maps) bit-exact
    against the oracle's plain loops, for every receiver and sender."""
    from paper_conf_ipps_nisassvs18_b200.spmv import spmv_colmap_pack_index, spmv_halo_colmap
    if case == "lap96":
        A = matgen.laplacian5(96)
    elif case == "rmat12":
        A = matgen.rmat(12, seed=46)
    else:
        lens = np.random.default_rng(46).integers(0, 9, 4000)
        lens[100:900] = 0
        A = matgen.from_lengths(lens, 4000, seed=46)
    dA = sp.CSR.from_host(A)
    splits = sp.partition(dA, P)
    for k in range(P):
        cm, counts, S = spmv_halo_colmap(dA, splits, k)
        cmo, cnto, So = oracle.halo_colmap(A, splits, k)
        assert S == So and np.array_equal(counts, cnto)
        assert np.array_equal(cm.cpu().numpy(), cmo)
        for snd in range(P):
            idx = spmv_colmap_pack_index(cm, splits, snd, S).cpu().numpy()
            assert np.array_equal(idx, oracle.halo_pack_index(cmo, splits, snd, So)), (k, snd)


@pytest.mark.parametrize("ptr", [torch.int32, torch.int64], ids=["i32", "i64"])
@pytest.mark.parametrize("case", ["sparse_rows", "no_empty", "all_empty", "lap_foreign"])
def test_compress_rows_bit_exact(sp, case, ptr):
    """spmv_compress_rows (A33) equals the oracle's compressed rows bit for bit, and
    spmv_scatter puts a gathered vector back (dst[idx[q]] = src[q])."""
    from paper_conf_ipps_nisassvs18_b200.dist import HaloPlan
    from paper_conf_ipps_nisassvs18_b200.spmv import partition, spmv_compress_rows, spmv_gather, spmv_scatter, spmv_slice_split
    rng = np.random.default_rng(41)
    if case == "lap_foreign":                       # a rank's foreign block of a 4-way Laplacian split
        dA = sp.CSR.from_host(matgen.laplacian5(96))
        splits = partition(dA, 4)
        plan = HaloPlan(dA, splits, 1)
        F = spmv_slice_split(dA, splits, 1, 1, plan.colmap, plan.S)
        A = matgen.HostCSR(F.row_ptr.cpu().numpy().astype(np.int64), F.col.cpu().numpy(), F.val.cpu().numpy(),
                           F.n_rows, F.n_cols)
    else:
        lens = {"sparse_rows": np.where(rng.random(70000) < 0.01, rng.integers(1, 9, 70000), 0),
                "no_empty": rng.integers(1, 5, 3000), "all_empty": np.zeros(5000, np.int64)}[case]
        A = matgen.from_lengths(lens, 4000, seed=42)
    dA = sp.CSR.from_host(A, ptr_dtype=ptr)
    rows, rp = spmv_compress_rows(dA)
    orows, orp = oracle.compress_rows(A)
    assert rows.dtype == torch.int32 and rp.dtype == ptr
    assert np.array_equal(rows.cpu().numpy().astype(np.int64), orows)
    assert np.array_equal(rp.cpu().numpy().astype(np.int64), orp)
    y = torch.from_numpy(matgen.vector(A.n_rows, 43, 1)).cuda()
    yc = torch.empty(rows.numel(), dtype=torch.float64, device="cuda")
    spmv_gather(y, rows, yc)
    z = torch.zeros_like(y)
    spmv_scatter(yc, rows, z)
    torch.cuda.synchronize()
    keep = np.zeros(A.n_rows, bool)
    keep[orows] = True
    assert np.array_equal(z.cpu().numpy()[keep], y.cpu().numpy()[keep])
    assert not z.cpu().numpy()[~keep].any()
