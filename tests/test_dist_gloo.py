"""Multi-process logic of the row-partitioned SpMV on CPU (gloo, world size 2 and 3),
SURVEY §4 T4': partition + remap + padded slots + all-gather of x + a per-shard SpMV,
compared with the unpartitioned product.  The per-shard SpMV here is the ORACLE (test
harness only); the GPU path runs the same ShardLayout / all_gather_slots plumbing with
libspmv shards (bench.py --gpus N, tests/test_gpu_dist.py)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import matgen
import oracle
from paper_conf_ipps_nisassvs18_b200.dist import ShardLayout, all_gather_slots


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, case, q, compress=False):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        if case == "rmat":
            A = matgen.rmat(11, seed=31)
        elif case == "lap":
            A = matgen.laplacian5(40)
        else:                                    # empty rows and a long row
            lens = np.random.default_rng(5).integers(0, 7, 3000)
            lens[100:400] = 0
            lens[2000] = 2500
            A = matgen.from_lengths(lens, 3000, seed=33)
        x = matgen.vector(A.n_cols, 32, 1)
        y = matgen.vector(A.n_rows, 32, 2)
        splits = oracle.partition(A, world)
        lay = ShardLayout(splits, rank)
        if compress:
            # only columns some row references are exchanged
            cm, S = oracle.partition_colmap(A, splits)
            js = np.nonzero(cm[lay.r0:lay.r1] >= 0)[0]
            slot = torch.zeros(S, dtype=torch.float64)
            slot[: js.size] = torch.from_numpy(x[lay.r0 + js].copy())
            gathered = torch.zeros(world * S, dtype=torch.float64)
            all_gather_slots(gathered, slot)
            rp, col, val = oracle.slice_remap_colmap(A, splits, rank, cm)
            shard = matgen.HostCSR(rp, col, val, lay.rows, world * S)
        else:
            # every rank holds only its x slice; the gathered vector is built by the collective
            slot = lay.pack_x(torch.from_numpy(x[lay.r0:lay.r1].copy()))
            gathered = torch.zeros(world * lay.S, dtype=torch.float64)
            all_gather_slots(gathered, slot)
            rp, col, val = oracle.slice_remap(A, splits, rank)
            shard = matgen.HostCSR(rp, col, val, lay.rows, world * lay.S)
        y_local = oracle.spmv_csr(shard, gathered.numpy(), 1.25, -0.5, y[lay.r0:lay.r1])
        # slot_of agrees with the remap
        for k in range(0, A.nnz, max(1, A.nnz // 50)):
            r = int(np.searchsorted(A.row_ptr, k, side="right")) - 1
            if lay.r0 <= r < lay.r1 and not compress:
                assert col[k - A.row_ptr[lay.r0]] == lay.slot_of(int(A.col[k]))
        # assemble y for the check (padded equal-count gather)
        yslot = lay.pack_x(torch.from_numpy(y_local))
        yall = torch.zeros(world * lay.S, dtype=torch.float64)
        all_gather_slots(yall, yslot)
        if rank == 0:
            full = np.concatenate([yall[k * lay.S: k * lay.S + int(splits[k + 1] - splits[k])].numpy()
                                   for k in range(world)])
            ref = oracle.spmv_csr(A, x, 1.25, -0.5, y)
            q.put(bool(np.array_equal(full, ref)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("compress", [False, True])
@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("case", ["rmat", "lap", "ragged"])
def test_partitioned_spmv_gloo(world, case, compress):
    if compress and case == "lap":
        pytest.skip("every column of the Laplacian is referenced")
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, case, q, compress)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
        assert p.exitcode == 0
    assert q.get(timeout=10) is True


def test_layout_host_logic():
    splits = np.array([0, 3, 3, 10], dtype=np.int64)     # an empty middle part
    lay = ShardLayout(splits, 2)
    assert (lay.P, lay.S, lay.r0, lay.r1, lay.rows) == (3, 7, 3, 10, 7)
    assert lay.slot_of(0) == 0 and lay.slot_of(2) == 2
    assert lay.slot_of(3) == 2 * 7 + 0 and lay.slot_of(9) == 2 * 7 + 6
    v = lay.pack_x(torch.arange(7, dtype=torch.float64))
    assert v.tolist() == list(range(7))
    lay0 = ShardLayout(splits, 0)
    assert lay0.pack_x(torch.ones(3, dtype=torch.float64)).tolist() == [1, 1, 1, 0, 0, 0, 0]


class OracleHaloIndex:
    """The halo plan's index maps from the oracle (CPU test stand-in for libspmv's
    spmv_halo_colmap / spmv_colmap_pack_index, which are pinned to it on the GPU)."""

    @staticmethod
    def colmap(A, splits, k):
        return oracle.halo_colmap(A, splits, k)

    @staticmethod
    def pack(colmap, splits, rank, S):
        return oracle.halo_pack_index(colmap, splits, rank, S)


def _halo_worker(rank, world, port, case, q):
    """HaloPlan over gloo: pack, all_to_all_single, own + foreign blocks
    (oracle SpMV per block), integer regime so the split sum is exact."""
    from paper_conf_ipps_nisassvs18_b200.dist import HaloPlan
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        if case == "lap":
            A = matgen.laplacian5(37)
        elif case == "band":
            A = matgen.window(900, 900, 9, 0.8, seed=7, mode=0, kind="int")
        else:
            A = matgen.rmat(10, seed=41, kind="int")
        x = matgen.vector(A.n_cols, 9, 1, "int")
        y = matgen.vector(A.n_rows, 9, 2, "int")
        splits = oracle.partition(A, world)
        lay = ShardLayout(splits, rank)
        plan = HaloPlan(A, splits, rank, index=OracleHaloIndex)
        x_own = torch.from_numpy(x[lay.r0:lay.r1].copy())
        send = x_own[plan.send_index.to(torch.int64)].contiguous()          # spmv_gather's job on the GPU
        recv = torch.zeros(plan.recv_len, dtype=torch.float64)
        plan.exchange(send, recv)
        # own / foreign blocks of this rank's rows (test-side construction)
        a, b = int(A.row_ptr[lay.r0]), int(A.row_ptr[lay.r1])
        cols, vals = A.col[a:b], A.val[a:b]
        rows = np.repeat(np.arange(lay.rows), np.diff(A.row_ptr[lay.r0:lay.r1 + 1]))
        mine = (cols >= lay.r0) & (cols < lay.r1)
        cm = np.asarray(plan.colmap)
        assert np.all(cm[cols[~mine]] >= 0)

        def block(sel, c, ncols):
            rp = np.zeros(lay.rows + 1, np.int64)
            np.add.at(rp, rows[sel] + 1, 1)
            return matgen.HostCSR(np.cumsum(rp), c.astype(np.int32), vals[sel], lay.rows, ncols)
        own = block(mine, cols[mine] - lay.r0, lay.rows)
        foreign = block(~mine, cm[cols[~mine]], plan.recv_len)
        yl = oracle.spmv_csr(own, x_own.numpy(), 2.0, -1.0, y[lay.r0:lay.r1])
        yl = oracle.spmv_csr(foreign, recv.numpy(), 2.0, 1.0, yl)
        ref = oracle.spmv_csr(A, x, 2.0, -1.0, y)[lay.r0:lay.r1]
        ok = bool(np.array_equal(yl, ref))
        # halo volume: a banded matrix receives only its neighbours' band rows
        if case == "lap":
            ok = ok and plan.S <= 37
        q.put(ok)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("case", ["lap", "band", "rmat"])
def test_halo_exchange_gloo(world, case):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_halo_worker, args=(r, world, port, case, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    assert all(res), res
