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
