"""World size 2 through the real kernels (§8(a) a14/a15, §8(e)): two processes share
cuda:0 and talk over gloo (the collectives stage through host memory -- NCCL refuses two
ranks on one device), so DistSpMV / HaloSpMV run their full step -- pack, exchange,
shard SpMV, own/foreign overlap blocks -- across real ranks.  Compared with the oracle:
bit-exact in the integer regime (P5), within the north_star bound otherwise.  The
rank-local R-MAT construction (GPU generator, values for the rank's rows only) is
checked against the host generator's matrix through the same comparison."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import matgen
import oracle

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _check(y, A, x, y0, alpha, beta, exact, tol=1e-12):
    if exact:
        ref = oracle.spmv_csr(A, x, alpha, beta, y0)
        return bool(np.array_equal(y, ref)), "bit-exact"
    ref, bound = oracle.spmv_csr(A, x, alpha, beta, y0, with_bound=True)
    ok, ratio, nbad = oracle.check_tolerance(y, ref, bound, tol)
    return bool(ok), f"max ratio {ratio:.3g}, {nbad} rows out"


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    try:
        dist.init_process_group("gloo", rank=rank, world_size=world, timeout=__import__("datetime").timedelta(seconds=120))
    except Exception:                                   # report the rendezvous failure (retried)
        import traceback
        q.put((rank, [("exception", False, traceback.format_exc())]))
        return
    out = []
    try:
        import paper_conf_ipps_nisassvs18_b200 as sp
        from paper_conf_ipps_nisassvs18_b200.dist import DistSpMV, HaloSpMV

        def step(op, A, x, y, alpha, beta, reps=2):
            lay = op.layout
            xl = torch.from_numpy(x[lay.r0:lay.r1].copy()).cuda()
            for _ in range(reps):                         # the second step reuses every buffer
                yl = torch.from_numpy(y[lay.r0:lay.r1].copy()).cuda()
                op.run(alpha, beta, yl, x_local=xl)
            torch.cuda.synchronize()
            return op.gather_y(yl).cpu().numpy()

        cases = [("rmat11_int", matgen.rmat(11, seed=51, kind="int"), "int", True),
                 ("rmat11", matgen.rmat(11, seed=52), "f64", False),
                 ("ragged", matgen.from_lengths(np.r_[np.zeros(300, np.int64), np.full(2000, 7),
                                                      [2400], np.zeros(200, np.int64)], 2501, seed=53), "f64", False)]
        for name, A, kind, exact in cases:
            x = matgen.vector(A.n_cols, 54, 1, kind)
            y = matgen.vector(A.n_rows, 54, 2, kind)
            dA = sp.CSR.from_host(A)
            for fmt in ("csr", "merge", "csr5", "coo", "hyb"):
                for compress in (False, True):
                    for overlap in (False, True):
                        op = DistSpMV(dA, fmt, compress=compress, overlap=overlap)
                        got = step(op, A, x, y, 1.5 if not exact else 2.0, -0.5 if not exact else -1.0)
                        ok, how = _check(got, A, x, y, 1.5 if not exact else 2.0, -0.5 if not exact else -1.0, exact)
                        out.append((f"dist {name} {fmt} compress={compress} overlap={overlap}", ok, how))
        # halo exchange on a banded matrix (integer regime: bit-exact)
        A = matgen.laplacian5(64, kind="int")
        x = matgen.vector(A.n_cols, 55, 1, "int")
        y = matgen.vector(A.n_rows, 55, 2, "int")
        for fmt in ("csr", "ell", "csr5", "coo", "hyb", "merge"):
            for foreign in ("full", "compressed", "auto"):
                op = HaloSpMV(sp.CSR.from_host(A), fmt, foreign=foreign)
                ok, how = _check(step(op, A, x, y, 2.0, -1.0), A, x, y, 2.0, -1.0, True)
                # compressed: the foreign block runs over its 64 boundary rows only (A33)
                shape = (op.frows is None) if foreign == "full" else \
                    (op.frows is not None and op.frows.numel() == 64) if foreign == "compressed" else True
                out.append((f"halo lap64 {fmt} S={op.plan.S} foreign={foreign}", ok and op.plan.S <= 64 and shape, how))
        # rank-local R-MAT: GPU generator, values of the rank's rows only
        for kind, exact in (("int", True), ("f64", False)):
            Ah = matgen.rmat(12, seed=56, kind=kind)
            x = matgen.vector(Ah.n_cols, 57, 1, kind)
            y = matgen.vector(Ah.n_rows, 57, 2, kind)
            for compress, overlap in ((True, True), (False, False)):
                op = DistSpMV.from_rmat(12, "csr5", compress=compress, overlap=overlap, kind=kind, seed=56)
                ok, how = _check(step(op, Ah, x, y, 1.0, 1.0), Ah, x, y, 1.0, 1.0, exact)
                out.append((f"from_rmat 12 {kind} compress={compress} overlap={overlap} nnz={op.nnz_total}",
                            ok and op.nnz_total == Ah.nnz, how))
        q.put((rank, out))
    except Exception as e:                                  # surface the failure to the test
        import traceback
        q.put((rank, [("exception", False, traceback.format_exc())]))
        raise e
    finally:
        dist.destroy_process_group()


def _rendezvous_failure(res):
    """A rank failed before any check ran, on the rendezvous itself (the port taken between
    _free_port and init, a refused connection): worth one more attempt on a new port."""
    for lst in res.values():
        for name, ok, how in lst:
            if name == "exception" and not ok and any(
                    k in how for k in ("Address already in use", "EADDRINUSE", "Connection refused",
                                       "Connection reset", "ECONNREFUSED", "timed out")):
                return True
    return False


def test_world2_two_ranks_one_gpu():
    ctx = mp.get_context("spawn")
    for attempt in range(3):
        q = ctx.Queue()
        port = _free_port()
        procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
        for p in procs:
            p.start()
        res = dict(q.get(timeout=900) for _ in procs)
        for p in procs:
            p.join(timeout=120)
        if not _rendezvous_failure(res):
            break
    bad = [(r, c) for r, lst in res.items() for c in lst if not c[1]]
    assert not bad, bad
    assert all(len(lst) == len(res[0]) for lst in res.values())
