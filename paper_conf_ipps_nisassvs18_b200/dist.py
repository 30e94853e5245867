"""Row-partitioned multi-GPU SpMV.

The rows of a square matrix are split at nnz-balanced merge-path diagonals
(``spmv_partition``: splits[k] = row coordinate of the merge path of row ends and
nonzeros at diagonal floor(k*(n_rows+nnz)/P), the decomposition of the merge-based
CSR of PAPER.md:103).  Rank k owns rows [splits[k], splits[k+1]) of A, y and x.
Each SpMV step packs the rank's x slice into its slot, exchanges the slots and runs
the rank's shard (columns rewritten by ``spmv_slice_remap`` to slots of the gathered
vector: column j owned by rank o lives at o*S + (j - splits[o]), or through the
compressed / halo column maps).  y stays sharded (for a square A the y slice is the
next step's x slice).

Exchanges:
  * all-gather of equal-count slots (``all_gather_into_tensor`` on NCCL over
    NVLink/NVSwitch), dense or compressed to the referenced columns, optionally
    overlapped with the rank's own-column block (``DistSpMV``);
  * point-to-point halo (``all_to_all_single``) for banded matrices (``HaloSpMV``).
On a gloo group (CPU tests, and the GPU tests that run two ranks on one device) the
same collectives are staged through host memory.

Only plumbing lives here; every index map and every product is a libspmv kernel.
``ShardLayout`` is pure host logic shared with the gloo CPU tests.
"""
from __future__ import annotations

import time
from dataclasses import dataclass
from typing import Optional

import numpy as np
import torch
import torch.distributed as dist

from .spmv import (CSR, convert, partition, slice_remap, spmv_colmap_pack_index, spmv_compress_rows, spmv_gather, spmv_halo_colmap, spmv_scatter,
                   spmv_partition_colmap, spmv_slice_remap_colmap, spmv_slice_split)


@dataclass
class ShardLayout:
    """Ownership of rows / x slots for one rank of a P-way row partition."""
    splits: np.ndarray
    rank: int

    @property
    def P(self) -> int:
        return int(self.splits.size - 1)

    @property
    def S(self) -> int:
        """Slot size of the gathered x: the largest part."""
        return int(np.max(np.diff(self.splits))) if self.P else 0

    @property
    def r0(self) -> int:
        return int(self.splits[self.rank])

    @property
    def r1(self) -> int:
        return int(self.splits[self.rank + 1])

    @property
    def rows(self) -> int:
        return self.r1 - self.r0

    def local_slice(self, v):
        """This rank's rows of a full-length vector."""
        return v[self.r0:self.r1]

    def pack_x(self, x_local, out=None):
        """x_local (rows) -> padded slot of length S (zeros past the owned rows)."""
        if out is None:
            out = x_local.new_zeros(self.S)
        out[: self.rows] = x_local
        if self.rows < self.S:
            out[self.rows:] = 0
        return out

    def slot_of(self, j: int) -> int:
        """Gathered-x slot of global column j (the remap applied by spmv_slice_remap)."""
        o = int(np.searchsorted(self.splits, j, side="right")) - 1
        o = min(o, self.P - 1)
        return o * self.S + (j - int(self.splits[o]))


def is_nccl(group=None) -> bool:
    return dist.get_backend(group) == "nccl"


def all_gather_slots(x_gathered: torch.Tensor, x_slot: torch.Tensor, group=None):
    """Equal-count all-gather of the padded slots.  NCCL: all_gather_into_tensor on the
    device; gloo: list all_gather of host tensors (CUDA tensors staged through host)."""
    if is_nccl(group):
        dist.all_gather_into_tensor(x_gathered, x_slot, group=group)
        return x_gathered
    src = x_slot.cpu() if x_slot.is_cuda else x_slot
    out = torch.empty(x_gathered.numel(), dtype=x_gathered.dtype) if x_gathered.is_cuda else x_gathered
    parts = list(out.view(dist.get_world_size(group), -1).unbind(0))
    dist.all_gather(parts, src, group=group)
    if x_gathered.is_cuda:
        x_gathered.copy_(out)
    return x_gathered


def all_to_all_slots(recv: torch.Tensor, send: torch.Tensor, out_splits, in_splits, group=None, async_op=False):
    """all_to_all_single with uneven splits (halo).  gloo: CUDA tensors staged through host."""
    if is_nccl(group):
        return dist.all_to_all_single(recv, send, output_split_sizes=list(out_splits),
                                      input_split_sizes=list(in_splits), group=group, async_op=async_op)
    s = send.cpu() if send.is_cuda else send
    r = torch.empty(recv.numel(), dtype=recv.dtype) if recv.is_cuda else recv
    dist.all_to_all_single(r, s, output_split_sizes=list(out_splits), input_split_sizes=list(in_splits), group=group)
    if recv.is_cuda:
        recv.copy_(r)
    return None


def _agree(splits: np.ndarray, group, device) -> None:
    """Every rank computed the same partition (deterministic kernel, same matrix)."""
    t = torch.tensor(splits, dtype=torch.int64)
    if is_nccl(group):
        t = t.to(device)
    t0 = t.clone()
    dist.broadcast(t0, src=dist.get_global_rank(group, 0) if group is not None else 0, group=group)
    if not torch.equal(t, t0):
        raise RuntimeError("ranks disagree on the row partition (different matrices?)")


class RowRangeCSR(CSR):
    """A square matrix whose row_ptr and col are complete but whose values exist only for
    the nonzeros [k0, k0 + val.numel()) -- one rank's rows.  Everything the partition,
    column-map and own-shard calls read (row_ptr everywhere, col everywhere for the
    column maps, values only inside the rank's rows) is present; the value pointer
    handed to libspmv is offset so that nonzero k maps to val[k - k0]."""

    def __init__(self, row_ptr: torch.Tensor, col: torch.Tensor, val_local: torch.Tensor, n: int, k0: int):
        self.row_ptr, self.col, self.val = row_ptr.contiguous(), col.contiguous(), val_local.contiguous()
        self.n_rows = self.n_cols = int(n)
        self.nnz = int(col.numel())
        self.k0 = int(k0)

    def as_c(self):
        c = super().as_c()
        if self.val.numel():
            c.vals = self.val.data_ptr() - self.k0 * self.val.element_size()
        elif self.nnz:
            c.vals = self.col.data_ptr()     # no values yet: only for calls that never read them
        return c

    def bytes(self) -> int:
        return self.row_ptr.numel() * self.row_ptr.element_size() + self.nnz * 4 + \
            self.val.numel() * self.val.element_size()


class DistSpMV:
    """One rank's part of y = alpha*A*x + beta*y for a row-partitioned square A.

    ``A`` holds at least this rank's rows' values (a full ``CSR`` built identically on every
    rank, or a ``RowRangeCSR`` from ``from_rmat``); the partition kernel is deterministic and
    rank 0's splits are broadcast and checked.
    ``compress=True`` exchanges only the columns some row references:
    slots of S' = max referenced columns per part, packed every step by ``spmv_gather``.
    ``overlap=True`` splits the shard into its own-column block, run on the rank's x slice
    while the all-gather is in flight, and its foreign-column block, run (accumulating,
    beta = 1) once the gather lands.
    """

    def __init__(self, A: CSR, fmt: str = "csr5", group=None, compress: bool = False, overlap: bool = False,
                 **convert_opts):
        if A.n_rows != A.n_cols:
            raise ValueError("DistSpMV needs a square matrix (x is owned like y)")
        self.group = group
        P = dist.get_world_size(group)
        rank = dist.get_rank(group)
        dev = A.row_ptr.device
        splits = partition(A, P)
        _agree(splits, group, dev)
        self.layout = ShardLayout(splits, rank)
        self.compress, self.overlap, self.fmt = compress, overlap, fmt
        colmap = None
        if compress:
            colmap, S = spmv_partition_colmap(A, splits)
            self.shard = spmv_slice_remap_colmap(A, splits, rank, colmap, S)
            self.pack_idx = spmv_colmap_pack_index(colmap, splits, rank, S)
        else:
            self.shard, S = slice_remap(A, splits, rank)
            assert S == self.layout.S
            self.pack_idx = None
        self.slot = S
        self.dtype = A.val.dtype
        self.handle = convert(self.shard, fmt, **convert_opts)
        if overlap:
            lay = self.layout
            self.own = convert(spmv_slice_split(A, splits, rank, 0), fmt, **convert_opts)
            self.foreign = convert(spmv_slice_split(A, splits, rank, 1, colmap, S), fmt, **convert_opts)
        self.x_own = torch.zeros(self.layout.rows, dtype=self.dtype, device=dev)
        self.x_slot = torch.zeros(S, dtype=self.dtype, device=dev)
        self.x_gathered = torch.zeros(P * S, dtype=self.dtype, device=dev)
        self.nccl = is_nccl(group)

    @classmethod
    def from_rmat(cls, scale: int, fmt: str = "csr5", group=None, compress: bool = True, overlap: bool = True,
                  kind: str = "f64", dtype=torch.float64, seed=None, edge_factor: int = 16, **convert_opts):
        """Rank-local construction of an R-MAT operator ("generated on
        the GPU, each rank builds identically and keeps its shard"): the GPU generator builds
        row_ptr and col on this rank's device, the partition comes from row_ptr, values are
        materialised for this rank's rows only, and everything but the shard is dropped."""
        import matgen
        from matgen.gpu import DeviceRMAT
        seed = matgen.SEEDS["rmat24"] if seed is None else seed
        g = DeviceRMAT(scale, edge_factor, seed)
        col = g.col()
        probe = RowRangeCSR(g.row_ptr, col, torch.empty(0, dtype=dtype, device=col.device), g.n, 0)
        splits = partition(probe, dist.get_world_size(group))
        rank = dist.get_rank(group)
        r0, r1 = int(splits[rank]), int(splits[rank + 1])
        k0, k1 = (int(v) for v in g.row_ptr[[r0, r1]].tolist())
        A = RowRangeCSR(g.row_ptr, col, g.values(k0, k1, kind=kind, dtype=dtype), g.n, k0)
        g.release()
        op = cls(A, fmt, group=group, compress=compress, overlap=overlap, **convert_opts)
        op.nnz_total, op.generated = g.nnz, dict(scale=scale, seed=seed, edge_factor=edge_factor, kind=kind)
        return op

    @property
    def rows(self) -> int:
        return self.layout.rows

    def exchange_bytes(self) -> int:
        """Bytes each rank receives per step."""
        return (self.layout.P - 1) * self.slot * self.x_slot.element_size()

    def set_x(self, x_local: torch.Tensor):
        """Stage this rank's x slice (length rows): the own copy and the padded / compressed slot
        (``spmv_gather``)."""
        self.x_own.copy_(x_local)
        if self.compress:
            spmv_gather(self.x_own, self.pack_idx, self.x_slot)
        else:
            self.layout.pack_x(self.x_own, out=self.x_slot)

    def exchange(self, async_op: bool = False):
        """All-gather the x slots (the one collective of a step); NCCL work handle or None."""
        if async_op and self.nccl:
            return dist.all_gather_into_tensor(self.x_gathered, self.x_slot, group=self.group, async_op=True)
        all_gather_slots(self.x_gathered, self.x_slot, self.group)
        return None

    def run(self, alpha, beta, y_local: torch.Tensor, x_local: Optional[torch.Tensor] = None):
        """y_local <- alpha*(A x)[r0:r1] + beta*y_local.  With x_local the step packs it first
        (pack -> exchange -> SpMV); without, the slot staged by the last set_x is reused."""
        if x_local is not None:
            self.set_x(x_local)
        if self.overlap:
            work = self.exchange(async_op=True)
            self.own.run(alpha, self.x_own, beta, y_local)        # overlaps the exchange
            if work is not None:
                work.wait()                                       # compute stream waits for the gather
            self.foreign.run(alpha, self.x_gathered, 1.0, y_local)
            return y_local
        self.exchange()
        self.handle.run(alpha, self.x_gathered, beta, y_local)
        return y_local

    def run_local(self, alpha, beta, y_local: torch.Tensor):
        """The step's compute alone (no pack, no exchange): for the overlap accounting."""
        if self.overlap:
            self.own.run(alpha, self.x_own, beta, y_local)
            self.foreign.run(alpha, self.x_gathered, 1.0, y_local)
        else:
            self.handle.run(alpha, self.x_gathered, beta, y_local)
        return y_local

    def local_bytes(self) -> int:
        """Algorithmic bytes of this rank's SpMV kernels per step."""
        if self.overlap:
            return self.own.info()["bytes_per_run"] + self.foreign.info()["bytes_per_run"] - \
                self.rows * self.x_own.element_size() * 2        # y read/written once, not twice
        return self.handle.info()["bytes_per_run"]

    def launches(self) -> int:
        n = self.own.launches() + self.foreign.launches() if self.overlap else self.handle.launches()
        return n + (1 if self.compress else 0)

    def gather_y(self, y_local: torch.Tensor) -> torch.Tensor:
        """Assemble the full y on every rank (verification only; untimed)."""
        P, S = self.layout.P, self.layout.S
        buf = torch.zeros(P * S, dtype=y_local.dtype, device=y_local.device)
        slot = self.layout.pack_x(y_local)
        all_gather_slots(buf, slot, self.group)
        return torch.cat([buf[k * S: k * S + int(self.layout.splits[k + 1] - self.layout.splits[k])]
                          for k in range(P)])


# ---------------------------------------------------------------------- halo exchange

class LibspmvHaloIndex:
    """Index maps of the halo plan from libspmv (``spmv_halo_colmap`` +
    ``spmv_colmap_pack_index``) on the matrix's device."""

    @staticmethod
    def colmap(A, splits, k):
        return spmv_halo_colmap(A, splits, k)

    @staticmethod
    def pack(colmap, splits, rank, S):
        return spmv_colmap_pack_index(colmap, splits, rank, S)


class HaloPlan:
    """Point-to-point halo exchange for a row partition: receiver k gets,
    from each owner o != k, exactly the x entries of o's rows that k's rows reference,
    padded to S_k = max_o (count from o).  Receiver k's buffer holds slot o at
    [o*S_k, o*S_k + count); ``colmap`` maps each foreign column j referenced by this rank to
    its buffer position (-1 elsewhere), the layout ``spmv_slice_split(which=1, colmap)``
    remaps the foreign block through.  A banded matrix (LAP) exchanges its 2 x band rows
    per rank instead of the whole x.  The index maps come from ``index`` (default: the
    libspmv calls; the CPU gloo tests pass the oracle's); a step is one ``spmv_gather`` pack
    + one all_to_all_single."""

    def __init__(self, A, splits, rank: int, index=LibspmvHaloIndex):
        self.splits = np.asarray(splits, np.int64)
        self.P, self.rank = int(self.splits.size - 1), int(rank)
        self.slots = []                  # S_k per receiver
        self.sent_counts = []
        send = []                        # this rank's pack indices, per receiver, padded to S_k
        for k in range(self.P):
            cm, counts, S = index.colmap(A, self.splits, k)
            if k == self.rank:
                self.colmap, self.S, self.recv_counts = cm, int(S), np.asarray(counts)
            idx = torch.as_tensor(index.pack(cm, self.splits, self.rank, S))
            self.slots.append(int(S))
            self.sent_counts.append(int(idx.numel()))
            pad = torch.zeros(int(S), dtype=torch.int32, device=idx.device)
            pad[: idx.numel()] = idx.to(torch.int32)
            send.append(pad)
        self.send_index = torch.cat(send)                       # length sum_k S_k

    @property
    def recv_len(self) -> int:
        return self.P * self.S

    def exchange_bytes(self, elem: int) -> int:
        """Bytes this rank receives per step (padded slots, self excluded)."""
        return (self.P - 1) * self.S * elem

    def exchange(self, send_buf: torch.Tensor, recv_buf: torch.Tensor, group=None, async_op: bool = False):
        return all_to_all_slots(recv_buf, send_buf, [self.S] * self.P, self.slots, group=group, async_op=async_op)


def _compressed_faster(full, comp, rows, yf, n_rows, n_cols, reps: int = 5) -> bool:
    """A33 choice on this rank: the foreign block over every row (one run) or over its
    non-empty rows (gather, run, scatter) -- whichever takes less device time (CUDA events
    around `reps` back-to-back steps, after a warm-up; scratch vectors)."""
    dt = yf.dtype
    y = torch.zeros(n_rows, dtype=dt, device=yf.device)
    x = torch.zeros(max(n_cols, 1), dtype=dt, device=yf.device)
    s = torch.cuda.current_stream()

    def t(fn):
        fn()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        for _ in range(reps):
            fn()
        b.record(s)
        b.synchronize()
        return a.elapsed_time(b)

    def run_comp():
        spmv_gather(y, rows, yf)
        comp.run(1.0, x, 1.0, yf)
        spmv_scatter(yf, rows, y)

    return t(run_comp) < t(lambda: full.run(1.0, x, 1.0, y))


class HaloSpMV:
    """Row-partitioned y = alpha*A*x + beta*y with a halo exchange instead of the x
    all-gather.  Own-column block on the rank's x slice (overlapping
    the exchange on NCCL), foreign-column block on the received halo (beta = 1)."""

    def __init__(self, A: CSR, fmt: str = "csr", group=None, foreign: str = "auto", **convert_opts):
        """foreign: "auto" (A33: the faster of the two on this rank), "full" (the foreign
        block over every row) or "compressed" (over its non-empty rows)."""
        if A.n_rows != A.n_cols:
            raise ValueError("HaloSpMV needs a square matrix (x is owned like y)")
        if foreign not in ("auto", "full", "compressed"):
            raise ValueError(foreign)
        self.group = group
        P = dist.get_world_size(group)
        rank = dist.get_rank(group)
        splits = partition(A, P)
        _agree(splits, group, A.row_ptr.device)
        self.layout = ShardLayout(splits, rank)
        self.fmt = fmt
        self.plan = HaloPlan(A, splits, rank)
        self.own = convert(spmv_slice_split(A, splits, rank, 0), fmt, **convert_opts)
        F = spmv_slice_split(A, splits, rank, 1, self.plan.colmap, self.plan.S)
        # A33: a banded matrix's foreign block holds a few thousand non-empty rows among the
        # rank's millions -- run it over those rows only (gather their y, SpMV with beta = 1,
        # scatter back: the same single rounding as the full block), not over every row --
        # when that is faster for this format and shard: the formats that walk every row
        # (CSR, ELL/HYB, merge) gain on large shards, the nonzero-driven ones (COO, CSR5)
        # already skip rows without work and lose the extra launches (tools/halo_local_time.py)
        dev, self.dtype = A.row_ptr.device, A.val.dtype
        rows, rp_c = spmv_compress_rows(F)
        self.frows, self.yf = None, torch.zeros(0, dtype=self.dtype, device=dev)
        self.foreign = convert(F, fmt, **convert_opts) if F.nnz > 0 else None
        if self.foreign is not None and foreign != "full" and (foreign == "compressed" or rows.numel() * 4 <= F.n_rows):
            comp = convert(CSR(rp_c, F.col, F.val, (rows.numel(), F.n_cols)), fmt, **convert_opts)
            yf = torch.zeros(rows.numel(), dtype=self.dtype, device=dev)
            if foreign == "compressed" or _compressed_faster(self.foreign, comp, rows, yf, F.n_rows, F.n_cols):
                self.foreign, self.frows, self.yf = comp, rows, yf
        self.x_own = torch.zeros(self.layout.rows, dtype=self.dtype, device=dev)
        self.send = torch.zeros(self.plan.send_index.numel(), dtype=self.dtype, device=dev)
        self.recv = torch.zeros(self.plan.recv_len, dtype=self.dtype, device=dev)
        self.nccl = is_nccl(group)
        self.overlap, self.compress = True, False

    @property
    def rows(self) -> int:
        return self.layout.rows

    def exchange_bytes(self) -> int:
        return self.plan.exchange_bytes(self.recv.element_size())

    def set_x(self, x_local: torch.Tensor):
        self.x_own.copy_(x_local)
        spmv_gather(self.x_own, self.plan.send_index, self.send)    # pack every receiver's halo

    def exchange(self, async_op: bool = False):
        return self.plan.exchange(self.send, self.recv, self.group, async_op=async_op and self.nccl)

    def run(self, alpha, beta, y_local: torch.Tensor, x_local: Optional[torch.Tensor] = None):
        if x_local is not None:
            self.set_x(x_local)
        work = self.exchange(async_op=True)
        self.own.run(alpha, self.x_own, beta, y_local)              # overlaps the exchange
        if work is not None:
            work.wait()
        self._foreign(alpha, y_local)
        return y_local

    def _foreign(self, alpha, y_local: torch.Tensor):
        if self.foreign is None:
            return
        if self.frows is None:
            self.foreign.run(alpha, self.recv, 1.0, y_local)
        elif self.frows.numel():
            spmv_gather(y_local, self.frows, self.yf)
            self.foreign.run(alpha, self.recv, 1.0, self.yf)
            spmv_scatter(self.yf, self.frows, y_local)

    def run_local(self, alpha, beta, y_local: torch.Tensor):
        self.own.run(alpha, self.x_own, beta, y_local)
        self._foreign(alpha, y_local)
        return y_local

    def local_bytes(self) -> int:
        V = self.x_own.element_size()
        b = self.own.info()["bytes_per_run"]
        if self.foreign is None:
            return b
        if self.frows is None:                  # y read + written once, by the own block
            return b + self.foreign.info()["bytes_per_run"] - self.rows * V * 2
        k = self.frows.numel()                  # + gather / scatter of the compressed rows' y
        return b + self.foreign.info()["bytes_per_run"] + k * (4 + V) * 2

    def launches(self) -> int:
        f = 0 if self.foreign is None else self.foreign.launches() + (2 if self.frows is not None else 0)
        return self.own.launches() + f + 1

    def gather_y(self, y_local: torch.Tensor) -> torch.Tensor:
        P, S = self.layout.P, self.layout.S
        buf = torch.zeros(P * S, dtype=y_local.dtype, device=y_local.device)
        all_gather_slots(buf, self.layout.pack_x(y_local), self.group)
        return torch.cat([buf[k * S: k * S + int(self.layout.splits[k + 1] - self.layout.splits[k])]
                          for k in range(P)])


def time_exchange(op, iters: int = 20) -> float:
    """Mean ms of the exchange alone (pack + collective), CUDA events on the current stream
    (NCCL collectives issued without async_op are ordered on it)."""
    s = torch.cuda.current_stream()
    for _ in range(3):
        op.exchange()
    torch.cuda.synchronize()
    if dist.is_initialized():
        dist.barrier(group=op.group)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    a.record(s)
    for _ in range(iters):
        op.exchange()
    b.record(s)
    torch.cuda.synchronize()
    wall = (time.perf_counter() - t0) * 1e3 / iters
    ev = a.elapsed_time(b) / iters
    return ev if op.nccl else wall
