"""Row-partitioned multi-GPU SpMV.

The rows of a square matrix are split at nnz-balanced merge-path diagonals
(``spmv_partition``: splits[k] = row coordinate of the merge path of row ends and
nonzeros at diagonal floor(k*(n_rows+nnz)/P), the decomposition of the merge-based
CSR of PAPER.md:103).  Rank k owns rows [splits[k], splits[k+1]) of A, y and x.
Each SpMV step all-gathers x -- one equal-count ``all_gather_into_tensor`` of the
rank-local slices padded to S = max part rows (NCCL over NVLink/NVSwitch) -- and runs
the rank's shard, whose columns ``spmv_slice_remap`` rewrote to slots of the
gathered vector: column j owned by rank o lives at o*S + (j - splits[o]).  y stays
sharded (for a square A the y slice is the next step's x slice).

Only plumbing lives here; all compute is in libspmv kernels.  ``ShardLayout`` is
pure host logic shared with the gloo CPU tests (tests/test_dist_gloo.py).
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Optional

import numpy as np
import torch
import torch.distributed as dist

from .spmv import (CSR, convert, partition, slice_remap, spmv_colmap_pack_index, spmv_gather,
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


def all_gather_slots(x_gathered: torch.Tensor, x_slot: torch.Tensor, group=None):
    """Equal-count all-gather of the padded slots (NCCL: all_gather_into_tensor; gloo,
    used only by the CPU tests, has no into-tensor variant on every build)."""
    if dist.get_backend(group) == "nccl":
        dist.all_gather_into_tensor(x_gathered, x_slot, group=group)
    else:
        parts = list(x_gathered.view(dist.get_world_size(group), -1).unbind(0))
        dist.all_gather(parts, x_slot, group=group)
    return x_gathered


class DistSpMV:
    """One rank's part of y = alpha*A*x + beta*y for a row-partitioned square A.

    ``A`` is the full matrix on this rank's GPU (every rank builds the same one; the
    partition kernel is deterministic and rank 0's splits are broadcast and checked).
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
        splits = partition(A, P)
        t = torch.tensor(splits, dtype=torch.int64, device=A.row_ptr.device)
        t0 = t.clone()
        dist.broadcast(t0, src=dist.get_global_rank(group, 0) if group is not None else 0, group=group)
        if not torch.equal(t, t0):
            raise RuntimeError("ranks disagree on the row partition (different matrices?)")
        self.layout = ShardLayout(splits, rank)
        self.compress = compress
        dev = A.row_ptr.device
        if compress:
            colmap, S = spmv_partition_colmap(A, splits)
            self.shard = spmv_slice_remap_colmap(A, splits, rank, colmap, S)
            self.pack_idx = spmv_colmap_pack_index(colmap, splits, rank, S)
        else:
            self.shard, S = slice_remap(A, splits, rank)
            assert S == self.layout.S
            self.pack_idx = None
        self.slot = S
        self.handle = convert(self.shard, fmt, **convert_opts)
        self.overlap = overlap
        self._A, self._colmap = A, (colmap if compress else None)
        if overlap:
            self.own, self.foreign = self.split_handles(fmt, **convert_opts)
            self.x_own = torch.zeros(self.layout.rows, dtype=A.val.dtype, device=dev)
        self.dtype = A.val.dtype
        self.x_slot = torch.zeros(S, dtype=self.dtype, device=dev)
        self.x_gathered = torch.zeros(P * S, dtype=self.dtype, device=dev)

    @property
    def rows(self) -> int:
        return self.layout.rows

    def split_handles(self, fmt: str, **convert_opts):
        """(own-column block, foreign-column block) of this rank's shard in format `fmt`."""
        lay = self.layout
        own = convert(spmv_slice_split(self._A, lay.splits, lay.rank, 0), fmt, **convert_opts)
        foreign = convert(spmv_slice_split(self._A, lay.splits, lay.rank, 1, self._colmap, self.slot), fmt,
                          **convert_opts)
        return own, foreign

    def exchange_async(self):
        """Start the all-gather; returns the work handle (NCCL) or None (completed)."""
        if dist.get_backend(self.group) == "nccl":
            return dist.all_gather_into_tensor(self.x_gathered, self.x_slot, group=self.group, async_op=True)
        self.exchange()
        return None

    def exchange_bytes(self) -> int:
        """Bytes each rank receives per step."""
        return (self.layout.P - 1) * self.slot * self.x_slot.element_size()

    def set_x(self, x_local: torch.Tensor):
        """Stage this rank's x slice (length rows) into its padded / compressed slot."""
        if self.overlap:
            self.x_own.copy_(x_local)
        if self.compress:
            spmv_gather(x_local, self.pack_idx, self.x_slot)
        else:
            self.layout.pack_x(x_local, out=self.x_slot)

    def exchange(self):
        """All-gather the x slots (the one collective of a step)."""
        torch.cuda.nvtx.range_push("DistSpMV.exchange")
        try:
            return all_gather_slots(self.x_gathered, self.x_slot, self.group)
        finally:
            torch.cuda.nvtx.range_pop()

    def run(self, alpha, beta, y_local: torch.Tensor, x_local: Optional[torch.Tensor] = None):
        """y_local <- alpha*(A x)[r0:r1] + beta*y_local; x_local (optional) replaces the slot."""
        if x_local is not None:
            self.set_x(x_local)
        if self.overlap and dist.get_backend(self.group) == "nccl":
            work = dist.all_gather_into_tensor(self.x_gathered, self.x_slot, group=self.group, async_op=True)
            self.own.run(alpha, self.x_own, beta, y_local)        # overlaps the exchange
            work.wait()                                           # compute stream waits for the gather
            self.foreign.run(alpha, self.x_gathered, 1.0, y_local)
            return y_local
        self.exchange()
        if self.overlap:
            self.own.run(alpha, self.x_own, beta, y_local)
            self.foreign.run(alpha, self.x_gathered, 1.0, y_local)
            return y_local
        self.handle.run(alpha, self.x_gathered, beta, y_local)
        return y_local

    def gather_y(self, y_local: torch.Tensor) -> torch.Tensor:
        """Assemble the full y on every rank (verification only; untimed)."""
        P, S = self.layout.P, self.layout.S
        buf = torch.zeros(P * S, dtype=y_local.dtype, device=y_local.device)
        slot = self.layout.pack_x(y_local)
        all_gather_slots(buf, slot, self.group)
        return torch.cat([buf[k * S: k * S + int(self.layout.splits[k + 1] - self.layout.splits[k])]
                          for k in range(P)])


# ---------------------------------------------------------------------- halo exchange

class HaloPlan:
    """Point-to-point halo exchange for a row partition: receiver k gets,
    from each owner o != k, exactly the x entries of o's rows that k's rows reference,
    padded to S_k = max_o (count from o).  Receiver k's buffer holds slot o at
    [o*S_k, o*S_k + count); `colmap` maps each foreign column j referenced by this rank to
    its buffer position (-1 elsewhere), the layout ``spmv_slice_split(which=1, colmap)``
    remaps the foreign block through.  A banded matrix (LAP) exchanges its 2 x band
    rows per rank instead of the whole x.  Built once with tensor index ops on the
    matrix's device (setup plumbing); a step is one ``spmv_gather`` pack + one
    all_to_all_single.  Pure index logic: the gloo tests run it on CPU tensors."""

    def __init__(self, row_ptr: torch.Tensor, col: torch.Tensor, n_cols: int, splits, rank: int):
        dev = col.device
        sp = torch.as_tensor(np.asarray(splits, np.int64), device=dev)
        P = int(sp.numel() - 1)
        self.P, self.rank, self.splits = P, rank, np.asarray(splits, np.int64)
        self.slots = []                  # S_k per receiver
        send = []                        # this rank's pack indices, per receiver, padded to S_k
        self.sent_counts = []
        self.colmap = torch.full((n_cols,), -1, dtype=torch.int32, device=dev)
        for k in range(P):
            a, b = int(row_ptr[int(self.splits[k])]), int(row_ptr[int(self.splits[k + 1])])
            cols = col[a:b].to(torch.int64)
            own = torch.searchsorted(sp, cols, right=True) - 1
            u = torch.unique(cols[own != k])                   # sorted foreign columns of k
            ou = torch.searchsorted(sp, u, right=True) - 1
            cnt = torch.bincount(ou, minlength=P) if u.numel() else torch.zeros(P, dtype=torch.int64, device=dev)
            S = max(int(cnt.max()), 1)
            self.slots.append(S)
            first = torch.cumsum(cnt, 0) - cnt                 # start of each owner's run in u
            pos = torch.arange(u.numel(), device=dev) - first[ou]
            if k == rank:
                self.colmap[u] = (ou * S + pos).to(torch.int32)
            mine = u[ou == rank] - int(self.splits[rank])
            self.sent_counts.append(int(mine.numel()))
            pad = torch.zeros(S, dtype=torch.int32, device=dev)
            pad[: mine.numel()] = mine.to(torch.int32)
            send.append(pad)
        self.send_index = torch.cat(send)                       # length sum_k S_k
        self.S = self.slots[rank]                               # this rank's receive slot

    @property
    def recv_len(self) -> int:
        return self.P * self.S

    def exchange_bytes(self, elem: int) -> int:
        """Bytes this rank receives per step (padded slots, self excluded)."""
        return (self.P - 1) * self.S * elem

    def exchange(self, send_buf: torch.Tensor, recv_buf: torch.Tensor, group=None, async_op: bool = False):
        return dist.all_to_all_single(recv_buf, send_buf, output_split_sizes=[self.S] * self.P,
                                      input_split_sizes=list(self.slots), group=group, async_op=async_op)


class HaloSpMV:
    """Row-partitioned y = alpha*A*x + beta*y with a halo exchange instead of the x
    all-gather.  Own-column block on the rank's x slice (overlapping
    the exchange on NCCL), foreign-column block on the received halo (beta = 1)."""

    def __init__(self, A: CSR, fmt: str = "csr", group=None, **convert_opts):
        if A.n_rows != A.n_cols:
            raise ValueError("HaloSpMV needs a square matrix (x is owned like y)")
        self.group = group
        P = dist.get_world_size(group)
        rank = dist.get_rank(group)
        splits = partition(A, P)
        self.layout = ShardLayout(splits, rank)
        self.plan = HaloPlan(A.row_ptr, A.col, A.n_cols, splits, rank)
        self.own = convert(spmv_slice_split(A, splits, rank, 0), fmt, **convert_opts)
        self.foreign = convert(spmv_slice_split(A, splits, rank, 1, self.plan.colmap, self.plan.S), fmt,
                               **convert_opts)
        dev, self.dtype = A.row_ptr.device, A.val.dtype
        self.x_own = torch.zeros(self.layout.rows, dtype=self.dtype, device=dev)
        self.send = torch.zeros(self.plan.send_index.numel(), dtype=self.dtype, device=dev)
        self.recv = torch.zeros(self.plan.recv_len, dtype=self.dtype, device=dev)

    @property
    def rows(self) -> int:
        return self.layout.rows

    def exchange_bytes(self) -> int:
        return self.plan.exchange_bytes(self.recv.element_size())

    def set_x(self, x_local: torch.Tensor):
        self.x_own.copy_(x_local)
        spmv_gather(self.x_own, self.plan.send_index, self.send)    # pack every receiver's halo

    def run(self, alpha, beta, y_local: torch.Tensor, x_local: Optional[torch.Tensor] = None):
        if x_local is not None:
            self.set_x(x_local)
        nccl = dist.get_backend(self.group) == "nccl"
        work = self.plan.exchange(self.send, self.recv, self.group, async_op=nccl)
        self.own.run(alpha, self.x_own, beta, y_local)              # overlaps the exchange
        if work is not None:
            work.wait()
        self.foreign.run(alpha, self.recv, 1.0, y_local)
        return y_local
