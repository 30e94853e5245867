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
