"""Row-partitioned multi-GPU SpMV: host-side plumbing only.

A is cut into contiguous, 8-row-aligned slices of equal size
``slice_rows = ceil(m / (8 P)) * 8`` (the last one padded with empty rows), one
per rank.  Each rank converts its slice (local rows, global columns) with
``spaden_convert_csr_to_bitmap`` and computes its slice of y with
``spaden_spmv``.  For iterated SpMV the replicated x is rebuilt with one
``all_gather_into_tensor`` per iteration (NCCL over NVLink/NVSwitch on GPUs;
gloo in the CPU tests) -- the only exchange step the method has.  Because every
block-row's summation order depends only on that block-row, the gathered
vector is bitwise equal to the single-GPU result.

Nothing here computes: the SpMV is passed in (the CUDA path in production, the
oracle in the CPU tests).
"""
from __future__ import annotations

from dataclasses import dataclass


@dataclass(frozen=True)
class RowPartition:
    m: int
    world: int

    @property
    def slice_rows(self) -> int:
        return -(-self.m // (8 * self.world)) * 8 if self.m else 0

    @property
    def padded(self) -> int:
        """Length of the gathered vector (>= m): world * slice_rows."""
        return self.slice_rows * self.world

    def range(self, rank: int) -> tuple[int, int]:
        r0 = min(self.m, rank * self.slice_rows)
        r1 = min(self.m, (rank + 1) * self.slice_rows)
        return r0, r1


def gather_slices(full, local, group=None):
    """full[world*slice] <- concat over ranks of local[slice] (in rank order)."""
    import torch.distributed as dist

    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size(group) == 1:
        if full.data_ptr() != local.data_ptr():
            full[: local.numel()].copy_(local)
        return full
    try:
        dist.all_gather_into_tensor(full, local, group=group)
    except (RuntimeError, NotImplementedError):  # backends without the fused collective
        parts = list(full.chunk(dist.get_world_size(group)))
        dist.all_gather(parts, local.contiguous(), group=group)
    return full


class IteratedSpMV:
    """x_{k+1} = alpha * A x_k + c  with A row-partitioned across ranks.

    ``local_spmv(x_full_view, y_slice, alpha, beta)`` computes this rank's rows
    ``y_slice = alpha * A_r x + beta * y_slice`` (the CUDA path: Matrix.spmv).
    ``c`` (scalar) is added through ``beta = 1`` on a pre-filled slice.
    """

    def __init__(self, part: RowPartition, n: int, local_spmv, x0, rank: int, group=None):
        import torch

        self.part, self.n, self.rank, self.group = part, n, rank, group
        self.local_spmv = local_spmv
        L = max(part.padded, n)
        self.x = torch.zeros(L, dtype=torch.float32, device=x0.device)
        self.x[: x0.numel()].copy_(x0)
        self.x_next = torch.zeros_like(self.x)
        self.r0, self.r1 = part.range(rank)

    def local_slot(self, buf):
        s = self.part.slice_rows
        return buf[self.rank * s:(self.rank + 1) * s]

    def step(self, alpha: float = 1.0, c: float | None = None):
        slot = self.local_slot(self.x_next)
        y = slot[: self.r1 - self.r0]
        if c is not None:
            y.fill_(c)
        self.local_spmv(self.x[: self.n], y, alpha, 0.0 if c is None else 1.0)
        gather_slices(self.x_next[: self.part.padded], slot, self.group)
        self.x, self.x_next = self.x_next, self.x
        return self.x
