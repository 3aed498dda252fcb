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

``FusedIteratedSpMV`` removes the separate collective:
each rank's SpMV epilogue stores its slice straight into every rank's next-x
buffer (``spaden_spmv_scatter``; peer pointers from torch symmetric memory, i.e.
NVLink-mapped allocations), followed by one device-side barrier per iteration.

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


def convert_slice(rowptr, colidx, values, n: int, storage=None, residual_max_popc: int = 0, group=None,
                  stream=None):
    """Convert this rank's row slice (local rows, global columns).  With the
    automatic hybrid choice (residual_max_popc = -1) and several ranks, the
    choice is taken from the WHOLE matrix's mean block fill: each rank counts
    its slice's blocks (spaden_count_blocks; Bnnz is additive over 8-row-aligned
    slices), one all-reduce sums (nnz, Bnnz), and every rank converts with that
    fill -- so all slices take the same t and y stays partition invariant."""
    import torch
    import torch.distributed as dist

    import paper_conf_icpp_cheny24_b200 as sp

    fill = 0.0
    if residual_max_popc < 0 and dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        cnt = torch.tensor([float(colidx.numel()), float(sp.count_blocks(rowptr, colidx, n, stream=stream))],
                           dtype=torch.float64, device=rowptr.device)
        dist.all_reduce(cnt, group=group)
        nnz, bnnz = float(cnt[0]), float(cnt[1])
        fill = min(64.0, nnz / bnnz) if bnnz > 0 else 64.0
    return sp.convert(rowptr, colidx, values, n, storage=storage, stream=stream,
                      residual_max_popc=residual_max_popc, auto_mean_fill=fill)


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
        self.gather_events = None  # (start, end) CUDA events around the all-gather (bench timing)

    def local_slot(self, buf):
        s = self.part.slice_rows
        return buf[self.rank * s:(self.rank + 1) * s]

    def step(self, alpha: float = 1.0, c: float | None = None):
        slot = self.local_slot(self.x_next)
        y = slot[: self.r1 - self.r0]
        if c is not None:
            y.fill_(c)
        self.local_spmv(self.x[: self.n], y, alpha, 0.0 if c is None else 1.0)
        ev = self.gather_events
        if ev is not None:
            ev[0].record()
        gather_slices(self.x_next[: self.part.padded], slot, self.group)
        if ev is not None:
            ev[1].record()
        self.x, self.x_next = self.x_next, self.x
        return self.x


class FusedIteratedSpMV:
    """Iterated SpMV with the all-gather fused into the SpMV epilogue (NEXT-2).

    Two x buffers (ping/pong), each replicated on every rank.  ``bufs[k][p]`` is
    rank p's copy of buffer k as seen from this rank (a peer tensor).  One step
    reads ``bufs[cur][rank][:n]`` and, through ``matrix.spmv_scatter``, writes
    rows [r0, r1) of y into ``bufs[1-cur][p][r0:r1]`` for every p; then
    ``barrier()``.  The single barrier per step covers both hazards: every slot
    of the next x is written before anyone reads it, and no rank writes into a
    buffer (step k+1 targets bufs[cur]) that a slower rank is still reading.

    ``matrix`` needs ``spmv_scatter(x, out_ptrs, out_offset, y=, alpha=, beta=)``.
    ``buffers`` = (bufs0, bufs1, barrier) injects the peer views (tests emulate
    several ranks on one device); by default they come from torch symmetric
    memory (world > 1) or are local tensors (world == 1 / no process group).
    """

    def __init__(self, part: RowPartition, n: int, matrix, x0, rank: int, group=None, buffers=None):
        import torch

        self.part, self.n, self.rank, self.group = part, n, rank, group
        self.matrix = matrix
        self.r0, self.r1 = part.range(rank)
        L = max(part.padded, n)
        if buffers is None:
            buffers = _symmetric_buffers(L, part.world, rank, group, x0.device)
        self.bufs = [list(buffers[0]), list(buffers[1])]
        self.barrier = buffers[2]
        if len(self.bufs[0]) != part.world or len(self.bufs[1]) != part.world:
            raise ValueError("need one peer view per rank")
        if part.world > 8:
            raise ValueError("spaden_spmv_scatter stores to at most 8 peers (one node)")
        self.cur = 0
        own = self.bufs[0][rank]
        own.zero_()
        own[: x0.numel()].copy_(x0)
        self.barrier()
        del torch

    @property
    def x(self):
        return self.bufs[self.cur][self.rank]

    def step(self, alpha: float = 1.0, c: float | None = None):
        dst = self.bufs[1 - self.cur]
        y, beta = None, 0.0
        if c is not None:
            y = dst[self.rank][self.r0:self.r1]
            y.fill_(c)
            beta = 1.0
        if self.r1 > self.r0:
            self.matrix.spmv_scatter(self.x[: self.n], [t.data_ptr() for t in dst], self.r0,
                                     y=y, alpha=alpha, beta=beta)
        self.barrier()
        self.cur = 1 - self.cur
        return self.x


def _symmetric_buffers(L: int, world: int, rank: int, group, device, force_symmetric: bool = False):
    """Two length-L fp32 buffers visible to every rank (peer views) + a barrier.
    ``force_symmetric`` takes the symmetric-memory path even for one rank (tests)."""
    import torch
    import torch.distributed as dist

    if (world == 1 and not force_symmetric) or not (dist.is_available() and dist.is_initialized()):
        if world != 1:
            raise RuntimeError("world > 1 needs an initialised process group")
        a = torch.zeros(L, dtype=torch.float32, device=device)
        b = torch.zeros(L, dtype=torch.float32, device=device)
        return [a], [b], (lambda: None)
    import torch.distributed._symmetric_memory as symm_mem

    grp = group if group is not None else dist.group.WORLD
    views = []
    handles = []
    for _ in range(2):
        t = symm_mem.empty(L, dtype=torch.float32, device=device)
        h = symm_mem.rendezvous(t, grp)
        handles.append((t, h))
        views.append([t if p == rank else h.get_buffer(p, (L,), torch.float32) for p in range(world)])
    h0 = handles[0][1]

    def barrier():
        h0.barrier(channel=0)

    barrier._keepalive = handles  # the allocations must outlive the views
    return views[0], views[1], barrier
