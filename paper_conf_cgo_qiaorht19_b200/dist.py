"""Row-band data parallelism across the GPUs of one node.

GPU g owns output rows [g*H/P, (g+1)*H/P).  One fused plan needs R =
plan.halo_rows input rows above and below its band (the accumulated vertical
stencil radius); those rows live on the neighbours g-1 and g+1 and are
exchanged with one point-to-point step per run (NCCL send/recv over
NVLink/NVSwitch via torch.distributed; gloo on CPU for tests).  The fused
kernels then run on the band through kf_run_band, applying border modes at the
GLOBAL image edges, so the banded result is bit-identical to a single-GPU run.

Plumbing only: the exchange is torch.distributed, the compute is libkfuse.
"""
from __future__ import annotations

from dataclasses import dataclass

import torch
import torch.distributed as dist


@dataclass
class Band:
    rank: int
    world: int
    height: int         # global image height
    halo: int           # R
    row0: int           # owned output rows [row0, row1)
    row1: int
    in0: int            # rows held in the input buffer [in0, in1)
    in1: int

    @property
    def rows(self) -> int:
        return self.row1 - self.row0

    @property
    def top(self) -> int:          # halo rows above the band actually present
        return self.row0 - self.in0

    @property
    def bottom(self) -> int:
        return self.in1 - self.row1


def partition(height: int, world: int, rank: int, halo: int) -> Band:
    """Balanced contiguous row bands; the halo is clipped at the global edges."""
    r0 = height * rank // world
    r1 = height * (rank + 1) // world
    if halo > r1 - r0 and world > 1:
        raise ValueError(f"band of {r1 - r0} rows is thinner than the halo {halo}")
    return Band(rank, world, height, halo, r0, r1, max(0, r0 - halo), min(height, r1 + halo))


def exchange_halos(buf: torch.Tensor, band: Band, group=None) -> None:
    """buf holds rows [in0, in1) of the global image (first dim = rows); the
    owned rows [row0, row1) are valid.  Fills the top/bottom halo rows from the
    neighbours: one batched send/recv step (no collective)."""
    if band.world == 1 or band.halo == 0:
        return
    ops = []
    t, b, n = band.top, band.bottom, band.rows
    if band.rank > 0:
        ops.append(dist.P2POp(dist.isend, buf[t:t + band.halo].contiguous(), band.rank - 1, group))
        ops.append(dist.P2POp(dist.irecv, buf[0:t], band.rank - 1, group))
    recv_bottom = None
    if band.rank < band.world - 1:
        ops.append(dist.P2POp(dist.isend, buf[t + n - band.halo:t + n].contiguous(), band.rank + 1, group))
        recv_bottom = buf[t + n:t + n + b]
        ops.append(dist.P2POp(dist.irecv, recv_bottom, band.rank + 1, group))
    for req in dist.batch_isend_irecv(ops):
        req.wait()


def split_rows(band: Band) -> tuple[tuple[int, int], list[tuple[int, int]]]:
    """Output rows of a band that need no halo row -- the core [row0 + t, row1 - b)
    with t (b) = R when a neighbour exists above (below), else 0 -- and the edge
    strips that do.  The core can run while the halo rows are in flight."""
    t = band.halo if band.rank > 0 else 0
    b = band.halo if band.rank < band.world - 1 else 0
    c0, c1 = band.row0 + t, band.row1 - b
    if c0 >= c1:
        return (band.row0, band.row0), [(band.row0, band.row1)]
    edges = [(r0, r1) for r0, r1 in ((band.row0, c0), (c1, band.row1)) if r1 > r0]
    return (c0, c1), edges


def run_step_overlapped(plan, band: Band, inputs, outputs, side_stream, group=None) -> None:
    """One multi-GPU step with the exchange hidden behind the band's core rows
    (SURVEY §8(e) "overlap"): the halo send/recv is posted first (NCCL runs on its
    own stream), the core rows run on `side_stream` meanwhile, then the current
    stream waits for the halo rows and computes the edge strips.  Output is
    bit-identical to exchange_halos + run_band (border modes act at the global
    edges in every call)."""
    cur = torch.cuda.current_stream()
    (c0, c1), edges = split_rows(band)
    side_stream.wait_stream(cur)                      # inputs of this step are ready
    reqs = []
    if band.world > 1 and band.halo > 0:
        reqs = _post_halos(inputs, band, group)
    if c1 > c0:
        with torch.cuda.stream(side_stream):
            outs = [o[c0 - band.row0:c1 - band.row0] for o in outputs]
            plan.run_band(c0, c1, inputs, band.in0, band.in1, outs, side_stream)
    for r in reqs:
        r.wait()
    for r0, r1 in edges:
        outs = [o[r0 - band.row0:r1 - band.row0] for o in outputs]
        plan.run_band(r0, r1, inputs, band.in0, band.in1, outs, cur)
    cur.wait_stream(side_stream)


def _post_halos(inputs, band: Band, group=None) -> list:
    ops = []
    t, b, n = band.top, band.bottom, band.rows
    for buf in inputs:
        if band.rank > 0:
            ops.append(dist.P2POp(dist.isend, buf[t:t + band.halo], band.rank - 1, group))
            ops.append(dist.P2POp(dist.irecv, buf[0:t], band.rank - 1, group))
        if band.rank < band.world - 1:
            ops.append(dist.P2POp(dist.isend, buf[t + n - band.halo:t + n], band.rank + 1, group))
            ops.append(dist.P2POp(dist.irecv, buf[t + n:t + n + b], band.rank + 1, group))
    return dist.batch_isend_irecv(ops) if ops else []


def run_band(plan, band: Band, inputs, outputs, stream=None) -> None:
    """inputs: device tensors holding rows [in0, in1) (halo exchanged);
    outputs: device tensors of band.rows rows."""
    plan.run_band(band.row0, band.row1, inputs, band.in0, band.in1, outputs, stream)
