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
    if plan.num_launches > 1:
        # a multi-block plan keeps its intermediates in one workspace: the core
        # and edge calls must not overlap (kfuse.h), so the core runs on `cur`
        side_stream = cur
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


# ---------------------------------------------------------------------------
# Halo rows over peer memory (NVLink P2P through CUDA IPC mappings): the north
# star's "read from peer memory over NVLink" path.  No host collective per
# step: three stream-ordered kernels of libkfuse (kf_peer_signal / _pull /
# _wait) synchronise through monotonic device counters, so a whole step --
# signal, core rows, halo pull, edge strips -- is plain launches on ONE stream
# and can be captured into a CUDA graph.  The exchange latency hides behind
# the core rows: a neighbour's signal is issued before its own core kernel.

# counter slots (uint32) of each rank
_READY_ABOVE, _READY_BELOW, _SEEN_ABOVE, _SEEN_BELOW, _ACK_ABOVE, _ACK_BELOW, _SENT, _ERR = range(8)


class PeerHalo:
    """Maps the neighbours' input buffers and counters into this process
    (torch.multiprocessing's CUDA IPC reductions, exchanged once with
    all_gather_object) and runs the band steps over them.

    bufs: this rank's rotating input buffer SETS.  A set is one tensor (a
    one-input pipeline) or a list with one tensor per pipeline input; each
    tensor holds rows [in0, in1) of its global image (first dim = rows).  Every
    rank must pass the same number of sets of the same shape, and call step()
    the same number of times with the same set indices, in the same order."""

    def __init__(self, band: Band, bufs, group=None, spin_limit: int = 1 << 27):
        from torch.multiprocessing.reductions import reduce_tensor
        self.band, self.spin = band, spin_limit
        self.bufs = [list(s) if isinstance(s, (list, tuple)) else [s] for s in bufs]
        if len({len(s) for s in self.bufs}) != 1 or not 1 <= len(self.bufs[0]) <= 8:
            raise ValueError("every buffer set must hold the same number (1..8) of input tensors")
        dev = self.bufs[0][0].device
        self.ctr = torch.zeros(8, dtype=torch.int32, device=dev)
        if band.world == 1:   # no neighbours: nothing to share
            self.up = self.down = None
            return
        mine = {"ctr": reduce_tensor(self.ctr), "bufs": [[reduce_tensor(t) for t in s] for s in self.bufs],
                "top": band.top, "rows": band.rows}
        every = [None] * band.world
        dist.all_gather_object(every, mine, group=group)

        def open_(red):
            fn, args = red
            return fn(*args)

        def peer(r):
            d = every[r]
            return {"ctr": open_(d["ctr"]), "bufs": [[open_(x) for x in s] for s in d["bufs"]], "top": d["top"],
                    "rows": d["rows"]}

        self.up = peer(band.rank - 1) if band.rank > 0 and band.top > 0 else None
        self.down = peer(band.rank + 1) if band.rank < band.world - 1 and band.bottom > 0 else None
        # the pull/signal kernels run on this rank's GPU and touch the
        # neighbours' memory directly: enable the P2P path (NVLink) explicitly
        from . import kfuse as K
        dev = dev.index
        for nb in (self.up, self.down):
            if nb is not None:
                K.peer_enable(dev, nb["ctr"].device.index)

    def _c(self, slot: int, ctr=None) -> int:
        return (self.ctr if ctr is None else ctr).data_ptr() + 4 * slot

    def errors(self) -> int:
        """Non-zero when a wait timed out (a neighbour never signalled)."""
        return int(self.ctr[_ERR].item())

    def signal(self, stream) -> None:
        """This step's own rows are ready (everything queued before on `stream`)."""
        from . import kfuse as K
        flags = []
        if self.up:
            flags.append(self._c(_READY_BELOW, self.up["ctr"]))
        if self.down:
            flags.append(self._c(_READY_ABOVE, self.down["ctr"]))
        K.peer_signal(flags, self._c(_SENT), stream)

    def pull(self, s: int, stream) -> None:
        """Copies the neighbours' boundary rows of buffer set s into the halo rows."""
        from . import kfuse as K
        b, bset = self.band, self.bufs[s]
        dst, src, nb, flag, seen, ack = [], [], [], [], [], []
        if self.up:   # one segment per neighbour, one copy per input image
            u = self.up
            for i, buf in enumerate(bset):
                rb = buf[0].numel() * buf.element_size()
                dst.append(buf.data_ptr())
                src.append(u["bufs"][s][i].data_ptr() + (u["top"] + u["rows"] - b.top) * rb)
                nb.append(b.top * rb)
            flag.append(self._c(_READY_ABOVE))
            seen.append(self._c(_SEEN_ABOVE))
            ack.append(self._c(_ACK_BELOW, u["ctr"]))
        if self.down:
            d = self.down
            for i, buf in enumerate(bset):
                rb = buf[0].numel() * buf.element_size()
                dst.append(buf.data_ptr() + (b.top + b.rows) * rb)
                src.append(d["bufs"][s][i].data_ptr() + d["top"] * rb)
                nb.append(b.bottom * rb)
            flag.append(self._c(_READY_BELOW))
            seen.append(self._c(_SEEN_BELOW))
            ack.append(self._c(_ACK_ABOVE, d["ctr"]))
        K.peer_pull(dst, src, nb, flag, seen, ack, self._c(_ERR), self.spin, stream, copies=len(bset))

    def wait_consumed(self, stream) -> None:
        """Before the own rows are overwritten: both neighbours pulled every step signalled."""
        from . import kfuse as K
        cnt = ([self._c(_ACK_ABOVE)] if self.up else []) + ([self._c(_ACK_BELOW)] if self.down else [])
        K.peer_wait(cnt, [self._c(_SENT)] * len(cnt), self._c(_ERR), self.spin, stream)

    def step(self, plan, s: int, outputs, stream, side=None) -> None:
        """One band step on buffer set s: the core rows on `stream` while `side`
        (a second stream, forked from `stream`) signals, pulls the halo rows and
        computes the edge strips -- they read only the pulled and the own rows and
        write rows disjoint from the core's, so the whole exchange hides behind
        the core; `stream` joins `side` at the end.  Bit-identical to
        exchange_halos + run_band.  With side=None everything runs on `stream`,
        in the order signal, core, pull, edges.  Without neighbours it is just
        the core."""
        b = self.band
        (c0, c1), edges = split_rows(b)
        ins = self.bufs[s]
        exch = self.up is not None or self.down is not None
        if plan.num_launches > 1:
            side = None   # one workspace per plan: core and edges must not overlap (kfuse.h)

        def run_edges(st):
            for r0, r1 in edges:
                plan.run_band(r0, r1, ins, b.in0, b.in1, [o[r0 - b.row0:r1 - b.row0] for o in outputs], st)

        if exch and side is not None:
            side.wait_stream(stream)          # the own rows of this step are ready
            self.signal(side)
            self.pull(s, side)
            run_edges(side)
        elif exch:
            self.signal(stream)
        if c1 > c0:
            plan.run_band(c0, c1, ins, b.in0, b.in1, [o[c0 - b.row0:c1 - b.row0] for o in outputs], stream)
        if exch and side is not None:
            stream.wait_stream(side)
        else:
            if exch:
                self.pull(s, stream)
            run_edges(stream)

    def close(self) -> None:
        """Drops the peer mappings.  Call on every rank (synchronised) before any
        rank frees the buffers it exported."""
        self.up = self.down = None
        torch.cuda.synchronize()
