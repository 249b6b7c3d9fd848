"""Row-band decomposition host logic on CPU: partition() and the
halo-row exchange over torch.distributed with the gloo backend, world sizes 2
and 3 (two processes per test, 127.0.0.1 rendezvous).  The banded kernels
themselves are covered by tests/test_gpu_parity.py::test_bands_bit_identical."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from kf_inputs import gen
from paper_conf_cgo_qiaorht19_b200 import dist as KD


def _free_port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def test_partition_covers_rows_once():
    for H in (1, 7, 97, 4096):
        for world in (1, 2, 3, 8):
            if world > H:
                continue
            bands = [KD.partition(H, world, r, 0) for r in range(world)]
            rows = [y for b in bands for y in range(b.row0, b.row1)]
            assert rows == list(range(H))
            assert max(b.rows for b in bands) - min(b.rows for b in bands) <= 1


def test_partition_halo_clipped_at_global_edges():
    b0 = KD.partition(100, 4, 0, 3)
    b3 = KD.partition(100, 4, 3, 3)
    b1 = KD.partition(100, 4, 1, 3)
    assert (b0.in0, b0.top, b0.bottom) == (0, 0, 3)
    assert (b3.in1, b3.bottom, b3.top) == (100, 0, 3)
    assert (b1.in0, b1.in1) == (22, 53)


def test_partition_rejects_band_thinner_than_halo():
    with pytest.raises(ValueError):
        KD.partition(8, 4, 1, 3)


def _worker(rank, world, port, H, W, halo, q, posted=False, n_inputs=1):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        band = KD.partition(H, world, rank, halo)
        fulls = [gen.image_f32(9 + 13 * j, W, H) for j in range(n_inputs)]
        bufs = []
        for full in fulls:
            buf = torch.full((band.in1 - band.in0, W), float("nan"))
            buf[band.top:band.top + band.rows] = torch.from_numpy(full[band.row0:band.row1])
            bufs.append(buf)
        if posted:   # the overlapped step's non-blocking post (dist.run_step_overlapped), all inputs at once
            for r in KD._post_halos(bufs, band):
                r.wait()
        else:
            for buf in bufs:
                KD.exchange_halos(buf, band)
        ok = all(bool(np.array_equal(b.numpy(), f[band.in0:band.in1])) for b, f in zip(bufs, fulls))
        q.put((rank, ok))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("posted", [False, True])
@pytest.mark.parametrize("world,H,halo,n_inputs", [(2, 37, 2, 1), (3, 50, 6, 1), (2, 9, 4, 1), (2, 37, 2, 2),
                                                   (3, 50, 3, 3)])
def test_exchange_halos_gloo(world, H, halo, n_inputs, posted):
    """After one exchange every rank holds exactly rows [in0, in1) of every global
    input image (multi-input pipelines exchange each input's halo rows)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, H, 23, halo, q, posted, n_inputs))
             for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in procs)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert all(res[r] for r in range(world)), res


@pytest.mark.parametrize("H,world,halo", [(97, 3, 2), (100, 4, 6), (9, 2, 4), (50, 1, 3), (12, 3, 2)])
def test_split_rows_core_and_edges(H, world, halo):
    """The core rows need no halo row ([row0+R, row1-R) reads only owned rows) and
    core + edge strips cover the band exactly once."""
    for rank in range(world):
        try:
            b = KD.partition(H, world, rank, halo)
        except ValueError:
            continue
        (c0, c1), edges = KD.split_rows(b)
        rows = list(range(c0, c1)) + [y for r0, r1 in edges for y in range(r0, r1)]
        assert sorted(rows) == list(range(b.row0, b.row1))
        if c1 > c0:
            lo = c0 - halo if rank > 0 else max(0, c0 - halo)
            hi = c1 + halo if rank < world - 1 else min(H, c1 + halo)
            assert (rank == 0 or lo >= b.row0) and (rank == world - 1 or hi <= b.row1)
