"""Row sharding for C5: band / halo arithmetic and the all-gather glue,
exercised on CPU with the gloo backend at world size 2 and 3.  The per-band compute in
these tests is the oracle (injected here; the product runs liborion's kernel instead), so
the check is: bands + halos + gather reproduce the full-image result exactly."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_middleware_hayeslcsz16_b200 import shard


@pytest.mark.parametrize("H,P,halo", [(16384, 8, 6), (100, 3, 6), (7, 4, 3), (2, 5, 6), (256, 1, 6)])
def test_bands_partition_rows_and_clip_halos(H, P, halo):
    bands = [shard.band(r, P, H, halo) for r in range(P)]
    covered = []
    for b in bands:
        assert b.rows_per_rank == -(-H // P)
        assert 0 <= b.row_begin <= b.row_end <= H
        assert b.src_begin == max(0, b.row_begin - halo) and b.src_end == min(H, b.row_end + halo)
        covered += list(range(b.row_begin, b.row_end))
    assert covered == list(range(H))
    with pytest.raises(ValueError):
        shard.band(P, P, H, halo)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, W, H, kind, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    halo = 3 if kind == "knn" else 6
    b = shard.band(rank, world, H, halo)
    slab = synth.noisy_rgba(W, H, seed=5, sigma=0.13, row_begin=b.src_begin, row_end=b.src_end)
    out = torch.zeros((b.rows_per_rank, W, 3), dtype=torch.float64)
    if b.rows:
        o, _, _ = oracle.denoise(kind, slab, height=H, row0=b.src_begin, y_begin=b.row_begin, y_end=b.row_end)
        out[: b.rows] = torch.from_numpy(o)
    full = torch.empty((world * b.rows_per_rank, W, 3), dtype=torch.float64)
    shard.gather_bands(out, full)
    if rank == 0:
        q.put(full[:H].numpy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,H,kind", [(2, 37, "nlm"), (3, 20, "knn")])
def test_gloo_sharded_equals_full_image(world, H, kind):
    W = 23
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, W, H, kind, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = q.get(timeout=300)
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    full, _, _ = oracle.denoise(kind, synth.noisy_rgba(W, H, seed=5, sigma=0.13))
    assert np.array_equal(got, full)


def _chunk_worker(rank, world, port, H, W, chunks, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    b = shard.band(rank, world, H, 6)
    out = torch.full((b.rows_per_rank, W), -1.0)
    out[: b.rows] = torch.arange(b.row_begin, b.row_end, dtype=torch.float32)[:, None] + torch.zeros(W)
    full = torch.zeros((world * b.rows_per_rank, W))
    per = -(-b.rows_per_rank // chunks)
    for c in range(chunks):
        r0, r1 = min(b.rows_per_rank, c * per), min(b.rows_per_rank, (c + 1) * per)
        if r0 < r1:
            shard.gather_rows(out, full, b.rows_per_rank, r0, r1)
    if rank == 0:
        q.put(full[:H].numpy())
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,H,chunks", [(2, 37, 3), (3, 20, 4)])
def test_chunked_gather_places_rows(world, H, chunks):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_chunk_worker, args=(r, world, port, H, 5, chunks, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = q.get(timeout=300)
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    assert np.array_equal(got, np.repeat(np.arange(H, dtype=np.float32)[:, None], 5, axis=1))


@pytest.mark.parametrize("H,P,chunks", [(4096, 3, 4), (37, 3, 4), (16384, 8, 4), (5, 4, 3), (100, 7, 2)])
def test_chunk_plan_is_the_same_on_every_rank(H, P, chunks):
    # the gathered rows [r0, r1) must not depend on the rank (collectives match), and the image rows
    # [k0, k1) of the chunks tile each band exactly
    plans = [shard.chunk_plan(shard.band(r, P, H, 6), chunks) for r in range(P)]
    assert all([(p[0], p[1]) for p in pl] == [(p[0], p[1]) for p in plans[0]] for pl in plans)
    for r, pl in enumerate(plans):
        b = shard.band(r, P, H, 6)
        rows = [k for _, _, k0, k1 in pl for k in range(k0, k1)]
        assert rows == list(range(b.rows))


def _halo_worker(rank, world, port, H, W, halo, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    bands = [shard.band(r, world, H, halo) for r in range(world)]
    b = bands[rank]
    # this rank's next slab: its band rows hold the global row index, the halo rows -1 (not exchanged yet)
    nxt = torch.full((b.src_rows, W), -1.0)
    nxt[b.row_begin - b.src_begin:b.row_end - b.src_begin] = \
        torch.arange(b.row_begin, b.row_end, dtype=torch.float32)[:, None] + torch.zeros(W)
    shard.exchange_halos_gather(nxt, b, bands, halo)
    q.put((rank, nxt.numpy()))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world,H,halo", [(2, 37, 4), (3, 40, 4), (4, 61, 4)])
def test_stencil_halo_exchange_fallback(world, H, halo):
    # the all-gather fallback of the C3 halo exchange (the kernels' fan-out stores do the same over
    # NVLink): after it every slab holds the global rows [src_begin, src_end) -- its neighbours'
    # boundary rows in its halo
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_halo_worker, args=(r, world, port, H, 6, halo, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    for r in range(world):
        b = shard.band(r, world, H, halo)
        want = np.repeat(np.arange(b.src_begin, b.src_end, dtype=np.float32)[:, None], 6, axis=1)
        assert np.array_equal(got[r], want), r


def test_global_row_pointer_and_neighbours():
    bands = [shard.band(r, 4, 100, 4) for r in range(4)]
    assert shard.halo_neighbours(0, 4, bands) == (None, 1)
    assert shard.halo_neighbours(2, 4, bands) == (1, 3)
    assert shard.halo_neighbours(3, 4, bands) == (2, None)
    b = bands[2]                      # rows 50..75, slab from row 46
    assert shard.global_row_ptr(1 << 40, b, 64) + 46 * 64 * 4 == 1 << 40
