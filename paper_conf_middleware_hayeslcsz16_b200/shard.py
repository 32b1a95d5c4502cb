"""Row-sharded multi-GPU composition of the hot path (config C5).

Each rank owns an equal band of output rows, generates its input slab plus the
R_eff-row halo in place (the generator's hash and the clamping use GLOBAL
coordinates, so a slab is bit-identical to the same rows of the full image), runs
its own Orion tuner on that slab (per-GPU tuning), and one NCCL
``all_gather_into_tensor`` over NVLink collects the output bands -- the only
inter-GPU exchange of the configuration.

Two ways to gather: (1) NCCL all-gathers of row chunks on a side stream, overlapping
the next chunk's kernel (``gather_rows``); (2) the kernels' fan-out epilogue
(``orion_args.fanout``): with the full images in symmetric memory (``FanoutImage``), each
rank's kernel stores every output pixel straight into every rank's image over NVLink as
its tiles complete, and a device-side barrier closes the step -- compute and exchange in
one kernel, no collective call.

Host-side logic only (partitioning, halo arithmetic, the gather glue); all pixel
work happens in liborion's kernels.  The gather glue takes any process group, so
it is exercised with ``gloo`` on CPU tensors in tests/test_shard.py.
"""
from __future__ import annotations

from dataclasses import dataclass


@dataclass(frozen=True)
class Band:
    rank: int
    world: int
    height: int
    rows_per_rank: int   # equal band height (the last band may be partly past the image)
    row_begin: int       # first output row owned (global)
    row_end: int         # one past the last output row owned (global, clipped to height)
    src_begin: int       # first input row the kernel reads (global, halo included, clamped)
    src_end: int         # one past the last input row read

    @property
    def rows(self) -> int:
        return self.row_end - self.row_begin

    @property
    def src_rows(self) -> int:
        return self.src_end - self.src_begin


def band(rank: int, world: int, height: int, halo: int) -> Band:
    """Rank `rank`'s output band and the input rows (with `halo` rows each side) it needs."""
    if world < 1 or not 0 <= rank < world or height < 1 or halo < 0:
        raise ValueError("bad band request")
    per = -(-height // world)
    r0 = min(height, rank * per)
    r1 = min(height, r0 + per)
    return Band(rank, world, height, per, r0, r1, max(0, r0 - halo), min(height, r1 + halo))


def chunk_plan(b: Band, chunks: int):
    """Row chunks of a band for the overlapped gather: [(r0, r1, k0, k1)] with [r0, r1) the band-relative
    rows EVERY rank gathers (cut from the equal band height, so the collectives match across ranks
    even when the last band is shorter) and [k0, k1) the rows of the image inside it (empty for the
    last rank's padding rows)."""
    per = -(-b.rows_per_rank // max(1, chunks))
    plan = []
    for c in range(max(1, chunks)):
        r0, r1 = min(b.rows_per_rank, c * per), min(b.rows_per_rank, (c + 1) * per)
        if r0 < r1:
            plan.append((r0, r1, min(b.rows, r0), min(b.rows, r1)))
    return plan


def gather_rows(out_band, full_out, rows_per_rank: int, r0: int, r1: int, group=None):
    """all_gather rows [r0, r1) of every rank's band straight into their places in
    `full_out` (rank k's rows land at k * rows_per_rank + [r0, r1)).  Issue it on a side
    stream right after the kernel that produced those rows, so the collective of one chunk
    overlaps the compute of the next (kernel splitting, feeding the exchange)."""
    import torch.distributed as dist
    world = dist.get_world_size(group)
    views = [full_out[k * rows_per_rank + r0:k * rows_per_rank + r1] for k in range(world)]
    src = out_band[r0:r1].contiguous()
    if full_out.is_cuda and dist.get_backend(group) != "nccl":
        host = [v.new_empty(v.shape, device="cpu") for v in views]
        dist.all_gather(host, src.cpu(), group=group)
        for v, h in zip(views, host):
            v.copy_(h)
        return full_out
    dist.all_gather(views, src, group=group)
    return full_out


def gather_bands(out_band, full_out, group=None):
    """all_gather the equal-height output bands into `full_out` (world * rows_per_rank rows).

    `out_band`: (rows_per_rank, ...) tensor of this rank (rows past the image are padding);
    `full_out`: (world * rows_per_rank, ...) tensor; rows [0, height) hold the image after.
    """
    import torch.distributed as dist
    if full_out.is_cuda and dist.get_backend(group) != "nccl":
        # control-flow checks on a single-GPU box (gloo): stage through host memory
        host = full_out.new_empty(full_out.shape, device="cpu")
        dist.all_gather_into_tensor(host, out_band.contiguous().cpu(), group=group)
        full_out.copy_(host)
        return full_out
    dist.all_gather_into_tensor(full_out, out_band.contiguous(), group=group)
    return full_out


class FanoutImage:
    """The full output image of a row-sharded frame in symmetric memory: every rank holds one,
    and ``ptrs`` are all ranks' device addresses (peer memory over NVLink), in rank order --
    the fan-out list of ``orion.with_fanout``.  ``barrier()`` (device-side, on the current
    stream) orders every rank's stores before anyone reads its image."""

    def __init__(self, shape, device, group=None):
        import torch
        import torch.distributed as dist
        import torch.distributed._symmetric_memory as symm_mem
        self.tensor = symm_mem.empty(*shape, dtype=torch.float32, device=device)
        self.handle = symm_mem.rendezvous(self.tensor, group or dist.group.WORLD)
        self.ptrs = [int(p) for p in self.handle.buffer_ptrs]

    def barrier(self):
        self.handle.barrier()


# ---- the thermal stencil row-sharded with a per-launch halo exchange ------------------------------
# Each rank holds its band of a W x H grid plus `halo` rows per side (two such slabs, ping-pong) and
# the same slab of the power map.  A launch advancing `halo` steps writes the band into its next
# slab and, through orion_args.fanout, its first / last `halo` rows into the neighbours' next slabs
# (the kernel's halo exchange); one device barrier per launch orders those stores before any rank
# reads them.  Host-side logic only: pointer arithmetic and the fallback exchange.

def halo_neighbours(rank: int, world: int, bands):
    """(upper, lower) neighbour ranks whose next slabs receive this band's first / last rows, or
    None at the grid's edge (or when the neighbour's band is empty)."""
    up = rank - 1 if rank > 0 and bands[rank - 1].rows else None
    down = rank + 1 if rank + 1 < world and bands[rank + 1].rows else None
    return up, down


def global_row_ptr(base_ptr: int, b: Band, width: int, elem: int = 4) -> int:
    """Address such that global row y of the slab starting at b.src_begin sits at ptr + y * width."""
    return base_ptr - b.src_begin * width * elem


def exchange_halos_gather(nxt, b: Band, bands, halo: int, group=None):
    """Fallback halo exchange (no symmetric memory, e.g. gloo): every rank contributes its band's
    first and last `halo` rows of `nxt` (a (b.src_rows, W) slab), all ranks gather them, and each
    copies its neighbours' rows into its own halo rows -- the same rows the kernel's fan-out stores."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    rank = dist.get_rank(group)
    W = nxt.shape[1]
    mine = torch.zeros((2, halo, W), dtype=nxt.dtype, device=nxt.device)
    if b.rows:
        o = b.row_begin - b.src_begin
        mine[0] = nxt[o:o + halo]
        mine[1] = nxt[o + b.rows - halo:o + b.rows]
    host = nxt.is_cuda and dist.get_backend(group) != "nccl"
    src = mine.cpu() if host else mine
    allr = [torch.empty_like(src) for _ in range(world)]
    dist.all_gather(allr, src, group=group)
    up, down = halo_neighbours(rank, world, bands)
    if up is not None:           # rows [row_begin - halo, row_begin): the upper band's last rows
        nxt[b.row_begin - halo - b.src_begin:b.row_begin - b.src_begin] = allr[up][1].to(nxt.device)
    if down is not None:         # rows [row_end, row_end + halo): the lower band's first rows
        nxt[b.row_end - b.src_begin:b.row_end + halo - b.src_begin] = allr[down][0].to(nxt.device)
    return nxt


class SymmetricSlabs:
    """Two (rows x W) float32 slabs per rank in symmetric memory (every rank's addresses known):
    the ping-pong grids of a row-sharded stencil whose kernels store halo rows into peers."""

    def __init__(self, rows: int, width: int, device, group=None):
        import torch
        import torch.distributed as dist
        import torch.distributed._symmetric_memory as symm_mem
        self.tensors, self.handles, self.ptrs = [], [], []
        for _ in range(2):
            t = symm_mem.empty(rows, width, dtype=torch.float32, device=device)
            h = symm_mem.rendezvous(t, group or dist.group.WORLD)
            self.tensors.append(t)
            self.handles.append(h)
            self.ptrs.append([int(p) for p in h.buffer_ptrs])

    def barrier(self):
        self.handles[0].barrier()
