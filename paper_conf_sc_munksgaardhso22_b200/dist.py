"""Multi-GPU drivers (one process per GPU, torch.distributed for the plumbing).

Two partitionings, only where the path shards (DESIGN.md §1 rows a7/a8):

* batch (config 4): independent pairs -> contiguous pair ranges per rank, each rank runs ONE
  nw_fill_batch launch over its range.  No collective on the data path; a barrier and a MAX
  all-reduce of the elapsed device time only for timing.
* column strips (config 5): one huge pair, rank g owns global columns (col0_g, col0_g + w_g].
  Rank g's band 0 reads its left border from its local `halo_in` buffer, and its last band
  stores its right column straight into rank g+1's `halo_in` over NVLink (peer pointer from
  torch symmetric memory), entry by entry as rows complete — the border push is fused into
  the wavefront kernel.  The tags are the call's epoch, so halos never need resetting; one
  barrier per call keeps call e+1 from overwriting entries a peer still reads for call e.

The host-side logic (ranges, bounds, local-matrix layout, epochs) is plain Python, covered by
world_size-2 gloo tests on CPU (tests/test_dist_cpu.py).
"""
from __future__ import annotations

from dataclasses import dataclass


def pair_range(batch: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous [lo, hi) block of pairs for `rank` (the last rank takes the remainder...
    spread so sizes differ by at most one)."""
    if world < 1 or not 0 <= rank < world or batch < 0:
        raise ValueError("bad pair_range arguments")
    base, extra = divmod(batch, world)
    lo = rank * base + min(rank, extra)
    return lo, lo + base + (1 if rank < extra else 0)


@dataclass(frozen=True)
class Strip:
    rank: int
    world: int
    col0: int   # global column of local column 0 (the halo / left border column)
    w: int      # local interior columns (global columns col0+1 .. col0+w)


def strip_bounds(n: int, world: int, align: int = 128) -> list[Strip]:
    """Column strips of an n-column matrix: widths multiples of `align` (the band width) except
    the last, as even as possible."""
    if world < 1 or n < 0:
        raise ValueError("bad strip_bounds arguments")
    units = -(-n // align) if n else 0
    base, extra = divmod(units, world)
    out, c = [], 0
    for g in range(world):
        u = base + (1 if g < extra else 0)
        w = min(u * align, n - c)
        out.append(Strip(g, world, c, max(w, 0)))
        c += max(w, 0)
    assert c == n
    return out


def shard_strip(n: int, world: int, rank: int, tile: int = 0) -> Strip:
    """Rank's strip of the config-5 pipeline: a strip that pushes a halo must end on a band
    boundary (nw.h, else NW_ECOMM), so the widths are multiples of the band width of `tile`
    (not a fixed 128) and only the last strip is ragged."""
    from . import nw_band_width
    return strip_bounds(n, world, align=nw_band_width(tile))[rank]


class EpochCounter:
    """Per-call tag shared by all ranks (every rank calls next() once per collective call)."""

    def __init__(self, start: int = 0):
        self.e = start

    def next(self) -> int:
        self.e = (self.e % 0xFFFFFFFF) + 1
        return self.e


def local_strip_problem(n: int, p: int, seed: int, strip: Strip, device):
    """Rank-local (n+1, w+1) score / ref of the global seeded problem (inputs.device_problem's
    recipe restricted to the strip's columns): local column 0 = global column col0."""
    import inputs
    return inputs.device_strip(n, p, strip.col0, strip.w, seed=seed, device=device)


class StripShard:
    """One rank of the column-strip pipeline over NVLink (config 5)."""

    def __init__(self, n: int, p: int, seed: int, group=None, tile: int = 0):
        import torch
        import torch.distributed as dist
        import torch.distributed._symmetric_memory as symm_mem
        self.n, self.p, self.tile = n, p, tile
        self.group = group or dist.group.WORLD
        self.rank, self.world = dist.get_rank(self.group), dist.get_world_size(self.group)
        self.device = torch.device("cuda", torch.cuda.current_device())
        self.strip = shard_strip(n, self.world, self.rank, tile)
        self.score, self.ref = local_strip_problem(n, p, seed, self.strip, self.device)
        self.halo = symm_mem.empty(n + 2, dtype=torch.int64, device=self.device)  # n+2 entries (nw.h)
        self.halo.zero_()
        torch.cuda.synchronize()
        self.hdl = symm_mem.rendezvous(self.halo, self.group)
        self.halo_out = self.hdl.buffer_ptrs[self.rank + 1] if self.rank + 1 < self.world else None
        self.epochs = EpochCounter()

    def fill(self, stream=None):
        from . import nw_fill_sharded
        e = self.epochs.next()
        nw_fill_sharded(self.score, self.ref, self.p, halo_in=self.halo if self.rank > 0 else None,
                        halo_out=self.halo_out, epoch=e, halo_out_is_peer=True, tile=self.tile,
                        stream=stream)
        return e

    def barrier(self):
        self.hdl.barrier()
