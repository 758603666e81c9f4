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
    import numpy as np
    import torch

    import inputs
    a, b = inputs.gen_pair(n, seed)
    table = torch.from_numpy(inputs.blosum62()).to(device=device, dtype=torch.int32)
    ta = torch.from_numpy(a.astype(np.int64)).to(device)
    tb = torch.from_numpy(b[strip.col0:strip.col0 + strip.w].astype(np.int64)).to(device)
    w = strip.w
    score = torch.empty((n + 1, w + 1), dtype=torch.int32, device=device)
    ref = torch.zeros((n + 1, w + 1), dtype=torch.int32, device=device)
    rows_b = table[:, tb]
    for i0 in range(0, n, 4096):
        i1 = min(n, i0 + 4096)
        ref[1 + i0:1 + i1, 1:] = rows_b[ta[i0:i1]]
    cols = torch.arange(strip.col0, strip.col0 + w + 1, device=device, dtype=torch.int64)
    score[0] = (cols * (-p)).to(torch.int32)
    if strip.rank == 0:
        score[:, 0] = (torch.arange(n + 1, device=device, dtype=torch.int64) * (-p)).to(torch.int32)
    else:
        score[1:, 0] = inputs.SENTINEL   # never read: the halo carries the left border
    score[1:, 1:] = inputs.SENTINEL
    return score, ref


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
        self.strip = strip_bounds(n, self.world)[self.rank]
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
