"""Multi-process host logic of the multi-GPU paths, world_size 2 over gloo on the CPU.

* batch sharding: pair_range partitions the batch, no collective on the data path;
* column strips: strip_bounds + local_strip_problem build each rank's local problem exactly as
  the global seeded problem restricted to its columns, and the strip pipeline — rank g receives
  its left border column from rank g-1 (gloo send/recv here, NVLink peer stores on the GPU),
  fills its strip, forwards its right column — reproduces the full matrix.  The fills use the
  CPU oracle (a local strip embedded in a square buffer: columns depend only on columns to
  their left), so this checks the decomposition, not the kernel;
* epochs agree across ranks; timings reduce with MAX.
"""
import os
import socket

import numpy as np
import pytest

torch = pytest.importorskip("torch")
import torch.distributed as dist  # noqa: E402
import torch.multiprocessing as mp  # noqa: E402


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, n, p, q):
    import sys
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import inputs
    import oracle
    from paper_conf_sc_munksgaardhso22_b200 import dist as nwdist
    try:
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
        # ---- batch sharding
        lo, hi = nwdist.pair_range(4096, world, rank)
        rng = torch.tensor([lo, hi])
        allr = [torch.zeros(2, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(allr, rng)
        spans = sorted(tuple(int(x) for x in r) for r in allr)
        assert spans[0][0] == 0 and spans[-1][1] == 4096
        assert all(spans[i][1] == spans[i + 1][0] for i in range(world - 1))
        # ---- column strips
        strips = nwdist.strip_bounds(n, world, align=64)
        st = strips[rank]
        ls, lr = nwdist.local_strip_problem(n, p, inputs.SEED, st, "cpu")
        ls, lr = ls.numpy(), lr.numpy()
        gs, gr = inputs.make_problem(n, p)
        np.testing.assert_array_equal(lr[1:, 1:], gr[1:, st.col0 + 1:st.col0 + st.w + 1])
        np.testing.assert_array_equal(ls[0], gs[0, st.col0:st.col0 + st.w + 1])
        if rank > 0:                                  # the halo arrives from the left rank
            left = torch.zeros(n + 1, dtype=torch.int32)
            dist.recv(left, src=rank - 1)
            ls[1:, 0] = left.numpy()[1:]
        pad = np.full((n + 1, n + 1), inputs.SENTINEL, dtype=np.int32)
        rpad = np.zeros((n + 1, n + 1), dtype=np.int32)
        pad[:, : st.w + 1] = ls
        rpad[:, : st.w + 1] = lr
        oracle.nw_ref(pad, rpad, p)
        mine = pad[:, : st.w + 1]
        if rank + 1 < world:
            dist.send(torch.from_numpy(mine[:, st.w].copy()), dst=rank + 1)
        full = oracle.nw_ref(gs.copy(), gr, p)
        np.testing.assert_array_equal(mine[:, 1:], full[:, st.col0 + 1:st.col0 + st.w + 1])
        # ---- epochs agree, timing = max over ranks
        ec = nwdist.EpochCounter()
        es = torch.tensor([ec.next() for _ in range(5)])
        alle = [torch.zeros(5, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(alle, es)
        assert all(torch.equal(alle[0], e) for e in alle)
        t = torch.tensor([float(rank + 1)])
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        assert t.item() == world
        dist.barrier()
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


@pytest.mark.parametrize("n", [200, 333])
def test_dist_world2_gloo(n):
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, n, 10, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    res = dict(q.get(timeout=120) for _ in range(world))
    for pr in procs:
        pr.join(timeout=60)
    assert res == {0: "ok", 1: "ok"}, res


def test_pair_range_and_strip_bounds():
    from paper_conf_sc_munksgaardhso22_b200 import dist as nwdist
    for B, G in [(4096, 1), (4096, 8), (10, 3), (3, 8)]:
        rs = [nwdist.pair_range(B, G, g) for g in range(G)]
        assert rs[0][0] == 0 and rs[-1][1] == B
        assert max(h - l for l, h in rs) - min(h - l for l, h in rs) <= 1
    for n, G in [(65536, 2), (65536, 8), (1000, 3), (100, 4)]:
        ss = nwdist.strip_bounds(n, G)
        assert sum(s.w for s in ss) == n and ss[0].col0 == 0
        assert all(ss[i].col0 + ss[i].w == ss[i + 1].col0 for i in range(G - 1))
        assert all(s.w % 128 == 0 for s, nx in zip(ss, ss[1:]) if nx.w > 0)   # only the last is ragged
    assert [s.w for s in nwdist.strip_bounds(65536, 8)] == [8192] * 8


@pytest.mark.parametrize("tile", [0, 16, 64])
@pytest.mark.parametrize("n,G", [(40000, 2), (32768, 3), (32768, 5), (32768, 6), (32768, 7), (65536, 8), (1000, 3)])
def test_shard_strip_band_aligned(n, G, tile):
    """Round-1 advisor finding: StripShard cut strips on 128-column units while a halo-pushing
    strip must be a multiple of the band width (256 at tile 0), so e.g. n = 40000 on 2 GPUs got
    NW_ECOMM.  shard_strip aligns to nw_band_width(tile)."""
    import paper_conf_sc_munksgaardhso22_b200 as nwb
    from paper_conf_sc_munksgaardhso22_b200 import dist as nwdist
    W = nwb.nw_band_width(tile)
    ss = [nwdist.shard_strip(n, G, g, tile) for g in range(G)]
    assert sum(s.w for s in ss) == n and ss[0].col0 == 0
    assert all(ss[i].col0 + ss[i].w == ss[i + 1].col0 for i in range(G - 1))
    assert all(s.w % W == 0 for s in ss[:-1])

