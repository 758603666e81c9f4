"""Pin P7 — schedule invariants, run on the exact host-side schedule functions the kernels use
(nw_diag_lmad for the per-diagonal kernels, nw_strip_map for the persistent kernel).

From the paper (PAPER.md P:546-566 NW LMADs W / Rvert / Rhoriz; Fig. 9, the proof
that W ∩ Rvert = ∅ which licenses the in-place update):
  * per tile anti-diagonal d: W_d ∩ (Rvert_d ∪ Rhoriz_d) = ∅,
  * every read of diagonal d lies on the borders or in some W_{d'} with d' < d,
  * the W_d partition the interior (every cell written exactly once).
For the band schedule: every interior cell is computed exactly once, and each of its three
inputs is either a border cell or computed strictly earlier in the partial order the kernel
enforces (same band: earlier step; left neighbour band: handed off row by row).
"""
import numpy as np
import pytest

import paper_conf_sc_munksgaardhso22_b200 as nwb


def lmad_cells(off, dims):
    """Flat offsets of the LMAD off + {(n1:s1), ...} (eq. 1)."""
    idx = np.array([off], dtype=np.int64)
    for cnt, stride in dims:
        idx = (idx[:, None] + np.arange(cnt, dtype=np.int64)[None, :] * stride).ravel()
    return idx


@pytest.mark.parametrize("n,b", [(16, 16), (32, 16), (48, 16), (64, 16), (96, 32), (128, 32), (128, 64), (320, 64)])
def test_diag_lmads_disjoint_and_partition(n, b):
    if b not in (16, 32, 64):
        pytest.skip("library tiles are 16/32/64")
    N = n + 1
    q = n // b
    written = np.zeros((N, N), dtype=np.int32)
    when = np.full((N, N), -1, dtype=np.int64)
    for d in range(2 * q - 1):
        cnt, base, w_off, s0, s1, s2, rv_off, rv_s, rh_off, rh_s = nwb.nw_diag_lmad(n, N, b, d)
        assert (w_off, rv_off, rh_off) == (base + N + 1, base, base + 1)
        W = lmad_cells(w_off, [(cnt, s0), (b, s1), (b, s2)])
        Rv = lmad_cells(rv_off, [(cnt, s0), (b + 1, rv_s)])
        Rh = lmad_cells(rh_off, [(cnt, s0), (b, rh_s)])
        assert len(np.intersect1d(W, np.concatenate([Rv, Rh]))) == 0        # Fig. 9: W ∩ R = ∅
        wi, wj = np.divmod(W, N)
        assert wi.min() >= 1 and wj.min() >= 1 and wi.max() <= n and wj.max() <= n
        for R in (Rv, Rh):                                                   # reads: border or earlier
            ri, rj = np.divmod(R, N)
            interior = (ri >= 1) & (rj >= 1)
            assert (when[ri[interior], rj[interior]] >= 0).all()
            assert (when[ri[interior], rj[interior]] < d).all()
        written[wi, wj] += 1
        when[wi, wj] = d
    assert (written[1:, 1:] == 1).all() and (written[0] == 0).all() and (written[:, 0] == 0).all()


def test_diag_lmad_matches_paper_first_half():
    # PAPER.md P:549-552 for i < q: W = i*b + n + 1 + {(i+1 : n*b - b), (b : n), (b : 1)}
    # with the paper's n = row length = our N.
    n, b = 64, 16
    N = n + 1
    for d in range(n // b):
        cnt, base, w_off, s0, s1, s2, *_ = nwb.nw_diag_lmad(n, N, b, d)
        assert cnt == d + 1 and base == d * b and w_off == d * b + N + 1
        assert (s0, s1, s2) == (N * b - b, N, 1)


def strip_schedule(n, width, tile):
    """when[i, j] = (band, step) at which the persistent kernel computes cell (i, j)."""
    W = nwb.nw_band_width(tile)
    nb = -(-width // W)
    band_of = np.full((n + 1, width + 1), -1, dtype=np.int64)
    step_of = np.full((n + 1, width + 1), -1, dtype=np.int64)
    count = np.zeros((n + 1, width + 1), dtype=np.int64)
    for band in range(nb):
        for step in range(n + 31):
            for lane in range(32):
                r, c, k = nwb.nw_strip_map(n, width, tile, band, step, lane)
                for x in range(k):
                    count[r, c + x] += 1
                    band_of[r, c + x] = band
                    step_of[r, c + x] = step
    return band_of, step_of, count


@pytest.mark.parametrize("n,width,tile", [(5, 5, 0), (40, 40, 16), (70, 70, 64), (33, 130, 0), (64, 200, 32)])
def test_strip_schedule_exactly_once_and_ordered(n, width, tile):
    band_of, step_of, count = strip_schedule(n, width, tile)
    assert (count[1:, 1:] == 1).all() and (count[0] == 0).all() and (count[:, 0] == 0).all()
    W = nwb.nw_band_width(tile)
    for i in range(1, n + 1):
        for j in range(1, width + 1):
            b, s = band_of[i, j], step_of[i, j]
            for (pi, pj) in ((i - 1, j - 1), (i - 1, j), (i, j - 1)):
                if pi == 0 or pj == 0:
                    continue                                # border input
                pb, ps = band_of[pi, pj], step_of[pi, pj]
                if pb == b:
                    # same band: an earlier step, or the same step inside the lane's own chain
                    # (a lane computes its K cells of one row left to right within a step)
                    lane = lambda col: ((col - 1) % W) // (W // 32)  # noqa: E731
                    same_chain = ps == s and pi == i and pj == j - 1 and lane(pj) == lane(j)
                    assert ps < s or same_chain, ((i, j), (pi, pj))
                else:
                    # left band: the value crosses as the band's last column, row by row
                    assert pb == b - 1 and pj == b * W, ((i, j), (pi, pj))
    # lane skew: within a band, row r is computed by lane t at step r - 1 + t
    r, c, k = nwb.nw_strip_map(n, width, tile, 0, 10, 3)
    assert r == 8 and c == 1 + 3 * (W // 32)


def test_strip_map_rejects_bad_args():
    with pytest.raises(ValueError):
        nwb.nw_strip_map(10, 10, 0, 5, 0, 0)       # band beyond width
    with pytest.raises(ValueError):
        nwb.nw_strip_map(10, 10, 0, 0, 0, 32)      # lane 32
