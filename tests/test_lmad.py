"""The paper's static LMAD non-overlap test (Fig. 8 / Theorem; NEXT-4).

Pins, none of which re-uses the checker's arithmetic:
L1  Fig. 9: W ∩ Rvert = ∅ and W ∩ Rhoriz = ∅ are PROVEN for the paper's NW
    LMADs (n = q·b + 1, q >= 2, b >= 1, every diagonal block count i + 1), and brute-force
    enumeration of the point sets agrees.
L2  soundness: on random small LMAD pairs, every "proven disjoint" answer is confirmed by
    enumerating both point sets; overlapping pairs are never proven.
L4  the persistent kernel's bands (wave_band_lmads): every band's writes miss its reads, the
    next band's writes miss this band's reads and writes (brute force agrees on small n), and
    the true dependency (band k+1 reads band k's last column) is not proven disjoint.
L3  the schedule the diagonal kernels run (nw_diag_lmad of the C ABI, host-only): every tile
    anti-diagonal's write set is proven disjoint from its read sets, while the NEXT diagonal's
    Rvert / Rhoriz do overlap W (they read what W wrote) and are not proven.
"""
import random

import pytest

import paper_conf_sc_munksgaardhso22_b200 as nwb
from paper_conf_sc_munksgaardhso22_b200.lmad import (Lmad, non_overlap, nw_diag_lmads, nw_schedule_proofs,
                                                    wave_band_lmads, wave_schedule_proofs)


def points(L):
    pts = {L.offset}
    for n, s in L.dims:
        pts = {p + i * s for p in pts for i in range(n)}
    return pts if all(n > 0 for n, _ in L.dims) else set()


@pytest.mark.parametrize("q,b", [(2, 1), (2, 4), (3, 2), (4, 3), (5, 8), (8, 16)])
def test_fig9_nw_example(q, b):
    n = q * b + 1                            # the paper's n: row length
    for i in range(q - 1):
        W = Lmad(i * b + n + 1, ((i + 1, n * b - b), (b, n), (b, 1)))
        Rv = Lmad(i * b, ((i + 1, n * b - b), (b + 1, n)))
        Rh = Lmad(i * b + 1, ((i + 1, n * b - b), (b, 1)))
        assert non_overlap(W, Rv) and non_overlap(W, Rh)
        assert not (points(W) & points(Rv)) and not (points(W) & points(Rh))


def test_soundness_random():
    rng = random.Random(7)
    proven = refused_overlap = 0
    for _ in range(3000):
        def rand_lmad():
            dims = tuple((rng.randint(1, 4), rng.choice([1, 2, 3, 5, 7, 12, -3, 20])) for _ in range(rng.randint(1, 3)))
            return Lmad(rng.randint(-30, 60), dims)
        A, B = rand_lmad(), rand_lmad()
        disjoint = not (points(A) & points(B))
        got = non_overlap(A, B)
        if got:
            assert disjoint, (A, B)
            proven += 1
        if not disjoint:
            refused_overlap += 1
    assert proven > 300 and refused_overlap > 300


@pytest.mark.parametrize("n,tile", [(64, 16), (96, 32), (256, 64), (1024, 16), (1024, 64)])
def test_kernel_schedule_proven(n, tile):
    res = nw_schedule_proofs(nwb.lib(), n, tile)
    assert len(res) == 2 * (n // tile) - 1
    assert all(wv and wh for _, wv, wh in res), [r for r in res if not (r[1] and r[2])]


@pytest.mark.parametrize("n,tile", [(64, 16), (96, 32)])
def test_next_diagonal_reads_are_not_disjoint(n, tile):
    L = nwb.lib()
    q = n // tile
    for d in range(2 * q - 2):
        W, _, _ = nw_diag_lmads(L, n, n + 1, tile, d)
        _, Rv1, Rh1 = nw_diag_lmads(L, n, n + 1, tile, d + 1)
        assert points(W) & (points(Rv1) | points(Rh1))          # d+1 consumes d's results
        assert not (non_overlap(W, Rv1) and non_overlap(W, Rh1))


@pytest.mark.parametrize("n,width", [(40, 8), (100, 32), (1000, 128), (32768, 256), (33000, 256)])
def test_wave_bands_proven(n, width):
    res = wave_schedule_proofs(n, width)
    assert all(all(r) for r in res), [k for k, r in enumerate(res) if not all(r)]
    if n <= 100:
        for k in range(len(res) - 1):
            W, Rl, Rt = wave_band_lmads(n, n + 1, width, k)
            W1, Rl1, _ = wave_band_lmads(n, n + 1, width, k + 1)
            assert not (points(W) & (points(Rl) | points(Rt) | points(W1)))
            assert not (points(W1) & (points(Rl) | points(Rt)))
            assert points(W) & points(Rl1)                    # k+1 reads k's last column
            assert not non_overlap(W, Rl1)


def test_wave_bands_use_the_library_width():
    for tile in (0, 16, 64):
        w = nwb.nw_band_width(tile)
        assert all(all(r) for r in wave_schedule_proofs(4096, w))
