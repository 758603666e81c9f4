"""LMADs and the paper's static non-overlap test (NEXT-4, host side).

An LMAD (linear memory access descriptor, §II-B) is an offset plus a list of
(count : stride) dimensions; it denotes the flat element offsets
    t + sum_k i_k * s_k,   0 <= i_k < n_k.
``non_overlap(L1, L2)`` is the procedure of Fig. 8 on concrete integers:

1. normalise to positive strides and give both LMADs the same strides (adding count-1
   dimensions, "dimensions of length 0 can be introduced");
2. distribute the offset difference t1 - t2 over the strides, largest stride first, with a
   positive sign: a positive part raises I1's interval bounds, a negative part I2's
   (P:1491-1500 and footnote 27) -> two sums of intervals [l..u] * s;
3. Theorem (Non-Overlap): if neither sum has overlapping dimensions
   (s_i > sum_{j<i} u_j s_j for strides in increasing order) the sets are disjoint when some
   pair of matching intervals is disjoint;
4. otherwise split the interval that overflows into its last point and the rest
   on both sides and recurse on the four pairs (Fig. 8); a split that is impossible fails.

The answer True is a proof of disjointness; False means "not proven" (the test is sufficient,
not necessary).  ``nw_schedule_proofs`` applies it to the NW tile LMADs the diagonal kernels use
(``nw_diag_lmad`` of the C ABI), i.e. Fig. 9 for every anti-diagonal of a concrete
(n, b): W_d ∩ Rvert_d = ∅ and W_d ∩ Rhoriz_d = ∅, the condition that makes the in-place update
legal.  Host-side analysis only; nothing here runs on the data path.
"""
from __future__ import annotations

from dataclasses import dataclass


@dataclass(frozen=True)
class Lmad:
    offset: int
    dims: tuple  # ((count, stride), ...)


def _normalise(L: Lmad) -> Lmad:
    t, dims = L.offset, []
    for n, s in L.dims:
        if n <= 0:
            return Lmad(t, ((0, 1),))
        if n == 1 or s == 0:
            continue
        if s < 0:
            t += (n - 1) * s
            s = -s
        dims.append((n, s))
    return Lmad(t, tuple(dims))


def _intervals(L1: Lmad, L2: Lmad):
    """Steps 1-2: matching strides (increasing) and the two lists of [l, u] bounds."""
    strides = sorted({s for _, s in L1.dims} | {s for _, s in L2.dims} | {1})

    def base(L):
        iv = {s: [0, 0] for s in strides}
        for n, s in L.dims:
            if iv[s][1] != 0:              # two dimensions of one stride: not a sum of intervals
                return None
            iv[s] = [0, n - 1]
        return iv

    I1, I2 = base(L1), base(L2)
    if I1 is None or I2 is None:
        return None
    delta = L1.offset - L2.offset
    for s in reversed(strides):         # distribute, largest stride first, positive sign
        c = abs(delta) // s
        tgt = I1 if delta > 0 else I2
        tgt[s][0] += c
        tgt[s][1] += c
        delta -= c * s if delta > 0 else -c * s
    assert delta == 0
    return strides, I1, I2


def _first_overflow(strides, I):
    """Index (into strides) of the interval to split, or None if no dimension overlaps."""
    acc = 0
    for k, s in enumerate(strides):
        if k > 0 and s <= acc:
            # the largest lower-stride interval with a non-trivial range produced the overflow
            for j in range(k - 1, -1, -1):
                if I[strides[j]][1] > I[strides[j]][0]:
                    return j
            return None
        acc += I[s][1] * s
    return None


def _to_lmad(strides, iv) -> Lmad:
    return Lmad(sum(iv[s][0] * s for s in strides),
                tuple((iv[s][1] - iv[s][0] + 1, s) for s in strides if iv[s][1] > iv[s][0]))


def _split(strides, I, j):
    """I = (I with dim j's upper bound - 1)  ∪  (I with dim j = its last point), as LMADs."""
    s = strides[j]
    rest = {k: list(v) for k, v in I.items()}
    rest[s][1] -= 1
    last = {k: list(v) for k, v in I.items()}
    last[s][0] = last[s][1]
    return _to_lmad(strides, rest), _to_lmad(strides, last)


def non_overlap(L1: Lmad, L2: Lmad, depth: int = 8) -> bool:
    """Fig. 8: True proves L1 ∩ L2 = ∅; False = not proven."""
    L1, L2 = _normalise(L1), _normalise(L2)
    if any(n == 0 for n, _ in L1.dims + L2.dims):
        return True                     # an empty LMAD overlaps nothing
    r = _intervals(L1, L2)
    if r is None:
        return False
    strides, I1, I2 = r
    o1, o2 = _first_overflow(strides, I1), _first_overflow(strides, I2)
    ok1 = all(strides[k] > sum(I1[s][1] * s for s in strides[:k]) for k in range(1, len(strides)))
    ok2 = all(strides[k] > sum(I2[s][1] * s for s in strides[:k]) for k in range(1, len(strides)))
    if ok1 and ok2:
        return any(I1[s][1] < I2[s][0] or I2[s][1] < I1[s][0] for s in strides)
    if depth == 0:
        return False
    if (not ok1 and o1 is None) or (not ok2 and o2 is None):
        return False                    # splitAnOverlappingDimensionInto2LMADs = Fail
    # a side without overlapping dimensions is kept whole (Fig. 8 splits both; same proof)
    A = _split(strides, I1, o1) if not ok1 else (_to_lmad(strides, I1),)
    B = _split(strides, I2, o2) if not ok2 else (_to_lmad(strides, I2),)
    return all(non_overlap(a, b, depth - 1) for a in A for b in B)


def nw_diag_lmads(lib, n: int, ld: int, tile: int, d: int):
    """(W, Rvert, Rhoriz) of tile anti-diagonal d, from the C ABI's nw_diag_lmad."""
    import ctypes
    out = (ctypes.c_int64 * 10)()
    if lib.nw_diag_lmad(n, ld, tile, d, out) != 0:
        raise ValueError("nw_diag_lmad: bad arguments")
    cnt, _base, w_off, s0, s1, s2, rv_off, rv_s1, rh_off, rh_s1 = list(out)
    b = tile
    W = Lmad(w_off, ((cnt, s0), (b, s1), (b, s2)))
    Rvert = Lmad(rv_off, ((cnt, s0), (b + 1, rv_s1)))
    Rhoriz = Lmad(rh_off, ((cnt, s0), (b, rh_s1)))
    return W, Rvert, Rhoriz


def nw_schedule_proofs(lib, n: int, tile: int, ld: int | None = None):
    """For every anti-diagonal d of the (n, tile) schedule: (d, W∩Rvert=∅ proven, W∩Rhoriz=∅ proven)."""
    ld = n + 1 if ld is None else ld
    q = -(-n // tile)
    res = []
    for d in range(2 * q - 1):
        W, Rv, Rh = nw_diag_lmads(lib, n, ld, tile, d)
        res.append((d, non_overlap(W, Rv), non_overlap(W, Rh)))
    return res


def wave_band_lmads(n: int, ld: int, width: int, k: int):
    """(W, Rleft, Rtop) of band k of the persistent kernel (csrc/nw_wave.cuh): columns
    c0 = k*width + 1 .. c1 = min((k+1)*width, n), all rows.  The band writes the interior of its
    columns, reads the column left of it (rows 0..n: the border, or band k-1's last column) and
    row 0 of its columns."""
    c0, c1 = k * width + 1, min((k + 1) * width, n)
    W = Lmad(ld + c0, ((n, ld), (c1 - c0 + 1, 1)))
    Rleft = Lmad(c0 - 1, ((n + 1, ld),))
    Rtop = Lmad(c0, ((c1 - c0 + 1, 1),))
    return W, Rleft, Rtop


def wave_schedule_proofs(n: int, width: int, ld: int | None = None):
    """The persistent kernel runs neighbouring bands concurrently, in place.  Legal iff, for every
    band k: its writes miss its own reads (W_k ∩ Rleft_k = W_k ∩ Rtop_k = ∅), no two bands write
    one cell (W_k ∩ W_k+1 = ∅), and band k+1 never overwrites what band k still reads
    (W_k+1 ∩ Rleft_k = W_k+1 ∩ Rtop_k = ∅).  Returns one tuple of five proofs per band."""
    ld = n + 1 if ld is None else ld
    nb = -(-n // width)
    res = []
    for k in range(nb):
        W, Rl, Rt = wave_band_lmads(n, ld, width, k)
        if k + 1 < nb:
            W1 = wave_band_lmads(n, ld, width, k + 1)[0]
            nxt = (non_overlap(W, W1), non_overlap(W1, Rl), non_overlap(W1, Rt))
        else:
            nxt = (True, True, True)
        res.append((non_overlap(W, Rl), non_overlap(W, Rt)) + nxt)
    return res
