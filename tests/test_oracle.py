"""Pins for the CPU oracle (oracle/nw_ref.c) — none of them re-types the oracle's loop.

Each pin is chosen so that a plausible slip in the oracle (a dropped term, a wrong sign,
a swapped index, a transposed operand, an off-by-one on the borders) fails at least one:

P1  hand-worked example (tests/golden/appendix_b.txt): cell function, BLOSUM62 lookup,
    orientation (a down the rows, b across the columns), borders.
P2  brute-force enumeration of ALL alignment paths for n <= 8 — the definition of the
    global-alignment score with linear gaps (what the paper's Fig. 2 loop computes,
    PAPER.md P:371-381), both for the standard borders and for arbitrary
    borders (paths leave a border cell immediately; reading R5).
P3  closed form for a constant ref.
P4  invariants: borders untouched, lower/upper bounds, monotone border.
P5  metamorphic: transpose symmetry (BLOSUM62 is symmetric), border shift.
P6  independent formulation: each row as a max-plus prefix scan (numpy).
    plus: the streaming oracle equals the full oracle; int32 overflow is reported.
"""
import sys

import numpy as np
import pytest

import inputs
import oracle

sys.setrecursionlimit(10000)


# ---------------------------------------------------------------- P1
def test_hand_example(golden):
    g = golden("appendix_b.txt")
    p = int(g["p"])
    a, b = inputs.encode(g["a"]), inputs.encode(g["b"])
    n = len(a)
    ref = inputs.build_ref(a, b)
    np.testing.assert_array_equal(ref, np.array(g["ref"], dtype=np.int32))
    score = inputs.init_borders(inputs.aligned_matrix(n), p)
    inputs.fill_interior(score, inputs.SENTINEL)
    oracle.nw_ref(score, ref, p)
    np.testing.assert_array_equal(score, np.array(g["score"], dtype=np.int32))


# ---------------------------------------------------------------- P2
def brute_force(ref, row0, col0, p, n):
    """max over every monotone lattice path that starts on a border cell, steps off it
    immediately, and ends at (i, j): border value + sum of step scores
    (diagonal step into (i,j): +ref[i][j]; vertical or horizontal step: -p).
    Pure enumeration — no memoisation, no recurrence."""
    best = [[None] * (n + 1) for _ in range(n + 1)]

    def walk(i, j, acc):
        if best[i][j] is None or acc > best[i][j]:
            best[i][j] = acc
        if i < n and j < n:
            walk(i + 1, j + 1, acc + int(ref[i + 1][j + 1]))
        if i < n:
            walk(i + 1, j, acc - p)
        if j < n:
            walk(i, j + 1, acc - p)

    for k in range(n + 1):            # start on row 0 at (0, k)
        if k + 1 <= n:
            walk(1, k + 1, int(row0[k]) + int(ref[1][k + 1]))
        if k >= 1:
            walk(1, k, int(row0[k]) - p)
    for k in range(1, n + 1):         # start on column 0 at (k, 0)
        if k + 1 <= n:
            walk(k + 1, 1, int(col0[k]) + int(ref[k + 1][1]))
        walk(k, 1, int(col0[k]) - p)
    return best


def _check_brute(n, p, seed, family, border_seed=None):
    score, ref = inputs.make_problem(n, p, seed=seed, family=family, border_seed=border_seed)
    row0, col0 = score[0].copy(), score[:, 0].copy()
    oracle.nw_ref(score, ref, p)
    best = brute_force(ref, row0, col0, p, n)
    for i in range(1, n + 1):
        for j in range(1, n + 1):
            assert score[i, j] == best[i][j], (n, p, seed, family, i, j)


@pytest.mark.parametrize("n", [1, 2, 3, 4, 5])
@pytest.mark.parametrize("p", [0, 1, 3, 10])
@pytest.mark.parametrize("family", ["random", "homologous"])
def test_brute_force_small(n, p, family):
    for seed in range(3):
        _check_brute(n, p, 100 + seed, family)


@pytest.mark.parametrize("n,p,seed", [(6, 10, 1), (6, 1, 2), (7, 3, 3), (8, 10, 7), (8, 0, 8)])
def test_brute_force_up_to_8(n, p, seed):
    _check_brute(n, p, seed, "random")


@pytest.mark.parametrize("n,p,seed", [(1, 10, 5), (3, 10, 5), (4, 1, 6), (5, 3, 7), (6, 10, 8)])
def test_brute_force_arbitrary_borders(n, p, seed):
    _check_brute(n, p, seed, "random", border_seed=seed)


# ---------------------------------------------------------------- P3
@pytest.mark.parametrize("c", [-25, -20, -4, 0, 5, 9])
@pytest.mark.parametrize("p", [0, 1, 10])
def test_constant_ref_closed_form(c, p):
    n = 37
    score, ref = inputs.make_problem(n, p, family="const", const_ref=c)
    oracle.nw_ref(score, ref, p)
    i = np.arange(n + 1)[:, None]
    j = np.arange(n + 1)[None, :]
    if c + 2 * p > 0:
        expect = np.minimum(i, j) * c - np.abs(i - j) * p
    else:
        expect = -(i + j) * p
    np.testing.assert_array_equal(score, expect.astype(np.int32))


# ---------------------------------------------------------------- P4
@pytest.mark.parametrize("n,p", [(64, 10), (100, 1), (257, 3)])
def test_bounds_and_borders(n, p):
    score, ref = inputs.make_problem(n, p, seed=11)
    row0, col0 = score[0].copy(), score[:, 0].copy()
    oracle.nw_ref(score, ref, p)
    np.testing.assert_array_equal(score[0], row0)
    np.testing.assert_array_equal(score[:, 0], col0)
    assert (score != inputs.SENTINEL).all()
    M = int(ref[1:, 1:].max())
    i = np.arange(n + 1)[:, None]
    j = np.arange(n + 1)[None, :]
    lower = -(i + j) * p
    upper = np.maximum(np.minimum(i, j) * (M + 2 * p), 0) - (i + j) * p
    assert (score >= lower).all() and (score <= upper).all()
    if p > 0:
        assert (np.diff(score[0]) < 0).all() and (np.diff(score[:, 0]) < 0).all()


# ---------------------------------------------------------------- P5
@pytest.mark.parametrize("n,p", [(50, 10), (129, 3)])
def test_transpose_symmetry(n, p):
    a, b = inputs.gen_pair(n, 21)
    b62 = inputs.blosum62()
    assert (b62 == b62.T).all()
    s1 = inputs.init_borders(inputs.aligned_matrix(n), p)
    s2 = inputs.init_borders(inputs.aligned_matrix(n), p)
    oracle.nw_ref(s1, inputs.build_ref(a, b), p)
    oracle.nw_ref(s2, inputs.build_ref(b, a), p)
    np.testing.assert_array_equal(s1, s2.T)


@pytest.mark.parametrize("K", [-1000, 1, 12345])
def test_border_shift(K):
    n, p = 70, 10
    s1, ref = inputs.make_problem(n, p, seed=3, border_seed=4)
    s2 = s1.copy()
    s2[0, :] += K
    s2[1:, 0] += K
    oracle.nw_ref(s1, ref, p)
    oracle.nw_ref(s2, ref, p)
    np.testing.assert_array_equal(s2.astype(np.int64) - s1, np.full(s1.shape, K))


# ---------------------------------------------------------------- P6
def maxplus_scan_rows(score0: np.ndarray, ref: np.ndarray, p: int) -> np.ndarray:
    """Row i as a max-plus prefix scan:  t[j] = max(s[i-1][j-1] + ref[i][j], s[i-1][j] - p)
    (t[0] = s[i][0]),  s[i][j] = max_{k<=j} (t[k] + k p) - j p."""
    s = score0.astype(np.int64).copy()
    n = s.shape[0] - 1
    k = np.arange(n + 1, dtype=np.int64) * p
    for i in range(1, n + 1):
        t = np.empty(n + 1, dtype=np.int64)
        t[0] = s[i, 0]
        t[1:] = np.maximum(s[i - 1, :-1] + ref[i, 1:n + 1], s[i - 1, 1:] - p)
        s[i, :] = np.maximum.accumulate(t + k) - k
    return s


@pytest.mark.parametrize("n,p,family", [(31, 10, "random"), (512, 10, "random"),
                                        (2048, 10, "random"), (777, 1, "homologous"),
                                        (300, 0, "random")])
def test_maxplus_scan_formulation(n, p, family):
    score, ref = inputs.make_problem(n, p, seed=5, family=family)
    expect = maxplus_scan_rows(score, ref, p)
    oracle.nw_ref(score, ref, p)
    np.testing.assert_array_equal(score, expect)


def test_maxplus_scan_arbitrary_borders():
    n, p = 300, 10
    score, ref = inputs.make_problem(n, p, seed=9, border_seed=10)
    expect = maxplus_scan_rows(score, ref, p)
    oracle.nw_ref(score, ref, p)
    np.testing.assert_array_equal(score, expect)


# ---------------------------------------------------------------- streaming + overflow
@pytest.mark.parametrize("chunk", [1, 7, 64])
def test_stream_equals_full(chunk):
    n, p = 300, 10
    score, ref = inputs.make_problem(n, p, seed=13, border_seed=14)
    full = oracle.nw_ref(score.copy(), ref, p)
    st = oracle.NwRefStream(n, p, score[0])
    rows = [score[0:1]]
    for i0 in range(1, n + 1, chunk):
        i1 = min(n + 1, i0 + chunk)
        rows.append(st.rows(ref[i0:i1], score[i0:i1, 0]))
    np.testing.assert_array_equal(np.concatenate(rows), full)
    np.testing.assert_array_equal(st.last(), full[n])
    st.close()


def test_pitched_layout():
    n, p = 97, 10
    a, b = inputs.gen_pair(n, 17)
    s1 = inputs.init_borders(inputs.aligned_matrix(n), p)
    s2 = inputs.init_borders(inputs.aligned_matrix(n, ld=n + 20), p)
    oracle.nw_ref(s1, inputs.build_ref(a, b), p)
    oracle.nw_ref(s2, inputs.build_ref(a, b, ld=n + 7), p)
    np.testing.assert_array_equal(s1, s2[:, : n + 1])


def test_overflow_reported():
    n = 3
    score = inputs.aligned_matrix(n)
    ref = inputs.aligned_matrix(n)
    ref[1:, 1:] = 1 << 30
    with pytest.raises(OverflowError):
        oracle.nw_ref(score, ref, 0)
