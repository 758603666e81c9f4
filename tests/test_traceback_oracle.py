"""Pins for the traceback oracle (oracle/nw_ref.c nw_traceback_ref).

The paper stops at the score matrix (Fig. 2); the traceback recovers the
alignment it scores, with the tie rule diagonal > up > left (reading R12).  Pins:

T1  hand example (tests/golden/appendix_b_traceback.txt).
T2  brute force, n <= 6: enumerate EVERY alignment (monotone path from the origin), keep the
    optimal ones, and take the lexicographically smallest op sequence read from (n, n)
    backwards with diagonal < up < left.  The oracle's ops must be that sequence.  Families
    with many ties (ref in {-1, 0, 1}, p in {0, 1}) exercise the tie rule.
T3  any size: the ops form a valid global alignment (n a-residues, n b-residues) whose score,
    summed independently from ref and p, equals score[n][n].
T4  a matrix that is not a fill is rejected.
"""
import itertools

import numpy as np
import pytest

import inputs
import oracle


def test_hand_example(golden):
    g = golden("appendix_b_traceback.txt")
    p = int(g["p"])
    a, b = inputs.encode(g["a"]), inputs.encode(g["b"])
    n = len(a)
    ref = inputs.build_ref(a, b)
    score = inputs.init_borders(inputs.aligned_matrix(n), p)
    oracle.nw_ref(score, ref, p)
    np.testing.assert_array_equal(oracle.nw_traceback_ref(score, ref, p), np.array(g["ops"][0], dtype=np.uint8))


def path_score(ops, ref, p):
    i = j = 0
    s = 0
    for o in ops:
        if o == 0:
            i += 1; j += 1; s += int(ref[i][j])
        elif o == 1:
            i += 1; s -= p
        else:
            j += 1; s -= p
    return i, j, s


def all_alignments(n):
    """Every monotone path (0,0) -> (n,n) as a forward op tuple (pure enumeration)."""
    out = []

    def rec(i, j, acc):
        if i == n and j == n:
            out.append(tuple(acc))
            return
        if i < n and j < n:
            rec(i + 1, j + 1, acc + [0])
        if i < n:
            rec(i + 1, j, acc + [1])
        if j < n:
            rec(i, j + 1, acc + [2])

    rec(0, 0, [])
    return out


def _problem(n, p, seed, family):
    rng = np.random.default_rng(seed)
    if family == "ties":
        ref = np.zeros((n + 1, n + 1), dtype=np.int32)
        ref[1:, 1:] = rng.integers(-1, 2, size=(n, n))
        score = inputs.init_borders(inputs.aligned_matrix(n), p)
    else:
        score, ref = inputs.make_problem(n, p, seed=seed, family=family)
    return score, ref


@pytest.mark.parametrize("n", [1, 2, 3, 4, 5, 6])
@pytest.mark.parametrize("p,family", [(0, "ties"), (1, "ties"), (10, "random"), (3, "homologous")])
@pytest.mark.parametrize("seed", [1, 2])
def test_brute_force_tie_rule(n, p, family, seed):
    score, ref = _problem(n, p, seed, family)
    oracle.nw_ref(score, ref, p)
    paths = all_alignments(n)
    scores = [path_score(q, ref, p)[2] for q in paths]
    best = max(scores)
    want = min(tuple(reversed(q)) for q, s in zip(paths, scores) if s == best)
    got = oracle.nw_traceback_ref(score, ref, p)
    assert tuple(reversed(got.tolist())) == want
    assert best == score[n, n]


@pytest.mark.parametrize("n,p,family", [(64, 10, "random"), (300, 1, "random"), (1000, 10, "homologous"),
                                        (513, 0, "random")])
def test_alignment_scores_the_corner(n, p, family):
    score, ref = _problem(n, p, 7, family)
    oracle.nw_ref(score, ref, p)
    ops = oracle.nw_traceback_ref(score, ref, p)
    assert n <= len(ops) <= 2 * n and set(np.unique(ops).tolist()) <= {0, 1, 2}
    assert path_score(ops.tolist(), ref, p) == (n, n, int(score[n, n]))


def test_not_a_fill_rejected():
    n, p = 16, 10
    score, ref = _problem(n, p, 3, "random")
    oracle.nw_ref(score, ref, p)
    score[n, n] += 1000
    with pytest.raises(ValueError):
        oracle.nw_traceback_ref(score, ref, p)
