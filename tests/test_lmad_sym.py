"""The symbolic NonOverlap test (Fig. 8 / Theorem / Fig. 9; NEXT-4).

Pins, none of which re-uses the prover's arithmetic:
S1  footnote 27: the offset difference nb - b - n - 1 is distributed exactly as the
    paper says (+1 to I1 at stride nb - b, +1 to I2 at strides n and 1).  tests/golden/fig9_symbolic.txt.
S2  Fig. 9: the two sums of intervals and the four split pieces are the ones the paper prints
    (same fixture), and W ∩ Rvert = ∅ is PROVEN for all q >= 2, b >= 2, i >= 0 and for all
    q >= 3, b >= 1, i >= 0; W ∩ Rhoriz = ∅ for all q >= 2, b >= 1, i >= 0.
S3  Fig. 9's premise "2 <= q, 1 <= b, 0 <= i" admits q = 2, b = 1, i = 2, where brute
    force finds a common element (offset 6), so the prover must refuse that assumption set; on
    the anti-diagonals that exist at q = 2 (i <= q - 1) enumeration shows the claim holds
    (reading R17).
S4  soundness by brute force: at sampled symbol values every proven pair is disjoint by
    enumeration of both point sets; random symbolic LMAD pairs the prover accepts are disjoint
    at every sampled instance.
S5  the LMADs proven are the ones the kernels use: the diagonal kernels' nw_diag_lmad (C ABI)
    equals diag_lmads at (cnt, b, base, N), and wave_bands equals lmad.wave_band_lmads.
S6  the persistent kernel's band schedule (csrc/nw_wave.cuh): all five in-place legality
    conditions PROVEN for every n, W, k, w1 and pitch padding at once; the true dependency
    (band k+1 reads band k's last column) is not proven and overlaps by enumeration.
"""
import ctypes
import os
import random

import pytest

import paper_conf_sc_munksgaardhso22_b200 as nwb
from paper_conf_sc_munksgaardhso22_b200.lmad import nw_diag_lmads, wave_band_lmads
from paper_conf_sc_munksgaardhso22_b200.lmad_sym import (Assume, Poly, diag_lmads, fig9, lmad, offset_split, prove, sym, syms,
                                                        wave_band_assumptions, wave_band_proofs, wave_bands)

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "fig9_symbolic.txt")
q, b, i, n = syms("q b i n")
NAMES = {"q": q, "b": b, "i": i, "n": n}


def points(L):
    pts = {L.offset}
    for c, s in L.dims:
        pts = {p + k * s for p in pts for k in range(c)}
    return pts if all(c > 0 for c, _ in L.dims) else set()


def expr(s):
    return Poly.lift(eval(s, {"__builtins__": {}}, NAMES))


def golden():
    rows = {}
    for line in open(GOLDEN):
        if not line.strip() or line.startswith("#"):
            continue
        name, body = (x.strip() for x in line.split("|", 1))
        rows[name] = body
    return rows


def parse_intervals(body):
    """'n*b-b: 0 .. i ; n: 1 .. b ; 1: 1 .. b' -> {stride: (lo, hi)} with n = q b + 1."""
    A = Assume({"n": q * b + 1}, {})
    out = {}
    for part in body.split(";"):
        st, rng = part.split(":")
        lo, hi = rng.split("..")
        out[A.norm(expr(st))] = (A.norm(expr(lo)), A.norm(expr(hi)))
    return out


def as_dict(strides, I):
    return {s: (l, u) for s, (l, u) in zip(strides, I)}


FIG9 = Assume({"n": q * b + 1}, {"q": 2, "b": 2, "i": 0})


# ---- S1 -----------------------------------------------------------------------------------
def test_footnote27_distribution():
    body = golden()["footnote27"]
    t0s, i1s, i2s = (x.strip() for x in body.split(";"))
    t0 = expr(t0s.split("=", 1)[1])
    strides = [n * b - b, n, Poly.lift(1)]
    A = Assume({}, {"n": 2, "b": 1})       # footnote 27 keeps n free
    to1, to2 = offset_split(t0, strides, A)

    def amounts(s):
        d = {}
        for kv in s.split("+=", 1)[1].split(","):
            k, v = kv.split(":")
            d[expr(k)] = expr(v)
        return [d[x] for x in strides]

    assert to1 == amounts(i1s) and to2 == amounts(i2s)


# ---- S2 -----------------------------------------------------------------------------------
def test_fig9_sums_of_intervals_and_split_match_the_paper():
    W, Rv, _ = fig9()
    pr = prove(W, Rv, FIG9)
    assert pr.ok
    root, g = pr.root, golden()
    assert as_dict(root.strides, root.I1) == parse_intervals(g["W_I"])
    assert as_dict(root.strides, root.I2) == parse_intervals(g["Rvert_I"])
    assert root.verdict == "split"
    assert [as_dict(root.strides, I) for I in root.split1] == [parse_intervals(g["W1_I"]), parse_intervals(g["W2_I"])]
    assert [as_dict(root.strides, I) for I in root.split2] == [parse_intervals(g["Rvert1_I"]), parse_intervals(g["Rvert2_I"])]
    # "W1 ∩ Rvert2 = ∅ holds because [1..b-1]·n ∩ [0..0]·n = ∅"; the other three
    # pairs by their stride-1 intervals
    verdicts = [c.verdict for c in root.children]
    assert verdicts[1] == f"disjoint@{q * b + 1}"
    assert verdicts[0] == verdicts[2] == verdicts[3] == "disjoint@1"


@pytest.mark.parametrize("lower", [{"q": 2, "b": 2, "i": 0}, {"q": 3, "b": 1, "i": 0}])
def test_fig9_w_rvert_proven(lower):
    W, Rv, _ = fig9()
    assert prove(W, Rv, Assume({"n": q * b + 1}, lower)).ok


@pytest.mark.parametrize("lower", [{"q": 2, "b": 1, "i": 0}, {"q": 2, "b": 2, "i": 0}])
def test_fig9_w_rhoriz_proven(lower):
    W, _, Rh = fig9()
    assert prove(W, Rh, Assume({"n": q * b + 1}, lower)).ok


# ---- S3 -----------------------------------------------------------------------------------
def test_fig9_premise_edge_case():
    W, Rv, _ = fig9()
    assert not prove(W, Rv, Assume({"n": q * b + 1}, {"q": 2, "b": 1, "i": 0})).ok
    env = {"q": 2, "b": 1, "i": 2, "n": 3}
    assert points(W.at(env)) & points(Rv.at(env)) == {6}      # the premise admits an overlap
    for ii in range(2):                                          # the diagonals of a q = 2 grid
        env = {"q": 2, "b": 1, "i": ii, "n": 3}
        assert not points(W.at(env)) & points(Rv.at(env))


# ---- S4 -----------------------------------------------------------------------------------
def test_fig9_proofs_hold_at_instances():
    W, Rv, Rh = fig9()
    for qq in range(2, 7):
        for bb in range(1, 6):
            for ii in range(0, 7):
                env = {"q": qq, "b": bb, "i": ii, "n": qq * bb + 1}
                if bb >= 2 or qq >= 3:
                    assert not points(W.at(env)) & points(Rv.at(env)), env
                assert not points(W.at(env)) & points(Rh.at(env)), env


def test_soundness_random_symbolic_pairs():
    rng = random.Random(11)
    x, y = syms("x y")
    A = Assume({}, {"x": 1, "y": 0})
    terms = [Poly.lift(1), Poly.lift(2), x, x + 1, 2 * x, x + y + 1, x * x]
    proven = 0
    for _ in range(600):
        def rand():
            dims = tuple((rng.choice([Poly.lift(1), Poly.lift(2), x, x + 1, y + 1]), rng.choice(terms))
                         for _ in range(rng.randint(1, 3)))
            return lmad(rng.randint(0, 6) + rng.randint(0, 2) * x + rng.randint(0, 1) * y, *dims)
        L1, L2 = rand(), rand()
        if prove(L1, L2, A).ok:
            proven += 1
            for _ in range(8):
                env = A.sample(rng, hi=4)
                assert not points(L1.at(env)) & points(L2.at(env)), (L1, L2, env)
    assert proven >= 10          # (random pairs mostly overlap or share a stride twice)


# ---- S5 -----------------------------------------------------------------------------------
@pytest.mark.parametrize("nn,tile,pad", [(64, 16, 0), (96, 32, 3), (128, 8, 1)])
def test_diag_kernel_lmads_are_the_proven_ones(nn, tile, pad):
    L = nwb.lib()
    N = nn + 1 + pad
    qq = nn // tile
    for d in range(2 * qq - 1):
        got = nw_diag_lmads(L, nn, N, tile, d)
        out = (ctypes.c_int64 * 10)()
        assert L.nw_diag_lmad(nn, N, tile, d, out) == 0
        cnt, base = out[0], out[1]
        want = diag_lmads(c=Poly.lift(cnt), b=Poly.lift(tile), base=Poly.lift(base), N=Poly.lift(N))
        assert tuple(w.at({}) for w in want) == got
    # and the symbolic proof covers every diagonal of every grid (both triangles, padded pitch)
    g = sym("g")
    Wd, Rv, Rh = diag_lmads()
    for lower in ({"q": 2, "b": 2, "c": 1, "base": 0, "g": 0}, {"q": 3, "b": 1, "c": 1, "base": 0, "g": 0}):
        A = Assume({"N": q * b + 1 + g}, lower)
        assert prove(Wd, Rv, A).ok and prove(Wd, Rh, A).ok


def test_wave_band_lmads_match_the_concrete_ones():
    rng = random.Random(5)
    A = wave_band_assumptions(pitch_pad=False)
    for _ in range(40):
        env = A.sample(rng, hi=5)
        Wk, Rl, Rt, Wk1 = wave_bands()
        nn, ld, W, k = env["n"], env["ld"], env["W"], env["k"]
        cW, cRl, cRt = wave_band_lmads(nn, ld, W, k)
        assert (Wk.at(env), Rl.at(env), Rt.at(env)) == (cW, cRl, cRt)
        # band k+1's width is w1 = min(W, n - (k+1) W) when it is the last band
        if env["r"] == 0:
            assert Wk1.at(env) == wave_band_lmads(nn, ld, W, k + 1)[0]


# ---- S6 -----------------------------------------------------------------------------------
def test_wave_band_schedule_proven_symbolically():
    res = wave_band_proofs()
    assert all(p.ok for p in res.values()), {k: p.root.verdict if p.root else p.reason for k, p in res.items()}
    rng = random.Random(3)
    A = wave_band_assumptions()
    Wk, Rl, Rt, Wk1 = wave_bands()
    for _ in range(30):
        env = A.sample(rng, hi=4)
        pts = [points(L.at(env)) for L in (Wk, Rl, Rt, Wk1)]
        assert not pts[0] & (pts[1] | pts[2] | pts[3]) and not pts[3] & (pts[1] | pts[2])


def test_wave_band_true_dependency_not_proven():
    k, Wd, ld = sym("k"), sym("W"), sym("ld")
    Wk = wave_bands()[0]
    Rleft_next = lmad((k + 1) * Wd, (sym("n") + 1, ld))
    A = wave_band_assumptions()
    assert not prove(Wk, Rleft_next, A).ok
    env = A.sample(random.Random(1), hi=3)
    assert points(Wk.at(env)) & points(Rleft_next.at(env))
