"""The paper's non-overlap test on SYMBOLIC LMADs (NEXT-4, host side).

``lmad.py`` runs Fig. 8 on concrete integers.  This module runs the same procedure when offsets,
counts and strides are polynomials in symbols (q, b, i, n, ...), which is how the paper states and
proves its NW example (Fig. 9): a proof here holds for EVERY value of the symbols
allowed by the assumptions, not only for the sizes a test enumerates.

Pieces, each following the paper's text:

* ``Poly`` — integer polynomials in named symbols (the "computer algebra support for subtracting
  the offsets").
* ``Assume`` — the assumptions of a proof: equalities as substitutions (n = q b + 1) and integer
  lower bounds (2 <= q, 1 <= b, 0 <= i).  ``Assume.pos(e)`` proves e > 0 for all admitted
  values: shift every symbol to its lower bound (v = lo + v', v' >= 0) and check that the expanded
  polynomial has non-negative coefficients and a positive constant.  Sound (a sufficient test),
  not complete: False means "not proven".
* distribution of the offset difference (P:1495-1500 and footnote 27): t1 - t2 is
  divided by the strides, largest leading term first; each quotient monomial adds to the interval
  bounds of I1 when its sign is positive and, made positive, to I2's when it is negative.  Since all
  symbols are >= 0, each side only ever gains non-negative amounts, so l >= 0 holds (Theorem
  premise).
* the Theorem (Non-Overlap): both sums of intervals have no overlapping dimensions
  (s_k > sum_{j<k} u_j s_j in some common order of the dimensions) and some pair of matching
  intervals is disjoint (u1_j < l2_j or u2_j < l1_j).  The order is the strides sorted by size
  (provable comparisons, then degree); other orders are tried when that one fails (the theorem
  holds for any fixed order in which the conditions hold: mixed-radix uniqueness).
* the split heuristic (Fig. 8): the interval below the first overflowing stride is
  rewritten as its last point plus the rest; the last point's offset is redistributed over the
  strides (Fig. 9: [0..b]·n -> [0..b-1]·n ∪ {b·n}, and b·n = (nb - b) + b), and all pairs of
  pieces are proven recursively.

``prove`` returns a ``Proof`` tree that records every sum-of-intervals and split, so tests can
compare the intermediate forms with the ones Fig. 9 prints.  ``fig9`` builds the paper's NW LMADs;
``wave_bands`` the persistent kernel's bands (csrc/nw_wave.cuh), for which ``wave_band_proofs``
proves the in-place legality conditions symbolically.  Host-side analysis only.
"""
from __future__ import annotations

import itertools
from dataclasses import dataclass, field


# ---------------------------------------------------------------------------- polynomials
class Poly:
    """Integer polynomial: {monomial: coefficient}, a monomial a sorted tuple of (symbol, exp)."""

    __slots__ = ("t",)

    def __init__(self, terms=None):
        self.t = {m: c for m, c in (terms or {}).items() if c != 0}

    @staticmethod
    def lift(x) -> "Poly":
        if isinstance(x, Poly):
            return x
        if isinstance(x, int):
            return Poly({(): x})
        raise TypeError(f"not a polynomial: {x!r}")

    # arithmetic
    def __add__(self, o):
        o = Poly.lift(o)
        r = dict(self.t)
        for m, c in o.t.items():
            r[m] = r.get(m, 0) + c
        return Poly(r)

    __radd__ = __add__

    def __neg__(self):
        return Poly({m: -c for m, c in self.t.items()})

    def __sub__(self, o):
        return self + (-Poly.lift(o))

    def __rsub__(self, o):
        return Poly.lift(o) - self

    def __mul__(self, o):
        o = Poly.lift(o)
        r = {}
        for m1, c1 in self.t.items():
            for m2, c2 in o.t.items():
                m = _mono_mul(m1, m2)
                r[m] = r.get(m, 0) + c1 * c2
        return Poly(r)

    __rmul__ = __mul__

    def __pow__(self, k: int):
        r = Poly.lift(1)
        for _ in range(k):
            r = r * self
        return r

    def __eq__(self, o):
        return isinstance(o, (Poly, int)) and (self - o).is_zero()

    def __hash__(self):
        return hash(frozenset(self.t.items()))

    # inspection
    def is_zero(self) -> bool:
        return not self.t

    def is_const(self) -> bool:
        return all(m == () for m in self.t)

    def const(self) -> int:
        return self.t.get((), 0)

    def symbols(self) -> set:
        return {v for m in self.t for v, _ in m}

    def degree(self) -> int:
        return max((_deg(m) for m in self.t), default=0)

    def leading(self):
        """Leading (monomial, coefficient) in graded lexicographic order."""
        m = max(self.t, key=_mono_key)
        return m, self.t[m]

    def subs(self, env: dict) -> "Poly":
        r = Poly.lift(0)
        for m, c in self.t.items():
            term = Poly.lift(c)
            for v, e in m:
                term = term * (Poly.lift(env[v]) ** e if v in env else Poly({((v, e),): 1}))
            r = r + term
        return r

    def split_sign(self):
        """(P+, P-) with self = P+ - P-, both with non-negative coefficients."""
        return (Poly({m: c for m, c in self.t.items() if c > 0}),
                Poly({m: -c for m, c in self.t.items() if c < 0}))

    def __repr__(self):
        if not self.t:
            return "0"
        parts = []
        for m in sorted(self.t, key=_mono_key, reverse=True):
            c = self.t[m]
            mono = "*".join(v if e == 1 else f"{v}^{e}" for v, e in m)
            if not mono:
                parts.append(str(c))
            elif c == 1:
                parts.append(mono)
            elif c == -1:
                parts.append("-" + mono)
            else:
                parts.append(f"{c}*{mono}")
        return " + ".join(parts).replace("+ -", "- ")


def sym(name: str) -> Poly:
    return Poly({((name, 1),): 1})


def syms(names: str):
    return tuple(sym(v) for v in names.split())


def _deg(m) -> int:
    return sum(e for _, e in m)


def _mono_key(m):
    return (_deg(m), m)


def _mono_mul(a, b):
    d = dict(a)
    for v, e in b:
        d[v] = d.get(v, 0) + e
    return tuple(sorted(d.items()))


def _mono_div(a, b):
    """a / b if b divides a, else None."""
    d = dict(a)
    for v, e in b:
        if d.get(v, 0) < e:
            return None
        d[v] -= e
    return tuple(sorted((v, e) for v, e in d.items() if e))


# ---------------------------------------------------------------------------- assumptions
@dataclass
class Assume:
    """Equalities as substitutions (applied first) and integer lower bounds >= 0 on the symbols
    that remain.  Every remaining symbol needs a bound (an unbounded symbol proves nothing)."""
    subs: dict = field(default_factory=dict)
    lower: dict = field(default_factory=dict)

    def __post_init__(self):
        assert all(isinstance(v, int) and v >= 0 for v in self.lower.values()), "symbols are >= 0"

    def norm(self, e) -> Poly:
        return Poly.lift(e).subs(self.subs) if self.subs else Poly.lift(e)

    def nonneg(self, e) -> bool:
        p = self.norm(e)
        if not p.symbols() <= set(self.lower):
            return False
        shifted = p.subs({v: sym(v) + lo for v, lo in self.lower.items() if lo})
        return all(c >= 0 for c in shifted.t.values())

    def pos(self, e) -> bool:
        return self.nonneg(Poly.lift(e) - 1)

    def zero(self, e) -> bool:
        return self.norm(e).is_zero()

    def sample(self, rng, hi: int = 6) -> dict:
        """Concrete values of every symbol (bounded symbols drawn from [lo, lo + hi], then the
        substitutions evaluated), for brute-force checks of a proof."""
        env = {v: rng.randint(lo, lo + hi) for v, lo in self.lower.items()}
        for v, e in self.subs.items():
            env[v] = Poly.lift(e).subs(env).const()
        return env


# ---------------------------------------------------------------------------- LMADs
@dataclass(frozen=True)
class SymLmad:
    """offset + {(count : stride), ...} with polynomial entries (eq. (1), §II-B)."""
    offset: Poly
    dims: tuple

    def at(self, env: dict):
        """The concrete LMAD (lmad.Lmad) at symbol values env."""
        from .lmad import Lmad
        ev = lambda e: Poly.lift(e).subs(env).const()
        return Lmad(ev(self.offset), tuple((ev(c), ev(s)) for c, s in self.dims))


def lmad(offset, *dims) -> SymLmad:
    return SymLmad(Poly.lift(offset), tuple((Poly.lift(c), Poly.lift(s)) for c, s in dims))


@dataclass
class Node:
    """One step of the proof: the two sums of intervals over the common strides, the verdict,
    and (when neither was non-overlapping) the split pieces and their sub-proofs."""
    strides: list
    I1: list  # [[l, u], ...] aligned with strides
    I2: list
    verdict: str = ""       # "disjoint@<stride>", "split", "fail: ..."
    order: list | None = None
    split1: tuple | None = None  # pieces of I1 (I1 itself if it had no overlapping dimension)
    split2: tuple | None = None
    children: list = field(default_factory=list)

    def ok(self) -> bool:
        if self.verdict.startswith("disjoint"):
            return True
        if self.verdict == "split":
            return all(c.ok() for c in self.children)
        return False


@dataclass
class Proof:
    ok: bool
    root: Node | None
    reason: str = ""


def _normalise(L: SymLmad, A: Assume):
    """Positive strides; count-1 and stride-0 dimensions dropped."""
    t, dims = A.norm(L.offset), []
    for c, s in L.dims:
        c, s = A.norm(c), A.norm(s)
        if not A.nonneg(c):
            return None, f"count {c} not provably >= 0"
        if c == 1 or s.is_zero():
            continue
        if A.pos(s):
            dims.append((c, s))
        elif A.pos(-s):
            t = t + (c - 1) * s
            dims.append((c, -s))
        else:
            return None, f"stride {s} of unknown sign"
    return SymLmad(t, tuple(dims)), ""


def _sort_strides(strides, A: Assume):
    """Increasing size: provable comparisons, degree / leading term as the tie-break."""
    out = sorted(strides, key=lambda s: (s.degree(), _mono_key(s.leading()[0])))
    for _ in range(len(out)):
        for k in range(len(out) - 1):
            if A.pos(out[k] - out[k + 1]):
                out[k], out[k + 1] = out[k + 1], out[k]
    return out


def _distribute(delta: Poly, strides, A: Assume):
    """delta = sum_k c_k * strides[k] (multivariate division, largest leading term first; the
    constant stride 1 takes the remainder).  Returns the quotients, or None."""
    q = [Poly.lift(0) for _ in strides]
    rem = delta
    order = sorted(range(len(strides)), key=lambda k: _mono_key(strides[k].leading()[0]), reverse=True)
    for k in order:
        s = strides[k]
        if s == 1:
            continue
        ms, cs = s.leading()
        while True:
            cand = [(m, c) for m, c in rem.t.items() if _mono_div(m, ms) is not None and c % cs == 0]
            if not cand:
                break
            m, c = max(cand, key=lambda mc: _mono_key(mc[0]))
            qt = Poly({_mono_div(m, ms): c // cs})
            q[k] = q[k] + qt
            rem = rem - qt * s
    k1 = [k for k, s in enumerate(strides) if s == 1]
    if not k1:
        return None if not rem.is_zero() else q
    q[k1[0]] = q[k1[0]] + rem
    return q


def offset_split(delta, strides, A: Assume):
    """Footnote 27: the offset difference t1 - t2 distributed over the strides ->
    (amounts added to I1's intervals, amounts added to I2's), aligned with `strides`; None if it
    does not divide out."""
    q = _distribute(A.norm(delta), [A.norm(s) for s in strides], A)
    if q is None:
        return None
    parts = [c.split_sign() for c in q]
    return [p for p, _ in parts], [m for _, m in parts]


def _intervals(L1: SymLmad, L2: SymLmad, A: Assume):
    """Steps 1-2 of Fig. 8: matching strides and the two sums of intervals [l, u]."""
    strides = []
    for _, s in L1.dims + L2.dims + ((None, Poly.lift(1)),):
        if not any(A.zero(s - x) for x in strides):
            strides.append(s)
    strides = _sort_strides(strides, A)

    def base(L):
        iv = [[Poly.lift(0), Poly.lift(0)] for _ in strides]
        for c, s in L.dims:
            k = next(k for k, x in enumerate(strides) if A.zero(s - x))
            if not iv[k][1].is_zero():
                return None  # two dimensions of one stride
            iv[k][1] = c - 1
        return iv

    I1, I2 = base(L1), base(L2)
    if I1 is None or I2 is None:
        return None
    q = _distribute(A.norm(L1.offset - L2.offset), strides, A)
    if q is None:
        return None
    for k, c in enumerate(q):
        pos, neg = c.split_sign()     # symbols >= 0: both parts are >= 0
        I1[k] = [I1[k][0] + pos, I1[k][1] + pos]
        I2[k] = [I2[k][0] + neg, I2[k][1] + neg]
    return strides, I1, I2


def _no_overlap_in(order, I, A: Assume) -> int | None:
    """None if I has no overlapping dimension in this order, else the first overflowing index."""
    acc = Poly.lift(0)
    for pos_, k in enumerate(order):
        s, (_, u) = k[0], I[k[1]]
        if pos_ > 0 and not A.pos(s - acc):
            return pos_
        acc = acc + u * s
    return None


def _renorm(strides, I, A: Assume):
    """Redistribute a sum of intervals' lower corner over the strides (Fig. 9's W^2 / Rvert^2:
    [b..b]·n becomes +1 on nb - b and +b on 1)."""
    off = sum((iv[0] * s for iv, s in zip(I, strides)), Poly.lift(0))
    q = _distribute(A.norm(off), strides, A)
    if q is None or any(not A.nonneg(c) for c in q):
        return [list(iv) for iv in I]
    return [[c, c + (iv[1] - iv[0])] for c, iv in zip(q, I)]


def _split(strides, order, I, at, A: Assume):
    """Fig. 8 splitAnOverlappingDimensionInto2LMADs: the non-trivial interval right below the
    overflow at position `at` -> (rest, last point); None = Fail."""
    for pos_ in range(at - 1, -1, -1):
        k = order[pos_][1]
        l, u = I[k]
        if not A.zero(u - l):
            rest = [list(iv) for iv in I]
            rest[k] = [l, u - 1]
            last = [list(iv) for iv in I]
            last[k] = [u, u]
            return rest, _renorm(strides, last, A)
    return None


def _prove(strides, I1, I2, A: Assume, depth: int) -> Node:
    node = Node(strides, I1, I2)
    if not all(A.nonneg(l) for l, _ in I1 + I2):
        node.verdict = "fail: a lower bound not provably >= 0"
        return node
    base_order = [(s, k) for k, s in enumerate(strides)]
    orders = [base_order] + [list(o) for o in itertools.permutations(base_order) if list(o) != base_order]
    for order in orders:
        if _no_overlap_in(order, I1, A) is None and _no_overlap_in(order, I2, A) is None:
            node.order = [s for s, _ in order]
            for k, s in enumerate(strides):
                (l1, u1), (l2, u2) = I1[k], I2[k]
                if A.pos(l2 - u1) or A.pos(l1 - u2):
                    node.verdict = f"disjoint@{s}"
                    return node
            node.verdict = "fail: no disjoint pair of intervals"
            return node
    if depth == 0:
        node.verdict = "fail: depth"
        return node
    o1, o2 = _no_overlap_in(base_order, I1, A), _no_overlap_in(base_order, I2, A)
    P1 = (I1,) if o1 is None else _split(strides, base_order, I1, o1, A)
    P2 = (I2,) if o2 is None else _split(strides, base_order, I2, o2, A)
    if P1 is None or P2 is None:
        node.verdict = "fail: split"
        return node
    node.verdict, node.split1, node.split2 = "split", P1, P2
    for a in P1:
        for b in P2:
            node.children.append(_prove(strides, a, b, A, depth - 1))
    return node


def prove(L1: SymLmad, L2: SymLmad, A: Assume, depth: int = 4) -> Proof:
    """Fig. 8 NonOverlap on symbolic LMADs: ok = True proves L1 ∩ L2 = ∅ for all symbol values
    the assumptions admit."""
    N1, why1 = _normalise(L1, A)
    N2, why2 = _normalise(L2, A)
    if N1 is None or N2 is None:
        return Proof(False, None, why1 or why2)
    r = _intervals(N1, N2, A)
    if r is None:
        return Proof(False, None, "not a pair of sums of intervals with matching strides")
    root = _prove(*r, A, depth)
    return Proof(root.ok(), root)


# ---------------------------------------------------------------------------- the NW LMADs
def fig9(q=None, b=None, i=None, n=None):
    """PAPER.md P:548-552 (and Fig. 9): the anti-diagonal-i slices of the flat
    n·n array, n = q b + 1 the row length: (W, Rvert, Rhoriz)."""
    q, b, i, n = (sym(v) if x is None else x for v, x in zip("qbin", (q, b, i, n)))
    W = lmad(i * b + n + 1, (i + 1, n * b - b), (b, n), (b, 1))
    Rvert = lmad(i * b, (i + 1, n * b - b), (b + 1, n))
    Rhoriz = lmad(i * b + 1, (i + 1, n * b - b), (b, 1))
    return W, Rvert, Rhoriz


def diag_lmads(c=None, b=None, base=None, N=None):
    """The diagonal kernels' slices (csrc/nw_diag.cuh diag_lmad, nw_diag_lmad of the C ABI) for a
    diagonal of c tiles at `base`, pitch N: the same shapes as Fig. 9 with i + 1 -> c and the
    diagonal's corner as the offset (upper-left triangle: base = i b; lower-right: base =
    e b N + (q - 1) b)."""
    c, b, base, N = (sym(v) if x is None else x for v, x in zip(("c", "b", "base", "N"), (c, b, base, N)))
    W = lmad(base + N + 1, (c, N * b - b), (b, N), (b, 1))
    Rvert = lmad(base, (c, N * b - b), (b + 1, N))
    Rhoriz = lmad(base + 1, (c, N * b - b), (b, 1))
    return W, Rvert, Rhoriz


def wave_bands(k=None, W=None, w1=None, ld=None, n=None):
    """The persistent kernel's bands (csrc/nw_wave.cuh; lmad.wave_band_lmads): band k covers
    columns kW+1 .. kW+W of every row 1..n (pitch ld), band k+1 the next w1 <= W columns.
    Returns (W_k, Rleft_k, Rtop_k, W_k+1)."""
    k, Wd, w1, ld, n = (sym(v) if x is None else x for v, x in zip(("k", "W", "w1", "ld", "n"), (k, W, w1, ld, n)))
    Wk = lmad(ld + k * Wd + 1, (n, ld), (Wd, 1))
    Rleft = lmad(k * Wd, (n + 1, ld))
    Rtop = lmad(k * Wd + 1, (Wd, 1))
    Wk1 = lmad(ld + (k + 1) * Wd + 1, (n, ld), (w1, 1))
    return Wk, Rleft, Rtop, Wk1


def wave_band_assumptions(pitch_pad: bool = True) -> Assume:
    """Band k full (it has a successor), band k+1 of width 1 <= w1 <= W, n >= (k+1)W + w1 rows
    and columns: W = w1 + u, ld = n + 1 + g (g >= 0: a padded pitch)."""
    k, w1, u, r, g = syms("k w1 u r g")
    Wd = w1 + u
    n = (k + 1) * Wd + w1 + r
    subs = {"W": Wd, "n": n, "ld": n + 1 + (g if pitch_pad else 0)}
    lower = {"k": 0, "w1": 1, "u": 0, "r": 0}
    if pitch_pad:
        lower["g"] = 0
    return Assume(subs, lower)


def wave_band_proofs(A: Assume | None = None) -> dict:
    """In-place legality of running neighbouring bands concurrently (lmad.wave_schedule_proofs,
    now for all n, W, k at once): name -> Proof."""
    A = A or wave_band_assumptions()
    Wk, Rl, Rt, Wk1 = wave_bands()
    return {
        "W_k ∩ Rleft_k": prove(Wk, Rl, A),
        "W_k ∩ Rtop_k": prove(Wk, Rt, A),
        "W_k ∩ W_k+1": prove(Wk, Wk1, A),
        "W_k+1 ∩ Rleft_k": prove(Wk1, Rl, A),
        "W_k+1 ∩ Rtop_k": prove(Wk1, Rt, A),
    }
