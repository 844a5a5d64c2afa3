"""Python-int oracle for the G1 / G2 MSM — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this module.  The product path never does.

What it computes is the plain definition (§2.1):

    s . P = sum_{i=0}^{N-1} s_i (x) P_i

in the group E(F_p): y^2 = x^3 + a x + b (§2.1) with the
chord-and-tangent group law in AFFINE coordinates, PMUL by left-to-right
binary double-and-add ("split into a series of PADD in order of the integer's
bit sequence"), and a sequential sum.  No windows, no buckets,
no projective coordinates, no Montgomery form: nothing here resembles the
Pippenger pipeline of the CUDA path.

The identity O is represented as None internally and encoded as (0, 0) on the
wire (reading R5).  Python ints are exact, so no rounding question
arises.
"""

from __future__ import annotations

from typing import Iterable, Optional, Sequence, Tuple

from .curves import Curve, get

Point = Optional[Tuple[int, int]]   # None = identity O


def inv_mod(x: int, p: int) -> int:
    if x % p == 0:
        raise ZeroDivisionError("inverse of 0")
    return pow(x, -1, p)


class Fp:
    """F_p on Python ints (G1)."""

    def __init__(self, p: int):
        self.p = p
        self.zero, self.one = 0, 1

    def add(self, x, y): return (x + y) % self.p
    def sub(self, x, y): return (x - y) % self.p
    def mul(self, x, y): return x * y % self.p
    def neg(self, x): return (-x) % self.p
    def inv(self, x): return inv_mod(x, self.p)
    def small(self, k: int): return k % self.p
    def elem(self, v): return v % self.p


class Fp2:
    """F_p^2 = F_p[u]/(u^2 - beta), elements (c0, c1) = c0 + c1 u (G2).  The
    product is the schoolbook polynomial product reduced by u^2 = beta."""

    def __init__(self, p: int, beta: int):
        self.p, self.beta = p, beta
        self.zero, self.one = (0, 0), (1, 0)

    def add(self, x, y): return ((x[0] + y[0]) % self.p, (x[1] + y[1]) % self.p)
    def sub(self, x, y): return ((x[0] - y[0]) % self.p, (x[1] - y[1]) % self.p)
    def neg(self, x): return ((-x[0]) % self.p, (-x[1]) % self.p)

    def mul(self, x, y):
        p = self.p
        return ((x[0] * y[0] + self.beta * x[1] * y[1]) % p, (x[0] * y[1] + x[1] * y[0]) % p)

    def inv(self, x):
        # (x0 + x1 u)^-1 = (x0 - x1 u) / (x0^2 - beta x1^2), the norm lies in F_p
        p = self.p
        nrm = (x[0] * x[0] - self.beta * x[1] * x[1]) % p
        ni = inv_mod(nrm, p)
        return (x[0] * ni % p, (-x[1]) * ni % p)

    def small(self, k: int): return (k % self.p, 0)
    def elem(self, v): return (v[0] % self.p, v[1] % self.p)


def field(c) -> "Fp | Fp2":
    c = get(c)
    return Fp2(c.p, c.beta) if c.deg == 2 else Fp(c.p)


def on_curve(c: Curve, P: Point) -> bool:
    if P is None:
        return True
    F = field(c)
    x, y = P
    rhs = F.add(F.add(F.mul(F.mul(x, x), x), F.mul(F.elem(c.a), x)), F.elem(c.b))
    return F.mul(y, y) == rhs


def neg(c: Curve, P: Point) -> Point:
    if P is None:
        return None
    return (P[0], field(c).neg(P[1]))


def add(c: Curve, P: Point, Q: Point) -> Point:
    """Affine chord-and-tangent addition with every exceptional case explicit
    ("PADD ... including point doubling", PAPER.md:116 footnote 2), over F_p
    (G1) or F_p^2 (G2)."""
    F = field(c)
    if P is None:
        return Q
    if Q is None:
        return P
    x1, y1 = P
    x2, y2 = Q
    if x1 == x2:
        if F.add(y1, y2) == F.zero:      # P == -Q (covers y == 0 doubling too)
            return None
        num = F.add(F.mul(F.small(3), F.mul(x1, x1)), F.elem(c.a))   # tangent
        lam = F.mul(num, F.inv(F.add(y1, y1)))
    else:
        lam = F.mul(F.sub(y2, y1), F.inv(F.sub(x2, x1)))             # chord
    x3 = F.sub(F.sub(F.mul(lam, lam), x1), x2)
    y3 = F.sub(F.mul(lam, F.sub(x1, x3)), y1)
    return (x3, y3)


def mul(c: Curve, k: int, P: Point) -> Point:
    """PMUL k (x) P by left-to-right binary double-and-add."""
    if k < 0:
        return mul(c, -k, neg(c, P))
    R: Point = None
    for bit in bin(k)[2:] if k else "":
        R = add(c, R, R)
        if bit == "1":
            R = add(c, R, P)
    return R


def msm(c, points: Sequence[Point], scalars: Iterable[int]) -> Point:
    """Q = sum_i k_i (x) P_i, the definition."""
    c = get(c)
    Q: Point = None
    for P, k in zip(points, scalars):
        if k == 0 or P is None:
            continue
        Q = add(c, Q, mul(c, k, P))
    return Q


def generator(c) -> Point:
    c = get(c)
    return (c.gx, c.gy)


# ---- wire encoding (the ABI's: little-endian u32 limbs, identity = (0,0)) ----

def encode_point(c, P: Point) -> list:
    """x || y; a G2 coordinate is c0 || c1 (each L limbs)."""
    c = get(c)
    L = c.limbs
    if P is None:
        return [0] * (2 * c.coord_limbs)
    if c.deg == 2:
        return [w for v in (P[0][0], P[0][1], P[1][0], P[1][1]) for w in int_to_limbs(v, L)]
    return int_to_limbs(P[0], L) + int_to_limbs(P[1], L)


def decode_point(c, limbs: Sequence[int]) -> Point:
    c = get(c)
    L = c.limbs
    v = [limbs_to_int(limbs[i * L:(i + 1) * L]) for i in range(2 * c.deg)]
    if not any(v):
        return None
    if c.deg == 2:
        return ((v[0], v[1]), (v[2], v[3]))
    return (v[0], v[1])


def int_to_limbs(v: int, n: int) -> list:
    if v < 0 or v >> (32 * n):
        raise ValueError("value does not fit")
    return [(v >> (32 * i)) & 0xFFFFFFFF for i in range(n)]


def limbs_to_int(limbs: Sequence[int]) -> int:
    v = 0
    for i, w in enumerate(limbs):
        v |= int(w) << (32 * i)
    return v
