"""Python-int oracle for the G1 MSM — TEST INFRASTRUCTURE ONLY.

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


def on_curve(c: Curve, P: Point) -> bool:
    if P is None:
        return True
    x, y = P
    return (y * y - (x * x * x + c.a * x + c.b)) % c.p == 0


def neg(c: Curve, P: Point) -> Point:
    if P is None:
        return None
    return (P[0], (-P[1]) % c.p)


def add(c: Curve, P: Point, Q: Point) -> Point:
    """Affine chord-and-tangent addition with every exceptional case explicit
    ("PADD ... including point doubling", PAPER.md:116 footnote 2)."""
    p = c.p
    if P is None:
        return Q
    if Q is None:
        return P
    x1, y1 = P
    x2, y2 = Q
    if x1 == x2:
        if (y1 + y2) % p == 0:          # P == -Q (covers y == 0 doubling too)
            return None
        lam = (3 * x1 * x1 + c.a) * inv_mod(2 * y1, p) % p   # tangent
    else:
        lam = (y2 - y1) * inv_mod(x2 - x1, p) % p             # chord
    x3 = (lam * lam - x1 - x2) % p
    y3 = (lam * (x1 - x3) - y1) % p
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
    c = get(c)
    L = c.limbs
    if P is None:
        return [0] * (2 * L)
    return int_to_limbs(P[0], L) + int_to_limbs(P[1], L)


def decode_point(c, limbs: Sequence[int]) -> Point:
    c = get(c)
    L = c.limbs
    x = limbs_to_int(limbs[:L])
    y = limbs_to_int(limbs[L:2 * L])
    if x == 0 and y == 0:
        return None
    return (x, y)


def int_to_limbs(v: int, n: int) -> list:
    if v < 0 or v >> (32 * n):
        raise ValueError("value does not fit")
    return [(v >> (32 * i)) & 0xFFFFFFFF for i in range(n)]


def limbs_to_int(limbs: Sequence[int]) -> int:
    v = 0
    for i, w in enumerate(limbs):
        v |= int(w) << (32 * i)
    return v
