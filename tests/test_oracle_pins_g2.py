"""Pins for the G2 oracle (`-m "not gpu"`), SURVEY.md §8(f) NEXT-3.

G2 is the order-r subgroup of the sextic twist E'(F_p^2): y^2 = x^3 + b' over
F_p^2 = F_p[u]/(u^2 + 1) (GZKP's MSM optimisations apply "to both
G1 and G2"; reading R14).  Nothing here retypes the oracle's
formulas; each plausible mistake fails at least one test:
  * wrong F_p^2 product (sign of beta, swapped cross terms)
        -> Frobenius x^p = conj(x), x^(p^2 - 1) = 1, C == Python
  * wrong twist coefficient b'           -> b' (9 + u) = 3 / b' = 4 (1 + u), G2 on E'
  * wrong generator or group law         -> r G2 = O and G2 != O; cofactor h r R = O
  * group law over F_p^2 (chord/tangent, exceptional cases)
        -> toy E(F_p^2) point count = the Weil count from E(F_p), Lagrange
  * MSM sum / encoding                   -> closed form, brute force, C == Python
"""

import random

import numpy as np
import pytest

import oracle
import synth
from oracle import curves, ref
from oracle.curves import Curve

G2 = [curves.BN254_G2, curves.BLS12_381_G2]


def _pow2(F, x, e):
    r = F.one
    while e:
        if e & 1:
            r = F.mul(r, x)
        x = F.mul(x, x)
        e >>= 1
    return r


def _sqrt2(F, a):
    """Square root in F_p^2 (u^2 = -1, p = 3 mod 4): Adj & Rodriguez-Henriquez,
    Algorithm 9.  Returns None for a non-square."""
    p = F.p
    a1 = _pow2(F, a, (p - 3) // 4)
    alpha = F.mul(a1, F.mul(a1, a))
    x0 = F.mul(a1, a)
    if alpha == (p - 1, 0):
        x = F.mul((0, 1), x0)
    else:
        x = F.mul(_pow2(F, F.add(F.one, alpha), (p - 1) // 2), x0)
    return x if F.mul(x, x) == a else None


def _random_twist_point(c, rng):
    F = ref.field(c)
    while True:
        x = (rng.randrange(c.p), rng.randrange(c.p))
        rhs = F.add(F.mul(F.mul(x, x), x), c.b)
        y = _sqrt2(F, rhs)
        if y is not None:
            return (x, y)


@pytest.mark.parametrize("c", G2, ids=lambda c: c.name)
def test_fp2_frobenius_and_order(c):
    # u^2 = -1 is a non-residue (p = 3 mod 4), so x^p is the conjugate and the
    # multiplicative group has order p^2 - 1: both fail for a wrong product.
    assert c.p % 4 == 3 and c.beta == c.p - 1
    F = ref.field(c)
    rng = random.Random(7)
    for _ in range(4):
        x = (rng.randrange(1, c.p), rng.randrange(1, c.p))
        assert _pow2(F, x, c.p) == (x[0], (-x[1]) % c.p)
        assert _pow2(F, x, c.p * c.p - 1) == F.one
        assert F.mul(x, F.inv(x)) == F.one


@pytest.mark.parametrize("c", G2, ids=lambda c: c.name)
def test_fp2_c_oracle_equals_python(c):
    F = ref.field(c)
    rng = random.Random(11)
    vals = [(0, 0), (1, 0), (0, 1), (c.p - 1, c.p - 1)] + [(rng.randrange(c.p), rng.randrange(c.p))
                                                           for _ in range(40)]
    for x in vals:
        for y in vals[:6] + [vals[-1]]:
            assert oracle.fp2_mul(c, x, y) == F.mul(x, y)


def test_twist_coefficients():
    p = curves.BN254.p
    b0, b1 = curves.BN254_G2.b
    # b' = 3 / (9 + u)  <=>  b' (9 + u) = 3 (EIP-197's twist of y^2 = x^3 + 3)
    assert ((9 * b0 - b1) % p, (b0 + 9 * b1) % p) == (3, 0)
    assert curves.BLS12_381_G2.b == (4, 4)          # 4 (1 + u)


@pytest.mark.parametrize("c", G2, ids=lambda c: c.name)
def test_g2_generator_on_twist_and_order_r(c):
    G = (c.gx, c.gy)
    assert ref.on_curve(c, G)
    assert ref.mul(c, c.r, G) is None
    assert ref.mul(c, c.r - 1, G) == ref.neg(c, G)
    assert ref.mul(c, 2, G) is not None
    # C oracle agrees: r G = O, (r-1) G = -G
    Gl = oracle.generator_limbs(c)
    k = np.array([ref.int_to_limbs(c.r, c.scalar_limbs), ref.int_to_limbs(c.r - 1, c.scalar_limbs)],
                 dtype=np.uint32)
    out = oracle.mul_each(c, Gl, k, 2)
    assert not out[0].any()
    assert ref.decode_point(c, list(out[1])) == ref.neg(c, G)


@pytest.mark.parametrize("c", G2, ids=lambda c: c.name)
def test_g2_cofactor(c):
    # #E'(F_p^2) = h r: a random twist point is killed by h r but not by r or h
    R = _random_twist_point(c, random.Random(3))
    assert ref.on_curve(c, R)
    assert ref.mul(c, c.cofactor * c.r, R) is None
    assert ref.mul(c, c.r, R) is not None
    cleared = ref.mul(c, c.cofactor, R)
    assert cleared is not None and ref.mul(c, c.r, cleared) is None


# ---- toy curve over F_p^2: brute-force enumeration against the Weil count ----
TOY_P = 103          # p = 3 mod 4: u^2 = -1 gives F_p^2
TOY_B = 5


def _toy2(a: int, b: int) -> Curve:
    return Curve(name="toy2", cid=-1, p=TOY_P, r=0, a=(a, 0), b=(b, 0), gx=(0, 0), gy=(0, 0),
                 cofactor=1, scalar_bits=16, deg=2, beta=TOY_P - 1)


@pytest.mark.parametrize("a", [0, 2])
def test_toy_fp2_enumeration_weil(a):
    """E: y^2 = x^3 + a x + 5 defined over F_103.  Over F_p^2 the group order
    must be p^2 + 1 - (t^2 - 2p) with t = p + 1 - #E(F_p) (Weil), and every
    point is killed by it (Lagrange)."""
    p = TOY_P
    n1 = 1 + sum(1 for x in range(p) for y in range(p) if (y * y - (x ** 3 + a * x + TOY_B)) % p == 0)
    t = p + 1 - n1
    n2_weil = p * p + 1 - (t * t - 2 * p)
    c = _toy2(a, TOY_B)
    F = ref.field(c)
    squares = {}
    for y0 in range(p):
        for y1 in range(p):
            squares.setdefault(F.mul((y0, y1), (y0, y1)), []).append((y0, y1))
    pts = [None]
    for x0 in range(p):
        for x1 in range(p):
            x = (x0, x1)
            rhs = F.add(F.add(F.mul(F.mul(x, x), x), F.mul((a, 0), x)), (TOY_B, 0))
            pts.extend((x, y) for y in squares.get(rhs, []))
    assert len(pts) == n2_weil
    rng = random.Random(5)
    for P in rng.sample(pts[1:], 25):
        assert ref.on_curve(c, P)
        assert ref.mul(c, n2_weil, P) is None
    # associativity / commutativity on random triples (exceptional cases included)
    for _ in range(300):
        P, Q, R = (rng.choice(pts) for _ in range(3))
        assert ref.add(c, ref.add(c, P, Q), R) == ref.add(c, P, ref.add(c, Q, R))
        assert ref.add(c, P, Q) == ref.add(c, Q, P)
    # the C oracle's F_p^2 group law agrees with Python's on the toy
    for _ in range(200):
        P, Q = rng.choice(pts), rng.choice(pts)
        if rng.random() < 0.2:
            Q = P
        got = oracle.ec_add(c, np.array(ref.encode_point(c, P), dtype=np.uint32),
                            np.array(ref.encode_point(c, Q), dtype=np.uint32))
        assert ref.decode_point(c, list(got)) == ref.add(c, P, Q)


# ---- MSM on G2 -----------------------------------------------------------------
@pytest.mark.parametrize("c", G2, ids=lambda c: c.name)
def test_g2_closed_form_and_c_equals_python(c):
    n = 24
    d = synth.dlogs(c.name, n, synth.dlog_seed(c.name))
    k = synth.scalars(c.name, n, synth.scalar_seed(7))
    pts = oracle.points_from_dlogs(c, d)
    got = oracle.msm(c, pts, k)
    assert np.array_equal(got, oracle.closed_form(c, k, d))
    P = [ref.decode_point(c, list(row)) for row in pts]
    assert all(ref.on_curve(c, q) for q in P)
    kk = [ref.limbs_to_int(row) for row in k]
    assert ref.encode_point(c, ref.msm(c, P[:6], kk[:6])) == list(oracle.msm(c, pts[:6], k[:6]))


@pytest.mark.parametrize("c", G2, ids=lambda c: c.name)
def test_g2_brute_force_small_scalars(c):
    rng = random.Random(9)
    G = (c.gx, c.gy)
    P = [G, ref.add(c, G, G), ref.neg(c, G), None, G]
    ks = [rng.randrange(0, 16) for _ in P]
    want = None
    for Pi, ki in zip(P, ks):
        for _ in range(ki):
            want = ref.add(c, want, Pi)
    pts = np.array([ref.encode_point(c, q) for q in P], dtype=np.uint32)
    k = np.zeros((len(P), c.scalar_limbs), dtype=np.uint32)
    k[:, 0] = ks
    assert ref.decode_point(c, list(oracle.msm(c, pts, k))) == want
