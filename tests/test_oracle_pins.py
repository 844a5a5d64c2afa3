"""Pins for the oracle (`-m "not gpu"`): checks against what the paper and the
mathematics fix, never against the oracle's own formulas retyped.

Each plausible oracle mistake fails at least one test here:
  * wrong constant (p, r, a, b, G)        -> primality / on-curve / r*G = O / Hasse
  * wrong chord or tangent formula         -> EIP-196 2G vector, toy enumeration
  * dropped a*x term (MNT4 has a = 2)      -> toy_a2 group order / associativity
  * wrong exceptional case (P == -Q, O)    -> toy enumeration, (r-1)G = -G
  * double-and-add bit order / index       -> toy k*P by repeated addition
  * Knuth-D qhat correction, EEA inverse   -> Python-int remainders / inverses
  * MSM sum / threading / encoding         -> closed form, brute force, C == Python
"""

import os
import random

import numpy as np
import pytest

import oracle
import synth
from oracle import curves, ref

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
BIG = [curves.BN254, curves.BLS12_381, curves.MNT4_753]
TOYS = [curves.TOY_A0, curves.TOY_A2]


def is_probable_prime(n: int, rounds: int = 40) -> bool:
    if n < 2:
        return False
    for sp in (2, 3, 5, 7, 11, 13, 17, 19, 23, 29, 31, 37):
        if n % sp == 0:
            return n == sp
    d, s = n - 1, 0
    while d % 2 == 0:
        d //= 2
        s += 1
    rng = random.Random(12345)
    for _ in range(rounds):
        a = rng.randrange(2, n - 1)
        x = pow(a, d, n)
        if x in (1, n - 1):
            continue
        for _ in range(s - 1):
            x = x * x % n
            if x == n - 1:
                break
        else:
            return False
    return True


# ------------------------------------------------------------ curve constants

@pytest.mark.parametrize("c", BIG + TOYS, ids=lambda c: c.name)
def test_moduli_prime(c):
    assert is_probable_prime(c.p)
    assert is_probable_prime(c.r)


@pytest.mark.parametrize("c", BIG + TOYS, ids=lambda c: c.name)
def test_generator_on_curve_and_order(c):
    G = ref.generator(c)
    assert ref.on_curve(c, G)
    assert ref.mul(c, c.r, G) is None                    # r*G = O
    assert ref.mul(c, c.r - 1, G) == ref.neg(c, G)       # (r-1)*G = -G
    assert ref.mul(c, c.r + 1, G) == G


@pytest.mark.parametrize("c", BIG + TOYS, ids=lambda c: c.name)
def test_hasse_bound(c):
    # #E = h*r must satisfy |p + 1 - #E| <= 2 sqrt(p) (Hasse); the group order is
    # unique in that interval when r > 4 sqrt(p), which pins the cofactor too.
    from math import isqrt
    n = c.cofactor * c.r
    assert (p1 := c.p + 1 - n) * p1 <= 4 * c.p
    if c.r * c.r > 16 * c.p:
        assert 4 * isqrt(c.p) < c.r


@pytest.mark.parametrize("c", BIG, ids=lambda c: c.name)
def test_identity_encoding_unambiguous(c):
    # (0,0) encodes O: it must not be a curve point (b != 0 for all three).
    assert (c.b % c.p) != 0
    assert not ref.on_curve(c, (0, 0))


def test_bls_cofactor_clearing():
    # h*P for a random curve point P lands in the order-r subgroup.
    c = curves.BLS12_381
    x = 5
    while True:
        rhs = (x ** 3 + c.a * x + c.b) % c.p
        y = pow(rhs, (c.p + 1) // 4, c.p)          # p = 3 mod 4
        if y * y % c.p == rhs:
            break
        x += 1
    P = (x, y)
    assert ref.on_curve(c, P)
    Q = ref.mul(c, c.cofactor, P)
    assert ref.mul(c, c.r, Q) is None
    assert ref.mul(c, c.r, P) is not None            # P itself is not in G1


# ------------------------------------------------------ known multiples (EIP-196)

def _golden_xy(name):
    vals = {}
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            k, v = line.split()
            vals[k] = int(v)
    return vals["x"], vals["y"]


def test_bn254_eip196_double():
    c = curves.BN254
    want = _golden_xy("bn254_eip196_double.txt")
    G = ref.generator(c)
    assert ref.add(c, G, G) == want
    assert ref.mul(c, 2, G) == want
    got = oracle.ec_add("bn254", oracle.generator_limbs("bn254"), oracle.generator_limbs("bn254"))
    assert ref.decode_point(c, got) == want


@pytest.mark.parametrize("c", BIG, ids=lambda c: c.name)
def test_double_equals_add_chain(c):
    G = ref.generator(c)
    P = G
    for k in range(2, 12):
        P = ref.add(c, P, G)                 # chord additions only
        assert ref.mul(c, k, G) == P         # double-and-add


# --------------------------------------------------------------- toy curves

@pytest.mark.parametrize("c", TOYS, ids=lambda c: c.name)
def test_toy_enumeration_group_order(c):
    squares = {}
    for y in range(c.p):
        squares.setdefault(y * y % c.p, []).append(y)
    pts = [None]
    for x in range(c.p):
        for y in squares.get((x ** 3 + c.a * x + c.b) % c.p, []):
            pts.append((x, y))
    assert len(pts) == c.r                   # #E(F_p) = r (prime order, cofactor 1)
    # every non-identity point has order r
    rng = random.Random(7)
    for P in rng.sample(pts[1:], 20):
        assert ref.mul(c, c.r, P) is None
        assert ref.mul(c, 1, P) == P


@pytest.mark.parametrize("c", TOYS, ids=lambda c: c.name)
def test_toy_group_axioms(c):
    G = ref.generator(c)
    rng = random.Random(3)
    pts = [ref.mul(c, rng.randrange(c.r), G) for _ in range(60)]
    for i in range(40):
        P, Q, R = pts[i], pts[i + 1], pts[i + 2]
        assert ref.add(c, ref.add(c, P, Q), R) == ref.add(c, P, ref.add(c, Q, R))
        assert ref.add(c, P, Q) == ref.add(c, Q, P)
        assert ref.on_curve(c, ref.add(c, P, Q))
        assert ref.add(c, P, ref.neg(c, P)) is None
        assert ref.add(c, P, None) == P


@pytest.mark.parametrize("c", TOYS, ids=lambda c: c.name)
def test_toy_mul_by_repeated_addition_all_k(c):
    G = ref.generator(c)
    acc = None
    for k in range(c.r + 1):
        assert ref.mul(c, k, G) == acc, k
        acc = ref.add(c, acc, G)
    # the C oracle's double-and-add over every k as well
    ks = np.arange(c.r + 1, dtype=np.uint32).reshape(-1, 1)
    out = oracle.mul_each(c.name, oracle.generator_limbs(c.name), ks)
    acc = None
    for k in range(c.r + 1):
        assert ref.decode_point(c, out[k]) == acc, k
        acc = ref.add(c, acc, G)


# --------------------------------------------------- bignum / field internals

def test_knuth_d_against_python_ints():
    rng = random.Random(11)
    for _ in range(3000):
        n = rng.randrange(1, 25)
        m = rng.randrange(n, 2 * n + 1)
        v = rng.getrandbits(32 * n) | (1 << (32 * n - 1 - rng.randrange(0, 32)))
        v |= 1
        u = rng.getrandbits(32 * m)
        if rng.random() < 0.3:               # force qhat-correction shapes
            q = rng.getrandbits(32 * (m - n))
            u = (q * v + rng.randrange(v)) % (1 << (32 * m))
        if v >> (32 * n):
            continue
        assert oracle.bn_mod(u, m, v, n) == u % v


@pytest.mark.parametrize("c", BIG + TOYS, ids=lambda c: c.name)
def test_field_mul_inv_against_python_ints(c):
    rng = random.Random(c.cid)
    edge = [0, 1, 2, c.p - 1, c.p - 2, (c.p - 1) // 2, (1 << (c.p.bit_length() - 1)) % c.p]
    vals = edge + [rng.randrange(c.p) for _ in range(150)]
    for x in vals:
        y = rng.choice(vals)
        assert oracle.fp_mul(c, x, y) == x * y % c.p
        if x:
            assert oracle.fp_inv(c, x) == pow(x, -1, c.p)


# ------------------------------------------------------------- oracle MSM

def _rand_points(c, n, seed):
    rng = random.Random(seed)
    G = ref.generator(c)
    a = [rng.randrange(1, c.r) for _ in range(n)]
    return [ref.mul(c, ai, G) for ai in a], a


@pytest.mark.parametrize("c", [curves.BN254, curves.BLS12_381], ids=lambda c: c.name)
def test_closed_form_python(c):
    pts, a = _rand_points(c, 24, 5)
    rng = random.Random(6)
    k = [rng.randrange(c.r) for _ in range(24)]
    want = ref.mul(c, sum(x * y for x, y in zip(k, a)) % c.r, ref.generator(c))
    assert ref.msm(c, pts, k) == want


def test_brute_force_small_scalars():
    # k_i <= 15: MSM by repeated addition only (no doubling formula used at all
    # except where P_i + P_i occurs inside the repeated sum).
    c = curves.BN254
    pts, _ = _rand_points(c, 6, 9)
    ks = [0, 1, 2, 7, 15, 3]
    acc = None
    for P, k in zip(pts, ks):
        for _ in range(k):
            acc = ref.add(c, acc, P)
    assert ref.msm(c, pts, ks) == acc
    L = c.limbs
    P = np.array([ref.encode_point(c, q) for q in pts], dtype=np.uint32)
    K = np.zeros((6, c.scalar_limbs), dtype=np.uint32)
    K[:, 0] = ks
    assert ref.decode_point(c, oracle.msm("bn254", P, K)) == acc


@pytest.mark.parametrize("c", BIG + TOYS, ids=lambda c: c.name)
def test_c_oracle_equals_python_oracle(c):
    n = 4 if c is curves.MNT4_753 else 12
    rng = random.Random(c.cid + 1)
    G = ref.generator(c)
    pts = [ref.mul(c, rng.randrange(1, c.r), G) for _ in range(n)]
    pts[1] = None                                  # identity input
    pts[2] = pts[3]                                # duplicate point
    ks = [rng.randrange(1 << c.scalar_bits) for _ in range(n)]
    ks[0] = 0
    ks[2] = (c.r - ks[3] % c.r) % c.r              # k2*P + k3*P = O (P2 == P3)
    P = np.array([ref.encode_point(c, q) for q in pts], dtype=np.uint32)
    K = np.array([ref.int_to_limbs(k, c.scalar_limbs) for k in ks], dtype=np.uint32)
    want = ref.msm(c, pts, ks)
    for nt in (1, 3):
        assert ref.decode_point(c, oracle.msm(c, P, K, nthreads=nt)) == want


@pytest.mark.parametrize("c", [curves.BN254, curves.BLS12_381, curves.TOY_A2], ids=lambda c: c.name)
def test_c_oracle_closed_form_seeded(c):
    n = 64
    d = synth.dlogs(c.name, n, synth.dlog_seed(c.name))
    pts = oracle.points_from_dlogs(c.name, d)
    k = synth.scalars(c.name, n, 77)
    got = oracle.msm(c.name, pts, k)
    assert np.array_equal(got, oracle.closed_form(c.name, k, d))
    # linearity: MSM(k) + MSM(k') = MSM(k + k') for small k' so no overflow
    k2 = synth.scalars(c.name, n, 78, dist="all_one")
    both = oracle.ec_add(c.name, got, oracle.msm(c.name, pts, k2))
    ksum = k.copy()
    carry = np.ones(n, dtype=np.uint64)
    for i in range(k.shape[1]):
        t = k[:, i].astype(np.uint64) + carry
        ksum[:, i] = (t & 0xFFFFFFFF).astype(np.uint32)
        carry = t >> np.uint64(32)
    assert np.array_equal(both, oracle.msm(c.name, pts, ksum))


def test_dot_mod_exact():
    rng = random.Random(1)
    c = curves.BLS12_381
    n = 300
    k = [rng.randrange(c.r) for _ in range(n)]
    a = [rng.randrange(c.r) for _ in range(n)]
    K = np.array([ref.int_to_limbs(x, 8) for x in k], dtype=np.uint32)
    A = np.array([ref.int_to_limbs(x, 8) for x in a], dtype=np.uint32)
    assert oracle.dot_mod(K, A, c.r) == sum(x * y for x, y in zip(k, a)) % c.r
    # several chunks (the float64 partial products are summed across chunks)
    assert oracle.dot_mod(K, A, c.r, chunk=7) == sum(x * y for x, y in zip(k, a)) % c.r


def test_dot_mod_tiled_and_extreme_limbs():
    """a_i = dlogs[i mod m] (SURVEY.md §8(d) tiling) and all-ones limbs, where
    a chunk's float64 sums are largest (every 16-bit half 0xffff)."""
    rng = random.Random(2)
    c = curves.MNT4_753
    n, m = 1000, 37
    k = [rng.randrange(c.r) for _ in range(n)]
    a = [rng.randrange(c.r) for _ in range(m)]
    K = np.array([ref.int_to_limbs(x, 24) for x in k], dtype=np.uint32)
    A = np.array([ref.int_to_limbs(x, 24) for x in a], dtype=np.uint32)
    want = sum(k[i] * a[i % m] for i in range(n)) % c.r
    assert oracle.dot_mod(K, A, c.r) == want
    assert oracle.dot_mod(K, A, c.r, chunk=64) == want
    big = np.full((3000, 24), 0xFFFFFFFF, dtype=np.uint32)
    assert oracle.dot_mod(big, big, c.r) == (3000 * ((1 << 768) - 1) ** 2) % c.r


def test_msm_empty_and_zero():
    for c in (curves.BN254, curves.TOY_A0):
        L = c.limbs
        assert oracle.msm(c, np.zeros((0, 2 * L), np.uint32), np.zeros((0, c.scalar_limbs), np.uint32)).sum() == 0
        pts = oracle.points_from_dlogs(c.name, synth.dlogs(c.name, 5, 1))
        assert oracle.msm(c, pts, synth.scalars(c.name, 5, 1, "all_zero")).sum() == 0
