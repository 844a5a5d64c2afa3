"""GPU field and group-law parity (`-m gpu`).

Field: the CUDA Montgomery/EEA kernels vs Python integers (the textbook
definition a*b mod p, a^-1 mod p) on random and edge values.
Group law: the XYZZ madd / add / dbl / mdbl kernels (projective inputs, not
just Z = 1) vs the oracle's affine chord-and-tangent law, including the
exceptional cases P == Q, P == -Q and O."""

import random

import numpy as np
import pytest

from oracle import curves, ref
from tests.gpu_util import dev, host, int_limbs, limbs_int, require_cuda

pytestmark = pytest.mark.gpu
ALL = [curves.BN254, curves.BLS12_381, curves.MNT4_753, curves.TOY_A0, curves.TOY_A2]


def _edge_values(c):
    L = c.limbs
    R = 1 << (32 * L)
    e = [0, 1, 2, 3, c.p - 1, c.p - 2, (c.p - 1) // 2, (c.p + 1) // 2, R % c.p, (R - 1) % c.p,
         (1 << (c.p.bit_length() - 1)) % c.p, pow(R, -1, c.p), pow(R, 2, c.p)]
    return [v % c.p for v in e]


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_field_ops(c):
    gz = require_cuda()
    rng = random.Random(c.cid * 7 + 1)
    L = c.limbs
    edge = _edge_values(c)
    n = 20000 if c.limbs <= 12 else 4000
    a = edge + [rng.randrange(c.p) for _ in range(n)]
    b = list(reversed(edge)) + [rng.randrange(c.p) for _ in range(n)]
    # all edge x edge pairs too
    for x in edge:
        for y in edge:
            a.append(x)
            b.append(y)
    A, B = dev(int_limbs(a, L)), dev(int_limbs(b, L))
    mul = host(gz.field_op(c.name, 0, A, B))
    add = host(gz.field_op(c.name, 1, A, B))
    sub = host(gz.field_op(c.name, 2, A, B))
    rt = host(gz.field_op(c.name, 4, A, B))
    sq = host(gz.field_op(c.name, 5, A, B))
    dfp = host(gz.field_op(c.name, 6, A, B))       # FP64 (DFP) product where available
    coop = host(gz.field_op(c.name, 8, A, B))      # lane-split product (8 lanes per product)
    for i in range(len(a)):
        assert limbs_int(sq[i]) == a[i] * a[i] % c.p, (i, a[i])
        assert limbs_int(dfp[i]) == a[i] * b[i] % c.p, ("dfp", i, a[i], b[i])
        assert limbs_int(mul[i]) == a[i] * b[i] % c.p, (i, a[i], b[i])
        assert limbs_int(coop[i]) == a[i] * b[i] % c.p, ("coop", i, a[i], b[i])
        assert limbs_int(add[i]) == (a[i] + b[i]) % c.p, i
        assert limbs_int(sub[i]) == (a[i] - b[i]) % c.p, i
        assert limbs_int(rt[i]) == a[i], i
    nz = [x for x in a if x][:3000]
    inv = host(gz.field_op(c.name, 3, dev(int_limbs(nz, L)), dev(int_limbs(nz, L))))
    bg = host(gz.field_op(c.name, 7, dev(int_limbs(nz, L)), dev(int_limbs(nz, L))))   # binary-GCD inverse
    for i, x in enumerate(nz):
        assert limbs_int(inv[i]) == pow(x, -1, c.p), (i, x)
        assert limbs_int(bg[i]) == pow(x, -1, c.p), ("bingcd", i, x)
    assert not host(gz.field_op(c.name, 7, dev(int_limbs([0], L)), dev(int_limbs([0], L)))).any()


@pytest.mark.parametrize("c", [curves.BN254, curves.BLS12_381, curves.MNT4_753], ids=lambda c: c.name)
def test_bingcd_inverse_stress(c):
    """The constant-time binary-GCD inverse (Pornin's bound of
    ceil((2 len p - 1) / 31) outer iterations) on many random values and on
    values with long runs of zero / one bits: x x^-1 = 1 (mod p)."""
    gz = require_cuda()
    rng = random.Random(99 + c.cid)
    L = c.limbs
    n = 1 << (17 if L <= 12 else 14)
    xs = [rng.randrange(1, c.p) for _ in range(n)]
    xs += [(1 << k) % c.p for k in range(c.p.bit_length())]
    xs += [((1 << k) - 1) % c.p or 1 for k in range(1, c.p.bit_length())]
    xs += [c.p - (1 << k) for k in range(c.p.bit_length() - 1)]
    X = dev(int_limbs(xs, L))
    got = host(gz.field_op(c.name, 7, X, X))
    for i, x in enumerate(xs):
        assert limbs_int(got[i]) * x % c.p == 1, (i, x)


def _points(c, k, seed):
    rng = random.Random(seed)
    G = ref.generator(c)
    return [ref.mul(c, rng.randrange(1, c.r), G) for _ in range(k)]


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_group_ops(c):
    gz = require_cuda()
    k = 24 if c is curves.MNT4_753 else 64
    P = _points(c, k, 1)
    Q = _points(c, k, 2)
    # exceptional pairs: P == Q, P == -Q, O on either side
    P += [P[0], P[1], None, P[2], None]
    Q += [P[0], ref.neg(c, P[1]), Q[0], None, None]
    enc = lambda pts: np.array([ref.encode_point(c, x) for x in pts], dtype=np.uint32)
    dP, dQ = dev(enc(P)), dev(enc(Q))
    madd = host(gz.ec_op(c.name, 0, dP, dQ))
    add = host(gz.ec_op(c.name, 1, dP, dQ))
    dbl = host(gz.ec_op(c.name, 2, dP, dQ))
    mdbl = host(gz.ec_op(c.name, 3, dP, dQ))
    for i in range(len(P)):
        want = ref.add(c, P[i], Q[i])
        assert ref.decode_point(c, madd[i]) == want, ("madd", i)
        assert ref.decode_point(c, add[i]) == want, ("add", i)
        d = ref.add(c, P[i], P[i])
        assert ref.decode_point(c, dbl[i]) == d, ("dbl", i)
        assert ref.decode_point(c, mdbl[i]) == d, ("mdbl", i)


@pytest.mark.parametrize("c", ALL, ids=lambda c: c.name)
def test_fixed_base_generator_matches_oracle(c):
    gz = require_cuda()
    import oracle
    import synth
    d = synth.dlogs(c.name, 40 if c is curves.MNT4_753 else 200, 99)
    d[0] = 0
    d[1, :] = 0
    d[1, 0] = 1
    got = host(gz.fixed_base_mul(c.name, dev(d)))
    want = oracle.points_from_dlogs(c.name, d)
    assert np.array_equal(got, want)
