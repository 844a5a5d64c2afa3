"""Pins for the NTT oracle (`-m "not gpu"`).

The oracle evaluates a_k = A(w_N^k) (§2.2) by Horner's rule.
Nothing here retypes that formula; each plausible mistake fails a test:
  * w_N not a primitive N-th root (wrong exponent, wrong g)  -> w^N = 1, w^(N/2) = -1
  * wrong evaluation order / index (A_i w^(ik) vs w^(-ik))   -> convolution theorem,
      delta and constant inputs, the closed form of a geometric series
  * wrong inverse scaling                                    -> INTT(NTT(A)) = A
  * C Horner (threaded) vs Python Horner                     -> equality on random inputs
"""

import random

import numpy as np
import pytest

import oracle
import synth
from oracle import curves, ntt, ref

FIELDS = [curves.BN254, curves.BLS12_381, curves.MNT4_753]


@pytest.mark.parametrize("c", FIELDS, ids=lambda c: c.name)
def test_root_of_unity_primitive(c):
    s = ntt.two_adicity(c.r)
    assert (c.r - 1) % (1 << s) == 0 and ((c.r - 1) >> s) & 1
    g = ntt.smallest_non_residue(c.r)
    assert pow(g, (c.r - 1) // 2, c.r) == c.r - 1          # Euler's criterion: a non-residue
    for log_n in (0, 1, 2, 5, 10, s):
        w = ntt.root_of_unity(c, log_n)
        n = 1 << log_n
        assert pow(w, n, c.r) == 1
        if log_n:
            assert pow(w, n // 2, c.r) == c.r - 1          # order exactly N
    with pytest.raises(ValueError):
        ntt.root_of_unity(c, s + 1)


def _cyclic_convolution(a, b, r):
    n = len(a)
    out = [0] * n
    for i in range(n):
        for j in range(n):
            out[(i + j) % n] = (out[(i + j) % n] + a[i] * b[j]) % r
    return out


@pytest.mark.parametrize("c", FIELDS, ids=lambda c: c.name)
@pytest.mark.parametrize("n", [1, 2, 8, 32])
def test_convolution_theorem(c, n):
    rng = random.Random(n)
    a = [rng.randrange(c.r) for _ in range(n)]
    b = [rng.randrange(c.r) for _ in range(n)]
    fa, fb = ntt.ntt(c, a), ntt.ntt(c, b)
    prod = [x * y % c.r for x, y in zip(fa, fb)]
    assert ntt.ntt(c, prod, inverse=True) == _cyclic_convolution(a, b, c.r)


@pytest.mark.parametrize("c", FIELDS, ids=lambda c: c.name)
def test_delta_constant_geometric(c):
    n = 16
    r = c.r
    w = ntt.root_of_unity(c, 4)
    # constant polynomial 1 -> all ones; delta at 0 (A = 1) and sum of all x^i
    assert ntt.ntt(c, [1] + [0] * (n - 1)) == [1] * n
    assert ntt.ntt(c, [1] * n) == [n % r] + [0] * (n - 1)      # geometric series vanishes off k = 0
    # x^j -> w^(jk)
    for j in (1, 3, 15):
        e = [0] * n
        e[j] = 1
        assert ntt.ntt(c, e) == [pow(w, j * k, r) for k in range(n)]


@pytest.mark.parametrize("c", FIELDS, ids=lambda c: c.name)
def test_inverse_round_trip(c):
    rng = random.Random(2)
    for n in (1, 4, 64):
        a = [rng.randrange(c.r) for _ in range(n)]
        assert ntt.ntt(c, ntt.ntt(c, a), inverse=True) == a
        assert ntt.ntt(c, ntt.ntt(c, a, inverse=True)) == a


@pytest.mark.parametrize("c", FIELDS, ids=lambda c: c.name)
def test_c_horner_equals_python(c):
    n = 200
    k = synth.scalars(c.name, n, 12)
    A = [ref.limbs_to_int(row) for row in k]
    rng = random.Random(4)
    xs = [0, 1, c.r - 1] + [rng.randrange(c.r) for _ in range(20)]
    assert oracle.poly_eval(c, k, xs, nthreads=3) == [ntt.horner(A, x, c.r) for x in xs]
