"""NTT parity (`-m gpu`): libgzkp.so's gzkp_ntt through
the C ABI against the oracle's definition a_k = A(w_N^k),
bit-exact (integer results, no tolerance).

Small N: the full oracle transform (Horner per output, oracle/ntt.py).
Multi-pass and large N: sampled outputs a_k computed one by one by the C
oracle's Horner evaluation (oracle.poly_eval), plus the round trip
INTT(NTT(A)) = A on the device.  Edge inputs: zeros, r - 1 everywhere, a delta,
in-place transforms."""

import random

import numpy as np
import pytest

import oracle
import synth
from oracle import curves, ntt, ref
from tests.gpu_util import dev, host, require_cuda

pytestmark = pytest.mark.gpu

FIELDS = ["bn254", "bls12_381", "mnt4_753"]


def _ints(rows):
    return [ref.limbs_to_int(r) for r in rows]


def _limbs(vals, Ls):
    return np.array([ref.int_to_limbs(v, Ls) for v in vals], dtype=np.uint32).reshape(-1, Ls)


@pytest.mark.parametrize("name", FIELDS)
def test_scalar_field_ops(name):
    gz = require_cuda()
    c = curves.get(name)
    r, Ls = c.r, c.scalar_limbs
    rng = random.Random(5)
    R = 1 << (32 * Ls)
    edge = [0, 1, 2, r - 1, r - 2, (r - 1) // 2, (r + 1) // 2, R % r, (R - 1) % r]
    a = edge + [rng.randrange(r) for _ in range(8000)]
    b = list(reversed(edge)) + [rng.randrange(r) for _ in range(8000)]
    for x in edge:
        for y in edge:
            a.append(x)
            b.append(y)
    A, B = dev(_limbs(a, Ls)), dev(_limbs(b, Ls))
    out = {op: _ints(host(gz.scalar_field_op(name, op, A, B))) for op in (0, 1, 2, 4, 5)}
    for i, (x, y) in enumerate(zip(a, b)):
        assert out[0][i] == x * y % r
        assert out[1][i] == (x + y) % r
        assert out[2][i] == (x - y) % r
        assert out[4][i] == x
        assert out[5][i] == x * x % r
    nz = [x for x in a if x][:3000]
    inv = _ints(host(gz.scalar_field_op(name, 3, dev(_limbs(nz, Ls)), dev(_limbs(nz, Ls)))))
    assert inv == [pow(x, -1, r) for x in nz]


@pytest.mark.parametrize("name", FIELDS)
@pytest.mark.parametrize("log_n", [0, 1, 2, 3, 5, 8, 10])
def test_ntt_small_full_oracle(name, log_n):
    gz = require_cuda()
    c = curves.get(name)
    n = 1 << log_n
    if c.scalar_limbs > 8 and log_n > 8:
        log_n, n = 8, 256
    k = synth.scalars(name, n, 40 + log_n)
    A = _ints(k)
    fwd = _ints(host(gz.ntt(name, dev(k))))
    assert fwd == ntt.ntt(c, A)
    inv = _ints(host(gz.ntt(name, dev(k), inverse=True)))
    assert inv == ntt.ntt(c, A, inverse=True)


def _sampled_check(gz, name, log_n, seed, samples=24, dist="uniform"):
    c = curves.get(name)
    n = 1 << log_n
    k = synth.scalars(name, n, seed, dist)
    D = dev(k)
    out = host(gz.ntt(name, D))
    w = ntt.root_of_unity(c, log_n)
    rng = np.random.Generator(np.random.PCG64(seed))
    idx = sorted(set([0, 1, n // 2, n - 1] + list(rng.choice(n, samples, replace=False))))
    want = oracle.poly_eval(c, k, [pow(w, int(j), c.r) for j in idx])
    assert _ints(out[idx]) == want, name
    back = host(gz.ntt(name, dev(out), inverse=True))
    assert np.array_equal(back, k)
    return k, out


@pytest.mark.parametrize("name,log_n", [("bn254", 11), ("bn254", 12), ("bn254", 17), ("bn254", 19),
                                        ("bls12_381", 13), ("bls12_381", 18), ("bls12_381", 20),
                                        ("mnt4_753", 9), ("mnt4_753", 12), ("mnt4_753", 17)])
def test_ntt_multipass_sampled(name, log_n):
    gz = require_cuda()
    _sampled_check(gz, name, log_n, 300 + log_n)


@pytest.mark.parametrize("name", ["bn254", "bls12_381", "mnt4_753"])
def test_ntt_edge_inputs(name):
    gz = require_cuda()
    c = curves.get(name)
    Ls = c.scalar_limbs
    for log_n in (4, 14):
        n = 1 << log_n
        z = np.zeros((n, Ls), dtype=np.uint32)
        assert not host(gz.ntt(name, dev(z))).any()
        m1 = _limbs([c.r - 1] * n, Ls)                   # -1 everywhere: a_0 = -N, rest 0
        got = _ints(host(gz.ntt(name, dev(m1))))
        assert got[0] == (-n) % c.r and not any(got[1:])
        delta = np.zeros((n, Ls), dtype=np.uint32)
        delta[1, 0] = 1                                   # A(x) = x: a_k = w^k
        w = ntt.root_of_unity(c, log_n)
        got = _ints(host(gz.ntt(name, dev(delta))))
        assert got[:64] == [pow(w, j, c.r) for j in range(min(n, 64))]
        assert got[-1] == pow(w, n - 1, c.r)


@pytest.mark.parametrize("name", ["bn254", "mnt4_753"])
def test_ntt_in_place(name):
    gz = require_cuda()
    for log_n in (6, 15):
        n = 1 << log_n
        k = synth.scalars(name, n, 9)
        D = dev(k)
        want = host(gz.ntt(name, D))
        gz.ntt(name, D, out=D)                            # in == out
        assert np.array_equal(host(D), want)
        gz.ntt(name, D, inverse=True, out=D)
        assert np.array_equal(host(D), k)


def test_ntt_bench_size_sampled():
    """BLS12-381 F_r at the bench size 2^24, the launch configuration bench.py
    times: 16 outputs re-derived by the oracle (Horner over all 2^24
    coefficients), plus the device round trip."""
    gz = require_cuda()
    _sampled_check(gz, "bls12_381", 24, 24, samples=12)


def test_ntt_errors():
    gz = require_cuda()
    with pytest.raises(gz.GzkpError):
        gz.lib()
        k = dev(np.zeros((3, 8), dtype=np.uint32))
        gz.ntt("bn254", k)
    assert gz.ntt_max_log("bn254") == 28 and gz.ntt_max_log("bls12_381") == 30
    assert gz.ntt_max_log("mnt4_753") == 30 and gz.ntt_max_log("toy_a0") == -1
