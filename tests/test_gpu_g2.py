"""G2 MSM parity (`-m gpu`): libgzkp.so through the C
ABI vs the oracle's F_p^2 definition, bit-exact.

G2 = the order-r subgroup of the sextic twist E'(F_p^2) (DESIGN.md
reading R14).  The CUDA path is the same Pippenger pipeline instantiated over
the Karatsuba F_p^2 of csrc/field2.cuh; the oracle multiplies schoolbook
(oracle/oracle.c fe_mul, oracle/ref.py Fp2)."""

import random

import numpy as np
import pytest

import oracle
import synth
from oracle import curves, ref
from tests.fixtures import oracle_msm_cached, oracle_points
from tests.gpu_util import dev, host, require_cuda

pytestmark = pytest.mark.gpu

G2 = [curves.BN254_G2, curves.BLS12_381_G2]
NAMES = [c.name for c in G2]


@pytest.fixture(autouse=True)
def _reset_config():
    yield
    try:
        import paper_conf_asplos_maxsm0k0zsh23_b200 as gz
        gz.set_config(0, 0)
    except Exception:
        pass


def _elems(c, vals):
    L = c.limbs
    return np.array([ref.int_to_limbs(v[0], L) + ref.int_to_limbs(v[1], L) for v in vals],
                    dtype=np.uint32).reshape(-1, 2 * L)


def _dec(c, rows):
    L = c.limbs
    return [(ref.limbs_to_int(r[:L]), ref.limbs_to_int(r[L:])) for r in rows]


@pytest.mark.parametrize("c", G2, ids=lambda c: c.name)
def test_fp2_field_ops(c):
    gz = require_cuda()
    F = ref.field(c)
    p = c.p
    rng = random.Random(c.cid)
    edge = [(0, 0), (1, 0), (0, 1), (p - 1, 0), (0, p - 1), (p - 1, p - 1), (1, p - 1), ((p - 1) // 2, (p + 1) // 2)]
    a = edge + [(rng.randrange(p), rng.randrange(p)) for _ in range(6000)]
    b = list(reversed(edge)) + [(rng.randrange(p), rng.randrange(p)) for _ in range(6000)]
    for x in edge:
        for y in edge:
            a.append(x)
            b.append(y)
    A, B = dev(_elems(c, a)), dev(_elems(c, b))
    mul = _dec(c, host(gz.field_op(c.name, 0, A, B)))
    add = _dec(c, host(gz.field_op(c.name, 1, A, B)))
    sub = _dec(c, host(gz.field_op(c.name, 2, A, B)))
    rt = _dec(c, host(gz.field_op(c.name, 4, A, B)))
    sq = _dec(c, host(gz.field_op(c.name, 5, A, B)))
    for i, (x, y) in enumerate(zip(a, b)):
        assert mul[i] == F.mul(x, y), (i, x, y)
        assert add[i] == F.add(x, y)
        assert sub[i] == F.sub(x, y)
        assert rt[i] == x
        assert sq[i] == F.mul(x, x)
    nz = [x for x in a if x != (0, 0)][:2000]
    inv = _dec(c, host(gz.field_op(c.name, 3, dev(_elems(c, nz)), dev(_elems(c, nz)))))
    for x, ix in zip(nz, inv):
        assert ix == F.inv(x)


@pytest.mark.parametrize("c", G2, ids=lambda c: c.name)
def test_g2_group_ops_vs_oracle(c):
    """XYZZ madd / add / dbl / mdbl over F_p^2 against the oracle's affine law,
    including P == Q, P == -Q and O."""
    gz = require_cuda()
    pts, _ = oracle_points(c.name, 64)
    P = [ref.decode_point(c, list(r)) for r in pts]
    rng = random.Random(3)
    A, B = [], []
    for i in range(200):
        x = P[rng.randrange(64)]
        kind = i % 5
        y = x if kind == 0 else (ref.neg(c, x) if kind == 1 else (None if kind == 2 else P[rng.randrange(64)]))
        if i % 17 == 0:
            x = None
        A.append(x)
        B.append(y)
    Al = np.array([ref.encode_point(c, q) for q in A], dtype=np.uint32)
    Bl = np.array([ref.encode_point(c, q) for q in B], dtype=np.uint32)
    for op in range(4):
        got = host(gz.ec_op(c.name, op, dev(Al), dev(Bl)))
        for i in range(len(A)):
            want = ref.add(c, A[i], B[i]) if op in (0, 1) else ref.add(c, A[i], A[i])
            assert ref.decode_point(c, list(got[i])) == want, (op, i)


@pytest.mark.parametrize("name,n", [("bn254_g2", 1), ("bn254_g2", 2), ("bn254_g2", 7), ("bn254_g2", 257),
                                    ("bn254_g2", 1024), ("bls12_381_g2", 1), ("bls12_381_g2", 5),
                                    ("bls12_381_g2", 300), ("bls12_381_g2", 1024)])
def test_g2_msm_uniform_vs_oracle(name, n):
    gz = require_cuda()
    pts, _ = oracle_points(name, max(n, 64))
    pts = pts[:n]
    k = synth.scalars(name, n, 900 + n)
    got = host(gz.msm(name, dev(pts), dev(k)))
    assert np.array_equal(got, oracle_msm_cached(name, pts, k))


@pytest.mark.parametrize("dist", ["zcash_like", "all_one", "r_minus_1", "single_hot", "small", "all_zero"])
@pytest.mark.parametrize("name", NAMES)
def test_g2_msm_distributions(name, dist):
    gz = require_cuda()
    n = 500
    pts, _ = oracle_points(name, 1024)
    pts = pts[:n]
    k = synth.scalars(name, n, 78, dist)
    assert np.array_equal(host(gz.msm(name, dev(pts), dev(k))), oracle_msm_cached(name, pts, k))


@pytest.mark.parametrize("name", NAMES)
def test_g2_identity_duplicates_cancellation(name):
    gz = require_cuda()
    c = curves.get(name)
    pts, _ = oracle_points(name, 256)
    pts = pts.copy()
    n = 256
    k = synth.scalars(name, n, 31)
    pts[3] = 0                                   # identity input points
    pts[40] = 0
    pts[10:20] = pts[9]                          # duplicates (same bucket, P == Q)
    k[10:20] = k[9]
    P51 = ref.decode_point(c, list(pts[51]))
    pts[50] = ref.encode_point(c, ref.neg(c, P51))   # P and -P with equal scalars
    k[50] = k[51]
    assert np.array_equal(host(gz.msm(name, dev(pts), dev(k))), oracle_msm_cached(name, pts, k))
    # a sum that is O: k P + k (-P)
    two = np.stack([pts[51], pts[50]])
    kk = np.stack([k[51], k[51]])
    assert not host(gz.msm(name, dev(two), dev(kk))).any()


@pytest.mark.parametrize("name", NAMES)
def test_g2_window_and_chunk_invariance(name):
    gz = require_cuda()
    pts, _ = oracle_points(name, 512)
    k = synth.scalars(name, 512, 5)
    want = oracle_msm_cached(name, pts, k)
    for wb in (3, 7, 11, 16):
        for chunk in (1, 16, 64):
            gz.set_config(wb, chunk)
            assert np.array_equal(host(gz.msm(name, dev(pts), dev(k))), want), (wb, chunk)


@pytest.mark.parametrize("name", NAMES)
def test_g2_prepared_weighted_and_sharding(name):
    gz = require_cuda()
    pts, _ = oracle_points(name, 700)
    k = synth.scalars(name, 700, 6)
    want = oracle_msm_cached(name, pts, k)
    for weighted, wb in ((True, 0), (True, 9), (False, 0)):
        h = gz.PreparedPoints(name, dev(pts), weighted=weighted, window_bits=wb)
        assert np.array_equal(host(h.msm(dev(k))), want), (weighted, wb)
        assert np.array_equal(h.msm_host(k), want)
        h.release()
    for G in (2, 3, 5):
        parts = []
        for g in range(G):
            lo, hi = gz.shard_range(700, G, g)
            parts.append(gz.msm_partial(name, dev(pts[lo:hi]), dev(k[lo:hi])))
        import torch
        assert np.array_equal(host(gz.combine_partials(name, torch.stack(parts))), want), G
    assert np.array_equal(gz.msm_host(name, pts, k), want)


@pytest.mark.parametrize("name", NAMES)
def test_g2_fixed_base_vs_oracle(name):
    gz = require_cuda()
    c = curves.get(name)
    d = synth.dlogs(name, 300, 4242)
    got = host(gz.fixed_base_mul(name, dev(d)))
    want = oracle.points_from_dlogs(c, d)
    assert np.array_equal(got, want)


@pytest.mark.parametrize("name,logn", [("bn254_g2", 18), ("bls12_381_g2", 17),
                                       # the benched G2 workloads (bench.py *_g2_2p20, planner c = 16)
                                       ("bn254_g2", 20), ("bls12_381_g2", 20)])
def test_g2_large_closed_form(name, logn):
    """Larger n: device-generated points a_i G2 (a 16-point sample re-derived by
    the oracle), MSM checked against the oracle's closed form
    (sum k_i a_i mod r) G2, for the standard and the weighted-point paths."""
    gz = require_cuda()
    c = curves.get(name)
    n = 1 << logn
    d = synth.dlogs(name, n, synth.dlog_seed(name))
    k = synth.scalars(name, n, synth.scalar_seed(20 + logn))
    D = dev(d)
    P = gz.fixed_base_mul(name, D)
    sample = np.random.Generator(np.random.PCG64(1)).choice(n, 16, replace=False)
    assert np.array_equal(host(P)[sample], oracle.points_from_dlogs(c, d[sample]))
    want = oracle.closed_form(c, k, d)
    gz.set_profiling(True)
    gz.profile_read(reset=True)
    assert np.array_equal(host(gz.msm(name, P, dev(k))), want)
    prof = gz.profile_read(reset=True)
    gz.set_profiling(False)
    assert prof["c"] == gz.window_bits(name, n)
    h = gz.PreparedPoints(name, P, weighted=True)
    assert np.array_equal(host(h.msm(dev(k))), want)
    h.release()
