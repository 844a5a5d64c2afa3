"""Seeded input generators: range, determinism, and the sparse preset's shape."""

import numpy as np
import pytest

import synth
from oracle import curves, ref


@pytest.mark.parametrize("name", ["bn254", "bls12_381", "mnt4_753", "toy_a0"])
def test_uniform_below_r_and_deterministic(name):
    c = curves.get(name)
    k = synth.scalars(name, 2000, 1)
    assert k.shape == (2000, c.scalar_limbs) and k.dtype == np.uint32
    assert np.array_equal(k, synth.scalars(name, 2000, 1))
    vals = [ref.limbs_to_int(row) for row in k[:300]]
    assert all(0 <= v < c.r for v in vals)
    assert max(vals).bit_length() == c.r.bit_length()      # top bits are exercised
    d = synth.dlogs(name, 500, 2)
    dv = [ref.limbs_to_int(row) for row in d]
    assert all(1 <= v < c.r for v in dv)


def test_zcash_like_fractions():
    k = synth.scalars("bls12_381", 100000, 5, "zcash_like")
    v0 = k[:, 0].astype(np.uint64)
    rest = k[:, 1:].any(axis=1)
    zero = (v0 == 0) & ~rest
    one = (v0 == 1) & ~rest
    assert abs(zero.mean() - 0.50) < 0.01
    assert abs(one.mean() - 0.40) < 0.01
    big = k[:, 2:].any(axis=1)
    assert abs(big.mean() - 0.05) < 0.005


def test_presets():
    n = 50
    for dist in synth.DISTS:
        k = synth.scalars("bn254", n, 3, dist)
        assert k.shape == (n, 8)
    assert synth.scalars("bn254", n, 3, "all_zero").sum() == 0
    r1 = synth.scalars("bn254", 2, 3, "r_minus_1")
    assert ref.limbs_to_int(r1[0]) == curves.BN254.r - 1
