"""Seeded synthetic inputs for the G1 MSM (shared by tests, smoke and bench).

This module holds NO part of the method's arithmetic: it only draws random
integers (scalars k_i and discrete logs a_i) from numpy's PCG64 and encodes
them as little-endian u32 limbs.  Turning a_i into points a_i * G is done by the
consumer: the oracle for the parity tests, the product's fixed-base kernel for
the benchmark.

Recipe:
  * seeds: scalars 1000 + config, discrete logs 2000 + curve id;
  * ``uniform``: uniform in [0, r) by rejection sampling b-bit integers
    (reading R4: "uniform 254/381/753-bit scalars" = uniform mod r);
  * ``zcash_like``: the sparse witness of PAPER.md:243-245 ("many 0s and 1s"):
    0 w.p. 0.50, 1 w.p. 0.40, uniform [2, 2^64) w.p. 0.05, uniform [0, r)
    w.p. 0.05 (reading R9);
  * adversarial presets for the edge-case tests.
"""

from __future__ import annotations

import numpy as np

# (scalar bits b, group order r) -- this module's own copy; only the range of
# the random draws depends on them.
ORDERS = {
    "bn254": (254, int("30644e72e131a029b85045b68181585d2833e84879b9709143e1f593f0000001", 16)),
    "bls12_381": (255, int("73eda753299d7d483339d80809a1d80553bda402fffe5bfeffffffff00000001", 16)),
    "mnt4_753": (753, int("1c4c62d92c41110229022eee2cdadb7f997505b8fafed5eb7e8f96c97d87307fdb925e8a0ed8d99d124d9a15af79db26c5c28c859a99b3eebca9429212636b9dff97634993aa4d6c381bc3f0057974ea099170fa13a4fd90776e240000001", 16)),
    "toy_a0": (14, 9967),
    "toy_a2": (14, 10091),
}
ORDERS["bn254_g2"] = ORDERS["bn254"]            # G2 shares r with G1
ORDERS["bls12_381_g2"] = ORDERS["bls12_381"]
CURVE_IDS = {"bn254": 0, "bls12_381": 1, "mnt4_753": 2, "toy_a0": 100, "toy_a2": 101,
             "bn254_g2": 3, "bls12_381_g2": 4}
NAMES = {v: k for k, v in CURVE_IDS.items()}

DISTS = ("uniform", "zcash_like", "full_bits", "all_zero", "all_one", "r_minus_1",
         "single_hot", "pow2", "small")


def _name(curve) -> str:
    if isinstance(curve, int):
        return NAMES[curve]
    return getattr(curve, "name", curve)


def scalar_limbs(curve) -> int:
    return (ORDERS[_name(curve)][0] + 31) // 32


def _int_to_limbs(v: int, n: int) -> np.ndarray:
    return np.array([(v >> (32 * i)) & 0xFFFFFFFF for i in range(n)], dtype=np.uint32)


def _ge(x: np.ndarray, bound: np.ndarray) -> np.ndarray:
    """Row-wise x >= bound for little-endian limb rows."""
    n, L = x.shape
    res = np.ones(n, dtype=bool)       # equal so far => >=
    decided = np.zeros(n, dtype=bool)
    for i in range(L - 1, -1, -1):
        gt = x[:, i] > bound[i]
        lt = x[:, i] < bound[i]
        res = np.where(~decided & gt, True, res)
        res = np.where(~decided & lt, False, res)
        decided |= gt | lt
    return res


def _uniform_below(rng: np.random.Generator, n: int, bits: int, bound: int) -> np.ndarray:
    """n integers uniform in [0, bound), bound <= 2^bits, as [n, ceil(bits/32)] u32."""
    L = (bits + 31) // 32
    top_mask = np.uint32((1 << (bits - 32 * (L - 1))) - 1) if bits % 32 else np.uint32(0xFFFFFFFF)
    bnd = _int_to_limbs(bound, L)
    out = np.empty((n, L), dtype=np.uint32)
    todo = np.arange(n)
    while todo.size:
        draw = rng.integers(0, 1 << 32, size=(todo.size, L), dtype=np.uint64).astype(np.uint32)
        draw[:, L - 1] &= top_mask
        ok = ~_ge(draw, bnd)
        out[todo[ok]] = draw[ok]
        todo = todo[~ok]
    return out


def scalars(curve, n: int, seed: int, dist: str = "uniform", c: int = 16) -> np.ndarray:
    """[n, Ls] u32 little-endian scalars."""
    name = _name(curve)
    bits, r = ORDERS[name]
    L = (bits + 31) // 32
    rng = np.random.Generator(np.random.PCG64(seed))
    if dist == "uniform":
        return _uniform_below(rng, n, bits, r)
    if dist == "full_bits":                       # any integer < 2^b (ABI allows it)
        return _uniform_below(rng, n, bits, 1 << bits)
    if dist == "zcash_like":
        u = rng.random(n)
        out = np.zeros((n, L), dtype=np.uint32)
        one = (u >= 0.50) & (u < 0.90)
        small = (u >= 0.90) & (u < 0.95)
        big = u >= 0.95
        out[one, 0] = 1
        ns = int(small.sum())
        if ns:
            hi = 1 << min(64, bits)
            v = rng.integers(2, hi, size=ns, dtype=np.uint64)
            out[small, 0] = (v & np.uint64(0xFFFFFFFF)).astype(np.uint32)
            if L > 1:
                out[small, 1] = (v >> np.uint64(32)).astype(np.uint32)
        nb = int(big.sum())
        if nb:
            out[big] = _uniform_below(rng, nb, bits, r)
        return out
    if dist == "all_zero":
        return np.zeros((n, L), dtype=np.uint32)
    if dist == "all_one":
        out = np.zeros((n, L), dtype=np.uint32)
        out[:, 0] = 1
        return out
    if dist == "r_minus_1":
        return np.tile(_int_to_limbs(r - 1, L), (n, 1))
    if dist == "single_hot":                      # one nonzero scalar
        out = np.zeros((n, L), dtype=np.uint32)
        if n:
            out[int(rng.integers(0, n))] = _uniform_below(rng, 1, bits, r)[0]
        return out
    if dist == "pow2":                            # random powers of two, incl. 2^(b-1)
        e = rng.integers(0, bits, size=n)
        out = np.zeros((n, L), dtype=np.uint32)
        out[np.arange(n), e // 32] = (np.uint32(1) << (e % 32).astype(np.uint32))
        return out
    if dist == "small":                           # digits that hit +-2^(c-1) and carries
        vals = rng.choice(np.array([1, 2, (1 << (c - 1)) - 1, 1 << (c - 1), (1 << (c - 1)) + 1,
                                    (1 << c) - 1, 1 << c], dtype=np.uint64), size=n)
        out = np.zeros((n, L), dtype=np.uint32)
        out[:, 0] = (vals & 0xFFFFFFFF).astype(np.uint32)
        if L > 1:
            out[:, 1] = (vals >> np.uint64(32)).astype(np.uint32)
        return out
    raise ValueError(f"unknown distribution {dist!r}")


def dlogs(curve, n: int, seed: int) -> np.ndarray:
    """Discrete logs a_i uniform in [1, r) as [n, Ls] u32 (points are a_i * G)."""
    name = _name(curve)
    bits, r = ORDERS[name]
    rng = np.random.Generator(np.random.PCG64(seed))
    out = _uniform_below(rng, n, bits, r - 1)
    # shift [0, r-1) -> [1, r): add one with carry
    carry = np.ones(n, dtype=np.uint64)
    for i in range(out.shape[1]):
        s = out[:, i].astype(np.uint64) + carry
        out[:, i] = (s & 0xFFFFFFFF).astype(np.uint32)
        carry = s >> np.uint64(32)
    return out


def scalar_seed(config: int) -> int:
    return 1000 + config


def dlog_seed(curve) -> int:
    return 2000 + {"bn254": 0, "bls12_381": 1, "mnt4_753": 2, "toy_a0": 3, "toy_a2": 4,
                   "bn254_g2": 5, "bls12_381_g2": 6}[_name(curve)]
