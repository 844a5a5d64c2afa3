"""Curve parameters for the ORACLE ONLY (test infrastructure).

This file is the oracle's own copy of the curve constants, written as hex
strings.  The CUDA product path keeps its own, separately generated copy
(`paper_conf_asplos_maxsm0k0zsh23_b200/csrc/curves.cuh`); the two share no code.

The paper names the curves only ("ALT-BN128, BLS12-381, MNT4753",
PAPER.md:279-287 §5.1, Table 1) and defines the point set
{(x, y) in F_q x F_q | y^2 = x^3 + a x + b} (§2.1).  The numeric
parameters are the published standard ones (reading R1); each one is
pinned in tests/test_oracle_pins.py by primality, the curve equation and the
group order, not by trusting this file.

Toy curves (test builds only): small prime-order curves on which
random buckets constantly hit the P == Q and P == -Q cases, so the group law
can be brute-forced.
"""

from dataclasses import dataclass


@dataclass(frozen=True)
class Curve:
    name: str
    cid: int          # id shared with the C ABI enum (gzkp_curve)
    p: int            # base field modulus q (PAPER.md:106 calls it F_q)
    r: int            # order of the G1 group = scalar field modulus (PAPER.md:105 F_r)
    a: object         # int for G1; (c0, c1) in F_p^2 for G2
    b: object
    gx: object
    gy: object
    cofactor: int     # #E(F_p) / r   (G2: #E'(F_p^2) / r)
    scalar_bits: int  # b = bit length of r: scalars are integers < 2^scalar_bits
    deg: int = 1      # 1: G1 over F_p; 2: G2 over F_p^2 = F_p[u]/(u^2 - beta)
    beta: int = 0     # deg 2 only

    @property
    def coord_limbs(self) -> int:
        """u32 limbs of one curve coordinate (deg F_p coordinates c0 || c1)."""
        return self.deg * self.limbs

    @property
    def limbs(self) -> int:
        """u32 limbs of one base-field coordinate in the ABI encoding
        (ceil(bits/32) rounded up to even: 8 / 12 / 24, and 2 for the toys)."""
        n = (self.p.bit_length() + 31) // 32
        return n + (n & 1)

    @property
    def scalar_limbs(self) -> int:
        return (self.scalar_bits + 31) // 32


def _h(s: str) -> int:
    return int(s, 16)


BN254 = Curve(
    name="bn254", cid=0,
    p=_h("30644e72e131a029b85045b68181585d97816a916871ca8d3c208c16d87cfd47"),
    r=_h("30644e72e131a029b85045b68181585d2833e84879b9709143e1f593f0000001"),
    a=0, b=3, gx=1, gy=2, cofactor=1, scalar_bits=254,
)

BLS12_381 = Curve(
    name="bls12_381", cid=1,
    p=_h("1a0111ea397fe69a4b1ba7b6434bacd764774b84f38512bf6730d2a0f6b0f6241eabfffeb153ffffb9feffffffffaaab"),
    r=_h("73eda753299d7d483339d80809a1d80553bda402fffe5bfeffffffff00000001"),
    a=0, b=4,
    gx=_h("17f1d3a73197d7942695638c4fa9ac0fc3688c4f9774b905a14e3a3f171bac586c55e83ff97a1aeffb3af00adb22c6bb"),
    gy=_h("08b3f481e3aaa0f1a09e30ed741d8ae4fcf5e095d5d00af600db18cb2c04b3edd03cc744a2888ae40caa232946c5e7e1"),
    cofactor=_h("396c8c005555e1568c00aaab0000aaab"), scalar_bits=255,
)

# MNT4-753 G1: a = 2, cofactor 1.  The libff generator could not be verified
# offline, so G = (1, y) with y the smaller square root of 1 + 2 + b
# (reading R2).  With cofactor 1 and r prime, any
# non-identity point generates the group (pinned: r*G = O in the tests).
MNT4_753 = Curve(
    name="mnt4_753", cid=2,
    p=_h("1c4c62d92c41110229022eee2cdadb7f997505b8fafed5eb7e8f96c97d87307fdb925e8a0ed8d99d124d9a15af79db117e776f218059db80f0da5cb537e38685acce9767254a4638810719ac425f0e39d54522cdd119f5e9063de245e8001"),
    r=_h("1c4c62d92c41110229022eee2cdadb7f997505b8fafed5eb7e8f96c97d87307fdb925e8a0ed8d99d124d9a15af79db26c5c28c859a99b3eebca9429212636b9dff97634993aa4d6c381bc3f0057974ea099170fa13a4fd90776e240000001"),
    a=2,
    b=_h("1373684a8c9dcae7a016ac5d7748d3313cd8e39051c596560835df0c9e50a5b59b882a92c78dc537e51a16703ec9855c77fc3d8bb21c8d68bb8cfb9db4b8c8fba773111c36c8b1b4e8f1ece940ef9eaad265458e06372009c9a0491678ef4"),
    gx=1,
    gy=_h("7b753d99cf6f828729cd4e81339b83589f644376b25812761ca069cc1aaff44973d9f1751bee9fab5b8ec89845d948e3f9854059d4a6049cb8e9039c96f7fa2fdf50d0add627081b1c88bddc1166e34ce99bfbcc08a2d39f3788b4f54125"),
    cofactor=1, scalar_bits=753,
)

# Toy prime-order curves (SURVEY.md §4 "Toy curve").  Generators are the
# smallest-x point with the smaller y; the tests enumerate the whole group.
TOY_A0 = Curve(name="toy_a0", cid=100, p=10099, r=9967, a=0, b=3,
               gx=0, gy=0, cofactor=1, scalar_bits=14)
TOY_A2 = Curve(name="toy_a2", cid=101, p=10007, r=10091, a=2, b=30,
               gx=0, gy=0, cofactor=1, scalar_bits=14)


def _toy_generator(c: Curve) -> Curve:
    # smallest x with x^3+ax+b a nonzero square; y = smaller root (brute force,
    # the field has ~10^4 elements).
    for x in range(c.p):
        rhs = (x * x * x + c.a * x + c.b) % c.p
        if rhs == 0:
            continue
        for y in range(1, (c.p + 1) // 2):
            if y * y % c.p == rhs:
                return Curve(**{**c.__dict__, "gx": x, "gy": y})
    raise ValueError("no point")


TOY_A0 = _toy_generator(TOY_A0)
TOY_A2 = _toy_generator(TOY_A2)

# ---- G2 (GZKP's MSM optimisations "apply to both G1 and G2";
# Groth16's B-query lives in G2).  G2 is the order-r subgroup of a sextic twist
# E'(F_p^2): y^2 = x^3 + b' over F_p^2 = F_p[u]/(u^2 + 1) (DESIGN.md reading
# R14).  b' and the generators are the standard published values (EIP-197 for
# BN254; the IETF pairing-friendly-curves draft / zkcrypto for BLS12-381);
# tests/test_oracle_pins.py pins them: b'(9 + u) = 3 resp. b' = 4(1 + u),
# G2 on E', r G2 = O, G2 != O.
BN254_G2 = Curve(
    name="bn254_g2", cid=3, p=BN254.p, r=BN254.r, a=(0, 0),
    b=(_h("2b149d40ceb8aaae81be18991be06ac3b5b4c5e559dbefa33267e6dc24a138e5"),
       _h("009713b03af0fed4cd2cafadeed8fdf4a74fa084e52d1852e4a2bd0685c315d2")),
    gx=(10857046999023057135944570762232829481370756359578518086990519993285655852781,
        11559732032986387107991004021392285783925812861821192530917403151452391805634),
    gy=(8495653923123431417604973247489272438418190587263600148770280649306958101930,
        4082367875863433681332203403145435568316851327593401208105741076214120093531),
    cofactor=2 * BN254.p - BN254.r, scalar_bits=254, deg=2, beta=BN254.p - 1,
)

BLS12_381_G2 = Curve(
    name="bls12_381_g2", cid=4, p=BLS12_381.p, r=BLS12_381.r, a=(0, 0), b=(4, 4),
    gx=(_h("024aa2b2f08f0a91260805272dc51051c6e47ad4fa403b02b4510b647ae3d1770bac0326a805bbefd48056c8c121bdb8"),
        _h("13e02b6052719f607dacd3a088274f65596bd0d09920b61ab5da61bbdc7f5049334cf11213945d57e5ac7d055d042b7e")),
    gy=(_h("0ce5d527727d6e118cc9cdc6da2e351aadfd9baa8cbdd3a76d429a695160d12c923ac9cc3baca289e193548608b82801"),
        _h("0606c4a02ea734cc32acd2b02bc28b99cb3e287e85a763af267492ab572e99ab3f370d275cec1da1aaa9075ff05f79be")),
    cofactor=_h("5d543a95414e7f1091d50792876a202cd91de4547085abaa68a205b2e5a7ddfa628f1cb4d9e82ef21537e293a6691ae1616ec6e786f0c70cf1c38e31c7238e5"),
    scalar_bits=255, deg=2, beta=BLS12_381.p - 1,
)

CURVES = {c.name: c for c in (BN254, BLS12_381, MNT4_753, TOY_A0, TOY_A2, BN254_G2, BLS12_381_G2)}
BY_ID = {c.cid: c for c in CURVES.values()}


def get(curve) -> Curve:
    if isinstance(curve, Curve):
        return curve
    if isinstance(curve, int):
        return BY_ID[curve]
    return CURVES[curve]
