"""Exact emulation of the FP64 ("DFP", §4.3) Montgomery
multiplication used by csrc/field_dfp.cuh.  Development aid, NOT the oracle.

Limbs: beta = 2^48, L = 2N/3 limbs (N u32 limbs -> 32N = 48L bits, so the
Montgomery radix R = 2^(32N) is identical to the u32 IMAD path and the two
products can be mixed inside one formula).

Every floating-point operation is modelled exactly: the real result is computed
with Fractions and rounded to 53 significant bits with the stated mode; the
emulator asserts that every step documented as exact really is exact, and
that the rounding-dependent steps (fma_rz "floors") behave as claimed.
"""
from fractions import Fraction as Fr
import random

BETA = 1 << 48
TWO52 = 1 << 52


def rnd(x: Fr, mode: str) -> Fr:
    """Round a non-negative or negative rational to a double (53-bit mantissa)."""
    if x == 0:
        return Fr(0)
    neg = x < 0
    ax = -x if neg else x
    e = ax.numerator.bit_length() - ax.denominator.bit_length()
    # find e with 2^e <= ax < 2^(e+1)
    while Fr(2) ** e > ax:
        e -= 1
    while Fr(2) ** (e + 1) <= ax:
        e += 1
    ulp = Fr(2) ** (e - 52)
    q = ax / ulp
    fl = q.numerator // q.denominator
    if mode == "rz" or q == fl:
        r = fl
    elif mode == "rn":
        rem = q - fl
        r = fl + (1 if rem > Fr(1, 2) or (rem == Fr(1, 2) and fl % 2) else 0)
    else:
        raise ValueError(mode)
    v = r * ulp
    return -v if neg else v


def exact(x: Fr) -> Fr:
    assert rnd(x, "rn") == x, "claimed-exact FP step is inexact"
    return x


def fma_rz(a, b, c):
    return rnd(a * b + c, "rz")


def fma_ex(a, b, c):
    return exact(a * b + c)


def add_ex(a, b):
    return exact(a + b)


def to_limbs48(v, L):
    return [Fr((v >> (48 * k)) & (BETA - 1)) for k in range(L)]


def dfp_mul(a_int, b_int, p, L):
    """Returns a*b*2^(-48L) mod p in [0, 2p) (Montgomery product)."""
    n0 = (-pow(p, -1, BETA)) % BETA
    A = to_limbs48(a_int, L)
    Bs = [x / BETA for x in to_limbs48(b_int, L)]          # pre-scaled b_j * 2^-48 (exact)
    Ps = [x / BETA for x in to_limbs48(p, L)]
    n0s = Fr(n0) / BETA
    # --- product: Hb[k] (biased by 2^52) gets floor(a_i b_j / beta) at k = i+j+1,
    #     F[k] the fraction frac(a_i b_j / beta) (its column value is F[k] * beta at k-1)
    Hb = [Fr(TWO52)] * (2 * L + 2)
    F = [Fr(0)] * (2 * L + 2)
    for i in range(L):
        for j in range(L):
            k = i + j + 1
            old = Hb[k]
            Hb[k] = fma_rz(A[i], Bs[j], old)
            assert TWO52 <= Hb[k] < 2 * TWO52
            d = add_ex(Hb[k], -old)
            F[k] = add_ex(F[k], fma_ex(A[i], Bs[j], -d))
            assert 0 <= F[k] < 32
    # --- normalise the product columns: Nk = (Hb[k]-2^52) + F[k+1]*beta + carry, limbs < beta
    Nn = [Fr(0)] * (2 * L + 1)
    carry = Fr(0)
    for k in range(2 * L):
        c = add_ex(add_ex(add_ex(Hb[k], -TWO52), F[k + 1] * BETA), carry)
        assert c < 2 ** 53
        q = add_ex(fma_rz(c, Fr(1, BETA), Fr(TWO52)), -TWO52)     # floor(c / beta)
        Nn[k] = fma_ex(q, -Fr(BETA), c)
        assert 0 <= Nn[k] < BETA
        carry = q
    Nn[2 * L] = carry
    # --- Montgomery reduction (SOS), fresh accumulators for the m_i p_j products
    Hb2 = [Fr(TWO52)] * (2 * L + 2)
    F2 = [Fr(0)] * (2 * L + 2)
    carry = Fr(0)
    for i in range(L):
        c = add_ex(add_ex(add_ex(Nn[i], add_ex(Hb2[i], -TWO52)), F2[i + 1] * BETA), carry)
        assert c < 2 ** 53
        # m = (c mod beta) * n0 mod beta
        q = add_ex(fma_rz(c, Fr(1, BETA), Fr(TWO52)), -TWO52)
        t = fma_ex(q, -Fr(BETA), c)
        h = add_ex(fma_rz(t, n0s, Fr(TWO52)), -TWO52)
        m = fma_ex(t, n0s, -h) * BETA
        assert m == int(m) and 0 <= m < BETA
        for j in range(L):
            k = i + j + 1
            old = Hb2[k]
            Hb2[k] = fma_rz(m, Ps[j], old)
            assert TWO52 <= Hb2[k] < 2 * TWO52
            d = add_ex(Hb2[k], -old)
            F2[k] = add_ex(F2[k], fma_ex(m, Ps[j], -d))
            assert 0 <= F2[k] < 32
        # column i is now a multiple of beta
        col = add_ex(add_ex(add_ex(Nn[i], add_ex(Hb2[i], -TWO52)), F2[i + 1] * BETA), carry)
        assert col % BETA == 0
        carry = col / BETA
        assert carry == int(carry) and carry < 2 ** 8
    # --- result columns L..2L, normalised
    out = []
    for k in range(L, 2 * L):
        c = add_ex(add_ex(add_ex(Nn[k], add_ex(Hb2[k], -TWO52)), F2[k + 1] * BETA), carry)
        assert c < 2 ** 53
        q = add_ex(fma_rz(c, Fr(1, BETA), Fr(TWO52)), -TWO52)
        out.append(fma_ex(q, -Fr(BETA), c))
        carry = q
    top = add_ex(add_ex(Nn[2 * L], add_ex(Hb2[2 * L], -TWO52)), carry)
    v = sum(int(x) << (48 * k) for k, x in enumerate(out)) + (int(top) << (48 * L))
    return v


if __name__ == "__main__":
    for name, p in [("bls12_381", 0x1a0111ea397fe69a4b1ba7b6434bacd764774b84f38512bf6730d2a0f6b0f6241eabfffeb153ffffb9feffffffffaaab),
                    ("mnt4_753", 0x1c4c62d92c41110229022eee2cdadb7f997505b8fafed5eb7e8f96c97d87307fdb925e8a0ed8d99d124d9a15af79db117e776f218059db80f0da5cb537e38685acce9767254a4638810719ac425f0e39d54522cdd119f5e9063de245e8001)]:
        N = (p.bit_length() + 31) // 32
        N += N & 1
        L = 2 * N // 3
        R = 1 << (48 * L)
        assert R == 1 << (32 * N)
        Rinv = pow(R, -1, p)
        rng = random.Random(5)
        vals = [0, 1, p - 1, p - 2, R % p, (R - 1) % p] + [rng.randrange(p) for _ in range(120 if L == 8 else 25)]
        for t in range(len(vals)):
            x = vals[t]
            y = vals[(t * 7 + 3) % len(vals)]
            v = dfp_mul(x, y, p, L)
            assert v < 2 * p and v % p == x * y * Rinv % p, (name, t)
        print(name, "L=%d ok (%d products)" % (L, len(vals)))
