"""Model of the constant-time optimised binary GCD inversion (Pornin, "Optimized
Binary GCD for Modular Inversion", 2020) as the device code implements it:
32-bit limbs, k - 1 = 31 inner divsteps per outer iteration on 64-bit
approximations, u/v kept in [0, m) with a Montgomery-style division by 2^31
per outer iteration, which keeps the invariants a = u y, b = v y (mod m)
exact, so b = 1 at the end gives v = y^-1 with no correction factor.

Run: python tools/emulate_bingcd.py  -- checks random and edge inputs against
pow(y, -1, m) for the curves' moduli."""

import random

K1 = 31          # inner iterations per outer iteration (k - 1)
MASK31 = (1 << 31) - 1


def outer_iters(m):
    return -(-(2 * m.bit_length() - 1) // K1)


def inv(y, m):
    a, b, u, v = y, m, 1, 0
    T = outer_iters(m)
    minv31 = (-pow(m, -1, 1 << 31)) % (1 << 31)          # -m^-1 mod 2^31
    for _ in range(T):
        n = max(a.bit_length(), b.bit_length(), 64)
        a_ = (a & MASK31) | ((a >> (n - 33)) << 31)        # 31 low bits + 33 top bits
        b_ = (b & MASK31) | ((b >> (n - 33)) << 31)
        f0, g0, f1, g1 = 1, 0, 0, 1
        for _ in range(K1):
            if a_ & 1:
                if a_ < b_:
                    a_, b_ = b_, a_
                    f0, g0, f1, g1 = f1, g1, f0, g0
                a_ -= b_
                f0 -= f1
                g0 -= g1
            a_ >>= 1
            f1 <<= 1
            g1 <<= 1
        na = a * f0 + b * g0
        nb = a * f1 + b * g1
        assert na % (1 << K1) == 0 and nb % (1 << K1) == 0
        na >>= K1
        nb >>= K1
        if na < 0:
            na, f0, g0 = -na, -f0, -g0
        if nb < 0:
            nb, f1, g1 = -nb, -f1, -g1
        a, b = na, nb
        # u, v <- (u f0 + v g0) / 2^31 mod m, (u f1 + v g1) / 2^31 mod m
        def mdiv(x):
            x %= m
            t = ((x & MASK31) * minv31) & MASK31
            r = (x + t * m) >> 31
            return r - m if r >= m else r
        u, v = mdiv(u * f0 + v * g0), mdiv(u * f1 + v * g1)
    assert a == 0, "did not converge"
    if b != 1:
        return 0
    # the modular division by 2^31 keeps the invariants a = u y, b = v y (mod m)
    # exact, so b = 1 gives v = y^-1 directly
    return v


def main():
    curves = {
        "bn254": 0x30644e72e131a029b85045b68181585d97816a916871ca8d3c208c16d87cfd47,
        "bls12_381": 0x1a0111ea397fe69a4b1ba7b6434bacd764774b84f38512bf6730d2a0f6b0f6241eabfffeb153ffffb9feffffffffaaab,
        "mnt4_753": int("1c4c62d92c41110229022eee2cdadb7f997505b8fafed5eb7e8f96c97d87307fdb925e8a0ed8d99d124d9a15af79db117e776f218059db80f0da5cb537e38685acce9767254a4638810719ac425f0e39d54522cdd119f5e9063de245e8001", 16),
    }
    rng = random.Random(7)
    for name, m in curves.items():
        cases = [1, 2, 3, m - 1, m - 2, (m - 1) // 2, (m + 1) // 2, 1 << (m.bit_length() - 2)]
        cases += [(1 << k) % m for k in range(0, m.bit_length(), 7)]
        cases += [((1 << k) - 1) % m for k in range(1, m.bit_length(), 5)]
        cases += [rng.randrange(1, m) for _ in range(3000 if m.bit_length() < 400 else 600)]
        for y in cases:
            if y % m == 0:
                continue
            got = inv(y, m)
            assert got == pow(y, -1, m), (name, y)
        print(name, "ok", len(cases), "cases, outer iterations", outer_iters(m))


if __name__ == "__main__":
    main()
