"""Carry-exact emulation of the PTX instruction sequence used by
csrc/field.cuh mont_mul (even/odd-split CIOS).  Development aid: checks that no
carry is dropped for the three production moduli, on random and extreme inputs.
It models mad.lo.cc / madc.hi.cc etc. bit-for-bit; it is NOT the oracle."""
import random, sys

M = 0xFFFFFFFF

class CC:
    def __init__(s): s.c = 0

def mont_mul(a, b, P, n0, N):
    cc = CC()
    def mad(lohi, x, y, z, cin, cout):
        prod = x * y
        t = (prod & M if lohi == 'lo' else prod >> 32) + z + (cc.c if cin else 0)
        if cout: cc.c = t >> 32
        else: assert t >> 32 == 0, "dropped carry"
        return t & M
    def add(x, y, cin, cout):
        t = x + y + (cc.c if cin else 0)
        if cout: cc.c = t >> 32
        else: assert t >> 32 == 0, "dropped carry (add)"
        return t & M

    E = [0] * N; O = [0] * N
    bi = b[0]
    for j in range(0, N, 2):
        E[j] = (a[j] * bi) & M; E[j+1] = (a[j] * bi) >> 32
        O[j] = (a[j+1] * bi) & M; O[j+1] = (a[j+1] * bi) >> 32
    def reduce(E, O):
        m = (E[0] * n0) & M
        for j in range(0, N, 2):   # O += m * p_odd
            O[j]   = mad('lo', P[j+1], m, O[j],   j > 0, True)
            O[j+1] = mad('hi', P[j+1], m, O[j+1], True, j + 2 < N)
        for j in range(0, N, 2):   # E += m * p_even
            E[j]   = mad('lo', P[j], m, E[j],   j > 0, True)
            E[j+1] = mad('hi', P[j], m, E[j+1], True, True)
        O[N-1] = add(O[N-1], 0, True, False)
        assert E[0] == 0
    reduce(E, O)
    for i in range(1, N):
        E, O = O, E                 # roles swap
        bi = b[i]
        E[0] = add(E[0], O[1], False, True)
        for j in range(0, N, 2):    # O_new[k] = a_odd*bi + O_old[k+2]
            z0 = O[j+2] if j + 2 < N else 0
            z1 = O[j+3] if j + 3 < N else 0
            O[j]   = mad('lo', a[j+1], bi, z0, True, True)
            O[j+1] = mad('hi', a[j+1], bi, z1, True, j + 2 < N)
        for j in range(0, N, 2):    # E += a_even*bi
            E[j]   = mad('lo', a[j], bi, E[j],   j > 0, True)
            E[j+1] = mad('hi', a[j], bi, E[j+1], True, True)
        O[N-1] = add(O[N-1], 0, True, False)
        reduce(E, O)
    r = [0] * N
    r[0] = add(E[1], O[0], False, True)
    for k in range(1, N - 1):
        r[k] = add(E[k+1], O[k], True, True)
    r[N-1] = add(O[N-1], 0, True, False)
    v = sum(x << (32 * k) for k, x in enumerate(r))
    return v

def limbs(v, N): return [(v >> (32 * i)) & M for i in range(N)]

for name, p in [("bn254", 0x30644e72e131a029b85045b68181585d97816a916871ca8d3c208c16d87cfd47),
                ("bls", 0x1a0111ea397fe69a4b1ba7b6434bacd764774b84f38512bf6730d2a0f6b0f6241eabfffeb153ffffb9feffffffffaaab),
                ("mnt4", 0x1c4c62d92c41110229022eee2cdadb7f997505b8fafed5eb7e8f96c97d87307fdb925e8a0ed8d99d124d9a15af79db117e776f218059db80f0da5cb537e38685acce9767254a4638810719ac425f0e39d54522cdd119f5e9063de245e8001),
                ("toy", 10099),
                # scalar fields F_r (NTT, NEXT-4): BLS12-381's r has a single spare bit
                ("r_bn254", 0x30644e72e131a029b85045b68181585d2833e84879b9709143e1f593f0000001),
                ("r_bls", 0x73eda753299d7d483339d80809a1d80553bda402fffe5bfeffffffff00000001),
                ("r_mnt4", 0x1c4c62d92c41110229022eee2cdadb7f997505b8fafed5eb7e8f96c97d87307fdb925e8a0ed8d99d124d9a15af79db26c5c28c859a99b3eebca9429212636b9dff97634993aa4d6c381bc3f0057974ea099170fa13a4fd90776e240000001)]:
    N = (p.bit_length() + 31) // 32; N += N & 1
    n0 = (-pow(p, -1, 1 << 32)) % (1 << 32)
    R = 1 << (32 * N); Rinv = pow(R, -1, p)
    P = limbs(p, N)
    rng = random.Random(1)
    vals = [0, 1, p - 1, p - 2, R % p, (R - 1) % p] + [rng.randrange(p) for _ in range(3000)]
    for t in range(3000):
        x = vals[t % len(vals)] if t < 50 else rng.choice(vals)
        y = rng.choice(vals) if t >= 6 else vals[t]
        v = mont_mul(limbs(x, N), limbs(y, N), P, n0, N)
        assert v < 2 * p
        assert v % p == x * y * Rinv % p, (name, x, y)
    print(name, "N=%d n0=%#x ok" % (N, n0))
