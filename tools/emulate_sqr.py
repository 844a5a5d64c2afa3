"""Carry-exact emulation of the PTX sequence for csrc/field.cuh F::sqr
(triangular product + doubling + diagonal + SOS reduction with deferred chain
carries).  Development aid, not the oracle."""
import random

M32 = 0xFFFFFFFF


class Ctx:
    def __init__(s):
        s.cc = 0

    def mad(s, hi, x, y, z, cin, cout):
        p = x * y
        t = ((p >> 32) if hi else (p & M32)) + z + (s.cc if cin else 0)
        if cout:
            s.cc = t >> 32
        else:
            assert t >> 32 == 0, "dropped carry (mad)"
        return t & M32

    def add(s, x, y, cin, cout):
        t = x + y + (s.cc if cin else 0)
        if cout:
            s.cc = t >> 32
        else:
            assert t >> 32 == 0, "dropped carry (add)"
        return t & M32


def sqr(a, P, n0, N):
    X = Ctx()
    EV = [0] * (2 * N + 2)
    OD = [0] * (2 * N + 2)
    # triangular product: row i multiplies a_i by a_{i+1..N-1}
    for i in range(N - 1):
        for par, acc in ((0, OD), (1, EV)):        # k even -> odd-start positions, k odd -> even-start
            ks = list(range(par, N - 1 - i, 2))
            if not ks:
                continue
            for idx, k in enumerate(ks):
                pos = 2 * i + 1 + k
                acc[pos] = X.mad(False, a[i], a[i + 1 + k], acc[pos], idx > 0, True)
                acc[pos + 1] = X.mad(True, a[i], a[i + 1 + k], acc[pos + 1], True, True)
            last = 2 * i + 1 + ks[-1] + 2
            acc[last] = X.add(acc[last], 0, True, False)
    # V = OD + EV
    V = [0] * (2 * N + 1)
    V[0] = X.add(OD[0], EV[0], False, True)
    for k in range(1, 2 * N):
        V[k] = X.add(OD[k], EV[k], True, True)
    V[2 * N] = X.add(OD[2 * N], EV[2 * N], True, False)
    assert V[2 * N] == 0
    # T = 2V (V < 2^(64N-1))
    T = [0] * (2 * N)
    for k in range(2 * N - 1, 0, -1):
        T[k] = ((V[k] << 1) | (V[k - 1] >> 31)) & M32
    T[0] = (V[0] << 1) & M32
    assert V[2 * N - 1] >> 31 == 0
    # + diagonal a_i^2 at (2i, 2i+1)
    for i in range(N):
        T[2 * i] = X.mad(False, a[i], a[i], T[2 * i], i > 0, True)
        T[2 * i + 1] = X.mad(True, a[i], a[i], T[2 * i + 1], True, i < N - 1)
    # SOS reduction with deferred carries C[pos], pos >= N
    C = [0] * (2 * N + 2)
    for i in range(N):
        m = (T[i] * n0) & M32
        for par in (0, 1):                          # p even limbs -> pos i+2k, p odd -> i+1+2k
            for k in range(N // 2):
                j = 2 * k + par
                pos = i + j
                T[pos] = X.mad(False, P[j], m, T[pos], k > 0, True)
                T[pos + 1] = X.mad(True, P[j], m, T[pos + 1], True, True)
            cpos = i + N + par
            C[cpos] = X.add(C[cpos], 0, True, False)
        assert T[i] == 0
    R = [0] * (N + 1)
    R[0] = X.add(T[N], C[N], False, True)
    for k in range(1, N):
        R[k] = X.add(T[N + k], C[N + k], True, True)
    R[N] = X.add(C[2 * N], C[2 * N + 1], True, False)
    v = sum(x << (32 * k) for k, x in enumerate(R))
    return v


def limbs(v, N):
    return [(v >> (32 * i)) & M32 for i in range(N)]


for name, p in [("bn254", 0x30644e72e131a029b85045b68181585d97816a916871ca8d3c208c16d87cfd47),
                ("bls", 0x1a0111ea397fe69a4b1ba7b6434bacd764774b84f38512bf6730d2a0f6b0f6241eabfffeb153ffffb9feffffffffaaab),
                ("mnt4", 0x1c4c62d92c41110229022eee2cdadb7f997505b8fafed5eb7e8f96c97d87307fdb925e8a0ed8d99d124d9a15af79db117e776f218059db80f0da5cb537e38685acce9767254a4638810719ac425f0e39d54522cdd119f5e9063de245e8001),
                ("toy", 10099),
                # scalar fields F_r (NTT, NEXT-4): BLS12-381's r has a single spare bit
                ("r_bn254", 0x30644e72e131a029b85045b68181585d2833e84879b9709143e1f593f0000001),
                ("r_bls", 0x73eda753299d7d483339d80809a1d80553bda402fffe5bfeffffffff00000001),
                ("r_mnt4", 0x1c4c62d92c41110229022eee2cdadb7f997505b8fafed5eb7e8f96c97d87307fdb925e8a0ed8d99d124d9a15af79db26c5c28c859a99b3eebca9429212636b9dff97634993aa4d6c381bc3f0057974ea099170fa13a4fd90776e240000001)]:
    N = (p.bit_length() + 31) // 32
    N += N & 1
    n0 = (-pow(p, -1, 1 << 32)) % (1 << 32)
    R = 1 << (32 * N)
    Rinv = pow(R, -1, p)
    P = limbs(p, N)
    rng = random.Random(2)
    vals = [0, 1, 2, p - 1, p - 2, (p - 1) // 2, R % p, (R - 1) % p] + [rng.randrange(p) for _ in range(4000)]
    for x in vals:
        v = sqr(limbs(x, N), P, n0, N)
        assert v < 2 * p, (name, x)
        assert v % p == x * x * Rinv % p, (name, x)
    print(name, "ok")
