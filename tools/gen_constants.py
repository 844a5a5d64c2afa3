"""Generate paper_conf_asplos_maxsm0k0zsh23_b200/csrc/curves.cuh.

PRODUCT-SIDE constants generator.  It holds its own hex copy of the standard
curve parameters (reading R1) and derives the Montgomery constants
(n0' = -p^-1 mod 2^32, R mod p, R^2 mod p, a*R mod p).  It does not import or
call anything under oracle/ (the oracle keeps its own copy in oracle/curves.py).

Run:  python tools/gen_constants.py   (output is committed)
"""

import os

CURVES = [
    # name, enum id, p, a, b, scalar bits (bit length of r), generator (x, y)
    ("BN254", 0,
     "30644e72e131a029b85045b68181585d97816a916871ca8d3c208c16d87cfd47", "0", "3", 254,
     ("1", "2")),
    ("BLS12_381", 1,
     "1a0111ea397fe69a4b1ba7b6434bacd764774b84f38512bf6730d2a0f6b0f6241eabfffeb153ffffb9feffffffffaaab",
     "0", "4", 255,
     ("17f1d3a73197d7942695638c4fa9ac0fc3688c4f9774b905a14e3a3f171bac586c55e83ff97a1aeffb3af00adb22c6bb",
      "08b3f481e3aaa0f1a09e30ed741d8ae4fcf5e095d5d00af600db18cb2c04b3edd03cc744a2888ae40caa232946c5e7e1")),
    ("MNT4_753", 2,
     "1c4c62d92c41110229022eee2cdadb7f997505b8fafed5eb7e8f96c97d87307fdb925e8a0ed8d99d124d9a15af79db117e776f218059db80f0da5cb537e38685acce9767254a4638810719ac425f0e39d54522cdd119f5e9063de245e8001",
     "2",
     "1373684a8c9dcae7a016ac5d7748d3313cd8e39051c596560835df0c9e50a5b59b882a92c78dc537e51a16703ec9855c77fc3d8bb21c8d68bb8cfb9db4b8c8fba773111c36c8b1b4e8f1ece940ef9eaad265458e06372009c9a0491678ef4",
     753,
     ("1",
      "7b753d99cf6f828729cd4e81339b83589f644376b25812761ca069cc1aaff44973d9f1751bee9fab5b8ec89845d948e3f9854059d4a6049cb8e9039c96f7fa2fdf50d0add627081b1c88bddc1166e34ce99bfbcc08a2d39f3788b4f54125")),
    # toy prime-order curves (test builds), generators = smallest x, smaller y
    ("TOY_A0", 100, "%x" % 10099, "0", "3", 14, None),
    ("TOY_A2", 101, "%x" % 10007, "2", "1e", 14, None),
]


# G2: the order-r subgroup of the sextic
# twist E'(F_p^2): y^2 = x^3 + b' over F_p^2 = F_p[u]/(u^2 + 1).  This script's
# own copy of the standard generators (EIP-197 for BN254; IETF draft /
# zkcrypto for BLS12-381).  b' = 3 / (9 + u) for BN254, 4 (1 + u) for BLS12-381.
G2_CURVES = [
    # name, enum id, base struct, b' as a function of p, generator ((x0, x1), (y0, y1)) decimal/hex
    ("BN254_G2", 3, "BN254",
     (("10857046999023057135944570762232829481370756359578518086990519993285655852781",
       "11559732032986387107991004021392285783925812861821192530917403151452391805634"),
      ("8495653923123431417604973247489272438418190587263600148770280649306958101930",
       "4082367875863433681332203403145435568316851327593401208105741076214120093531")), 10),
    ("BLS12_381_G2", 4, "BLS12_381",
     (("024aa2b2f08f0a91260805272dc51051c6e47ad4fa403b02b4510b647ae3d1770bac0326a805bbefd48056c8c121bdb8",
       "13e02b6052719f607dacd3a088274f65596bd0d09920b61ab5da61bbdc7f5049334cf11213945d57e5ac7d055d042b7e"),
      ("0ce5d527727d6e118cc9cdc6da2e351aadfd9baa8cbdd3a76d429a695160d12c923ac9cc3baca289e193548608b82801",
       "0606c4a02ea734cc32acd2b02bc28b99cb3e287e85a763af267492ab572e99ab3f370d275cec1da1aaa9075ff05f79be")), 16),
]


def f2mul(x, y, p):
    return ((x[0] * y[0] - x[1] * y[1]) % p, (x[0] * y[1] + x[1] * y[0]) % p)


def g2_twist_b(name, p):
    if name == "BN254_G2":           # 3 / (9 + u) = 3 (9 - u) / 82
        inv82 = pow(82, -1, p)
        return (27 * inv82 % p, (-3) * inv82 % p)
    return (4, 4)


# Scalar fields F_r (NTT): this script's
# own copy of r.  ROOT = g^((r-1) / 2^S) with S the 2-adicity of r - 1 and g the
# smallest quadratic non-residue (reading R15), so ROOT^(2^(S-1)) = -1.
FR_FIELDS = [
    ("FR_BN254", "30644e72e131a029b85045b68181585d2833e84879b9709143e1f593f0000001"),
    ("FR_BLS12_381", "73eda753299d7d483339d80809a1d80553bda402fffe5bfeffffffff00000001"),
    ("FR_MNT4_753", "1c4c62d92c41110229022eee2cdadb7f997505b8fafed5eb7e8f96c97d87307fdb925e8a0ed8d99d124d9a15af79db26c5c28c859a99b3eebca9429212636b9dff97634993aa4d6c381bc3f0057974ea099170fa13a4fd90776e240000001"),
]


def fr_root(r):
    S = 0
    while ((r - 1) >> S) & 1 == 0:
        S += 1
    g = 2
    while pow(g, (r - 1) // 2, r) != r - 1:
        g += 1
    w = pow(g, (r - 1) >> S, r)
    assert pow(w, 1 << (S - 1), r) == r - 1 and pow(w, 1 << S, r) == 1
    return S, g, w


def limbs(v, n):
    return [(v >> (32 * i)) & 0xFFFFFFFF for i in range(n)]


def arr(v, n):
    return "{" + ", ".join("0x%08xu" % x for x in limbs(v, n)) + "}"


def dfp_block(p, n):
    """FP64 (DFP) constants: 48-bit limbs of p pre-scaled by
    2^-48, and n0_48 = -p^-1 mod 2^48 pre-scaled by 2^-48 (all exact doubles).
    Only emitted when 32n is a multiple of 48 (same Montgomery radix)."""
    if (32 * n) % 48:
        return "  static constexpr bool HAS_DFP = false;\n"
    L = 32 * n // 48
    beta = 1 << 48
    n0 = (-pow(p, -1, beta)) % beta
    limbs48 = [(p >> (48 * k)) & (beta - 1) for k in range(L)]
    ps = ", ".join(float(x / beta).hex() for x in limbs48)
    for x in limbs48:
        assert float(x / beta) * beta == x
    assert float(n0 / beta) * beta == n0
    return (f"  static constexpr bool HAS_DFP = true;\n"
            f"  static constexpr int DFP_L = {L};    // 48-bit limbs, radix 2^(48 L) = 2^(32 N)\n"
            f"  GZ_HD static constexpr double P48S(int i) {{ constexpr double v[{L}] = {{{ps}}}; return v[i]; }}  // p limbs * 2^-48\n"
            f"  static constexpr double N048S = {float(n0 / beta).hex()};   // (-p^-1 mod 2^48) * 2^-48\n")


def toy_gen(p, a, b):
    for x in range(p):
        rhs = (x ** 3 + a * x + b) % p
        if rhs == 0:
            continue
        for y in range(1, (p + 1) // 2):
            if y * y % p == rhs:
                return x, y
    raise ValueError


def write_if_changed(dst, text):
    """Keep the mtime (and so the incremental build) when nothing changed."""
    try:
        with open(dst) as f:
            if f.read() == text:
                print("unchanged", dst)
                return
    except OSError:
        pass
    with open(dst, "w") as f:
        f.write(text)
    print("wrote", dst)


def main():
    out = []
    out.append("// GENERATED by tools/gen_constants.py -- do not edit.\n"
               "// Product-side curve constants (standard parameters, DESIGN.md reading R1).\n"
               "// Montgomery form: R = 2^(32 N); n0 = -p^-1 mod 2^32.\n"
               "#pragma once\n#include <cstdint>\n\n#ifndef GZ_HD\n#define GZ_HD __host__ __device__ __forceinline__\n#endif\n\nnamespace gzkp {\n")
    for name, cid, ph, ah, bh, sbits, gen in CURVES:
        p, a, b = int(ph, 16), int(ah, 16), int(bh, 16)
        n = (p.bit_length() + 31) // 32
        n += n & 1
        R = 1 << (32 * n)
        n0 = (-pow(p, -1, 1 << 32)) % (1 << 32)
        if gen is None:
            gx, gy = toy_gen(p, a, b)
        else:
            gx, gy = int(gen[0], 16), int(gen[1], 16)
        assert (gy * gy - gx ** 3 - a * gx - b) % p == 0, name
        ls = (sbits + 31) // 32
        out.append(f"struct {name} {{\n"
                   f"  static constexpr int ID = {cid};\n"
                   f"  static constexpr int N = {n};            // u32 limbs of p\n"
                   f"  static constexpr int NS = {ls};           // u32 limbs of a scalar\n"
                   f"  static constexpr int SCALAR_BITS = {sbits};\n"
                   f"  static constexpr int P_BITS = {p.bit_length()};\n"
                   f"  static constexpr uint32_t N0 = 0x{n0:08x}u;\n"
                   f"  static constexpr bool A_ZERO = {'true' if a == 0 else 'false'};\n"
                   f"  static constexpr uint32_t A_SMALL = {a if a < 2**32 else 0}u;  // a as an integer (0 or 2 here)\n"
                   f"  // limb accessors (constexpr functions fold to immediates after unrolling)\n"
                   f"  GZ_HD static constexpr uint32_t P(int i) {{ constexpr uint32_t v[N] = {arr(p, n)}; return v[i]; }}\n"
                   f"  GZ_HD static constexpr uint32_t ONE(int i) {{ constexpr uint32_t v[N] = {arr(R % p, n)}; return v[i]; }}  // R mod p\n"
                   f"  GZ_HD static constexpr uint32_t R2(int i) {{ constexpr uint32_t v[N] = {arr(R * R % p, n)}; return v[i]; }}  // R^2 mod p\n"
                   f"  GZ_HD static constexpr uint32_t A_MONT(int i) {{ constexpr uint32_t v[N] = {arr(a * R % p, n)}; return v[i]; }}\n"
                   f"  GZ_HD static constexpr uint32_t NP(int i) {{ constexpr uint32_t v[N] = {arr((-pow(p, -1, R)) % R, n)}; return v[i]; }}  // -p^-1 mod R\n"
                   f"  GZ_HD static constexpr uint32_t GX(int i) {{ constexpr uint32_t v[N] = {arr(gx, n)}; return v[i]; }}  // generator, canonical\n"
                   f"  GZ_HD static constexpr uint32_t GY(int i) {{ constexpr uint32_t v[N] = {arr(gy, n)}; return v[i]; }}\n"
                   + dfp_block(p, n) +
                   f"}};\n")
    bases = {c[0]: c for c in CURVES}
    for name, cid, base, gen, radix in G2_CURVES:
        _, _, ph, _, _, sbits, _ = bases[base]
        p = int(ph, 16)
        n = (p.bit_length() + 31) // 32
        n += n & 1
        (x0, x1), (y0, y1) = [[int(v, radix) for v in c] for c in gen]
        bt = g2_twist_b(name, p)
        lhs = f2mul((y0, y1), (y0, y1), p)
        x3 = f2mul(f2mul((x0, x1), (x0, x1), p), (x0, x1), p)
        assert lhs == ((x3[0] + bt[0]) % p, (x3[1] + bt[1]) % p), name
        ls = (sbits + 31) // 32
        w = 2 * n
        out.append(f"// G2 of {base}: F_p^2 coordinates c0 || c1 (u^2 = -1), N = 2 x {n} words\n"
                   f"struct {name} {{\n"
                   f"  using Base = {base};\n"
                   f"  static constexpr int ID = {cid};\n"
                   f"  static constexpr int N = {w};            // u32 words of one F_p^2 coordinate\n"
                   f"  static constexpr int NS = {ls};           // u32 limbs of a scalar\n"
                   f"  static constexpr int SCALAR_BITS = {sbits};\n"
                   f"  static constexpr int P_BITS = {p.bit_length()};\n"
                   f"  static constexpr bool A_ZERO = true;\n"
                   f"  static constexpr uint32_t A_SMALL = 0u;\n"
                   f"  GZ_HD static constexpr uint32_t A_MONT(int i) {{ constexpr uint32_t v[N] = {arr(0, w)}; return v[i]; }}\n"
                   f"  GZ_HD static constexpr uint32_t GX(int i) {{ constexpr uint32_t v[N] = {arr(x0 | (x1 << (32 * n)), w)}; return v[i]; }}  // generator, canonical\n"
                   f"  GZ_HD static constexpr uint32_t GY(int i) {{ constexpr uint32_t v[N] = {arr(y0 | (y1 << (32 * n)), w)}; return v[i]; }}\n"
                   f"  static constexpr bool HAS_DFP = false;\n"
                   f"}};\n")
    out.append("}  // namespace gzkp\n")
    dst = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                       "paper_conf_asplos_maxsm0k0zsh23_b200", "csrc", "curves.cuh")
    write_if_changed(dst, "\n".join(out))
    out = ["// GENERATED by tools/gen_constants.py -- do not edit.\n"
           "// Scalar fields F_r for the NTT (SURVEY.md §8(f) NEXT-4), Montgomery R = 2^(32 N).\n"
           "#pragma once\n#include <cstdint>\n\n#ifndef GZ_HD\n#define GZ_HD __host__ __device__ __forceinline__\n#endif\n\nnamespace gzkp {\n"]
    for name, rh in FR_FIELDS:
        r = int(rh, 16)
        n = (r.bit_length() + 31) // 32
        n += n & 1
        R = 1 << (32 * n)
        n0 = (-pow(r, -1, 1 << 32)) % (1 << 32)
        S, g, w = fr_root(r)
        out.append(f"// scalar field F_r ({r.bit_length()} bits) for the NTT; ROOT = {g}^((r-1)/2^{S}), canonical\n"
                   f"struct {name} {{\n"
                   f"  static constexpr int N = {n};            // u32 limbs of r\n"
                   f"  static constexpr int NS = {n};\n"
                   f"  static constexpr int P_BITS = {r.bit_length()};\n"
                   f"  static constexpr uint32_t N0 = 0x{n0:08x}u;\n"
                   f"  static constexpr int TWO_ADICITY = {S};\n"
                   f"  static constexpr bool A_ZERO = true;\n"
                   f"  static constexpr uint32_t A_SMALL = 0u;\n"
                   f"  GZ_HD static constexpr uint32_t P(int i) {{ constexpr uint32_t v[N] = {arr(r, n)}; return v[i]; }}  // r\n"
                   f"  GZ_HD static constexpr uint32_t ONE(int i) {{ constexpr uint32_t v[N] = {arr(R % r, n)}; return v[i]; }}  // R mod r\n"
                   f"  GZ_HD static constexpr uint32_t R2(int i) {{ constexpr uint32_t v[N] = {arr(R * R % r, n)}; return v[i]; }}  // R^2 mod r\n"
                   f"  GZ_HD static constexpr uint32_t A_MONT(int i) {{ constexpr uint32_t v[N] = {arr(0, n)}; return v[i]; }}\n"
                   f"  GZ_HD static constexpr uint32_t ROOT(int i) {{ constexpr uint32_t v[N] = {arr(w, n)}; return v[i]; }}  // primitive 2^S-th root\n"
                   f"  GZ_HD static constexpr uint32_t HALF(int i) {{ constexpr uint32_t v[N] = {arr((r + 1) // 2, n)}; return v[i]; }}  // 1/2 mod r\n"
                   f"  static constexpr bool HAS_DFP = false;\n"
                   f"}};\n")
    out.append("}  // namespace gzkp\n")
    dst = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                       "paper_conf_asplos_maxsm0k0zsh23_b200", "csrc", "fr_fields.cuh")
    write_if_changed(dst, "\n".join(out))


if __name__ == "__main__":
    main()
