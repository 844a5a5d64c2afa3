"""NTT oracle -- TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl
reference legs may import this module; the product never does.

What it computes is the definition of PAPER.md:128 (§2.2): for a polynomial
A(x) = sum_{i<N} A_i x^i with A_i in F_r, the N-NTT is the vector

    a = (A(1), A(w_N), ..., A(w_N^(N-1))),     a_k = sum_i A_i w_N^(i k),

with w_N a primitive N-th root of unity in F_r.  The inverse maps a back to A:
A_i = N^-1 sum_k a_k w_N^(-i k).  Here each a_k is the evaluation A(w_N^k) by
Horner's rule, i.e. the definition itself: O(N^2), no butterflies, no
Cooley-Tukey, nothing that resembles the GPU kernels.

Root of unity (the paper does not fix one; reading R15): with
r - 1 = 2^s t (t odd) and g the smallest quadratic non-residue mod r,
w_N = g^((r-1)/N) for N = 2^n <= 2^s.  Then w_N^(N/2) = g^((r-1)/2) = -1, so
w_N is primitive (pinned in tests/test_oracle_ntt.py).
"""

from __future__ import annotations

from typing import Sequence

from .curves import get


def two_adicity(r: int) -> int:
    s = 0
    while (r - 1) >> s & 1 == 0:
        s += 1
    return s


def smallest_non_residue(r: int) -> int:
    g = 2
    while pow(g, (r - 1) // 2, r) != r - 1:
        g += 1
    return g


def root_of_unity(curve, log_n: int) -> int:
    """w_N, N = 2^log_n, in the scalar field F_r of `curve`."""
    r = get(curve).r
    s = two_adicity(r)
    if log_n > s:
        raise ValueError(f"2^{log_n} does not divide r - 1 (2-adicity {s})")
    return pow(smallest_non_residue(r), (r - 1) >> log_n, r)


def horner(coeffs: Sequence[int], x: int, r: int) -> int:
    """A(x) mod r for A = sum_i coeffs[i] x^i."""
    acc = 0
    for c in reversed(coeffs):
        acc = (acc * x + c) % r
    return acc


def ntt(curve, coeffs: Sequence[int], inverse: bool = False) -> list:
    """The definition: a_k = A(w^k) (forward) or A_k = N^-1 a(w^-k) (inverse)."""
    r = get(curve).r
    n = len(coeffs)
    log_n = n.bit_length() - 1
    if n != 1 << log_n:
        raise ValueError("N must be a power of two")
    w = root_of_unity(curve, log_n)
    if inverse:
        w = pow(w, -1, r)
    out = [horner(coeffs, pow(w, k, r), r) for k in range(n)]
    if inverse:
        ninv = pow(n, -1, r)
        out = [v * ninv % r for v in out]
    return out
