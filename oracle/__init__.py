"""The CPU oracle for the G1 MSM — TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline and
``--impl reference`` legs may import this package.  The product package
(paper_conf_asplos_maxsm0k0zsh23_b200) never imports it, and it never imports
the product: the two share no code.

Two independent oracles live here:

* ``oracle.ref``  — Python ints, affine chord-and-tangent, double-and-add
  (tiny inputs; cross-checks the C oracle);
* ``liboracle.so`` (oracle.c) — the same definition in plain C with
  schoolbook bignums and Knuth-D remainders, threaded over the host cores.

Both compute the definition Q = sum_i k_i (x) P_i (§2.1).
Pins: tests/test_oracle_pins.py.
"""

from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

from . import curves, ref
from .curves import Curve, get

_HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(_HERE, "liboracle.so")
_SRC = os.path.join(_HERE, "oracle.c")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (plain -O2, no vectorisation tricks)."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + ".tmp.%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", "-pthread",
                               _SRC, "-o", tmp])
        os.replace(tmp, _SO)
    return _SO


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_SO)
        u32p = ctypes.POINTER(ctypes.c_uint32)
        for name, args in {
            "oracle_msm": [ctypes.c_int, u32p, u32p, u32p, u32p, ctypes.c_int, ctypes.c_uint64, u32p, ctypes.c_int],
            "oracle_mul_each": [ctypes.c_int, u32p, u32p, u32p, u32p, ctypes.c_int, ctypes.c_uint64, u32p, ctypes.c_int],
            "oracle_ec_add": [ctypes.c_int, u32p, u32p, u32p, u32p, u32p],
            "oracle_msm_ext": [ctypes.c_int, ctypes.c_int, u32p, u32p, u32p, u32p, u32p, ctypes.c_int,
                               ctypes.c_uint64, u32p, ctypes.c_int],
            "oracle_mul_each_ext": [ctypes.c_int, ctypes.c_int, u32p, u32p, u32p, u32p, u32p, ctypes.c_int,
                                    ctypes.c_uint64, u32p, ctypes.c_int],
            "oracle_ec_add_ext": [ctypes.c_int, ctypes.c_int, u32p, u32p, u32p, u32p, u32p, u32p],
            "oracle_fp2_mul": [ctypes.c_int, u32p, u32p, u32p, u32p, u32p],
            "oracle_poly_eval": [ctypes.c_int, u32p, u32p, ctypes.c_uint64, u32p, ctypes.c_int, u32p,
                                 ctypes.c_int],
            "oracle_fp_mul": [ctypes.c_int, u32p, u32p, u32p, u32p],
            "oracle_fp_inv": [ctypes.c_int, u32p, u32p, u32p],
            "oracle_bn_mod": [u32p, ctypes.c_int, u32p, ctypes.c_int, u32p],
        }.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = ctypes.c_int
        _lib = L
    return _lib


def default_threads() -> int:
    try:
        return max(1, len(os.sched_getaffinity(0)))
    except AttributeError:
        return os.cpu_count() or 1


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32))


def _u32(a) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.uint32)


def _consts(c: Curve):
    """(L, deg, p, beta, a) limb arrays for the C oracle."""
    L = c.limbs
    if c.deg == 2:
        a = ref.int_to_limbs(c.a[0] % c.p, L) + ref.int_to_limbs(c.a[1] % c.p, L)
        beta = ref.int_to_limbs(c.beta % c.p, L)
    else:
        a = ref.int_to_limbs(c.a % c.p, L)
        beta = [0] * L
    return L, c.deg, _u32(ref.int_to_limbs(c.p, L)), _u32(beta), _u32(a)


def msm(curve, points: np.ndarray, scalars: np.ndarray, nthreads: int | None = None) -> np.ndarray:
    """C oracle MSM.  points: [n, 2D] u32 canonical affine ((0,0) = O; D =
    deg * L limbs per coordinate); scalars: [n, Ls] u32 little-endian.
    Returns [2D] u32 (affine, (0,0) = O)."""
    c = get(curve)
    L, deg, p, beta, a = _consts(c)
    D = deg * L
    points = _u32(points).reshape(-1, 2 * D)
    scalars = _u32(scalars)
    n = points.shape[0]
    Ls = scalars.shape[1] if scalars.ndim == 2 else 1
    scalars = scalars.reshape(n, Ls)
    out = np.zeros(2 * D, dtype=np.uint32)
    rc = lib().oracle_msm_ext(L, deg, _p(p), _p(beta), _p(a), _p(points), _p(scalars), Ls, n, _p(out),
                              nthreads or default_threads())
    if rc:
        raise RuntimeError(f"oracle_msm failed: {rc}")
    return out


def mul_each(curve, P: np.ndarray, scalars: np.ndarray, nthreads: int | None = None) -> np.ndarray:
    """out[i] = k_i (x) P (C oracle).  Returns [n, 2D] u32."""
    c = get(curve)
    L, deg, p, beta, a = _consts(c)
    D = deg * L
    P = _u32(P).reshape(2 * D)
    scalars = _u32(scalars)
    n = scalars.shape[0]
    Ls = scalars.shape[1] if scalars.ndim == 2 else 1
    scalars = scalars.reshape(n, Ls)
    out = np.zeros((n, 2 * D), dtype=np.uint32)
    rc = lib().oracle_mul_each_ext(L, deg, _p(p), _p(beta), _p(a), _p(P), _p(scalars), Ls, n, _p(out),
                                   nthreads or default_threads())
    if rc:
        raise RuntimeError(f"oracle_mul_each failed: {rc}")
    return out


def generator_limbs(curve) -> np.ndarray:
    c = get(curve)
    return _u32(ref.encode_point(c, (c.gx, c.gy)))


def points_from_dlogs(curve, dlogs: np.ndarray, nthreads: int | None = None) -> np.ndarray:
    """P_i = a_i (x) G, the synthetic proving-key points with known discrete
    logs (SURVEY.md §8(d) "Points")."""
    return mul_each(curve, generator_limbs(curve), dlogs, nthreads)


def ec_add(curve, P: np.ndarray, Q: np.ndarray) -> np.ndarray:
    c = get(curve)
    L, deg, p, beta, a = _consts(c)
    out = np.zeros(2 * deg * L, dtype=np.uint32)
    rc = lib().oracle_ec_add_ext(L, deg, _p(p), _p(beta), _p(a), _p(_u32(P)), _p(_u32(Q)), _p(out))
    if rc:
        raise RuntimeError(f"oracle_ec_add failed: {rc}")
    return out


def fp_mul(curve, x: int, y: int) -> int:
    c = get(curve)
    L = c.limbs
    p = _u32(ref.int_to_limbs(c.p, L))
    out = np.zeros(L, dtype=np.uint32)
    X, Y = _u32(ref.int_to_limbs(x, L)), _u32(ref.int_to_limbs(y, L))
    if lib().oracle_fp_mul(L, _p(p), _p(X), _p(Y), _p(out)):
        raise RuntimeError("oracle_fp_mul failed")
    return ref.limbs_to_int(out)


def fp2_mul(curve, x, y):
    """x * y in the G2 curve's F_p^2 (C oracle); x, y = (c0, c1)."""
    c = get(curve)
    L, _, p, beta, _ = _consts(c)
    X = _u32(ref.int_to_limbs(x[0], L) + ref.int_to_limbs(x[1], L))
    Y = _u32(ref.int_to_limbs(y[0], L) + ref.int_to_limbs(y[1], L))
    out = np.zeros(2 * L, dtype=np.uint32)
    if lib().oracle_fp2_mul(L, _p(p), _p(beta), _p(X), _p(Y), _p(out)):
        raise RuntimeError("oracle_fp2_mul failed")
    return (ref.limbs_to_int(out[:L]), ref.limbs_to_int(out[L:]))


def fp_inv(curve, x: int) -> int:
    c = get(curve)
    L = c.limbs
    p = _u32(ref.int_to_limbs(c.p, L))
    out = np.zeros(L, dtype=np.uint32)
    X = _u32(ref.int_to_limbs(x, L))
    if lib().oracle_fp_inv(L, _p(p), _p(X), _p(out)):
        raise RuntimeError("oracle_fp_inv failed")
    return ref.limbs_to_int(out)


def bn_mod(u: int, m: int, v: int, n: int) -> int:
    U = _u32(ref.int_to_limbs(u, m))
    V = _u32(ref.int_to_limbs(v, n))
    out = np.zeros(n, dtype=np.uint32)
    if lib().oracle_bn_mod(_p(U), m, _p(V), n, _p(out)):
        raise RuntimeError("oracle_bn_mod failed")
    return ref.limbs_to_int(out)


def poly_eval(curve, coeffs: np.ndarray, xs, nthreads: int | None = None) -> list:
    """A(x) mod r for every x in xs (C oracle, Horner; the NTT definition,
    PAPER.md:128).  coeffs: [N, Ls] u32 canonical (< r) scalar-field values of
    `curve`."""
    c = get(curve)
    Ls = c.scalar_limbs
    coeffs = _u32(coeffs).reshape(-1, Ls)
    r = _u32(ref.int_to_limbs(c.r, Ls))
    X = _u32([ref.int_to_limbs(x % c.r, Ls) for x in xs]).reshape(-1, Ls)
    out = np.zeros((X.shape[0], Ls), dtype=np.uint32)
    if lib().oracle_poly_eval(Ls, _p(r), _p(coeffs), coeffs.shape[0], _p(X), X.shape[0], _p(out),
                              nthreads or default_threads()):
        raise RuntimeError("oracle_poly_eval failed")
    return [ref.limbs_to_int(row) for row in out]


def closed_form(curve, scalars: np.ndarray, dlogs: np.ndarray) -> np.ndarray:
    """sum_i k_i (a_i G) = (sum_i k_i a_i mod r) G  (SURVEY.md §8(c) pins).

    dlogs may hold fewer rows m than there are scalars: a_i = dlogs[i mod m]
    (the tiled point sets P_i = T[i mod m] of SURVEY.md §8(d))."""
    c = get(curve)
    s = dot_mod(scalars, dlogs, c.r)
    Ls = c.scalar_limbs
    k = _u32(ref.int_to_limbs(s, Ls)).reshape(1, Ls)
    return mul_each(c, generator_limbs(c), k, 1)[0]


def dot_mod(scalars: np.ndarray, dlogs: np.ndarray, r: int, chunk: int = 1 << 20) -> int:
    """(sum_i k_i a_{i mod m}) mod r, exactly, for u32-limb arrays (m = rows
    of dlogs).

    Both operands are split into 16-bit limbs and M[u, v] = sum_i k16[i, u]
    a16[i, v] is formed per chunk of <= 2^20 rows as a float64 matrix product:
    every product is < 2^32 and a chunk's sum < 2^52, so the float64 values
    are exact integers.  The chunks' matrices are added as Python ints, then
    total = sum_{u,v} M[u, v] 2^(16 (u + v))."""
    if chunk > (1 << 20):
        raise ValueError("chunk too large for exact float64 accumulation")
    scalars = _u32(scalars)
    dlogs = _u32(dlogs)
    n = scalars.shape[0]
    m = dlogs.shape[0]
    if n == 0:
        return 0
    if m == 0:
        raise ValueError("no discrete logs")
    a16_all = dlogs.view(np.uint16).astype(np.float64)           # [m, 2 La] little-endian halves
    acc = None
    for s0 in range(0, n, chunk):
        s1 = min(n, s0 + chunk)
        k16 = scalars[s0:s1].view(np.uint16).astype(np.float64)
        idx = np.arange(s0, s1) % m
        M = k16.T @ a16_all[idx]
        Mi = [[int(x) for x in row] for row in M]
        if acc is None:
            acc = Mi
        else:
            for u in range(len(acc)):
                for v in range(len(acc[u])):
                    acc[u][v] += Mi[u][v]
    total = 0
    for u, row in enumerate(acc):
        for v, x in enumerate(row):
            if x:
                total += x << (16 * (u + v))
    return total % r


__all__ = ["curves", "ref", "msm", "mul_each", "points_from_dlogs", "closed_form", "dot_mod",
           "ec_add", "fp_mul", "fp2_mul", "fp_inv", "poly_eval", "bn_mod", "build", "default_threads", "generator_limbs"]
