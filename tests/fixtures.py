"""Cached oracle-generated test inputs.

Points with known discrete logs are produced ONLY by the oracle
(oracle.points_from_dlogs); scalars and discrete logs only by synth.  The cache
(tests/.cache, git-ignored) just saves recomputation; a missing cache is
regenerated from the same seeds.
"""

from __future__ import annotations

import os

import numpy as np

import oracle
import synth

CACHE = os.path.join(os.path.dirname(os.path.abspath(__file__)), ".cache")


def oracle_points(curve: str, n: int, seed: int | None = None):
    """(points [n,2L] u32, dlogs [n,Ls] u32) with points_i = dlogs_i * G."""
    seed = synth.dlog_seed(curve) if seed is None else seed
    os.makedirs(CACHE, exist_ok=True)
    path = os.path.join(CACHE, f"pts_{curve}_{seed}_{n}.npz")
    if os.path.exists(path):
        z = np.load(path)
        return z["points"], z["dlogs"]
    d = synth.dlogs(curve, n, seed)
    pts = oracle.points_from_dlogs(curve, d)
    tmp = path + f".{os.getpid()}.tmp.npz"
    np.savez(tmp, points=pts, dlogs=d)
    os.replace(tmp, path)
    return pts, d


def oracle_msm_cached(curve: str, points: np.ndarray, scalars: np.ndarray):
    import hashlib
    os.makedirs(CACHE, exist_ok=True)
    h = hashlib.sha1(np.ascontiguousarray(points).tobytes()
                     + np.ascontiguousarray(scalars).tobytes()).hexdigest()[:20]
    path = os.path.join(CACHE, f"msm_{curve}_{h}.npy")
    if os.path.exists(path):
        return np.load(path)
    out = oracle.msm(curve, points, scalars)
    np.save(path, out)
    return out
