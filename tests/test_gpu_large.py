"""Full-size parity (`-m gpu`) at BASELINE.json's sizes, in the launch
configuration bench.py times (the same planner: window bits c and chunk size S
depend only on (curve, n), and the test asserts the c the call used).  The
oracle cannot run 2^20+ double-and-adds in seconds, so (SURVEY.md §8(c)
"Parity pins"):

* the points are a_i * G from the product's fixed-base kernel, and a sample of
  them is re-derived by the oracle one by one (pins the generator);
* for n > 2^22 the point set is tiled, P_i = T[i mod 2^22] (SURVEY.md §8(d)
  "For n > m = 2^22, tile"), which keeps the closed form exact;
* the MSM result must equal, byte for byte, the oracle's closed form
  (sum_i k_i a_{i mod m} mod r) * G (PAPER.md:122 is the definition).
"""

import numpy as np
import pytest

import oracle
import synth
from tests.gpu_util import dev, host, require_cuda

pytestmark = pytest.mark.gpu


def _points(gz, curve, m, seed_cfg):
    d = synth.dlogs(curve, m, synth.dlog_seed(curve))
    pts = gz.fixed_base_mul(curve, dev(d))
    # sampled generator check: the oracle recomputes 16 points one by one
    idx = np.random.default_rng(seed_cfg).choice(m, 16, replace=False)
    sample = host(pts[idx.tolist()])
    assert np.array_equal(sample, oracle.points_from_dlogs(curve, d[idx]))
    return d, pts


def _msm_checked(gz, curve, pts, k_dev, n):
    """One MSM through the C ABI with phase profiling on: returns the bytes and
    the window bits c the library used (must be the planner's, as in bench.py)."""
    gz.set_profiling(True)
    gz.profile_read(reset=True)
    got = host(gz.msm(curve, pts, k_dev))
    prof = gz.profile_read(reset=True)
    gz.set_profiling(False)
    assert prof["c"] == gz.window_bits(curve, n)
    return got, prof


@pytest.mark.parametrize("curve,log_n,cfg,dist", [
    ("bn254", 20, 2, "uniform"),         # configs[1]
    ("bls12_381", 22, 3, "uniform"),     # configs[2] (the headline bench workload)
    ("bls12_381", 20, 5, "zcash_like"),  # sparse preset (configs[4] shape at 2^20)
    ("mnt4_753", 16, 4, "uniform"),      # configs[3] shape at 2^16 (planner c = 13)
])
def test_closed_form_full_size(curve, log_n, cfg, dist):
    gz = require_cuda()
    n = 1 << log_n
    d, pts = _points(gz, curve, n, cfg)
    k = synth.scalars(curve, n, synth.scalar_seed(cfg), dist)
    got, _ = _msm_checked(gz, curve, pts, dev(k), n)
    want = oracle.closed_form(curve, k, d)
    assert np.array_equal(got, want)
    # the same MSM through prepared weighted points (NEXT-1), planner's c,
    # full table (M = 1) and Algorithm 1 checkpoints (M = 2, 3)
    for M in (1, 2, 3):
        h = gz.PreparedPoints(curve, pts, weighted=M)
        assert np.array_equal(host(h.msm(dev(k))), want), M
        h.release()


@pytest.mark.parametrize("curve,log_n,cfg,dist,tile_log", [
    # configs[4] (C5): BLS12-381 2^26 sparse/skewed -- bucket 1 of window 0
    # holds ~40 % of all points, the deepest heavy-bucket tree
    ("bls12_381", 26, 5, "zcash_like", 22),
    # the north_star target: bit-exact dense 2^26 (~1.07e9 bucket entries)
    ("bls12_381", 26, 6, "uniform", 22),
    # configs[3] (C4): MNT4-753 2^20 at the planner's c = 16 (48 windows)
    ("mnt4_753", 20, 4, "uniform", 20),
])
def test_bench_config_bit_exact(curve, log_n, cfg, dist, tile_log):
    """The benched workloads of bench.py at their full n, in their launch
    configuration, byte-equal to the oracle's closed form."""
    gz = require_cuda()
    import torch
    n = 1 << log_n
    m = 1 << tile_log
    d, T = _points(gz, curve, m, cfg)
    pts = T.repeat(n // m, 1) if n > m else T
    del T
    k = synth.scalars(curve, n, synth.scalar_seed(cfg), dist)
    got, prof = _msm_checked(gz, curve, pts, dev(k), n)
    if curve == "mnt4_753":
        assert prof["c"] == 16
    # every entry is a non-zero signed digit: E <= n W, and the dense case is
    # within a fraction of a percent of n W (1 - 2^-c of the digits are non-zero)
    W = -(-(oracle.curves.get(curve).scalar_bits + 1) // prof["c"])
    assert 0 < prof["entries"] <= n * W
    want = oracle.closed_form(curve, k, d)
    assert np.array_equal(got, want)
    del pts
    torch.cuda.empty_cache()


@pytest.mark.parametrize("curve,dist", [("mnt4_753", "uniform"), ("mnt4_753", "zcash_like")])
def test_mnt4_window_invariance_at_bench_c(curve, dist):
    """MNT4-753's standard path at the benched c = 16 (and c = 13, the 2^16
    plan, and small c) for several chunk sizes: same bytes as the closed form."""
    gz = require_cuda()
    from tests.fixtures import oracle_points
    n = 2000
    pts, d = oracle_points(curve, 2048)
    pts, d = pts[:n], d[:n]
    k = synth.scalars(curve, n, 33, dist)
    want = oracle.closed_form(curve, k, d)
    try:
        for c in (4, 13, 16, 18):
            for S in (1, 16, 64, 257):
                gz.set_config(c, S)
                assert np.array_equal(host(gz.msm(curve, dev(pts), dev(k))), want), (c, S)
    finally:
        gz.set_config(0, 0)
