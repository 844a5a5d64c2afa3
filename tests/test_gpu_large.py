"""Full-size parity (`-m gpu`) at BASELINE.json's sizes, in the launch
configuration bench.py times.  The oracle cannot run 2^20+ double-and-adds in
seconds, so (SURVEY.md §8(c) "Parity pins"):

* the points are a_i * G from the product's fixed-base kernel, and a sample of
  them is re-derived by the oracle one by one (pins the generator);
* the MSM result must equal the oracle's closed form (sum k_i a_i mod r) * G;
* linearity: MSM(k) + MSM(1) = MSM(k + 1) via the oracle's affine addition.
"""

import numpy as np
import pytest

import oracle
import synth
from tests.gpu_util import dev, host, require_cuda

pytestmark = pytest.mark.gpu


def _setup(gz, curve, n, seed_cfg, dist="uniform"):
    d = synth.dlogs(curve, n, synth.dlog_seed(curve))
    pts = gz.fixed_base_mul(curve, dev(d))
    k = synth.scalars(curve, n, synth.scalar_seed(seed_cfg), dist)
    # sampled generator check: the oracle recomputes 16 points one by one
    idx = np.random.default_rng(seed_cfg).choice(n, 16, replace=False)
    sample = host(pts[idx.tolist()])
    assert np.array_equal(sample, oracle.points_from_dlogs(curve, d[idx]))
    return d, pts, k


@pytest.mark.parametrize("curve,log_n,cfg,dist", [
    ("bn254", 20, 2, "uniform"),         # configs[1]
    ("bls12_381", 22, 3, "uniform"),     # configs[2]
    ("bls12_381", 20, 5, "zcash_like"),  # sparse preset (configs[4] shape at 2^20)
    ("mnt4_753", 16, 4, "uniform"),      # configs[3] shape at 2^16
])
def test_closed_form_full_size(curve, log_n, cfg, dist):
    gz = require_cuda()
    n = 1 << log_n
    d, pts, k = _setup(gz, curve, n, cfg, dist)
    got = host(gz.msm(curve, pts, dev(k)))
    want = oracle.closed_form(curve, k, d)
    assert np.array_equal(got, want)
    # the same MSM through prepared weighted points (NEXT-1), planner's c
    h = gz.PreparedPoints(curve, pts, weighted=True)
    assert np.array_equal(host(h.msm(dev(k))), want)
    h.release()
