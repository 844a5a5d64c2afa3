"""Parity of the alternate code paths (`-m gpu`), each in its own process
because the switches are read once per process:

* GZKP_DFP=1           hot loop with FP64 (DFP) products (NEXT-2 experiment)
* GZKP_PIPELINE=1      window-group pipeline on a side stream (halving groups)
* GZKP_PIPELINE=2      two equal window groups
* GZKP_ACCUM_THREADS=32  small accumulation CTAs
* GZKP_WINDOW_BITS / GZKP_SEGMENT  planner overrides
* GZKP_REDUCE_GROUPS=R  bucket reduction in R window sub-groups, the Horner
                       tail of each on its own stream
* GZKP_AFFINE_LEVELS=L  batch-affine tree levels before the XYZZ loop
                       (affine.cuh experiment; mnt4 and toy curves included)
* GZKP_ONES=0          the scalar-1 points stay in window 0's bucket 1 (the
                       default sums them apart, k_ones_sum)
* GZKP_SEG_COOP=0      one-thread segment chains in the bucket reduction
                       everywhere (the default runs small reductions on CoopS groups)
* GZKP_CANON=1         the canonical-input hot loop (no Montgomery conversion
                       pass; experiment, measured slower)
"""

import os
import subprocess
import sys

import pytest

from tests.gpu_util import require_cuda

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r"""
import sys, numpy as np
sys.path.insert(0, %r)
import synth
from tests.fixtures import oracle_points, oracle_msm_cached
import paper_conf_asplos_maxsm0k0zsh23_b200 as gz
ok = True
for curve, n, dist in (("bls12_381", 1024, "uniform"), ("bls12_381", 1000, "zcash_like"), ("bn254", 1024, "uniform"),
                       ("toy_a2", 2000, "uniform"), ("toy_a0", 3000, "uniform"), ("mnt4_753", 64, "uniform")):
    pts, _ = oracle_points(curve, {"toy_a2": 2048, "toy_a0": 4096, "mnt4_753": 64}.get(curve, 1024))
    pts = pts[:n]
    k = synth.scalars(curve, n, 91, dist)
    want = oracle_msm_cached(curve, pts, k)
    got = gz.to_numpy(gz.msm(curve, gz.to_device(pts), gz.to_device(k)))
    h = gz.PreparedPoints(curve, gz.to_device(pts), weighted=True)
    got_w = gz.to_numpy(h.msm(gz.to_device(k)))
    ok &= bool(np.array_equal(got, want)) and bool(np.array_equal(got_w, want))
print("VARIANT_OK" if ok else "VARIANT_FAIL")
""" % ROOT


@pytest.mark.parametrize("env", [{"GZKP_DFP": "1"}, {"GZKP_PIPELINE": "1"}, {"GZKP_PIPELINE": "2"}, {"GZKP_ACCUM_THREADS": "32"},
                                 {"GZKP_WINDOW_BITS": "11", "GZKP_SEGMENT": "5"},
                                 {"GZKP_DFP": "1", "GZKP_PIPELINE": "1", "GZKP_ACCUM_THREADS": "64"},
                                 {"GZKP_AFFINE_LEVELS": "3"}, {"GZKP_AFFINE_LEVELS": "12"},
                                 {"GZKP_AFFINE_LEVELS": "2", "GZKP_WINDOW_BITS": "5"},
                                 {"GZKP_REDUCE_GROUPS": "3"}, {"GZKP_REDUCE_GROUPS": "16"},
                                 {"GZKP_REDUCE_GROUPS": "2", "GZKP_PIPELINE": "1"},
                                 {"GZKP_CANON": "1"}, {"GZKP_CANON": "1", "GZKP_PIPELINE": "2"},
                                 {"GZKP_SEG_COOP": "0"}, {"GZKP_ONES": "0"}],
                         ids=lambda e: ",".join(f"{k}={v}" for k, v in e.items()))
def test_variant_parity(env):
    require_cuda()
    r = subprocess.run([sys.executable, "-c", SCRIPT], cwd=ROOT, env={**os.environ, **env},
                       capture_output=True, text=True, timeout=600)
    assert "VARIANT_OK" in r.stdout, r.stdout + r.stderr
