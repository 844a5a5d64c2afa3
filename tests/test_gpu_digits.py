"""Direct tests of the digit + sort stage (a2-a3) through the test hook
gzkp_debug_buckets (`-m gpu`): the bucket layout the accumulation consumes.

* PAPER.md:154 (§2.3, Figure 3): N = 8, k = 4, l = 256; in window w0 the points
  whose scalar's low hex digit is 5 (P0, P3, P5) land in bucket 5
  (tests/golden/fig3_bucket_example.txt).  Under the signed digits of DESIGN.md
  reading R7 the digit 0xA becomes -6 (+1 carried into w1), so bucket "A" of
  the figure is bucket 6 with a negative sign.
* Reconstruction: for every point i, the signed digits found in the buckets
  satisfy sum_t d_t 2^(c t) = k_i exactly, each window holds each point at
  most once, and no digit is zero (any c, any scalar preset).
"""

import os

import numpy as np
import pytest

import synth
from tests.gpu_util import dev, require_cuda

pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "fig3_bucket_example.txt")
NEG = 0x80000000


def _load_fig3():
    rows, expect = [], {}
    for line in open(GOLDEN):
        line = line.strip()
        if line.startswith("# expected:"):
            for part in line[len("# expected:"):].split(";"):
                k, v = part.split("=")
                expect[k.strip()] = [int(x) for x in v.split()]
        elif line and not line.startswith("#"):
            i, nib = line.split()
            rows.append((int(i), int(nib)))
    return rows, expect


def _buckets(off, vals, B, t):
    """{magnitude: sorted [(index, negative)]} of window t"""
    out = {}
    for j in range(B):
        lo, hi = int(off[t * B + j]), int(off[t * B + j + 1])
        if hi > lo:
            out[j + 1] = sorted((int(v) & ~NEG, bool(v & NEG)) for v in vals[lo:hi])
    return out


@pytest.mark.parametrize("curve", ["bn254", "bls12_381"])
def test_fig3_bucket_membership(curve):
    gz = require_cuda()
    rows, expect = _load_fig3()
    n = len(rows)
    k = synth.scalars(curve, n, 154)
    for i, nib in rows:                      # the figure fixes only the low hex digit
        k[i, 0] = (k[i, 0] & ~np.uint32(0xF)) | np.uint32(nib)
    off, vals = gz.debug_buckets(curve, dev(k), 4)
    B = 8
    w0 = _buckets(off, vals, B, 0)
    assert [i for i, neg in w0[5]] == expect["bucket5"] and not any(neg for _, neg in w0[5])
    # 0xA = 10 > 2^(k-1): signed digit -6, the figure's bucket A
    assert [i for i, neg in w0[6]] == expect["bucket10"] and all(neg for _, neg in w0[6])
    # the figure's 64 windows at k = 4 and l = 256: W = ceil((b+1)/c) = 64 for
    # b = 254 (BN254) and b = 255 (BLS12-381) (reading R7)
    assert (len(off) - 1) // B == 64


@pytest.mark.parametrize("curve,c", [("bn254", 2), ("bn254", 5), ("bn254", 16), ("bls12_381", 13),
                                     ("bls12_381", 16), ("bls12_381", 18), ("mnt4_753", 16), ("toy_a2", 3)])
@pytest.mark.parametrize("dist", ["uniform", "zcash_like", "r_minus_1", "full_bits", "small", "pow2"])
def test_digits_reconstruct_scalars(curve, c, dist):
    gz = require_cuda()
    n = 1500
    k = synth.scalars(curve, n, 9000 + c, dist, c=c)
    off, vals = gz.debug_buckets(curve, dev(k), c)
    B = 1 << (c - 1)
    M = len(off) - 1
    W = M // B
    assert M == W * B and np.all(np.diff(off.astype(np.int64)) >= 0)
    recon = [0] * n
    for t in range(W):
        seen = set()
        for j in range(B):
            lo, hi = int(off[t * B + j]), int(off[t * B + j + 1])
            for v in vals[lo:hi]:
                i = int(v) & ~NEG
                assert 0 <= i < n and i not in seen
                seen.add(i)
                d = -(j + 1) if int(v) & NEG else (j + 1)
                recon[i] += d << (c * t)
    want = [sum(int(w) << (32 * q) for q, w in enumerate(row)) for row in k]
    assert recon == want


def test_debug_checks_reject_bad_inputs():
    """GZKP_DEBUG_CHECKS=1 (read once per process, so a subprocess): a point off
    the curve, a coordinate >= p and a scalar >= 2^b each give
    GZKP_ERROR_INVALID_VALUE before any MSM work; valid inputs pass."""
    require_cuda()
    import subprocess
    import sys
    code = r'''
import sys, numpy as np
sys.path.insert(0, %r)
import paper_conf_asplos_maxsm0k0zsh23_b200 as gz, synth
from tests.fixtures import oracle_points
from tests.gpu_util import dev
pts, d = oracle_points("bls12_381", 64)
k = synth.scalars("bls12_381", 64, 3)
gz.msm("bls12_381", dev(pts), dev(k))                  # valid: passes
res = []
bad = pts.copy(); bad[7, 0] ^= 1                        # off the curve
bad2 = pts.copy(); bad2[9, :12] = [0xffffaaab, 0xb9feffff, 0xb153ffff, 0x1eabfffe, 0xf6b0f624, 0x6730d2a0,
                                   0xf38512bf, 0x64774b84, 0x434bacd7, 0x4b1ba7b6, 0x397fe69a, 0x1a0111ea]  # x = p
badk = k.copy(); badk[3, 7] |= 0x80000000               # bit 255 set: >= 2^b
for P, K in ((bad, k), (bad2, k), (pts, badk)):
    try:
        gz.msm("bls12_381", dev(P), dev(K)); res.append("ok")
    except gz.GzkpError as e:
        res.append(str(e))
h = None
try:
    h = gz.PreparedPoints("bls12_381", dev(bad)); res.append("ok")
except gz.GzkpError as e:
    res.append(str(e))
print("RESULT", res)
''' % os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, GZKP_DEBUG_CHECKS="1")
    out = subprocess.run([sys.executable, "-c", code], capture_output=True, text=True, env=env, timeout=600)
    assert out.returncode == 0, out.stderr[-3000:]
    line = [x for x in out.stdout.splitlines() if x.startswith("RESULT")][0]
    res = eval(line[len("RESULT "):])
    assert "not on the curve" in res[0]
    assert ">= p" in res[1]
    assert "scalar is >= 2^b" in res[2]
    assert "not on the curve" in res[3]
