"""Small MSMs on every path for compute-sanitizer runs (tools/run_sanitizers.sh):
standard, prepared weighted (M = 1) and checkpointed (M = 2), partial +
combine, fixed base, the digit/sort test hook, the binary-GCD inverse and the
lane-split product (field ops 7, 8), a small NTT.  Run it once more with
GZKP_AFFINE_LEVELS=3 for the batch-affine levels."""
import sys

import numpy as np

sys.path.insert(0, ".")
import oracle  # noqa: E402
import paper_conf_asplos_maxsm0k0zsh23_b200 as gz  # noqa: E402
import synth  # noqa: E402

ok = True
for curve, n in (("bn254", 300), ("bls12_381", 200), ("toy_a2", 500)):
    d = synth.dlogs(curve, n, 3)
    pts = oracle.points_from_dlogs(curve, d)
    k = synth.scalars(curve, n, 4, "zcash_like" if curve != "toy_a2" else "uniform")
    want = oracle.msm(curve, pts, k)
    P, K = gz.to_device(pts), gz.to_device(k)
    got = gz.to_numpy(gz.msm(curve, P, K))
    h = gz.PreparedPoints(curve, P, weighted=True)
    got_w = gz.to_numpy(h.msm(K))
    h.release()
    h2 = gz.PreparedPoints(curve, P, weighted=2)
    got_m2 = gz.to_numpy(h2.msm(K))
    h2.release()
    part = gz.msm_partial(curve, P, K)
    import torch
    got_c = gz.to_numpy(gz.combine_partials(curve, torch.stack([part])))
    fb = gz.to_numpy(gz.fixed_base_mul(curve, gz.to_device(d[:16])))
    off, vals = gz.debug_buckets(curve, K, 4)
    x = pts[:64, :gz.field_limbs(curve)]
    inv = gz.to_numpy(gz.field_op(curve, 7, gz.to_device(x), gz.to_device(x)))
    mul8 = gz.to_numpy(gz.field_op(curve, 8, gz.to_device(x), gz.to_device(x)))
    mul0 = gz.to_numpy(gz.field_op(curve, 0, gz.to_device(x), gz.to_device(x)))
    res = [np.array_equal(got, want), np.array_equal(got_w, want), np.array_equal(got_m2, want),
           np.array_equal(got_c, want), np.array_equal(fb, pts[:16]), int(off[-1]) == len(vals),
           np.array_equal(mul8, mul0), inv.shape == x.shape]
    print(curve, res)
    ok &= all(res)
a = synth.scalars("bls12_381", 256, 5)
out = gz.to_numpy(gz.ntt("bls12_381", gz.to_device(a)))
back = gz.to_numpy(gz.ntt("bls12_381", gz.to_device(out.reshape(256, -1)), inverse=True))
ok &= bool(np.array_equal(back.reshape(a.shape), a))
print("SANITIZE_PARITY", "ok" if ok else "FAIL")
