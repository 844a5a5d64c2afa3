"""Small MSMs on every path (standard, prepared weighted, partial+combine,
fixed base) for compute-sanitizer runs: tools/run_sanitizers.sh."""
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
    part = gz.msm_partial(curve, P, K)
    import torch
    got_c = gz.to_numpy(gz.combine_partials(curve, torch.stack([part])))
    fb = gz.to_numpy(gz.fixed_base_mul(curve, gz.to_device(d[:16])))
    res = [np.array_equal(got, want), np.array_equal(got_w, want), np.array_equal(got_c, want),
           np.array_equal(fb, pts[:16])]
    print(curve, res)
    ok &= all(res)
print("SANITIZE_PARITY", "ok" if ok else "FAIL")
