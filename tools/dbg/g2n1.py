import sys
sys.path.insert(0, ".")
import numpy as np, torch
import oracle, synth
import paper_conf_asplos_maxsm0k0zsh23_b200 as gz
for name, n in (("bls12_381_g2", 1), ("bls12_381_g2", 5), ("mnt4_753", 1), ("mnt4_753", 3)):
    d = synth.dlogs(name, 8, 3)
    pts = oracle.points_from_dlogs(name, d)[:n]
    k = synth.scalars(name, n, 900 + n)
    got = gz.to_numpy(gz.msm(name, gz.to_device(pts), gz.to_device(k)))
    torch.cuda.synchronize()
    print(name, n, np.array_equal(got, oracle.msm(name, pts, k)), flush=True)
