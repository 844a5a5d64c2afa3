import sys, numpy as np, torch
sys.path.insert(0, '.')
import oracle, synth
import paper_conf_asplos_maxsm0k0zsh23_b200 as gz
c = 'mnt4_753'
for n in (1, 4, 64, 1024):
    d = synth.dlogs(c, n, 7)
    a = gz.to_numpy(gz.fixed_base_mul(c, gz.to_device(d)))
    b = gz.to_numpy(gz.fixed_base_mul(c, gz.to_device(d)))
    w = oracle.points_from_dlogs(c, d[:min(n, 64)])
    bad = [i for i in range(min(n, 64)) if not np.array_equal(a[i], w[i])]
    print(n, "deterministic", np.array_equal(a, b), "bad", len(bad), bad[:10])
    # MSM path for the same k*G
    G = oracle.generator_limbs(c).reshape(1, -1)
    for i in range(min(n, 4)):
        m = gz.to_numpy(gz.msm(c, gz.to_device(G), gz.to_device(d[i:i+1])))
        print("   msm k*G == oracle", np.array_equal(m, w[i]), " fixed==oracle", np.array_equal(a[i], w[i]))
