import sys, numpy as np
sys.path.insert(0, '.')
import oracle
from oracle import ref, curves
import paper_conf_asplos_maxsm0k0zsh23_b200 as gz
c = 'mnt4_753'; C = curves.get(c)
ks = [1, 2, 3, 4, 5, 7, 1 << 40, (1 << 700) + 1]
d = np.array([ref.int_to_limbs(k, 24) for k in ks], dtype=np.uint32)
a = gz.to_numpy(gz.fixed_base_mul(c, gz.to_device(d)))
G = ref.generator(C)
for i, k in enumerate(ks):
    got = ref.decode_point(C, a[i]); want = ref.mul(C, k, G)
    print(k if k < 100 else hex(k)[:12], got == want, ref.on_curve(C, got) if got else None)
