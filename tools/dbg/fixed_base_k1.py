import sys, numpy as np
sys.path.insert(0, '.')
from oracle import ref, curves
import paper_conf_asplos_maxsm0k0zsh23_b200 as gz
c = 'mnt4_753'; C = curves.get(c); p = C.p; R = 1 << (32 * 24)
d = np.array([ref.int_to_limbs(1, 24)], dtype=np.uint32)
a = gz.to_numpy(gz.fixed_base_mul(c, gz.to_device(d)))[0]
x, y = ref.limbs_to_int(a[:24]), ref.limbs_to_int(a[24:])
print("x", hex(x)[:40], "y", hex(y)[:40])
for nm, f in [("R", R % p), ("Rinv", pow(R, -1, p)), ("R2", R * R % p), ("1", 1)]:
    print(nm, x == C.gx * f % p, y == C.gy * f % p)
# also via ec_op: G + O through madd, and 2G
G = np.array([ref.encode_point(C, (C.gx, C.gy))], dtype=np.uint32)
Z = np.zeros_like(G)
for op in range(4):
    o = gz.to_numpy(gz.ec_op(c, op, gz.to_device(G), gz.to_device(Z)))[0]
    print("ec_op", op, ref.decode_point(C, o) == (ref.add(C, (C.gx, C.gy), None) if op < 2 else ref.add(C, (C.gx, C.gy), (C.gx, C.gy))))
