"""Helpers for the `-m gpu` parity tests: the CUDA path is called through the
C ABI (libgzkp.so via the package binding); expected values come only from
the oracle (oracle/) on the same seeded inputs (synth/)."""

import numpy as np
import pytest

torch = pytest.importorskip("torch")


def require_cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import os

    import paper_conf_asplos_maxsm0k0zsh23_b200 as gz
    from paper_conf_asplos_maxsm0k0zsh23_b200 import build
    if not os.path.exists(gz.LIB_PATH):
        build.build()
    return gz


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint32).view(np.int32)).cuda()


def host(t):
    return t.cpu().numpy().view(np.uint32)


def int_limbs(values, n):
    return np.array([[(v >> (32 * i)) & 0xFFFFFFFF for i in range(n)] for v in values], dtype=np.uint32).reshape(-1, n)


def limbs_int(row):
    v = 0
    for i, w in enumerate(row):
        v |= int(w) << (32 * i)
    return v
