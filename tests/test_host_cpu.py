"""Host-side logic on CPU (`-m "not gpu"`): the binding's argument checks (they
must raise before the C library touches a host pointer), the bench's
multi-GPU self-launch command and rank check, and the Algorithm 1 / planner
bookkeeping exposed without a device."""

import os
import subprocess
import sys

import numpy as np
import pytest

import paper_conf_asplos_maxsm0k0zsh23_b200 as gz

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("pts_shape,sc_shape", [((10, 23), (10, 8)), ((10, 24), (10, 7)), ((10, 24), (9, 8)),
                                                ((10, 24, 1), (10, 8))])
def test_msm_host_rejects_bad_shapes(pts_shape, sc_shape):
    """BLS12-381: points [n, 24], scalars [n, 8]; anything else raises GzkpError
    (gzkp_msm_host would copy n * 96 and n * 32 bytes from the pointers)."""
    with pytest.raises(gz.GzkpError):
        gz.msm_host("bls12_381", np.zeros(pts_shape, np.uint32), np.zeros(sc_shape, np.uint32))


def test_host_u32_accepts_flat_rows():
    a = gz._host_u32(np.arange(48, dtype=np.uint32), 24, "x")
    assert a.shape == (2, 24)


def test_bench_relaunch_command():
    sys.path.insert(0, ROOT)
    import bench
    cmd = bench.relaunch_cmd(8, ["--gpus", "8", "--steps", "3"], 29511)
    assert cmd[1:3] == ["-m", "torch.distributed.run"]
    assert "--nproc-per-node=8" in cmd and "--master-addr=127.0.0.1" in cmd and "--master-port=29511" in cmd
    assert cmd[-4:] == ["--gpus", "8", "--steps", "3"]
    assert os.path.samefile(cmd[-5], os.path.join(ROOT, "bench.py"))


def test_bench_rejects_world_size_mismatch():
    env = dict(os.environ, WORLD_SIZE="2", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "4"], env=env,
                       capture_output=True, text=True, timeout=120)
    assert r.returncode != 0 and "WORLD_SIZE=2 but --gpus 4" in r.stderr


def test_window_bits_planner_ranges():
    """The planner's c (host-only call) stays in the range the sort supports."""
    for curve in ("bn254", "bls12_381", "mnt4_753", "bn254_g2", "bls12_381_g2"):
        for logn in (0, 5, 10, 16, 19, 20, 22, 26):
            c = gz.window_bits(curve, 1 << logn)
            assert 2 <= c <= 18, (curve, logn, c)
    # the benched configurations keep their measured window sizes
    assert gz.window_bits("bls12_381", 1 << 22) == 16 and gz.window_bits("bls12_381", 1 << 26) == 17
    assert gz.window_bits("bn254", 1 << 20) == 16 and gz.window_bits("mnt4_753", 1 << 20) == 16
