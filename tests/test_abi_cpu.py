"""CPU-only checks of the C-ABI boundary (`-m "not gpu"`): the library builds
for sm_100a, loads, exports every symbol include/gzkp.h declares, and its
host-only entry points (sizes, planner, status strings) answer correctly.
No compute call is made here (no GPU in this container)."""

import ctypes
import os
import re
import subprocess

import pytest

import paper_conf_asplos_maxsm0k0zsh23_b200 as gz
from paper_conf_asplos_maxsm0k0zsh23_b200 import build as gbuild

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "gzkp.h")


@pytest.fixture(scope="module")
def lib():
    gbuild.build()
    return gz.lib()


def declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"\b(gzkp_[a-z0-9_]+)\s*\(", src)
    return sorted(set(names))


def test_header_declares_core_entry_points():
    names = declared_functions()
    for must in ["gzkp_msm", "gzkp_msm_ex", "gzkp_msm_sharded", "gzkp_msm_partial", "gzkp_combine_partials",
                 "gzkp_points_prepare", "gzkp_msm_prepared", "gzkp_comm_init", "gzkp_nccl_unique_id"]:
        assert must in names


def test_every_declared_symbol_exported(lib):
    out = subprocess.run(["nm", "-D", "--defined-only", gz.LIB_PATH], capture_output=True, text=True, check=True).stdout
    exported = set(re.findall(r"\bT (gzkp_\w+)", out))
    missing = [n for n in declared_functions() if n not in exported]
    assert not missing, missing
    for n in declared_functions():
        assert hasattr(lib, n)


def test_library_is_sm100a(lib):
    out = subprocess.run(["cuobjdump", "--list-elf", gz.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_sizes(lib):
    assert lib.gzkp_field_bytes(0) == 32 and lib.gzkp_scalar_bytes(0) == 32
    assert lib.gzkp_field_bytes(1) == 48 and lib.gzkp_scalar_bytes(1) == 32
    assert lib.gzkp_field_bytes(2) == 96 and lib.gzkp_scalar_bytes(2) == 96
    assert lib.gzkp_partial_bytes(1) == 4 * 48
    assert lib.gzkp_field_bytes(100) == 8 and lib.gzkp_scalar_bytes(100) == 4
    assert lib.gzkp_field_bytes(7) == 0


def test_planner_host_only(lib):
    # window size grows with n and stays within the supported range
    cs = [gz.window_bits("bls12_381", 1 << k) for k in (4, 10, 16, 20, 22, 26)]
    assert all(2 <= c <= 18 for c in cs)
    assert cs == sorted(cs)
    assert gz.window_bits("bls12_381", 1 << 22) >= 12
    assert gz.workspace_bytes("bn254", 1 << 20) > (1 << 20) * 64
    gz.set_config(9, 17)
    assert gz.window_bits("bn254", 1 << 20) == 9
    gz.set_config(0, 0)
    with pytest.raises(gz.GzkpError):
        gz.set_config(40, 0)


def test_status_strings(lib):
    assert lib.gzkp_status_string(0) == b"success"
    assert lib.gzkp_status_string(5) == b"NCCL error"


def test_argument_errors_are_synchronous(lib):
    # NULL out / unknown curve are rejected before any CUDA call
    assert lib.gzkp_msm(7, None, None, 0, 16, None) == 2
    assert lib.gzkp_msm(0, None, None, 5, None, None) == 1
    assert lib.gzkp_msm(0, 16, 16, 5, 8, None) == 1          # misaligned out
    assert b"aligned" in lib.gzkp_last_error()


def test_no_cpu_fallback_in_product():
    # the product package never imports the oracle
    pkg = os.path.join(ROOT, "paper_conf_asplos_maxsm0k0zsh23_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                txt = open(os.path.join(dp, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt, f
                assert "oracle.c" not in txt, f
