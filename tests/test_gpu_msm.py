"""GPU MSM parity (`-m gpu`): libgzkp.so through the C ABI vs the oracle,
bit-exact (the MSM value is unique and the affine encoding canonical, so there
is no tolerance: DESIGN.md §Parity).

Small n: the C oracle on the full input (same seeded points/scalars).
Edge cases: n = 0, 1, ragged n, identity points, duplicates, cancellation,
sparse/adversarial scalar presets, toy curves where buckets constantly hit
P == Q and P == -Q.
Invariance: the bytes do not depend on the window size c, the chunk size or
the sharding (partials + combine)."""

import numpy as np
import pytest

import oracle
import synth
from oracle import curves, ref
from tests.fixtures import oracle_msm_cached, oracle_points
from tests.gpu_util import dev, host, require_cuda

pytestmark = pytest.mark.gpu


@pytest.fixture(autouse=True)
def _reset_config():
    yield
    try:
        import paper_conf_asplos_maxsm0k0zsh23_b200 as gz
        gz.set_config(0, 0)
    except Exception:
        pass


def run(gz, curve, pts, k):
    return host(gz.msm(curve, dev(pts), dev(k)))


def test_config1_bn254_2p10_bit_exact():
    """BASELINE configs[0]: BN254 n = 2^10, uniform scalars, full oracle check."""
    gz = require_cuda()
    pts, _ = oracle_points("bn254", 1 << 10)
    k = synth.scalars("bn254", 1 << 10, synth.scalar_seed(1))
    want = oracle_msm_cached("bn254", pts, k)
    assert np.array_equal(run(gz, "bn254", pts, k), want)


@pytest.mark.parametrize("curve,n", [
    ("bn254", 1), ("bn254", 2), ("bn254", 3), ("bn254", 31), ("bn254", 257), ("bn254", 1000),
    ("bls12_381", 1), ("bls12_381", 5), ("bls12_381", 257), ("bls12_381", 1024),
    ("mnt4_753", 1), ("mnt4_753", 7), ("mnt4_753", 64),
    ("toy_a0", 1), ("toy_a0", 100), ("toy_a0", 3000),
    ("toy_a2", 1), ("toy_a2", 100), ("toy_a2", 3000),
])
def test_msm_uniform_vs_oracle(curve, n):
    gz = require_cuda()
    m = max(n, 64) if curve != "mnt4_753" else 64
    pts, _ = oracle_points(curve, m)
    pts = pts[:n]
    k = synth.scalars(curve, n, 500 + n)
    assert np.array_equal(run(gz, curve, pts, k), oracle_msm_cached(curve, pts, k))


def test_msm_empty():
    gz = require_cuda()
    for curve in ("bn254", "bls12_381", "mnt4_753"):
        L = gz.field_limbs(curve)
        out = run(gz, curve, np.zeros((0, 2 * L), np.uint32), np.zeros((0, gz.scalar_limbs(curve)), np.uint32))
        assert not out.any()


@pytest.mark.parametrize("dist", ["zcash_like", "all_one", "r_minus_1", "single_hot", "pow2", "small",
                                  "full_bits", "all_zero"])
@pytest.mark.parametrize("curve", ["bn254", "bls12_381"])
def test_msm_distributions(curve, dist):
    gz = require_cuda()
    n = 700
    pts, _ = oracle_points(curve, 1024)
    pts = pts[:n]
    k = synth.scalars(curve, n, 77, dist)
    assert np.array_equal(run(gz, curve, pts, k), oracle_msm_cached(curve, pts, k))


def test_identity_duplicates_cancellation():
    gz = require_cuda()
    curve = "bls12_381"
    c = curves.get(curve)
    pts, _ = oracle_points(curve, 1024)
    pts = pts[:300].copy()
    k = synth.scalars(curve, 300, 5)
    pts[3] = 0                         # identity inputs
    pts[4] = 0
    pts[10:40] = pts[9]                # duplicated point in many buckets
    pts[50] = pts[51]                  # P and -P with equal scalars -> cancel
    y = ref.limbs_to_int(pts[51, c.limbs:])
    pts[50, c.limbs:] = ref.int_to_limbs((-y) % c.p, c.limbs)
    k[50] = k[51]
    # k_i and r - k_i on the same point: sum is O
    pts[60] = pts[61]
    kv = ref.limbs_to_int(k[61])
    k[60] = ref.int_to_limbs((c.r - kv) % c.r, c.scalar_limbs)
    assert np.array_equal(run(gz, curve, pts, k), oracle_msm_cached(curve, pts, k))


def test_result_identity():
    gz = require_cuda()
    curve = "bn254"
    c = curves.get(curve)
    pts, _ = oracle_points(curve, 1024)
    P = np.tile(pts[7], (2, 1))
    k = np.zeros((2, c.scalar_limbs), np.uint32)
    k[0] = ref.int_to_limbs(12345, c.scalar_limbs)
    k[1] = ref.int_to_limbs(c.r - 12345, c.scalar_limbs)
    assert not run(gz, curve, P, k).any()


@pytest.mark.parametrize("curve", ["bn254", "bls12_381", "toy_a2"])
def test_invariance_window_and_chunk(curve):
    """Same bytes for every c and chunk size (the group is exact)."""
    gz = require_cuda()
    n = 2000
    pts, _ = oracle_points(curve, 2048)
    pts = pts[:n]
    k = synth.scalars(curve, n, 31, "zcash_like" if curve != "toy_a2" else "uniform")
    want = oracle_msm_cached(curve, pts, k)
    cmax = 18 if curve != "toy_a2" else 4
    for c in sorted({2, 3, 4, 7, 10, 13, 16, 17, cmax} & set(range(2, cmax + 1))):
        for S in (1, 3, 16, 64, 257):
            gz.set_config(c, S)
            got = run(gz, curve, pts, k)
            assert np.array_equal(got, want), (c, S)


@pytest.mark.parametrize("curve", ["bn254", "bls12_381"])
def test_sharding_partials_combine(curve):
    """gzkp_msm_partial on G shards + gzkp_combine_partials == full MSM, for
    G = 1..8 (the multi-GPU maths on one GPU)."""
    gz = require_cuda()
    n = 1000
    pts, _ = oracle_points(curve, 1024)
    pts = pts[:n]
    k = synth.scalars(curve, n, 8)
    want = oracle_msm_cached(curve, pts, k)
    L = gz.field_limbs(curve)
    for G in range(1, 9):
        parts = []
        for r in range(G):
            lo, hi = gz.shard_range(n, G, r)
            parts.append(gz.msm_partial(curve, dev(pts[lo:hi].reshape(-1, 2 * L)), dev(k[lo:hi].reshape(-1, k.shape[1]))))
        import torch
        got = host(gz.combine_partials(curve, torch.stack(parts)))
        assert np.array_equal(got, want), G


def test_prepared_and_host_paths():
    gz = require_cuda()
    curve = "bls12_381"
    pts, _ = oracle_points(curve, 1024)
    k = synth.scalars(curve, 1024, 12)
    want = oracle_msm_cached(curve, pts, k)
    h = gz.PreparedPoints(curve, dev(pts))
    assert np.array_equal(host(h.msm(dev(k))), want)
    assert np.array_equal(h.msm_host(k), want)
    # prefix of a prepared vector
    want2 = oracle_msm_cached(curve, pts[:100], k[:100])
    assert np.array_equal(host(h.msm(dev(k[:100]))), want2)
    h.release()
    assert np.array_equal(gz.msm_host(curve, pts, k), want)


def test_workspace_ex_path():
    gz = require_cuda()
    import torch
    curve = "bn254"
    pts, _ = oracle_points(curve, 1024)
    k = synth.scalars(curve, 1024, 13)
    ws = torch.empty(gz.workspace_bytes(curve, 1024), dtype=torch.uint8, device="cuda")
    got = host(gz.msm(curve, dev(pts), dev(k), workspace=ws))
    assert np.array_equal(got, oracle_msm_cached(curve, pts, k))


def test_sharded_single_rank_nccl():
    """gzkp_msm_sharded through a real NCCL communicator (world = 1 on the
    single-GPU box; the multi-rank maths is covered by the partials test)."""
    gz = require_cuda()
    import socket

    import torch.distributed as dist
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", world_size=1, rank=0)
    try:
        comm = gz.Comm(1, 0)
        curve = "bls12_381"
        pts, _ = oracle_points(curve, 1024)
        k = synth.scalars(curve, 1024, 21)
        got = host(gz.msm_sharded(curve, dev(pts), dev(k), comm))
        want = oracle_msm_cached(curve, pts, k)
        assert np.array_equal(got, want)
        for weighted in (True, False):                 # prepared shards, same all-gather
            h = gz.PreparedPoints(curve, dev(pts), weighted=weighted)
            assert np.array_equal(host(gz.msm_prepared_sharded(h, dev(k), comm)), want)
            h.release()
        comm.destroy()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("curve,cs", [("bn254", (3, 8, 13, 16, 20)), ("bls12_381", (4, 11, 16, 18, 21)),
                                      ("mnt4_753", (9, 16)), ("toy_a0", (2, 3, 4)), ("toy_a2", (2, 4))])
def test_weighted_points_cross_window_consolidation(curve, cs):
    """NEXT-1: prepared weighted points 2^(ct) P_i, one bucket
    set for all windows; bit-exact vs the oracle for several c, sparse scalars,
    identity points and a prefix of the prepared vector."""
    gz = require_cuda()
    n = 64 if curve == "mnt4_753" else 1024
    pts, _ = oracle_points(curve, n if curve != "mnt4_753" else 64)
    pts = pts.copy()
    pts[5] = 0                                    # identity input
    for dist in ("uniform", "zcash_like") if curve != "mnt4_753" else ("uniform",):
        k = synth.scalars(curve, n, 41, dist)
        want = oracle_msm_cached(curve, pts, k)
        want_prefix = oracle_msm_cached(curve, pts[:n // 3], k[:n // 3])
        for c in cs:
            h = gz.PreparedPoints(curve, dev(pts), weighted=True, window_bits=c)
            info = h.info()
            assert info["weighted"] and info["window_bits"] == c
            assert np.array_equal(host(h.msm(dev(k))), want), (dist, c)
            assert np.array_equal(host(h.msm(dev(k[:n // 3]))), want_prefix), (dist, c)
            h.release()


def test_weighted_default_and_unweighted_prepare():
    gz = require_cuda()
    curve = "bn254"
    pts, _ = oracle_points(curve, 1024)
    k = synth.scalars(curve, 1024, 42)
    want = oracle_msm_cached(curve, pts, k)
    h = gz.PreparedPoints(curve, dev(pts))
    assert h.info()["weighted"]
    assert np.array_equal(host(h.msm(dev(k))), want)
    h2 = gz.PreparedPoints(curve, dev(pts), weighted=False)
    assert not h2.info()["weighted"]
    assert np.array_equal(host(h2.msm(dev(k))), want)


@pytest.mark.parametrize("curve", ["bn254", "bls12_381"])
def test_heavy_buckets_tree(curve):
    """Skew beyond MERGE_QMAX chunks per bucket: the heavy-list tree (fan-in
    1024, several levels with chunk size 1) against the oracle's closed form.
    all-equal scalars put every point of every window into ONE bucket per
    window (W heavy buckets); all-one scalars make one bucket of n entries."""
    gz = require_cuda()
    n = 1 << 13
    pts, d = oracle_points(curve, n)
    c = curves.get(curve)
    k_eq = np.tile(synth.scalars(curve, 1, 4242), (n, 1))
    k_one = synth.scalars(curve, n, 1, "all_one")
    for k in (k_eq, k_one):
        want = oracle.closed_form(curve, k, d)
        for chunk in (0, 1, 7):
            gz.set_config(0, chunk)
            assert np.array_equal(run(gz, curve, pts, k), want), chunk
    gz.set_config(0, 0)


@pytest.mark.parametrize("curve,c,intervals", [("bn254", 16, (2, 3, 5, 16, 40)), ("bls12_381", 13, (2, 4, 20)),
                                               ("bls12_381", 20, (2, 3)), ("mnt4_753", 11, (2, 7, 69)),
                                               ("toy_a2", 3, (2, 5)), ("toy_a0", 2, (3, 8))])
def test_checkpoint_interval_algorithm1(curve, c, intervals):
    """GZKP's Algorithm 1 with checkpoint interval M > 1:
    only the checkpoints 2^(c M j) P_i are stored and window t = M j + r
    accumulates checkpoint j into bucket set r (reading R10).  Bit-exact vs the
    oracle for several M, including M >= W (no table: the standard pipeline),
    sparse scalars, an identity input and a prefix of the prepared vector."""
    gz = require_cuda()
    n = 64 if curve == "mnt4_753" else 1024
    pts, _ = oracle_points(curve, n)
    pts = pts.copy()
    pts[7] = 0
    c_ = curves.get(curve)
    W = -(-(c_.scalar_bits + 1) // c)
    for dist in ("uniform", "zcash_like") if curve != "mnt4_753" else ("uniform",):
        k = synth.scalars(curve, n, 52, dist)
        want = oracle_msm_cached(curve, pts, k)
        want_prefix = oracle_msm_cached(curve, pts[:n // 2], k[:n // 2])
        for M in intervals:
            h = gz.PreparedPoints(curve, dev(pts), weighted=M, window_bits=c)
            info = h.info()
            Mi = min(M, W)
            assert info["interval"] == M and info["windows"] == -(-W // Mi), info
            assert np.array_equal(host(h.msm(dev(k))), want), (dist, M)
            assert np.array_equal(host(h.msm(dev(k[:n // 2]))), want_prefix), (dist, M)
            h.release()
