"""Multi-process execution of the sharded MSM on the GPU (`-m gpu`,
SURVEY.md §8(e); "sub-MSM tasks" per GPU).

* Two processes, one shard each, through the product's partial/combine ABI:
  every rank runs gzkp_msm_partial on its contiguous shard, the XYZZ partials
  (gzkp_partial_bytes each) cross the process boundary through a gloo
  all-gather, and every rank folds them in rank order with
  gzkp_combine_partials.  Runs on a single GPU (both ranks on cuda:0) and
  checks that both ranks hold identical bytes equal to the oracle.
* With >= 2 GPUs: two ranks on two GPUs through gzkp_msm_sharded and
  gzkp_msm_prepared_sharded, i.e. the real NCCL all-gather (skipped on a
  1-GPU box: NCCL refuses two ranks on one device).
"""

import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _inputs(curve, n):
    import synth
    from tests.fixtures import oracle_points
    pts, d = oracle_points(curve, 1024)
    idx = np.arange(n) % 1024
    k = synth.scalars(curve, n, 606, "zcash_like" if curve == "bls12_381" else "uniform")
    return pts[idx], d[idx], k


def _partials_worker(rank, world, port, curve, n, q):
    import sys
    sys.path.insert(0, ROOT)
    try:
        import torch
        import torch.distributed as dist

        import paper_conf_asplos_maxsm0k0zsh23_b200 as gz
        from tests.gpu_util import dev, host
        ndev = torch.cuda.device_count()
        torch.cuda.set_device(rank % ndev)
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", world_size=world, rank=rank)
        pts, _, k = _inputs(curve, n)
        lo, hi = gz.shard_range(n, world, rank)
        part = gz.msm_partial(curve, dev(pts[lo:hi]), dev(k[lo:hi]))
        torch.cuda.synchronize()
        mine = torch.from_numpy(host(part).view(np.int32).copy())
        parts = [torch.empty_like(mine) for _ in range(world)]
        dist.all_gather(parts, mine)                    # partial bytes cross the process boundary
        out = host(gz.combine_partials(curve, torch.stack(parts).cuda()))
        torch.cuda.synchronize()
        q.put((rank, out.tobytes(), None))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover - surfaced by the asserts
        import traceback
        q.put((rank, None, traceback.format_exc() + repr(e)))


def _nccl_worker(rank, world, port, curve, n, q):
    import sys
    sys.path.insert(0, ROOT)
    try:
        import torch
        import torch.distributed as dist

        import paper_conf_asplos_maxsm0k0zsh23_b200 as gz
        from tests.gpu_util import dev, host
        torch.cuda.set_device(rank)
        dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", world_size=world, rank=rank)
        comm = gz.Comm(world, rank)                     # NCCL unique id via the torch group
        pts, _, k = _inputs(curve, n)
        lo, hi = gz.shard_range(n, world, rank)
        outs = [host(gz.msm_sharded(curve, dev(pts[lo:hi]), dev(k[lo:hi]), comm)).tobytes()]
        for weighted in (True, False):
            h = gz.PreparedPoints(curve, dev(pts[lo:hi]), weighted=weighted)
            outs.append(host(gz.msm_prepared_sharded(h, dev(k[lo:hi]), comm)).tobytes())
            h.release()
        torch.cuda.synchronize()
        comm.destroy()
        q.put((rank, outs, None))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        import traceback
        q.put((rank, None, traceback.format_exc() + repr(e)))


def _spawn(target, world, *args):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=target, args=(r, world, port) + args + (q,)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=600) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
    for rank, _, err in res:
        assert err is None, f"rank {rank}: {err}"
    return sorted(res)


def _want(curve, n):
    import oracle
    pts, d, k = _inputs(curve, n)
    return oracle.closed_form(curve, k, d)


@pytest.mark.parametrize("curve,n,world", [("bn254", 3001, 2), ("bls12_381", 5000, 2), ("bls12_381", 4099, 3)])
def test_multiprocess_partials_gloo_exchange(curve, n, world):
    from tests.gpu_util import require_cuda
    require_cuda()
    res = _spawn(_partials_worker, world, curve, n)
    want = _want(curve, n).tobytes()
    for rank, out, _ in res:
        assert out == want, rank


def test_two_rank_nccl_sharded():
    from tests.gpu_util import require_cuda
    require_cuda()
    import torch
    if torch.cuda.device_count() < 2:
        pytest.skip("needs 2 GPUs (NCCL: one rank per device)")
    curve, n = "bls12_381", 6000
    res = _spawn(_nccl_worker, 2, curve, n)
    want = _want(curve, n).tobytes()
    for rank, outs, _ in res:
        for i, o in enumerate(outs):
            assert o == want, (rank, i)
