"""B200-native G1 multi-scalar multiplication (GZKP, ASPLOS '23 -> sm_100a).

Thin ctypes binding over libgzkp.so (include/gzkp.h).  Argument marshalling
only: every step of the MSM runs in the library's CUDA kernels.  PyTorch is
used for device memory, streams and process groups.  There is no CPU fallback:
if libgzkp.so is missing or no CUDA device is present the calls raise.
"""

from __future__ import annotations

import ctypes
import os
from typing import Optional

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# GZKP_LIB: an experiment build of the same library (build.py -D... --out ...)
LIB_PATH = os.environ.get("GZKP_LIB") or os.path.join(_HERE, "libgzkp.so")

CURVES = {"bn254": 0, "bls12_381": 1, "mnt4_753": 2, "toy_a0": 100, "toy_a2": 101,
          "bn254_g2": 3, "bls12_381_g2": 4}
NAMES = {v: k for k, v in CURVES.items()}

_lib = None


class GzkpError(RuntimeError):
    pass


def curve_id(curve) -> int:
    if isinstance(curve, int):
        if curve not in NAMES:
            raise ValueError(f"unknown curve id {curve}")
        return curve
    name = getattr(curve, "name", curve)
    return CURVES[name]


def lib():
    """Load libgzkp.so (raises if it was not built -- no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise GzkpError(f"{LIB_PATH} not built; run python -m paper_conf_asplos_maxsm0k0zsh23_b200.build")
        L = ctypes.CDLL(LIB_PATH)
        vp, sz, i32 = ctypes.c_void_p, ctypes.c_size_t, ctypes.c_int
        sigs = {
            "gzkp_field_bytes": ([i32], sz),
            "gzkp_scalar_bytes": ([i32], sz),
            "gzkp_partial_bytes": ([i32], sz),
            "gzkp_msm": ([i32, vp, vp, sz, vp, vp], i32),
            "gzkp_msm_workspace_bytes": ([i32, sz], sz),
            "gzkp_msm_ex": ([i32, vp, vp, sz, vp, vp, sz, vp], i32),
            "gzkp_msm_host": ([i32, vp, vp, sz, vp, vp], i32),
            "gzkp_points_prepare": ([i32, vp, sz, ctypes.POINTER(vp), vp], i32),
            "gzkp_points_prepare_ex": ([i32, vp, sz, i32, i32, ctypes.POINTER(vp), vp], i32),
            "gzkp_prepared_info": ([vp, ctypes.POINTER(i32), ctypes.POINTER(i32), ctypes.POINTER(i32),
                                    ctypes.POINTER(sz)], i32),
            "gzkp_msm_prepared": ([vp, vp, sz, vp, vp], i32),
            "gzkp_msm_prepared_host": ([vp, vp, sz, vp, vp], i32),
            "gzkp_points_release": ([vp], i32),
            "gzkp_msm_partial": ([i32, vp, vp, sz, vp, vp], i32),
            "gzkp_combine_partials": ([i32, vp, i32, vp, vp], i32),
            "gzkp_nccl_unique_id": ([ctypes.c_char_p], i32),
            "gzkp_comm_init": ([i32, i32, ctypes.c_char_p, ctypes.POINTER(vp)], i32),
            "gzkp_comm_destroy": ([vp], i32),
            "gzkp_msm_sharded": ([i32, vp, vp, sz, vp, vp, vp], i32),
            "gzkp_msm_prepared_sharded": ([vp, vp, sz, vp, vp, vp], i32),
            "gzkp_fixed_base_mul": ([i32, vp, sz, vp, vp], i32),
            "gzkp_field_op": ([i32, i32, vp, vp, vp, sz, vp], i32),
            "gzkp_ec_op": ([i32, i32, vp, vp, vp, sz, vp], i32),
            "gzkp_set_config": ([i32, i32], i32),
            "gzkp_window_bits": ([i32, sz], i32),
            "gzkp_set_profiling": ([i32], i32),
            "gzkp_profile_read": ([ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_uint64), i32], i32),
            "gzkp_ntt_max_log": ([i32], i32),
            "gzkp_ntt": ([i32, vp, vp, i32, i32, vp], i32),
            "gzkp_ntt_last_launches": ([], i32),
            "gzkp_scalar_field_op": ([i32, i32, vp, vp, vp, sz, vp], i32),
            "gzkp_release_stream": ([vp], i32),
            "gzkp_debug_buckets": ([i32, vp, sz, i32, ctypes.POINTER(ctypes.c_uint32), sz,
                                    ctypes.POINTER(ctypes.c_uint32), sz, vp], i32),
            "gzkp_status_string": ([i32], ctypes.c_char_p),
            "gzkp_last_error": ([], ctypes.c_char_p),
        }
        for name, (args, res) in sigs.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = res
        _lib = L
    return _lib


def _check(status: int, what: str):
    if status:
        L = lib()
        raise GzkpError(f"{what}: {L.gzkp_status_string(status).decode()} "
                        f"({L.gzkp_last_error().decode()})")


def field_limbs(curve) -> int:
    return lib().gzkp_field_bytes(curve_id(curve)) // 4


def scalar_limbs(curve) -> int:
    return lib().gzkp_scalar_bytes(curve_id(curve)) // 4


def window_bits(curve, n: int) -> int:
    return lib().gzkp_window_bits(curve_id(curve), n)


def workspace_bytes(curve, n: int) -> int:
    return lib().gzkp_msm_workspace_bytes(curve_id(curve), n)


def set_config(window_bits: int = 0, chunk_entries: int = 0):
    _check(lib().gzkp_set_config(window_bits, chunk_entries), "gzkp_set_config")


PHASES = ["sort", "accumulate", "merge", "reduce", "tail"]


def set_profiling(on: bool):
    _check(lib().gzkp_set_profiling(1 if on else 0), "gzkp_set_profiling")


def profile_read(reset: bool = True):
    """Summed per-phase device ms since the last reset (CUDA events recorded on
    the call's stream) and stats of the last call."""
    ms = (ctypes.c_double * 5)()
    st = (ctypes.c_uint64 * 4)()
    _check(lib().gzkp_profile_read(ms, st, 1 if reset else 0), "gzkp_profile_read")
    return {"phase_ms": dict(zip(PHASES, list(ms))), "calls": st[0], "launches": st[1],
            "entries": st[2], "c": st[3]}


# ------------------------------------------------------------ torch plumbing

def _torch():
    import torch
    return torch


def _stream_ptr(stream=None, device=None) -> int:
    """The raw cudaStream_t: `stream` if given, else the current stream of
    `device` (the device of the call's tensors), else of the current device."""
    torch = _torch()
    s = stream if stream is not None else torch.cuda.current_stream(device)
    return s.cuda_stream


def _on(t):
    """Context manager: make the tensor's GPU the current device for the call
    (the library launches on the current device)."""
    return _torch().cuda.device(t.device)


def _host_u32(a, cols: int, name: str) -> np.ndarray:
    """Contiguous [n, cols] u32 host array; the column count must match the
    curve (the C call copies n*cols*4 bytes from the pointer)."""
    a = np.ascontiguousarray(a, dtype=np.uint32)
    if a.ndim == 1 and a.size % cols == 0:
        a = a.reshape(-1, cols)
    if a.ndim != 2 or a.shape[1] != cols:
        raise GzkpError(f"{name}: expected shape [n, {cols}], got {a.shape}")
    return a


def _dev_u32(x, cols: int, name: str):
    """Return a contiguous int32 CUDA tensor viewed as [n, cols] u32 limbs."""
    torch = _torch()
    if isinstance(x, np.ndarray):
        x = torch.from_numpy(np.ascontiguousarray(x, dtype=np.uint32).view(np.int32))
    if not x.is_cuda:
        raise GzkpError(f"{name} must be a CUDA tensor (no CPU path)")
    if x.dtype in (torch.uint8,):
        x = x.view(torch.int32)
    if x.dtype not in (torch.int32, torch.uint32):
        raise GzkpError(f"{name}: expected int32/uint32/uint8 limbs, got {x.dtype}")
    if x.numel() % cols or (x.dim() == 2 and x.shape[1] != cols):
        raise GzkpError(f"{name}: expected [n, {cols}] u32 limbs, got shape {tuple(x.shape)}")
    x = x.contiguous().reshape(-1, cols)
    if x.data_ptr() % 16:
        raise GzkpError(f"{name} must be 16-byte aligned")
    return x


def to_device(a: np.ndarray, device="cuda"):
    torch = _torch()
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint32).view(np.int32)).to(device)


def to_numpy(t) -> np.ndarray:
    return t.detach().cpu().numpy().view(np.uint32)


def msm(curve, points, scalars, out=None, stream=None, workspace=None):
    """Q = sum_i scalars[i] * points[i] on the current CUDA device.

    points: [n, 2L] u32 limbs (canonical affine, (0,0) = O); scalars: [n, Ls].
    Returns a [2L] int32 CUDA tensor (canonical affine, little-endian limbs)."""
    torch = _torch()
    cid = curve_id(curve)
    L, Ls = field_limbs(cid), scalar_limbs(cid)
    P = _dev_u32(points, 2 * L, "points")
    K = _dev_u32(scalars, Ls, "scalars")
    n = P.shape[0]
    if K.shape[0] != n:
        raise GzkpError("points and scalars differ in length")
    if K.device != P.device:
        raise GzkpError("points and scalars are on different devices")
    if out is None:
        out = torch.empty(2 * L, dtype=torch.int32, device=P.device)
    with _on(P):
        if workspace is None:
            st = lib().gzkp_msm(cid, P.data_ptr(), K.data_ptr(), n, out.data_ptr(), _stream_ptr(stream, P.device))
        else:
            st = lib().gzkp_msm_ex(cid, P.data_ptr(), K.data_ptr(), n, out.data_ptr(), workspace.data_ptr(),
                                   workspace.numel() * workspace.element_size(), _stream_ptr(stream, P.device))
    _check(st, "gzkp_msm")
    return out


def msm_host(curve, points: np.ndarray, scalars: np.ndarray, out: Optional[np.ndarray] = None, stream=None):
    """MSM from HOST buffers: copies inside the call (the e2e path)."""
    cid = curve_id(curve)
    L, Ls = field_limbs(cid), scalar_limbs(cid)
    points = _host_u32(points, 2 * L, "points")
    scalars = _host_u32(scalars, Ls, "scalars")
    n = points.shape[0]
    if scalars.shape[0] != n:
        raise GzkpError("points and scalars differ in length")
    if out is None:
        out = np.zeros(2 * L, dtype=np.uint32)
    st = lib().gzkp_msm_host(cid, points.ctypes.data, scalars.ctypes.data, n, out.ctypes.data, _stream_ptr(stream))
    _check(st, "gzkp_msm_host")
    return out


class PreparedPoints:
    """Device-resident Montgomery copy of a fixed point vector."""

    def __init__(self, curve, points, stream=None, weighted=None, window_bits: int = 0):
        """weighted=None: library default (weighted-point table when it fits);
        True/False force GZKP's cross-window consolidation on/off; an int
        M >= 1 selects Algorithm 1's checkpoint interval M (1 = full table)."""
        self.curve = curve_id(curve)
        self.handle = None
        L = field_limbs(self.curve)
        P = _dev_u32(points, 2 * L, "points")
        self.n = P.shape[0]
        self.device = P.device
        h = ctypes.c_void_p()
        with _on(P):
            if weighted is None and window_bits == 0:
                _check(lib().gzkp_points_prepare(self.curve, P.data_ptr(), self.n, ctypes.byref(h),
                                                 _stream_ptr(stream, P.device)), "gzkp_points_prepare")
            else:
                if weighted is None or weighted is True:
                    interval = 1
                elif weighted is False:
                    interval = 0
                else:
                    interval = int(weighted)
                _check(lib().gzkp_points_prepare_ex(self.curve, P.data_ptr(), self.n, window_bits, interval,
                                                    ctypes.byref(h), _stream_ptr(stream, P.device)),
                       "gzkp_points_prepare_ex")
        self.handle = h

    def info(self):
        c, w, wt, b = ctypes.c_int(), ctypes.c_int(), ctypes.c_int(), ctypes.c_size_t()
        _check(lib().gzkp_prepared_info(self.handle, ctypes.byref(c), ctypes.byref(w), ctypes.byref(wt),
                                        ctypes.byref(b)), "gzkp_prepared_info")
        return {"window_bits": c.value, "windows": w.value, "weighted": bool(wt.value), "interval": wt.value,
                "bytes": b.value}

    def msm(self, scalars, out=None, stream=None):
        torch = _torch()
        L, Ls = field_limbs(self.curve), scalar_limbs(self.curve)
        K = _dev_u32(scalars, Ls, "scalars")
        if K.device != self.device:
            raise GzkpError("scalars must be on the prepared points' device")
        if K.shape[0] > self.n:
            raise GzkpError("more scalars than prepared points")
        if out is None:
            out = torch.empty(2 * L, dtype=torch.int32, device=K.device)
        with _on(K):
            _check(lib().gzkp_msm_prepared(self.handle, K.data_ptr(), K.shape[0], out.data_ptr(),
                                           _stream_ptr(stream, K.device)), "gzkp_msm_prepared")
        return out

    def msm_host(self, scalars: np.ndarray, out: Optional[np.ndarray] = None, stream=None):
        L, Ls = field_limbs(self.curve), scalar_limbs(self.curve)
        scalars = _host_u32(scalars, Ls, "scalars")
        if scalars.shape[0] > self.n:
            raise GzkpError("more scalars than prepared points")
        if out is None:
            out = np.zeros(2 * L, dtype=np.uint32)
        with _torch().cuda.device(self.device):
            _check(lib().gzkp_msm_prepared_host(self.handle, scalars.ctypes.data, scalars.shape[0], out.ctypes.data,
                                                _stream_ptr(stream, self.device)), "gzkp_msm_prepared_host")
        return out

    def release(self):
        if getattr(self, "handle", None):
            with _torch().cuda.device(self.device):
                lib().gzkp_points_release(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.release()
        except Exception:
            pass


def msm_partial(curve, points, scalars, out=None, stream=None):
    torch = _torch()
    cid = curve_id(curve)
    L, Ls = field_limbs(cid), scalar_limbs(cid)
    P = _dev_u32(points, 2 * L, "points")
    K = _dev_u32(scalars, Ls, "scalars")
    if K.shape[0] != P.shape[0] or K.device != P.device:
        raise GzkpError("points and scalars differ in length or device")
    if out is None:
        out = torch.empty(4 * L, dtype=torch.int32, device=P.device)
    with _on(P):
        _check(lib().gzkp_msm_partial(cid, P.data_ptr(), K.data_ptr(), P.shape[0], out.data_ptr(),
                                      _stream_ptr(stream, P.device)), "gzkp_msm_partial")
    return out


def combine_partials(curve, partials, out=None, stream=None):
    torch = _torch()
    cid = curve_id(curve)
    L = field_limbs(cid)
    Pt = _dev_u32(partials, 4 * L, "partials")
    if out is None:
        out = torch.empty(2 * L, dtype=torch.int32, device=Pt.device)
    with _on(Pt):
        _check(lib().gzkp_combine_partials(cid, Pt.data_ptr(), Pt.shape[0], out.data_ptr(),
                                           _stream_ptr(stream, Pt.device)), "gzkp_combine_partials")
    return out


def fixed_base_mul(curve, scalars, out=None, stream=None):
    """out[i] = scalars[i] * G (canonical affine) -- synthetic key generation."""
    torch = _torch()
    cid = curve_id(curve)
    L, Ls = field_limbs(cid), scalar_limbs(cid)
    K = _dev_u32(scalars, Ls, "scalars")
    if out is None:
        out = torch.empty((K.shape[0], 2 * L), dtype=torch.int32, device=K.device)
    with _on(K):
        _check(lib().gzkp_fixed_base_mul(cid, K.data_ptr(), K.shape[0], out.data_ptr(), _stream_ptr(stream, K.device)),
               "gzkp_fixed_base_mul")
    return out


def field_op(curve, op: int, a, b, stream=None):
    torch = _torch()
    cid = curve_id(curve)
    L = field_limbs(cid)
    A = _dev_u32(a, L, "a")
    B = _dev_u32(b, L, "b")
    out = torch.empty_like(A)
    with _on(A):
        _check(lib().gzkp_field_op(cid, op, A.data_ptr(), B.data_ptr(), out.data_ptr(), A.shape[0],
                                   _stream_ptr(stream, A.device)), "gzkp_field_op")
    return out


def ec_op(curve, op: int, P, Q, stream=None):
    torch = _torch()
    cid = curve_id(curve)
    L = field_limbs(cid)
    A = _dev_u32(P, 2 * L, "P")
    B = _dev_u32(Q, 2 * L, "Q")
    out = torch.empty_like(A)
    with _on(A):
        _check(lib().gzkp_ec_op(cid, op, A.data_ptr(), B.data_ptr(), out.data_ptr(), A.shape[0],
                                _stream_ptr(stream, A.device)), "gzkp_ec_op")
    return out


# ------------------------------------------------------ NTT over F_r (NEXT-4)

def ntt_max_log(curve) -> int:
    return lib().gzkp_ntt_max_log(curve_id(curve))


def ntt(curve, values, inverse: bool = False, out=None, stream=None):
    """N-NTT over the scalar field of `curve`: out[k] = A(w_N^k),
    or the inverse transform.  values: [N, Ls] u32 limbs (canonical < r) on
    the device, N a power of two.  out may alias values."""
    torch = _torch()
    cid = curve_id(curve)
    Ls = scalar_limbs(cid)
    A = _dev_u32(values, Ls, "values")
    n = A.shape[0]
    log_n = n.bit_length() - 1
    if n != 1 << log_n:
        raise GzkpError("NTT size must be a power of two")
    if out is None:
        out = torch.empty_like(A)
    with _on(A):
        _check(lib().gzkp_ntt(cid, A.data_ptr(), out.data_ptr(), log_n, 1 if inverse else 0,
                              _stream_ptr(stream, A.device)), "gzkp_ntt")
    return out


def ntt_last_launches() -> int:
    return lib().gzkp_ntt_last_launches()


def scalar_field_op(curve, op: int, a, b, stream=None):
    """Elementwise F_r ops (same op codes as field_op) -- tests only."""
    torch = _torch()
    cid = curve_id(curve)
    Ls = scalar_limbs(cid)
    A = _dev_u32(a, Ls, "a")
    B = _dev_u32(b, Ls, "b")
    out = torch.empty_like(A)
    with _on(A):
        _check(lib().gzkp_scalar_field_op(cid, op, A.data_ptr(), B.data_ptr(), out.data_ptr(), A.shape[0],
                                          _stream_ptr(stream, A.device)), "gzkp_scalar_field_op")
    return out


def debug_buckets(curve, scalars, window_bits: int, stream=None):
    """Test hook: the product's digit + sort stage alone (gzkp_debug_buckets).
    Returns (offsets [W 2^(c-1) + 1], vals [E]) as u32 numpy arrays: bucket
    key t 2^(c-1) + |d| - 1 owns vals[offsets[key]:offsets[key+1]], each
    val = point index | 0x80000000 for a negative digit."""
    cid = curve_id(curve)
    Ls = scalar_limbs(cid)
    K = _dev_u32(scalars, Ls, "scalars")
    n = K.shape[0]
    sbits = {0: 254, 1: 255, 2: 753, 3: 254, 4: 255, 100: 14, 101: 14}[cid]
    W = -(-(sbits + 1) // window_bits)
    M = W << (window_bits - 1)
    off = np.zeros(M + 1, dtype=np.uint32)
    vals = np.zeros(max(1, n * W), dtype=np.uint32)
    u32p = ctypes.POINTER(ctypes.c_uint32)
    with _on(K):
        _check(lib().gzkp_debug_buckets(cid, K.data_ptr(), n, window_bits, off.ctypes.data_as(u32p), off.size,
                                        vals.ctypes.data_as(u32p), vals.size, _stream_ptr(stream, K.device)),
               "gzkp_debug_buckets")
    return off, vals[:int(off[-1])]


def release_stream(stream=None):
    """Free the library's cached workspace and side stream for `stream` (call
    before destroying a stream the library was used on)."""
    _check(lib().gzkp_release_stream(_stream_ptr(stream)), "gzkp_release_stream")


# ------------------------------------------------------------- multi-GPU

def broadcast_unique_id(rank: int, group=None) -> bytes:
    """Rank 0 creates the NCCL unique id (gzkp_nccl_unique_id); the default
    torch process group carries the 128 bytes to every rank (plumbing only)."""
    torch = _torch()
    import torch.distributed as dist
    uid = ctypes.create_string_buffer(128)
    if rank == 0:
        _check(lib().gzkp_nccl_unique_id(uid), "gzkp_nccl_unique_id")
    t = torch.frombuffer(bytearray(uid.raw), dtype=torch.uint8).clone()
    if dist.get_backend(group) == "nccl":
        t = t.cuda()
    dist.broadcast(t, src=0, group=group)
    return bytes(t.cpu().numpy().tobytes())


class Comm:
    """NCCL communicator for gzkp_msm_sharded.  The 128-byte unique id is
    broadcast through the default torch process group (plumbing only)."""

    def __init__(self, world: int, rank: int, group=None):
        uid = ctypes.create_string_buffer(broadcast_unique_id(rank, group), 128)
        h = ctypes.c_void_p()
        _check(lib().gzkp_comm_init(world, rank, uid, ctypes.byref(h)), "gzkp_comm_init")
        self.handle = h
        self.world, self.rank = world, rank

    def destroy(self):
        if self.handle:
            lib().gzkp_comm_destroy(self.handle)
            self.handle = None


def shard_range(n: int, world: int, rank: int):
    """Contiguous slice [lo, hi) of rank `rank`."""
    per = (n + world - 1) // world if world else 0
    lo = min(n, rank * per)
    hi = min(n, (rank + 1) * per)
    return lo, hi


def msm_sharded(curve, points_local, scalars_local, comm: Comm, out=None, stream=None):
    torch = _torch()
    cid = curve_id(curve)
    L, Ls = field_limbs(cid), scalar_limbs(cid)
    P = _dev_u32(points_local, 2 * L, "points")
    K = _dev_u32(scalars_local, Ls, "scalars")
    if K.shape[0] != P.shape[0] or K.device != P.device:
        raise GzkpError("points and scalars differ in length or device")
    if out is None:
        out = torch.empty(2 * L, dtype=torch.int32, device=P.device)
    with _on(P):
        _check(lib().gzkp_msm_sharded(cid, P.data_ptr(), K.data_ptr(), P.shape[0], out.data_ptr(),
                                      _stream_ptr(stream, P.device), comm.handle), "gzkp_msm_sharded")
    return out


def msm_prepared_sharded(prepared: "PreparedPoints", scalars_local, comm: Comm, out=None, stream=None):
    """Collective MSM over per-rank prepared shards (one all-gather)."""
    torch = _torch()
    L, Ls = field_limbs(prepared.curve), scalar_limbs(prepared.curve)
    K = _dev_u32(scalars_local, Ls, "scalars")
    if K.shape[0] > prepared.n or K.device != prepared.device:
        raise GzkpError("scalars exceed the prepared shard or are on another device")
    if out is None:
        out = torch.empty(2 * L, dtype=torch.int32, device=K.device)
    with _on(K):
        _check(lib().gzkp_msm_prepared_sharded(prepared.handle, K.data_ptr(), K.shape[0], out.data_ptr(),
                                               _stream_ptr(stream, K.device), comm.handle), "gzkp_msm_prepared_sharded")
    return out


__all__ = ["CURVES", "GzkpError", "lib", "msm", "msm_host", "PreparedPoints", "msm_partial", "combine_partials",
           "fixed_base_mul", "field_op", "ec_op", "Comm", "msm_sharded", "msm_prepared_sharded", "shard_range", "set_config",
           "window_bits", "workspace_bytes", "set_profiling", "profile_read", "field_limbs", "scalar_limbs", "to_device",
           "to_numpy", "ntt", "ntt_max_log", "ntt_last_launches", "scalar_field_op", "release_stream",
           "debug_buckets"]
