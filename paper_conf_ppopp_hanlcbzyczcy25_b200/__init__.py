"""B200-native FlashFFTStencil hot path: Python binding over the C ABI (include/fftstencil.h).

    from paper_conf_ppopp_hanlcbzyczcy25_b200 import Plan
    plan = Plan((10240, 10240), weights, radius=1, T=8)       # host precompute + upload
    plan.run(u_in, u_out, total_steps=1000)                   # torch CUDA float64 tensors
    plan.run_host(h_in, h_out, total_steps=1000)              # numpy arrays (end to end)

Every step of the path runs in the CUDA kernels of libfftstencil.so; this module only
marshals arguments (torch is used for device memory and streams).  PAPER.md citations
live in include/fftstencil.h and csrc/.
"""
from __future__ import annotations

import ctypes

import numpy as np

from . import _native
from ._native import FftStencilError, Info, last_error

__all__ = ["Plan", "describe", "describe_dist", "export_aux", "e2e_schedule", "peer_schedule", "nccl_unique_id", "run_group", "FftStencilError"]


def _arrays(extents, weights, radius):
    ext = np.ascontiguousarray(np.asarray(extents, dtype=np.int64).reshape(-1))
    w = np.ascontiguousarray(np.asarray(weights, dtype=np.float64).reshape(-1))
    if w.size != (2 * int(radius) + 1) ** ext.size:
        raise ValueError(f"weights must have (2r+1)^ndim = {(2 * int(radius) + 1) ** ext.size} entries")
    return ext, w


def _current_device():
    """The CUDA device the C ABI binds a new plan to (the current one); None without torch/CUDA."""
    try:
        import torch
        return torch.cuda.current_device() if torch.cuda.is_available() else None
    except Exception:
        return None


def _i64p(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))


def _dp(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def describe(extents, weights, radius: int, T: int = 0, periodic: bool = False) -> dict:
    """Run the host plan builder only (no GPU needed) and return its geometry."""
    ext, w = _arrays(extents, weights, radius)
    info = Info()
    rc = _native.lib().fftstencil_describe_ex(int(ext.size), _i64p(ext), _dp(w), int(radius), int(T),
                                              _native.PERIODIC if periodic else 0, ctypes.byref(info))
    if rc != 0:
        raise FftStencilError(rc, last_error())
    return info.as_dict()


def describe_dist(extents, weights, radius: int, T: int, nranks: int, rank: int) -> dict:
    """Host-only slab geometry of one rank of the outer-axis decomposition."""
    ext, w = _arrays(extents, weights, radius)
    info = Info()
    rc = _native.lib().fftstencil_describe_dist(int(ext.size), _i64p(ext), _dp(w), int(radius), int(T),
                                                int(nranks), int(rank), ctypes.byref(info))
    if rc != 0:
        raise FftStencilError(rc, last_error())
    return info.as_dict()


def nccl_unique_id() -> bytes:
    """A fresh 128-byte ncclUniqueId (rank 0 creates it, then broadcasts it)."""
    buf = ctypes.create_string_buffer(128)
    rc = _native.lib().fftstencil_nccl_unique_id(buf)
    if rc != 0:
        raise FftStencilError(rc, last_error())
    return buf.raw


def run_group(plans, ins, outs, total_steps: int, stream=None) -> None:
    """Run loopback ranks (Plan(..., nranks=n, rank=k, nccl_id=None)) together on one GPU."""
    import torch
    n = len(plans)
    vp = ctypes.c_void_p
    P = (vp * n)(*[p._h.value for p in plans])
    I = (vp * n)(*[t.data_ptr() for t in ins])
    O = (vp * n)(*[t.data_ptr() for t in outs])
    for p, a, b in zip(plans, ins, outs):
        p._check_dev(a, "in")
        p._check_dev(b, "out")
    s = stream if stream is not None else torch.cuda.current_stream(ins[0].device)
    rc = _native.lib().fftstencil_run_group(P, I, O, n, int(total_steps), vp(s.cuda_stream))
    if rc != 0:
        raise FftStencilError(rc, last_error())


def export_aux(extents, weights, radius: int, T: int, which: int, axis: int = 0, t: int = 1) -> np.ndarray:
    """Host plan tables (see fftstencil_export_aux in include/fftstencil.h)."""
    ext, w = _arrays(extents, weights, radius)
    L = _native.lib()
    n = L.fftstencil_export_aux(int(ext.size), _i64p(ext), _dp(w), int(radius), int(T), int(which), int(axis),
                                int(t), None, 0)
    if n < 0:
        raise FftStencilError(int(n), last_error())
    out = np.empty(int(n), dtype=np.float64)
    m = L.fftstencil_export_aux(int(ext.size), _i64p(ext), _dp(w), int(radius), int(T), int(which), int(axis),
                                int(t), _dp(out), int(n))
    if m < 0:
        raise FftStencilError(int(m), last_error())
    return out


def peer_schedule(extents, weights, radius: int, T: int, nranks: int, rank: int, total_steps: int,
                  fused: bool = True, epoch0: int = 0) -> np.ndarray:
    """Op list of a peer-transport run of one rank, shape (n, 4) int64 (fftstencil_peer_schedule)."""
    ext, w = _arrays(extents, weights, radius)
    L = _native.lib()
    args = (int(ext.size), _i64p(ext), _dp(w), int(radius), int(T), int(nranks), int(rank), int(total_steps),
            int(bool(fused)), int(epoch0))
    n = L.fftstencil_peer_schedule(*args, None, 0)
    if n < 0:
        raise FftStencilError(int(n), last_error())
    out = np.zeros((int(n), 4), dtype=np.int64)
    m = L.fftstencil_peer_schedule(*args, out.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)), int(n))
    if m < 0:
        raise FftStencilError(int(m), last_error())
    return out


def e2e_schedule(extents, weights, radius: int, T: int, total_steps: int, chunks: int = 6,
                 depth: int = 16) -> np.ndarray:
    """Op list of the pipelined run_host, shape (n, 4) int64 (fftstencil_e2e_schedule)."""
    ext, w = _arrays(extents, weights, radius)
    L = _native.lib()
    n = L.fftstencil_e2e_schedule(int(ext.size), _i64p(ext), _dp(w), int(radius), int(T), int(total_steps),
                                  int(chunks), int(depth), None, 0)
    if n < 0:
        raise FftStencilError(int(n), last_error())
    out = np.zeros((int(n), 4), dtype=np.int64)
    m = L.fftstencil_e2e_schedule(int(ext.size), _i64p(ext), _dp(w), int(radius), int(T), int(total_steps),
                                  int(chunks), int(depth), _i64p(out), int(n))
    if m < 0:
        raise FftStencilError(int(m), last_error())
    return out


class Plan:
    """A FlashFFTStencil plan bound to the current CUDA device."""

    def __init__(self, extents, weights, radius: int, T: int = 0, nranks: int = 1, rank: int = 0,
                 nccl_id: bytes | None = None, loopback: bool = False, periodic: bool = False,
                 transport: str | None = None):
        """extents are GLOBAL.  nranks > 1: this process's rank of the outer-axis decomposition;
        pass the group's nccl_id (bytes from nccl_unique_id()), or loopback=True for a rank
        run with run_group on one device, or transport="peer" for the CUDA-IPC peer-memory
        transport (then exchange peer_handle() bytes and call peer_connect, or connect_peers()
        under torch.distributed).  in/out tensors then hold this rank's slab
        (rows [row_begin, row_end) of info())."""
        ext, w = _arrays(extents, weights, radius)
        self.global_extents = tuple(int(e) for e in ext)
        self.radius = int(radius)
        self._lib = _native.lib()
        if nranks == 1:
            h = self._lib.fftstencil_plan_create_ex(int(ext.size), _i64p(ext), _dp(w), int(radius), int(T),
                                                    _native.PERIODIC if periodic else 0)
        elif transport == "peer":
            h = self._lib.fftstencil_plan_create_dist_peer(int(ext.size), _i64p(ext), _dp(w), int(radius), int(T),
                                                           int(nranks), int(rank))
        else:
            if nccl_id is None and not loopback:
                raise ValueError("nranks > 1 needs nccl_id (or loopback=True)")
            idbuf = None if loopback else ctypes.create_string_buffer(bytes(nccl_id), 128)
            h = self._lib.fftstencil_plan_create_dist(int(ext.size), _i64p(ext), _dp(w), int(radius), int(T),
                                                      int(nranks), int(rank), idbuf)
        if not h:
            raise FftStencilError(_native.EINVAL, last_error())
        self._h = ctypes.c_void_p(h)
        self.device = _current_device()
        inf = self.info()
        self.extents = (inf["row_end"] - inf["row_begin"],) + self.global_extents[1:]

    # -- peer transport --
    def peer_handle(self) -> bytes:
        """This rank's FFTSTENCIL_PEER_HANDLE_BYTES handle blob (CUDA IPC handles + slab geometry)."""
        buf = ctypes.create_string_buffer(_native.PEER_HANDLE_BYTES)
        rc = self._lib.fftstencil_peer_handle(self._h, buf, _native.PEER_HANDLE_BYTES)
        if rc != 0:
            raise FftStencilError(rc, last_error())
        return buf.raw

    def peer_connect(self, lower: bytes | None, upper: bytes | None) -> None:
        """Open the neighbours' handles (None where there is no neighbour)."""
        lb = ctypes.create_string_buffer(bytes(lower), _native.PEER_HANDLE_BYTES) if lower is not None else None
        ub = ctypes.create_string_buffer(bytes(upper), _native.PEER_HANDLE_BYTES) if upper is not None else None
        rc = self._lib.fftstencil_peer_connect(self._h, lb, ub)
        if rc != 0:
            raise FftStencilError(rc, last_error())

    def connect_peers(self, group=None) -> None:
        """Exchange handles over torch.distributed (any backend) and connect to the neighbours."""
        import torch.distributed as dist
        inf = self.info()
        rank, world = inf["rank"], inf["nranks"]
        handles = [None] * world
        dist.all_gather_object(handles, self.peer_handle(), group=group)
        self.peer_connect(handles[rank - 1] if rank > 0 else None, handles[rank + 1] if rank < world - 1 else None)

    # -- lifetime --
    def close(self):
        if getattr(self, "_h", None):
            self._lib.fftstencil_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    # -- queries --
    def info(self) -> dict:
        info = Info()
        rc = self._lib.fftstencil_plan_info(self._h, ctypes.byref(info))
        if rc != 0:
            raise FftStencilError(rc, last_error())
        return info.as_dict()

    def set_profiling(self, enable: bool) -> None:
        rc = self._lib.fftstencil_set_profiling(self._h, int(bool(enable)))
        if rc != 0:
            raise FftStencilError(rc, last_error())

    def profile_read(self) -> dict:
        fm, bm = ctypes.c_double(), ctypes.c_double()
        fl, bl = ctypes.c_int64(), ctypes.c_int64()
        rc = self._lib.fftstencil_profile_read(self._h, ctypes.byref(fm), ctypes.byref(fl), ctypes.byref(bm),
                                               ctypes.byref(bl))
        if rc != 0:
            raise FftStencilError(rc, last_error())
        return {"fused_ms": fm.value, "fused_launches": fl.value, "band_ms": bm.value, "band_launches": bl.value}

    # -- execution --
    def _check_dev(self, t, name):
        import torch
        if not isinstance(t, torch.Tensor) or not t.is_cuda or t.dtype != torch.float64:
            raise TypeError(f"{name} must be a CUDA float64 torch tensor")
        if tuple(t.shape) != self.extents or not t.is_contiguous():
            raise ValueError(f"{name} must be contiguous with shape {self.extents}")
        if self.device is not None and t.device.index != self.device:
            raise ValueError(f"{name} is on cuda:{t.device.index}, the plan on cuda:{self.device}")

    def run(self, inp, out, total_steps: int, stream=None) -> None:
        """Enqueue total_steps time steps: out <- stencil^steps(inp) (asynchronous)."""
        import torch
        self._check_dev(inp, "inp")
        self._check_dev(out, "out")
        s = stream if stream is not None else torch.cuda.current_stream(inp.device)
        rc = self._lib.fftstencil_run(self._h, ctypes.c_void_p(inp.data_ptr()), ctypes.c_void_p(out.data_ptr()),
                                      int(total_steps), ctypes.c_void_p(s.cuda_stream))
        if rc != 0:
            raise FftStencilError(rc, last_error())

    def run_emit(self, inp, outs, emit_steps, stream=None) -> None:
        """outs[k] <- the state after emit_steps[k] time steps (flexible outputs, §4)."""
        import torch
        self._check_dev(inp, "inp")
        for o in outs:
            self._check_dev(o, "out")
        n = len(outs)
        steps = np.ascontiguousarray(np.asarray(emit_steps, dtype=np.int64))
        if steps.size != n:
            raise ValueError("one emit step per output")
        O = (ctypes.c_void_p * n)(*[o.data_ptr() for o in outs])
        s = stream if stream is not None else torch.cuda.current_stream(inp.device)
        rc = self._lib.fftstencil_run_emit(self._h, ctypes.c_void_p(inp.data_ptr()), _i64p(steps), n, O,
                                           ctypes.c_void_p(s.cuda_stream))
        if rc != 0:
            raise FftStencilError(rc, last_error())

    def run_raw(self, in_ptr: int, out_ptr: int, total_steps: int, stream_handle: int) -> None:
        rc = self._lib.fftstencil_run(self._h, ctypes.c_void_p(in_ptr), ctypes.c_void_p(out_ptr),
                                      int(total_steps), ctypes.c_void_p(stream_handle))
        if rc != 0:
            raise FftStencilError(rc, last_error())

    def run_host(self, h_in, h_out, total_steps: int, stream=None) -> None:
        """End to end with host buffers (numpy float64 or CPU torch tensors); synchronous."""
        def ptr(a, name):
            if isinstance(a, np.ndarray):
                if a.dtype != np.float64 or not a.flags.c_contiguous or tuple(a.shape) != self.extents:
                    raise ValueError(f"{name} must be C-contiguous float64 with shape {self.extents}")
                return a.ctypes.data
            import torch
            if isinstance(a, torch.Tensor) and not a.is_cuda and a.dtype == torch.float64:
                # the C side copies prod(extents) doubles from / into this buffer: a wrong
                # shape (e.g. a global grid passed to a slab plan) would run out of bounds
                if tuple(a.shape) != self.extents or not a.is_contiguous():
                    raise ValueError(f"{name} must be contiguous with shape {self.extents}")
                return a.data_ptr()
            raise TypeError(f"{name} must be a host float64 array")
        sh = 0
        if stream is not None:
            sh = stream.cuda_stream
        rc = self._lib.fftstencil_run_host(self._h, ctypes.c_void_p(ptr(h_in, "h_in")),
                                           ctypes.c_void_p(ptr(h_out, "h_out")), int(total_steps),
                                           ctypes.c_void_p(sh))
        if rc != 0:
            raise FftStencilError(rc, last_error())
