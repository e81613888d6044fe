"""ctypes binding of libfftstencil.so (include/fftstencil.h).  Argument marshalling only.

The shared object is the product: if it is missing this module raises -- there is no
Python or CPU fallback for any step of the path.
"""
from __future__ import annotations

import ctypes
import os

HERE = os.path.dirname(os.path.abspath(__file__))
SO_PATH = os.environ.get("FFTSTENCIL_LIB") or os.path.join(HERE, "libfftstencil.so")   # override: ablation builds

OK, EINVAL, ENOMEM, ECUDA, ENCCL, EUNSUPPORTED = 0, -1, -2, -3, -4, -5
PERIODIC = 1
CODES = {OK: "OK", EINVAL: "EINVAL", ENOMEM: "ENOMEM", ECUDA: "ECUDA", ENCCL: "ENCCL",
         EUNSUPPORTED: "EUNSUPPORTED"}

# every symbol include/fftstencil.h declares
EXPORTS = ("fftstencil_plan_create", "fftstencil_run", "fftstencil_run_host", "fftstencil_destroy",
           "fftstencil_plan_info", "fftstencil_last_error", "fftstencil_describe", "fftstencil_export_aux",
           "fftstencil_set_profiling", "fftstencil_profile_read", "fftstencil_plan_create_dist",
           "fftstencil_nccl_unique_id", "fftstencil_run_group", "fftstencil_describe_dist",
           "fftstencil_plan_create_ex", "fftstencil_describe_ex", "fftstencil_run_emit",
           "fftstencil_e2e_schedule", "fftstencil_plan_create_dist_peer", "fftstencil_peer_handle",
           "fftstencil_peer_connect", "fftstencil_peer_schedule")
PEER_HANDLE_BYTES = 256   # FFTSTENCIL_PEER_HANDLE_BYTES


class Info(ctypes.Structure):
    _fields_ = [
        ("ndim", ctypes.c_int),
        ("T", ctypes.c_int),
        ("radius", ctypes.c_int),
        ("halo", ctypes.c_int),
        ("tile", ctypes.c_int * 3),
        ("valid", ctypes.c_int * 3),
        ("pfa", ctypes.c_int * 2),
        ("extents", ctypes.c_int64 * 3),
        ("tiles", ctypes.c_int64),
        ("pairs", ctypes.c_int64),
        ("band_blocks", ctypes.c_int64),
        ("flops_per_cell_step", ctypes.c_double),
        ("mma_flops_per_pass", ctypes.c_double),
        ("smem_bytes", ctypes.c_size_t),
        ("device_bytes", ctypes.c_size_t),
        ("fused_grid", ctypes.c_int),
        ("last_run_launches", ctypes.c_int64),
        ("nranks", ctypes.c_int),
        ("rank", ctypes.c_int),
        ("row_begin", ctypes.c_int64),
        ("row_end", ctypes.c_int64),
        ("pair_begin", ctypes.c_int64),
        ("pair_end", ctypes.c_int64),
        ("interior_begin", ctypes.c_int64),
        ("interior_end", ctypes.c_int64),
        ("ghost_lo", ctypes.c_int64),
        ("ghost_hi", ctypes.c_int64),
        ("algo", ctypes.c_int),
        ("periodic", ctypes.c_int),
        ("engine", ctypes.c_int),
        ("alu_ops_per_pass", ctypes.c_double),
        ("last_run_pipelined", ctypes.c_int),
        ("last_run_chunks", ctypes.c_int),
        ("last_run_depth", ctypes.c_int),
        ("last_run_peer_fused", ctypes.c_int),
    ]

    def as_dict(self) -> dict:
        nd = self.ndim
        return {
            "ndim": nd, "T": self.T, "radius": self.radius, "halo": self.halo,
            "tile": list(self.tile)[:nd], "valid": list(self.valid)[:nd], "pfa": list(self.pfa),
            "extents": list(self.extents)[:nd], "tiles": self.tiles, "pairs": self.pairs,
            "band_blocks": self.band_blocks, "flops_per_cell_step": self.flops_per_cell_step,
            "mma_flops_per_pass": self.mma_flops_per_pass, "smem_bytes": self.smem_bytes,
            "device_bytes": self.device_bytes, "fused_grid": self.fused_grid,
            "last_run_launches": self.last_run_launches,
            "nranks": self.nranks, "rank": self.rank, "row_begin": self.row_begin, "row_end": self.row_end,
            "pair_begin": self.pair_begin, "pair_end": self.pair_end, "interior_begin": self.interior_begin,
            "interior_end": self.interior_end, "ghost_lo": self.ghost_lo, "ghost_hi": self.ghost_hi,
            "algo": ("dense", "factored", "unfused")[self.algo] if nd >= 2 else ("pfa", "factored")[self.algo],
            "periodic": bool(self.periodic),
            "engine": ("dmma", "alu")[self.engine], "alu_ops_per_pass": self.alu_ops_per_pass,
            "last_run_pipelined": bool(self.last_run_pipelined),
            "last_run_chunks": self.last_run_chunks, "last_run_depth": self.last_run_depth,
            "last_run_peer_fused": bool(self.last_run_peer_fused),
        }


_lib = None


def lib():
    """Load (once) and return the CDLL.  Raises if the extension was not built."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(SO_PATH):
        raise ImportError(f"{SO_PATH} is missing: build it with `python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build` "
                          "(there is no fallback path)")
    L = ctypes.CDLL(SO_PATH)
    i64p = ctypes.POINTER(ctypes.c_int64)
    dp = ctypes.POINTER(ctypes.c_double)
    vp = ctypes.c_void_p
    L.fftstencil_plan_create.argtypes = [ctypes.c_int, i64p, dp, ctypes.c_int, ctypes.c_int]
    L.fftstencil_plan_create.restype = vp
    L.fftstencil_run.argtypes = [vp, vp, vp, ctypes.c_int64, vp]
    L.fftstencil_run.restype = ctypes.c_int
    L.fftstencil_run_host.argtypes = [vp, vp, vp, ctypes.c_int64, vp]
    L.fftstencil_run_host.restype = ctypes.c_int
    L.fftstencil_destroy.argtypes = [vp]
    L.fftstencil_destroy.restype = None
    L.fftstencil_plan_info.argtypes = [vp, ctypes.POINTER(Info)]
    L.fftstencil_plan_info.restype = ctypes.c_int
    L.fftstencil_last_error.argtypes = []
    L.fftstencil_last_error.restype = ctypes.c_char_p
    L.fftstencil_describe.argtypes = [ctypes.c_int, i64p, dp, ctypes.c_int, ctypes.c_int, ctypes.POINTER(Info)]
    L.fftstencil_describe.restype = ctypes.c_int
    L.fftstencil_export_aux.argtypes = [ctypes.c_int, i64p, dp, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                        ctypes.c_int, ctypes.c_int, dp, ctypes.c_int64]
    L.fftstencil_export_aux.restype = ctypes.c_int64
    L.fftstencil_e2e_schedule.argtypes = [ctypes.c_int, i64p, dp, ctypes.c_int, ctypes.c_int, ctypes.c_int64,
                                          ctypes.c_int, ctypes.c_int, i64p, ctypes.c_int64]
    L.fftstencil_e2e_schedule.restype = ctypes.c_int64
    L.fftstencil_set_profiling.argtypes = [vp, ctypes.c_int]
    L.fftstencil_set_profiling.restype = ctypes.c_int
    L.fftstencil_profile_read.argtypes = [vp, dp, i64p, dp, i64p]
    L.fftstencil_profile_read.restype = ctypes.c_int
    L.fftstencil_plan_create_dist.argtypes = [ctypes.c_int, i64p, dp, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                              ctypes.c_int, vp]
    L.fftstencil_plan_create_dist.restype = vp
    L.fftstencil_plan_create_dist_peer.argtypes = [ctypes.c_int, i64p, dp, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                                   ctypes.c_int]
    L.fftstencil_plan_create_dist_peer.restype = vp
    L.fftstencil_peer_handle.argtypes = [vp, vp, ctypes.c_int64]
    L.fftstencil_peer_handle.restype = ctypes.c_int
    L.fftstencil_peer_schedule.argtypes = [ctypes.c_int, i64p, dp, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                           ctypes.c_int, ctypes.c_int64, ctypes.c_int, ctypes.c_int64, i64p,
                                           ctypes.c_int64]
    L.fftstencil_peer_schedule.restype = ctypes.c_int64
    L.fftstencil_peer_connect.argtypes = [vp, vp, vp]
    L.fftstencil_peer_connect.restype = ctypes.c_int
    L.fftstencil_nccl_unique_id.argtypes = [vp]
    L.fftstencil_nccl_unique_id.restype = ctypes.c_int
    L.fftstencil_run_group.argtypes = [ctypes.POINTER(vp), ctypes.POINTER(vp), ctypes.POINTER(vp), ctypes.c_int,
                                       ctypes.c_int64, vp]
    L.fftstencil_run_group.restype = ctypes.c_int
    L.fftstencil_describe_dist.argtypes = [ctypes.c_int, i64p, dp, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                           ctypes.c_int, ctypes.POINTER(Info)]
    L.fftstencil_describe_dist.restype = ctypes.c_int
    L.fftstencil_plan_create_ex.argtypes = [ctypes.c_int, i64p, dp, ctypes.c_int, ctypes.c_int, ctypes.c_int]
    L.fftstencil_plan_create_ex.restype = vp
    L.fftstencil_describe_ex.argtypes = [ctypes.c_int, i64p, dp, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                                         ctypes.POINTER(Info)]
    L.fftstencil_describe_ex.restype = ctypes.c_int
    L.fftstencil_run_emit.argtypes = [vp, vp, i64p, ctypes.c_int, ctypes.POINTER(vp), vp]
    L.fftstencil_run_emit.restype = ctypes.c_int
    _lib = L
    return L


def last_error() -> str:
    return lib().fftstencil_last_error().decode()


class FftStencilError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{CODES.get(code, code)}: {msg}")
        self.code = code
