"""CPU oracle for the FlashFFTStencil hot path -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline``
leg and ``--impl reference``) may import this package.  The product path
(``paper_conf_ppopp_hanlcbzyczcy25_b200``) never imports it and shares no code with it.

Contents
  stencil_run(...)    plain direct stencil, step by step, FP64 (C: stencil_oracle.c)
                      PAPER.md L93 (§2.2), Eq. 2, Fig. 2 left L111-L128, Eq. 10
  stencil_point(...)  the same definition for single cells (dependency-cone sub-box)
  stencil_run_py(...) the same definition as a pure-Python/numpy loop, tiny grids only
  spectrum.py         the stencil symbol sigma(theta) and powered spectrum S_t
                      (§4 Eq. 10, Alg. 1 line 2 L256)

Every function is pinned by tests/test_oracle.py against things other than itself
(hand expansions, closed forms, library routines on special cases, invariants).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "stencil_oracle.c")
_SO = os.path.join(_HERE, "libstencil_oracle.so")
_lock = threading.Lock()
_lib = None

# Plain FP64: no fast-math, no FMA contraction (reading Q17 in DESIGN.md).
CFLAGS = ["-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared", "-std=c11"]


def build(force: bool = False) -> str:
    """Compile the C oracle with gcc (called by __graft_entry__.build())."""
    if force or not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        tmp = _SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, _SRC, "-o", tmp])
        os.replace(tmp, _SO)
    return _SO


def _load():
    global _lib
    with _lock:
        if _lib is None:
            lib = ctypes.CDLL(build())
            i64p = ctypes.POINTER(ctypes.c_int64)
            dp = ctypes.POINTER(ctypes.c_double)
            lib.oracle_stencil_run.argtypes = [ctypes.c_int, i64p, dp, ctypes.c_int, ctypes.c_int64,
                                               ctypes.c_int, dp, dp, ctypes.c_int]
            lib.oracle_stencil_run.restype = ctypes.c_int
            lib.oracle_stencil_point.argtypes = [ctypes.c_int, i64p, dp, ctypes.c_int, ctypes.c_int64,
                                                 dp, ctypes.c_int64, i64p, dp, ctypes.c_int]
            lib.oracle_stencil_point.restype = ctypes.c_int
            lib.oracle_max_threads.argtypes = []
            lib.oracle_max_threads.restype = ctypes.c_int
            _lib = lib
    return _lib


def _dp(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def _ip(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))


def max_threads() -> int:
    return int(_load().oracle_max_threads())


def stencil_run(u0, weights, radius: int, steps: int, periodic: bool = False, nthreads: int = 0):
    """Return u after `steps` direct time steps (fixed ring unless periodic).

    u0: float64 array, ndim 1..3, C order, extents include the fixed ring.
    weights: (2r+1)^ndim float64, offset-cube row-major; weights[o+r] multiplies u[c+o].
    """
    u0 = np.ascontiguousarray(u0, dtype=np.float64)
    w = np.ascontiguousarray(weights, dtype=np.float64).reshape(-1)
    nd = u0.ndim
    if w.size != (2 * radius + 1) ** nd:
        raise ValueError("weights size does not match radius/ndim")
    ext = np.asarray(u0.shape, dtype=np.int64)
    out = np.empty_like(u0)
    rc = _load().oracle_stencil_run(nd, _ip(ext), _dp(w), int(radius), int(steps), int(bool(periodic)),
                                    _dp(u0), _dp(out), int(nthreads))
    if rc != 0:
        raise ValueError("oracle_stencil_run rejected its arguments")
    return out


def stencil_point(u0, weights, radius: int, steps: int, cells, nthreads: int = 0):
    """Fixed-ring values at the given cells (int array [npts, ndim]) after `steps` steps."""
    u0 = np.ascontiguousarray(u0, dtype=np.float64)
    w = np.ascontiguousarray(weights, dtype=np.float64).reshape(-1)
    nd = u0.ndim
    cells = np.ascontiguousarray(np.asarray(cells, dtype=np.int64).reshape(-1, nd))
    ext = np.asarray(u0.shape, dtype=np.int64)
    vals = np.empty(cells.shape[0], dtype=np.float64)
    rc = _load().oracle_stencil_point(nd, _ip(ext), _dp(w), int(radius), int(steps), _dp(u0),
                                      int(cells.shape[0]), _ip(cells), _dp(vals), int(nthreads))
    if rc != 0:
        raise ValueError("oracle_stencil_point rejected its arguments")
    return vals


def stencil_run_py(u0, weights, radius: int, steps: int, periodic: bool = False):
    """Pure-Python/numpy statement of the same definition (tiny grids only).

    Loops over cells and offsets exactly as L93 / Eq. 2 read (correlation form, Q1),
    ring cells held (Q2).  Used to cross-check the C oracle's indexing.
    """
    u = np.array(u0, dtype=np.float64)
    nd = u.ndim
    w = np.asarray(weights, dtype=np.float64).reshape((2 * radius + 1,) * nd)
    offsets = list(np.ndindex(*w.shape))
    for _ in range(steps):
        nxt = u.copy()
        for c in np.ndindex(*u.shape):
            if not periodic and any(c[a] < radius or c[a] >= u.shape[a] - radius for a in range(nd)):
                continue
            acc = 0.0
            for oi in offsets:
                p = tuple((c[a] + oi[a] - radius) % u.shape[a] for a in range(nd))
                acc += w[oi] * u[p]
            nxt[c] = acc
        u = nxt
    return u
