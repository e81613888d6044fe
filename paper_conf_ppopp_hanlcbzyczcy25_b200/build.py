"""Build libfftstencil.so in-tree: nvcc for sm_100a (+ g++ for the host plan builder).

    python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build [--force]

The shared object lands next to this file so it travels with the repo snapshot to the
GPU box (it is git-ignored, not gpurun-ignored).
"""
from __future__ import annotations

import concurrent.futures as cf
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
# Ablation builds: FFTSTENCIL_NVCC_DEFS="-DNAME=V ..." compiles a variant into its own object
# directory and .so (FFTSTENCIL_LIB selects it at load time, _native.py).
DEFS = os.environ.get("FFTSTENCIL_NVCC_DEFS", "").split()
_TAG = "".join(c if c.isalnum() else "_" for c in "".join(DEFS))
BUILD = os.path.join(HERE, "_build" + ("_" + _TAG if _TAG else ""))
SO = os.path.join(HERE, "libfftstencil.so" if not _TAG else f"libfftstencil_{_TAG}.so")
INCLUDE = os.path.join(ROOT, "include")

NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


def _nccl_dirs():
    """NCCL headers/library: the copy torch loads (pip nvidia-nccl), else the system one.
    Both carry the soname libnccl.so.2, so one NCCL is loaded per process."""
    try:
        import nvidia.nccl as nn   # noqa: F401
        base = list(nn.__path__)[0]
        inc, lib = os.path.join(base, "include"), os.path.join(base, "lib")
        if os.path.exists(os.path.join(inc, "nccl.h")) and os.path.exists(os.path.join(lib, "libnccl.so.2")):
            return inc, lib
    except Exception:
        pass
    return "/usr/include", "/usr/lib/x86_64-linux-gnu"


NCCL_INC, NCCL_LIB = _nccl_dirs()
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVFLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xptxas", "-v", *ARCH,
           "-I", INCLUDE, "-I", CSRC, "-I", NCCL_INC, *DEFS]
CXXFLAGS = ["-O2", "-std=c++17", "-fPIC", "-I", INCLUDE, "-I", CSRC, *DEFS]

CU = ["capi.cu", "kernel_fft2d.cu", "kernel_fft2d_ct.cu", "kernel_fft1d.cu", "kernel_fft1d_ct.cu", "kernel_fft3d.cu", "kernel_fft3d_ct.cu", "kernel_fft3d_bf.cu", "kernel_fft2d_bf.cu", "kernel_fft1d_bf.cu", "kernel_band.cu", "kernel_small1d.cu"]
CPP = ["plan.cpp"]
HEADERS = ["plan.h", "kernels.cuh", "device_common.cuh", "tma.cuh", "ct_line.cuh", "fft_radix.cuh"]


def _stale(obj: str, src: str) -> bool:
    if not os.path.exists(obj):
        return True
    t = os.path.getmtime(obj)
    deps = [src] + [os.path.join(CSRC, h) for h in HEADERS] + [os.path.join(INCLUDE, "fftstencil.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def _compile(src: str, force: bool):
    path = os.path.join(CSRC, src)
    obj = os.path.join(BUILD, src + ".o")
    if not force and not _stale(obj, path):
        return obj, ""
    if src.endswith(".cu"):
        cmd = [NVCC, *NVFLAGS, "-c", path, "-o", obj]
    else:
        cmd = ["g++", *CXXFLAGS, "-c", path, "-o", obj]
    res = subprocess.run(cmd, capture_output=True, text=True)
    if res.returncode != 0:
        raise RuntimeError(f"compile failed: {' '.join(cmd)}\n{res.stdout}\n{res.stderr}")
    return obj, res.stderr


def build(force: bool = False, verbose: bool = False) -> str:
    os.makedirs(BUILD, exist_ok=True)
    with cf.ThreadPoolExecutor(max_workers=min(8, os.cpu_count() or 2)) as ex:
        results = list(ex.map(lambda s: _compile(s, force), CU + CPP))
    objs = [o for o, _ in results]
    if verbose:
        for _, log in results:
            if log:
                sys.stderr.write(log)
    if force or not os.path.exists(SO) or any(os.path.getmtime(o) > os.path.getmtime(SO) for o in objs):
        tmp = SO + f".tmp{os.getpid()}"
        cmd = [NVCC, *ARCH, "-shared", "-o", tmp, *objs, "-lcudart", "-L", NCCL_LIB, "-l:libnccl.so.2",
               "-Xlinker", "-rpath", "-Xlinker", NCCL_LIB]
        res = subprocess.run(cmd, capture_output=True, text=True)
        if res.returncode != 0:
            raise RuntimeError(f"link failed: {' '.join(cmd)}\n{res.stdout}\n{res.stderr}")
        os.replace(tmp, SO)
    return SO


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
