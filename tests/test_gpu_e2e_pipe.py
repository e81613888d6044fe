"""GPU: the pipelined fftstencil_run_host (chunked H2D/D2H overlapped with row-skewed passes,
capi.cu run_host_pipelined) gives the same bits as fftstencil_run on device buffers, and meets
the oracle tolerance (BASELINE.json north_star: max abs err <= 1e-9 * max|u|).

The schedule only reorders whole outer tile rows of the same kernels (e2e), so the
comparison with the device path is bitwise.  Cases cover: passes P < depth Q (head and tail
overlap), P > 2Q (full middle passes), a remainder pass, r = 3, 3D, and K = 2 / 4 / 16 chunks.
"""
import math
import os

import numpy as np
import pytest

import oracle
from synth import workloads as wl

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def fs():
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    import paper_conf_ppopp_hanlcbzyczcy25_b200 as mod
    return mod


def _env(chunks, depth):
    old = {k: os.environ.get(k) for k in ("FFTSTENCIL_E2E_PIPE", "FFTSTENCIL_E2E_DEPTH")}
    os.environ["FFTSTENCIL_E2E_PIPE"] = str(chunks)
    if depth is None:
        os.environ.pop("FFTSTENCIL_E2E_DEPTH", None)
    else:
        os.environ["FFTSTENCIL_E2E_DEPTH"] = str(depth)
    return old


def _restore(old):
    for k, v in old.items():
        if v is None:
            os.environ.pop(k, None)
        else:
            os.environ[k] = v


CASES = [
    # extents, shape, r, T, steps, chunks K, depth Q (None = default 16)
    ((1500, 200), "star", 1, 11, 100, 16, None),   # P = 10 < Q: head and tail overlap
    ((800, 150), "box", 1, 4, 103, 4, 3),          # P = 26 > 2Q, remainder pass t = 3
    ((700, 130), "box", 3, 4, 50, 4, 2),           # r = 3 (h = 12), remainder t = 2
    ((420, 36, 40), "star", 1, 2, 9, 16, None),    # 3D, remainder t = 1
    ((200, 30, 33), "box", 1, 2, 12, 2, 1),        # 3D box, K = 2, Q = 1
    ((600, 97), "star", 1, 8, 1, 2, 4),            # one pass with t = 1
]


@pytest.mark.parametrize("ext,shape,r,T,steps,K,Q", CASES)
def test_pipelined_run_host_bitwise(fs, ext, shape, r, T, steps, K, Q):
    w = wl.seeded_weights(shape, len(ext), r)
    u0 = wl.grid(ext, 5 + len(ext))
    p = fs.Plan(ext, w, r, T)
    info = p.info()
    h, S = info["halo"], info["valid"][0]
    nt0 = math.ceil((ext[0] - 2 * h) / S)
    assert h <= S and nt0 >= 2 * K, "case must be eligible for the pipelined schedule"
    a = torch.from_numpy(u0).cuda()
    b = torch.empty_like(a)
    p.run(a, b, steps)
    torch.cuda.synchronize()
    dev = b.cpu().numpy()
    n_dev = p.info()["last_run_launches"]
    old = _env(K, Q)
    try:
        h_in = torch.from_numpy(u0).pin_memory()
        h_out = torch.full(u0.shape, np.nan, dtype=torch.float64).pin_memory()
        p.run_host(h_in.numpy(), h_out.numpy(), steps)
        n_pipe = p.info()["last_run_launches"]
        pi = p.info()
        assert pi["last_run_pipelined"]
        # default Q (capi.cu pipe_depth): 20 skewed passes for 3D plans, 16 otherwise
        assert (pi["last_run_chunks"], pi["last_run_depth"]) == (K, Q if Q is not None else (20 if len(ext) == 3 else 16))
        got = h_out.numpy().copy()
        # pageable host buffers take the same schedule
        out2 = np.full_like(u0, np.nan)
        p.run_host(u0, out2, steps)
    finally:
        _restore(old)
    assert n_pipe > n_dev, "the pipelined schedule was not taken"
    assert np.array_equal(got, dev)
    assert np.array_equal(out2, dev)
    if u0.size * steps <= 2e7:
        ref = oracle.stencil_run(u0, w, r, steps)
        assert float(np.abs(got - ref).max() / np.abs(ref).max()) <= 1e-9


def test_pipeline_off_and_ineligible_unchanged(fs):
    """FFTSTENCIL_E2E_PIPE=0, and grids with fewer than 2K outer tile rows, keep H2D, run, D2H."""
    ext = (300, 120)
    w = wl.seeded_weights("box", 2, 1)
    u0 = wl.grid(ext, 3)
    p = fs.Plan(ext, w, 1, 8)
    ref = oracle.stencil_run(u0, w, 1, 20)
    for k in ("0", "16"):
        old = _env(k, None)
        try:
            out = np.empty_like(u0)
            p.run_host(u0, out, 20)
        finally:
            _restore(old)
        assert float(np.abs(out - ref).max() / np.abs(ref).max()) <= 1e-9
