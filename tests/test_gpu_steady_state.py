"""GPU parity of the steady-state pipelined path of every default ALU kernel.

The fused kernels are persistent: a launch runs min(fused grid, pairs) CTAs of two groups,
and a group transforms pair p, p + 2 grid, ...  Only when a group owns two or more pairs does
it take the refill path: the next pair's TMA boxes are issued during the previous pair's last
pass, the mbarrier parity flips, and `fence.proxy.async` orders the generic-proxy reads of the
buffer before the async-proxy writes (kernel_fft2d_bf.cu / kernel_fft3d_bf.cu /
kernel_fft1d_bf.cu).  On a full B200 that needs more than 296 pairs per launch (292 in 1D),
which the small oracle cases of test_gpu_parity.py never reach.  Here:

  * FFTSTENCIL_MAX_CTAS caps the fused grid (test hook, capi.cu), so on small grids each group
    walks 4-20 pairs through the refill loop, with TMA and with cp.async staging;
  * uncapped grids with more than 296 (292) pairs per launch run the hardware's own
    persistent schedule;
  * signed, un-normalised weights (max|sigma| > 1) and signed inputs U(-1, 1).

Every case compares the whole grid element by element with the oracle (Eq. 7
L186-L188 stitching; Eq. 10 L290 temporal fusion), tolerance 1e-9 * max|u| (north_star).
"""
import numpy as np
import pytest

import oracle
from oracle import spectrum
from synth import workloads as wl

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

TOL = 1e-9


@pytest.fixture(scope="module")
def fs():
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    import paper_conf_ppopp_hanlcbzyczcy25_b200 as mod
    return mod


def run(fs, u0, w, r, T, steps):
    p = fs.Plan(u0.shape, w, r, T)
    a = torch.from_numpy(np.ascontiguousarray(u0)).cuda()
    b = torch.empty_like(a)
    p.run(a, b, steps)
    torch.cuda.synchronize()
    out = b.cpu().numpy()
    info = p.info()
    p.close()
    return out, info


def check(got, u0, w, r, steps, info):
    ref = oracle.stencil_run(u0, w, r, steps)
    err = float(np.abs(got - ref).max() / np.abs(ref).max())
    assert err <= TOL, (err, info)
    ring = np.ones(u0.shape, bool)
    ring[tuple(slice(r, e - r) for e in u0.shape)] = False
    assert np.array_equal(got[ring], u0[ring])
    return err


def pairs_per_group(info, ctas):
    return -(-(info["pair_end"] - info["pair_begin"]) // (2 * ctas))


# (extents, shape, r, T, steps, weights kind, env): each group walks >= 4 pairs at 1-2 CTAs
CAPPED = [
    # 2D default ALU kernel (64 x 64 tile, 4 x 16 butterflies): ragged tile counts, odd pairs
    ((300, 290), "box", 1, 8, 19, "seeded", {}),
    ((333, 270), "star", 1, 11, 25, "seeded", {}),
    ((260, 310), "box", 3, 4, 11, "seeded", {}),
    ((300, 290), "box", 1, 8, 19, "signed", {}),
    ((257, 301), "star", 2, 5, 13, "gain", {}),
    # 3D default ALU kernel (16^3 tile, radix-4 lines)
    ((60, 50, 45), "star", 1, 2, 5, "seeded", {}),
    ((52, 47, 61), "box", 1, 2, 7, "seeded", {}),
    ((60, 50, 45), "box", 1, 2, 5, "signed", {}),
    ((49, 58, 40), "star", 1, 1, 3, "gain", {}),
    # 1D default ALU kernel (4096 = 64 x 64 four-step); 64-aligned -> TMA staging
    ((65536,), "star", 2, 512, 1100, "seeded", {"FFTSTENCIL_ALGO": "factored"}),
    ((90001,), "star", 1, 300, 650, "seeded", {"FFTSTENCIL_ALGO": "factored"}),
    ((65536,), "star", 1, 1024, 2100, "signed_unit", {"FFTSTENCIL_ALGO": "factored"}),
]


@pytest.mark.parametrize("ctas", ["1", "2"])
@pytest.mark.parametrize("tma", ["1", "0"])
@pytest.mark.parametrize("ext,shape,r,T,steps,kind,env", CAPPED)
def test_capped_grid_multi_pair(fs, monkeypatch, ctas, tma, ext, shape, r, T, steps, kind, env):
    monkeypatch.setenv("FFTSTENCIL_MAX_CTAS", ctas)
    monkeypatch.setenv("FFTSTENCIL_TMA", tma)
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    w = wl.stencil_weights(shape, len(ext), r, kind)
    u0 = wl.signed_grid(ext, 3) if kind.startswith("signed") else wl.grid(ext, 3)
    got, info = run(fs, u0, w, r, T, steps)
    assert info["engine"] == "alu" and info["T"] == T
    assert pairs_per_group(info, int(ctas)) >= 4, info
    check(got, u0, w, r, steps, info)


# uncapped: more pairs per launch than 148 SMs x 2 groups (1D: the band leaves 146 SMs)
UNCAPPED = [
    ((2560, 2560), "box", 1, 0, None, "seeded", {}),            # auto T = 11: 1,891 pairs
    ((2600, 2333), "star", 3, 0, None, "seeded", {}),           # auto T = 4, ragged
    ((120, 120, 120), "star", 1, 0, None, "seeded", {}),        # 500 pairs
    ((130, 97, 120), "box", 1, 2, 5, "signed", {}),             # 440 pairs
    ((2400000,), "star", 1, 64, 131, "seeded", {"FFTSTENCIL_ALGO": "factored"}),   # 303 pairs
]


@pytest.mark.parametrize("tma", ["1", "0"])
@pytest.mark.parametrize("ext,shape,r,T,steps,kind,env", UNCAPPED)
def test_uncapped_many_pairs(fs, monkeypatch, tma, ext, shape, r, T, steps, kind, env):
    monkeypatch.setenv("FFTSTENCIL_TMA", tma)
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    w = wl.stencil_weights(shape, len(ext), r, kind)
    u0 = wl.signed_grid(ext, 5) if kind == "signed" else wl.grid(ext, 5)
    probe = fs.describe(ext, w, r, T)
    steps = steps or 2 * probe["T"] + 3
    got, info = run(fs, u0, w, r, T, steps)
    assert info["engine"] == "alu"
    assert info["pair_end"] - info["pair_begin"] > 2 * info["fused_grid"], info
    check(got, u0, w, r, steps, info)


@pytest.mark.parametrize("ext,shape,r,T,steps", [((180, 170), "box", 1, 8, 30), ((44, 40, 38), "star", 1, 2, 12),
                                                 ((150, 160), "star", 2, 4, 17)])
def test_signed_unnormalised_weights_grow(fs, ext, shape, r, T, steps):
    """|sigma| > 1 somewhere: the solution grows, and the relative tolerance still holds."""
    w = wl.signed_weights(shape, len(ext), r)
    sig = spectrum.symbol(w, r, [2.0 * np.pi * np.arange(64) / 64] * len(ext))
    assert np.abs(sig).max() > 1.0
    u0 = wl.signed_grid(ext, 9)
    got, info = run(fs, u0, w, r, T, steps)
    err = check(got, u0, w, r, steps, info)
    assert np.abs(got).max() > np.abs(u0).max(), "expected growth for max|sigma| > 1"
    assert err <= TOL


# the selectable engines' persistent loops too (DMMA factored 2D / 3D / 1D, dense 2D with its
# cp.async double buffer, dense 3D, PFA 1D): one CTA, so every CTA walks many pairs
ENGINE_CAPPED = [
    ((300, 290), "box", 1, 8, 19, {"FFTSTENCIL_ALGO": "factored", "FFTSTENCIL_ENGINE": "dmma"}),
    ((300, 290), "box", 1, 8, 19, {"FFTSTENCIL_ALGO": "factored", "FFTSTENCIL_ENGINE": "dmma", "FFTSTENCIL_TMA": "0"}),
    ((60, 50, 45), "star", 1, 2, 5, {"FFTSTENCIL_ALGO": "factored", "FFTSTENCIL_ENGINE": "dmma"}),
    ((65536,), "star", 2, 512, 1100, {"FFTSTENCIL_ALGO": "factored", "FFTSTENCIL_ENGINE": "dmma"}),
    ((260, 250), "star", 1, 8, 19, {"FFTSTENCIL_ALGO": "dense", "FFTSTENCIL_VARIANT": "1"}),
    ((260, 250), "star", 1, 8, 19, {"FFTSTENCIL_ALGO": "dense", "FFTSTENCIL_VARIANT": "0"}),
    ((60, 50, 45), "box", 1, 2, 5, {"FFTSTENCIL_ALGO": "dense"}),
    ((3001,), "star", 1, 8, 21, {"FFTSTENCIL_SMALL1D": "0"}),
]


@pytest.mark.parametrize("ext,shape,r,T,steps,env", ENGINE_CAPPED)
def test_capped_grid_other_engines(fs, monkeypatch, ext, shape, r, T, steps, env):
    monkeypatch.setenv("FFTSTENCIL_MAX_CTAS", "1")
    for k, v in env.items():
        monkeypatch.setenv(k, v)
    w = wl.seeded_weights(shape, len(ext), r)
    u0 = wl.grid(ext, 7)
    got, info = run(fs, u0, w, r, T, steps)
    assert info["pair_end"] - info["pair_begin"] >= 8, info
    check(got, u0, w, r, steps, info)
