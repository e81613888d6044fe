"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Acceptance (BASELINE.json north_star): max|u_gpu - u_oracle| <= 1e-9 * max|u_oracle| in
FP64 after the full step count.  Inputs are the seeded synthetic recipe of synth/.
"""
import numpy as np
import pytest

import oracle
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


def run_gpu(fs, u0, w, r, T, steps, plan=None):
    p = plan or fs.Plan(u0.shape, w, r, T)
    a = torch.from_numpy(u0).cuda()
    b = torch.empty_like(a)
    p.run(a, b, steps)
    torch.cuda.synchronize()
    return b.cpu().numpy(), p


def rel_err(got, ref):
    return float(np.abs(got - ref).max() / np.abs(ref).max())


CASES = [
    # (extents, shape, r, T, steps, weights kind)
    ((4096,), "star", 1, 8, 64, "seeded"),       # BASELINE configs[0]
    ((4096,), "star", 1, 8, 64, "classic"),
    ((1001,), "star", 2, 5, 13, "seeded"),
    ((333,), "star", 3, 4, 9, "seeded"),
    ((67,), "star", 1, 8, 17, "seeded"),
    ((57,), "star", 1, 3, 1, "seeded"),
    ((129, 131), "box", 1, 8, 19, "seeded"),
    ((200, 173), "star", 1, 4, 11, "seeded"),
    ((97, 101), "star", 3, 4, 11, "seeded"),
    ((120, 90), "box", 3, 2, 7, "seeded"),
    ((75, 88), "box", 1, 1, 5, "seeded"),
    ((150, 140), "box", 1, 16, 35, "seeded"),
    ((100, 100), "box", 2, 3, 10, "seeded"),
    ((64, 64), "star", 1, 12, 27, "classic"),
    ((40, 41), "box", 1, 2, 3, "classic"),
    ((257, 77), "box", 3, 3, 8, "seeded"),
    ((20, 23, 19), "box", 1, 2, 5, "seeded"),
    ((24, 30, 28), "star", 1, 2, 7, "seeded"),
    ((33, 17, 25), "box", 1, 1, 3, "seeded"),
    ((40, 40, 40), "star", 1, 3, 7, "classic"),
    ((36, 29, 31), "box", 2, 3, 7, "seeded"),
    ((30, 30, 30), "star", 1, 4, 9, "seeded"),
    ((25, 26, 27), "box", 3, 2, 4, "seeded"),
    ((45, 38, 41), "box", 1, 2, 2, "classic"),
]


@pytest.mark.parametrize("ext,shape,r,T,steps,kind", CASES)
def test_parity_vs_oracle(fs, ext, shape, r, T, steps, kind):
    w = wl.stencil_weights(shape, len(ext), r, kind)
    u0 = wl.grid(ext, 11)
    got, p = run_gpu(fs, u0, w, r, T, steps)
    ref = oracle.stencil_run(u0, w, r, steps)
    err = rel_err(got, ref)
    assert err <= TOL, (err, p.info())
    ring = np.ones(ext, bool)
    ring[tuple(slice(r, e - r) for e in ext)] = False
    assert np.array_equal(got[ring], u0[ring])


@pytest.mark.parametrize("ext,shape,r,T,steps,kind", [c for c in CASES if len(c[0]) == 2])
@pytest.mark.parametrize("variant", ["0", "1", "2"])
def test_parity_dense_kernel(fs, monkeypatch, ext, shape, r, T, steps, kind, variant):
    """The dense L x L DFT-GEMM kernel (all variants) stays parity-green beside the factored default."""
    monkeypatch.setenv("FFTSTENCIL_ALGO", "dense")
    monkeypatch.setenv("FFTSTENCIL_VARIANT", variant)
    w = wl.stencil_weights(shape, 2, r, kind)
    u0 = wl.grid(ext, 13)
    got, p = run_gpu(fs, u0, w, r, T, steps)
    assert p.info()["algo"] == "dense"
    ref = oracle.stencil_run(u0, w, r, steps)
    assert rel_err(got, ref) <= TOL


@pytest.mark.parametrize("ext,shape,r,T,steps,kind", CASES[::3])
def test_band_kernels_agree(fs, monkeypatch, ext, shape, r, T, steps, kind):
    """The cone-restricted band kernel equals the first (reference) band kernel bitwise."""
    w = wl.stencil_weights(shape, len(ext), r, kind)
    u0 = wl.grid(ext, 17)
    fast, _ = run_gpu(fs, u0, w, r, T, steps)
    monkeypatch.setenv("FFTSTENCIL_BAND", "reference")
    ref, _ = run_gpu(fs, u0, w, r, T, steps)
    assert np.array_equal(fast, ref)


@pytest.mark.parametrize("ext,shape,r,T,steps,kind", [c for c in CASES if len(c[0]) == 2][::2])
def test_parity_unfused_ablation(fs, monkeypatch, ext, shape, r, T, steps, kind):
    """NEXT-3: the unfused three-kernel pass (spectrum through HBM) computes the same result."""
    monkeypatch.setenv("FFTSTENCIL_ALGO", "unfused")
    w = wl.stencil_weights(shape, 2, r, kind)
    u0 = wl.grid(ext, 29)
    got, p = run_gpu(fs, u0, w, r, T, steps)
    assert p.info()["algo"] == "unfused"
    ref = oracle.stencil_run(u0, w, r, steps)
    assert rel_err(got, ref) <= TOL


@pytest.mark.parametrize("ext,r,T,steps", [((96, 90), 1, 4, 8), ((96, 90), 1, 4, 12), ((500,), 1, 8, 16),
                                           ((500,), 1, 8, 24)])
def test_in_place_aliasing(fs, ext, r, T, steps):
    w = wl.seeded_weights("box" if len(ext) == 2 else "star", len(ext), r)
    u0 = wl.grid(ext, 5)
    p = fs.Plan(ext, w, r, T)
    a = torch.from_numpy(u0).cuda()
    p.run(a, a, steps)
    torch.cuda.synchronize()
    ref = oracle.stencil_run(u0, w, r, steps)
    assert rel_err(a.cpu().numpy(), ref) <= TOL


def test_zero_steps_copies(fs):
    u0 = wl.grid((50, 60), 1)
    got, _ = run_gpu(fs, u0, wl.seeded_weights("box", 2, 1), 1, 4, 0)
    assert np.array_equal(got, u0)


def test_T_invariance(fs):
    """G4: the same 24 steps with T in {1,2,3,4,6,8,12} agree within tolerance."""
    ext = (140, 133)
    w = wl.seeded_weights("box", 2, 1)
    u0 = wl.grid(ext, 2)
    ref = oracle.stencil_run(u0, w, 1, 24)
    for T in (1, 2, 3, 4, 6, 8, 12):
        got, p = run_gpu(fs, u0, w, 1, T, 24)
        assert p.info()["T"] == T
        assert rel_err(got, ref) <= TOL, T


def test_semigroup(fs):
    ext = (111, 123)
    w = wl.seeded_weights("star", 2, 3)
    u0 = wl.grid(ext, 3)
    p = fs.Plan(ext, w, 3, 4)
    a = torch.from_numpy(u0).cuda()
    b = torch.empty_like(a)
    c = torch.empty_like(a)
    p.run(a, b, 7)
    p.run(b, c, 9)
    d = torch.empty_like(a)
    p.run(a, d, 16)
    torch.cuda.synchronize()
    assert rel_err(c.cpu().numpy(), d.cpu().numpy()) <= 1e-12


def test_constant_field(fs):
    u0 = np.full((130, 170), 0.625)
    got, _ = run_gpu(fs, u0, wl.seeded_weights("box", 2, 1), 1, 8, 40)
    np.testing.assert_allclose(got, u0, rtol=1e-12)


def test_plane_wave_fixed_grid(fs):
    """G2: away from the fixed ring (distance >= r*steps) a plane wave scales by sigma^steps."""
    n0, n1, r, steps = 300, 280, 1, 40
    w = wl.seeded_weights("box", 2, r)
    th = (2 * np.pi * 5 / n0, 2 * np.pi * 3 / n1)
    c0, c1 = np.meshgrid(np.arange(n0), np.arange(n1), indexing="ij")
    u0 = np.cos(th[0] * c0 + th[1] * c1)
    sig = sum(w[i, j] * np.exp(1j * ((i - r) * th[0] + (j - r) * th[1])) for i in range(3) for j in range(3))
    got, _ = run_gpu(fs, u0, w, r, 8, steps)
    m = r * steps + r
    ref = np.real(sig ** steps * np.exp(1j * (th[0] * c0 + th[1] * c1)))
    assert np.abs(got[m:-m, m:-m] - ref[m:-m, m:-m]).max() <= 1e-12


def test_run_host_matches_device(fs):
    ext = (90, 70)
    w = wl.seeded_weights("box", 2, 1)
    u0 = wl.grid(ext, 8)
    p = fs.Plan(ext, w, 1, 4)
    dev, _ = run_gpu(fs, u0, w, 1, 4, 13, plan=p)
    out = np.empty_like(u0)
    p.run_host(u0, out, 13)
    assert np.array_equal(out, dev)


def test_3d_T_invariance_and_constant(fs):
    ext = (34, 31, 29)
    w = wl.seeded_weights("star", 3, 1)
    u0 = wl.grid(ext, 21)
    ref = oracle.stencil_run(u0, w, 1, 12)
    for T in (1, 2, 3, 4, 6):
        got, p = run_gpu(fs, u0, w, 1, T, 12)
        assert p.info()["T"] == T
        assert rel_err(got, ref) <= TOL, T
    c = np.full(ext, 1.75)
    got, _ = run_gpu(fs, c, wl.seeded_weights("box", 3, 1), 1, 2, 9)
    np.testing.assert_allclose(got, c, rtol=1e-12)


def test_plans_with_different_band_sizes_coexist(fs):
    """Regression (compute-sanitizer memcheck): the band kernel's shared-memory attribute is
    per function; a later plan with a smaller band must not break an earlier one."""
    w1 = wl.seeded_weights("box", 2, 3)
    big = fs.Plan((300, 260), w1, 3, 4)
    small = fs.Plan((120, 100), wl.seeded_weights("box", 2, 1), 1, 1)
    u = wl.grid((300, 260), 9)
    a = torch.from_numpy(u).cuda()
    b = torch.empty_like(a)
    big.run(a, b, 9)
    torch.cuda.synchronize()
    ref = oracle.stencil_run(u, w1, 3, 9)
    assert rel_err(b.cpu().numpy(), ref) <= TOL
    del small


# ---------------------------------------------------------------- periodic mode + flexible outputs (NEXT-2)
PERIODIC_CASES = [((300,), "star", 1, 8, 21), ((130, 141), "box", 1, 4, 11), ((96, 90), "star", 3, 2, 7),
                  ((34, 30, 28), "box", 1, 2, 5), ((40, 33, 36), "star", 1, 3, 7)]


@pytest.mark.parametrize("algo", ["factored", "dense"])
@pytest.mark.parametrize("ext,shape,r,T,steps", PERIODIC_CASES)
def test_periodic_parity_vs_oracle(fs, monkeypatch, algo, ext, shape, r, T, steps):
    monkeypatch.setenv("FFTSTENCIL_ALGO", algo)
    w = wl.seeded_weights(shape, len(ext), r)
    u0 = wl.grid(ext, 19)
    p = fs.Plan(ext, w, r, T, periodic=True)
    assert p.info()["periodic"]
    a = torch.from_numpy(u0).cuda()
    b = torch.empty_like(a)
    p.run(a, b, steps)
    torch.cuda.synchronize()
    ref = oracle.stencil_run(u0, w, r, steps, periodic=True)
    assert rel_err(b.cpu().numpy(), ref) <= TOL


@pytest.mark.parametrize("name,steps", [("heat2d", 1000), ("box2d49p", 200), ("box3d27p", 100)])
def test_periodic_plane_wave_full_grid(fs, name, steps):
    """Oracle-free full-grid pin at the BASELINE size: on a periodic grid a plane wave
    cos(theta.c) becomes Re(sigma(theta)^s e^{i theta.c}) exactly."""
    wk = wl.CONFIGS[name]
    w = wk.weights()
    nd, r = wk.ndim, wk.radius
    n = wk.extents
    ks = (3, 5, 2)[:nd]
    th = [2 * np.pi * ks[a] / n[a] for a in range(nd)]
    idx = np.meshgrid(*[np.arange(e, dtype=np.float64) for e in n], indexing="ij", sparse=True)
    phase = sum(th[a] * idx[a] for a in range(nd))
    sig = 0j
    for off in np.ndindex(*w.shape):
        sig += w[off] * np.exp(1j * sum((off[a] - r) * th[a] for a in range(nd)))
    u0 = np.cos(phase)
    p = fs.Plan(n, w, r, 0, periodic=True)
    a = torch.from_numpy(np.ascontiguousarray(u0)).cuda()
    del u0
    b = torch.empty_like(a)
    p.run(a, b, steps)
    torch.cuda.synchronize()
    del a
    got = b.cpu().numpy()
    ref = np.real(sig ** steps * np.exp(1j * phase))
    assert np.abs(got - ref).max() <= 1e-9


def test_run_emit_matches_separate_runs(fs):
    ext = (150, 130)
    w = wl.seeded_weights("box", 2, 1)
    u0 = wl.grid(ext, 23)
    p = fs.Plan(ext, w, 1, 8)
    a = torch.from_numpy(u0).cuda()
    steps = [0, 5, 13, 13, 40]
    outs = [torch.empty_like(a) for _ in steps]
    p.run_emit(a, outs, steps)
    torch.cuda.synchronize()
    for s, o in zip(steps, outs):
        ref = oracle.stencil_run(u0, w, 1, s)
        assert rel_err(o.cpu().numpy(), ref) <= TOL, s


def test_invalid_arguments(fs):
    w = wl.seeded_weights("box", 2, 1)
    with pytest.raises(fs.FftStencilError):
        fs.Plan((2, 50), w, 1, 4)
    p = fs.Plan((50, 50), w, 1, 4)
    a = torch.zeros((50, 50), dtype=torch.float64, device="cuda")
    with pytest.raises(fs.FftStencilError):
        p.run(a, a, -1)
    with pytest.raises(ValueError):
        p.run(a, torch.zeros((50, 51), dtype=torch.float64, device="cuda"), 1)
    with pytest.raises(TypeError):
        p.run(a.float(), a, 1)


def test_launch_count_reported(fs):
    ext = (200, 200)
    p = fs.Plan(ext, wl.seeded_weights("box", 2, 1), 1, 8)
    a = torch.zeros(ext, dtype=torch.float64, device="cuda")
    b = torch.empty_like(a)
    p.run(a, b, 20)   # 2 full passes + 1 remainder pass: (fused + band) x 3 + 4 ring boxes
    assert p.info()["last_run_launches"] == 3 * 2 + 4


# ---------------------------------------------------------------- full BASELINE sizes
@pytest.mark.parametrize("name,T", [("heat2d", 0), ("box2d9p", 0), ("star2d13p", 0), ("box2d49p", 0),
                                    ("heat2d", 8), ("box2d9p", 8), ("box2d9p", 1), ("heat2d", 16)])
def test_full_size_sampled(fs, name, T):
    """10240^2 at parity steps 2T+3; T = 0 is bench.py's own plan (automatic T, the launch
    configuration it times); sampled cells (interior, band, ring, tile seams) against the
    oracle's single-cell evaluation."""
    wk = wl.CONFIGS[name]
    w = wk.weights()
    u0 = wk.grid()
    T_plan = fs.describe(wk.extents, w, wk.radius, T)["T"]
    steps = 2 * T_plan + 3
    got, p = run_gpu(fs, u0, w, wk.radius, T, steps)
    assert p.info()["T"] == T_plan
    info = p.info()
    rng = np.random.default_rng(17)
    n = np.array(wk.extents)
    cells = [rng.integers(0, n) for _ in range(150)]
    h, S = info["halo"], info["valid"][0]
    for k in range(6):       # tile seams, band and ring cells
        for v in (h + k * S - 1, h + k * S, wk.radius - 1, wk.radius, h - 1, h, n[0] - h, n[0] - h - 1):
            cells.append(np.array([v, (v * 7 + 13) % n[1]]))
    cells = np.clip(np.array(cells), 0, n - 1)
    ref = oracle.stencil_point(u0, w, wk.radius, steps, cells)
    vals = got[tuple(cells.T)]
    scale = np.abs(u0).max()
    assert np.abs(vals - ref).max() <= TOL * scale
    # invariants over the whole grid: finite, max principle (w >= 0, sum 1)
    assert np.isfinite(got).all()
    assert got.min() >= u0.min() - 1e-9 and got.max() <= u0.max() + 1e-9


@pytest.mark.parametrize("name,T", [("heat3d", 0), ("box3d27p", 0), ("heat3d", 1), ("box3d27p", 3)])
def test_full_size_3d_sampled(fs, name, T):
    """1024^3 at parity steps 2T+3 (T = 0: bench.py's automatic plan); sampled cells against
    the single-cell oracle."""
    wk = wl.CONFIGS[name]
    w = wk.weights()
    u0 = wk.grid()
    steps = 2 * fs.describe(wk.extents, w, wk.radius, T)["T"] + 3
    got, p = run_gpu(fs, u0, w, wk.radius, T, steps)
    info = p.info()
    rng = np.random.default_rng(23)
    n = np.array(wk.extents)
    cells = [rng.integers(0, n) for _ in range(120)]
    h, S = info["halo"], info["valid"][0]
    for k in range(4):
        for v in (h + k * S - 1, h + k * S, 0, 1, h - 1, h, n[0] - h, n[0] - 1):
            cells.append(np.array([v, (v * 7 + 13) % n[1], (v * 3 + 5) % n[2]]))
            cells.append(np.array([(v * 5 + 1) % n[0], v, (v * 11 + 2) % n[2]]))
            cells.append(np.array([(v * 5 + 1) % n[0], (v * 3 + 9) % n[1], v]))
    cells = np.clip(np.array(cells), 0, n - 1)
    ref = oracle.stencil_point(u0, w, wk.radius, steps, cells)
    vals = got[tuple(cells.T)]
    assert np.abs(vals - ref).max() <= TOL * np.abs(u0).max()
    assert np.isfinite(got).all()
    assert got.min() >= u0.min() - 1e-9 and got.max() <= u0.max() + 1e-9


# ---------------------------------------------------------------- factored 1D tile (4096 = 64 x 64)
CT1D_CASES = [((20000,), 1, 1024, 2051), ((4200,), 1, 1024, 1500), ((9001,), 3, 0, None),
              ((12345,), 2, 100, 250), ((300000,), 1, 500, 1003), ((70000,), 2, 37, 80), ((5000,), 1, 8, 3)]


@pytest.mark.parametrize("ext,r,T,steps", CT1D_CASES)
def test_factored_1d_parity(fs, monkeypatch, ext, r, T, steps):
    """kernel_fft1d_ct.cu: ragged tile counts, an odd pair, remainder passes, deep T."""
    monkeypatch.setenv("FFTSTENCIL_ALGO", "factored")
    w = wl.seeded_weights("star", 1, r)
    u0 = wl.grid(ext, 31)
    p = fs.Plan(ext, w, r, T)
    info = p.info()
    assert info["algo"] == "factored" and info["tile"] == [4096]
    steps = steps or 2 * info["T"] + 3
    got, _ = run_gpu(fs, u0, w, r, T, steps, plan=p)
    ref = oracle.stencil_run(u0, w, r, steps)
    assert rel_err(got, ref) <= TOL, (rel_err(got, ref), info)
    assert np.array_equal(got[:r], u0[:r]) and np.array_equal(got[-r:], u0[-r:])


def test_factored_1d_default_plan_parity(fs):
    """Auto plan on a long 1D grid: the factored tile at T = 1024, two full passes + a remainder."""
    ext, r = (1 << 20,), 1
    w = wl.seeded_weights("star", 1, r)
    u0 = wl.grid(ext, 37)
    got, p = run_gpu(fs, u0, w, r, 0, 2500)
    assert p.info()["algo"] == "factored" and p.info()["T"] == 1024
    ref = oracle.stencil_run(u0, w, r, 2500)
    assert rel_err(got, ref) <= TOL


@pytest.mark.parametrize("name", ["heat1d_512m", "1d7p_512m"])
def test_full_size_1d_sampled(fs, name):
    """Table 3's 1D size (2^29 cells), 1000 steps in the launch configuration bench.py times:
    sampled cells (interior, tile seams, band, ring) against the single-cell oracle."""
    wk = wl.CONFIGS[name]
    w = wk.weights()
    u0 = wk.grid()
    steps = 1000
    got, p = run_gpu(fs, u0, w, wk.radius, 0, steps)
    info = p.info()
    n = wk.extents[0]
    h, S = info["halo"], info["valid"][0]
    rng = np.random.default_rng(41)
    cells = list(rng.integers(0, n, 120))
    for k in (0, 1, 2, 1000, (n - 2 * h) // S - 1):
        cells += [h + k * S - 1, h + k * S]
    cells += [0, wk.radius - 1, wk.radius, h - 1, h, n - h - 1, n - h, n - 1, n // 2]
    cells = np.clip(np.array(cells), 0, n - 1).reshape(-1, 1)
    ref = oracle.stencil_point(u0, w, wk.radius, steps, cells)
    vals = got[cells[:, 0]]
    assert np.abs(vals - ref).max() <= TOL * np.abs(u0).max()
    assert np.isfinite(got).all()
    assert got.min() >= u0.min() - 1e-9 and got.max() <= u0.max() + 1e-9


def test_periodic_plane_wave_1d_long(fs):
    """Oracle-free pin of the periodic factored 1D path on 2^25 cells, 3000 steps."""
    n, steps = 1 << 25, 3000
    w = wl.CONFIGS["1d5p_512m"].weights()
    r = 2
    th = 2 * np.pi * 7 / n
    c = np.arange(n, dtype=np.float64)
    sig = sum(w[o] * np.exp(1j * (o - r) * th) for o in range(2 * r + 1))
    p = fs.Plan((n,), w, r, 0, periodic=True)
    assert p.info()["algo"] == "factored"
    a = torch.from_numpy(np.cos(th * c)).cuda()
    b = torch.empty_like(a)
    p.run(a, b, steps)
    torch.cuda.synchronize()
    ref = np.real(sig ** steps * np.exp(1j * th * c))
    assert np.abs(b.cpu().numpy() - ref).max() <= 1e-9


CASES_3D = [c for c in CASES if len(c[0]) == 3]


@pytest.mark.parametrize("engine,tma", [("dmma", "1"), ("alu", "1"), ("alu", "0")])
@pytest.mark.parametrize("ext,shape,r,T,steps,kind", CASES_3D)
def test_parity_3d_engines(fs, monkeypatch, engine, tma, ext, shape, r, T, steps, kind):
    """Both line-DFT engines of the factored 3D tile (DFT-8 GEMMs on DMMA; radix-4 FFTs on the
    FP64 ALU, TMA-swizzled and cp.async staging) against the oracle."""
    monkeypatch.setenv("FFTSTENCIL_ALGO", "factored")
    monkeypatch.setenv("FFTSTENCIL_ENGINE", engine)
    monkeypatch.setenv("FFTSTENCIL_TMA", tma)
    w = wl.stencil_weights(shape, len(ext), r, kind)
    u0 = wl.grid(ext, 12)
    got, p = run_gpu(fs, u0, w, r, T, steps)
    assert p.info()["engine"] == engine
    ref = oracle.stencil_run(u0, w, r, steps)
    assert rel_err(got, ref) <= TOL, (rel_err(got, ref), p.info())


CASES_2D = [c for c in CASES if len(c[0]) == 2]


@pytest.mark.parametrize("engine,tma", [("dmma", "1"), ("alu", "1"), ("alu", "0")])
@pytest.mark.parametrize("ext,shape,r,T,steps,kind", CASES_2D)
def test_parity_2d_engines(fs, monkeypatch, engine, tma, ext, shape, r, T, steps, kind):
    """Both line-DFT engines of the factored 2D tile (DFT-8 GEMMs on DMMA; radix-8 butterflies on
    the FP64 ALU, TMA-swizzled and cp.async staging) against the oracle."""
    monkeypatch.setenv("FFTSTENCIL_ALGO", "factored")
    monkeypatch.setenv("FFTSTENCIL_ENGINE", engine)
    monkeypatch.setenv("FFTSTENCIL_TMA", tma)
    w = wl.stencil_weights(shape, len(ext), r, kind)
    u0 = wl.grid(ext, 13)
    got, p = run_gpu(fs, u0, w, r, T, steps)
    assert p.info()["engine"] == engine and p.info()["algo"] == "factored"
    ref = oracle.stencil_run(u0, w, r, steps)
    assert rel_err(got, ref) <= TOL, (rel_err(got, ref), p.info())


CASES_1D_LONG = [((20000,), 1, 1024, 2100), ((9000,), 3, 352, 800), ((70000,), 2, 512, 1100), ((12345,), 1, 300, 700),
                 ((131072,), 1, 1024, 2100), ((40960,), 3, 352, 1000), ((65536,), 2, 512, 1200)]


@pytest.mark.parametrize("engine,tma", [("dmma", "1"), ("alu", "1"), ("alu", "0")])
@pytest.mark.parametrize("ext,r,T,steps", CASES_1D_LONG)
def test_parity_1d_engines(fs, monkeypatch, engine, tma, ext, r, T, steps):
    """Both line engines of the factored 1D tile (4096 = 64 x 64 four-step) against the oracle;
    64-aligned grids with 64-aligned valid lengths take the TMA staging path."""
    monkeypatch.setenv("FFTSTENCIL_ALGO", "factored")
    monkeypatch.setenv("FFTSTENCIL_ENGINE", engine)
    monkeypatch.setenv("FFTSTENCIL_TMA", tma)
    w = wl.seeded_weights("star", 1, r)
    u0 = wl.grid(ext, 14)
    got, p = run_gpu(fs, u0, w, r, T, steps)
    assert p.info()["engine"] == engine and p.info()["T"] == T
    ref = oracle.stencil_run(u0, w, r, steps)
    assert rel_err(got, ref) <= TOL, (rel_err(got, ref), p.info())


# ---------------------------------------------------------------- small 1D grids: one launch per run
SMALL1D_CASES = [c for c in CASES if len(c[0]) == 1] + [((8192,), "star", 3, 4, 41, "seeded"),
                                                       ((5000,), "star", 2, 6, 6, "classic")]


@pytest.mark.parametrize("small", ["1", "0"])
@pytest.mark.parametrize("ext,shape,r,T,steps,kind", SMALL1D_CASES)
def test_small1d_whole_run_parity(fs, monkeypatch, small, ext, shape, r, T, steps, kind):
    """The on-chip whole-run kernel (kernel_small1d.cu) and the per-pass driver both match the
    oracle; the whole-run path is one launch per fftstencil_run."""
    monkeypatch.setenv("FFTSTENCIL_SMALL1D", small)
    w = wl.stencil_weights(shape, 1, r, kind)
    u0 = wl.grid(ext, 13)
    got, p = run_gpu(fs, u0, w, r, T, steps)
    ref = oracle.stencil_run(u0, w, r, steps)
    assert rel_err(got, ref) <= TOL, p.info()
    if small == "1" and p.info()["algo"] == "pfa":
        assert p.info()["last_run_launches"] == 1


def test_small1d_in_place_and_zero_steps(fs):
    ext, r, T = (4096,), 1, 8
    w = wl.seeded_weights("star", 1, r)
    u0 = wl.grid(ext, 17)
    p = fs.Plan(ext, w, r, T)
    a = torch.from_numpy(u0).cuda()
    p.run(a, a, 64)   # in == out
    torch.cuda.synchronize()
    assert rel_err(a.cpu().numpy(), oracle.stencil_run(u0, w, r, 64)) <= TOL
    b = torch.empty_like(a)
    p.run(a, b, 0)
    torch.cuda.synchronize()
    assert torch.equal(a, b)


# ---------------------------------------------------------------- beyond 2^31 cells (int32 indices)
def _window_ref(u_dev, w, r, steps, cell, ext):
    """Oracle value at `cell` from the dependency cone only: the sub-box of radius
    r*steps + 2r around it (clipped to the grid, whose faces keep the true fixed ring); a
    window face inside the grid is treated as fixed by the oracle, and its error front moves r
    cells per step, so it stops 2r cells short of `cell`."""
    R = r * steps + 2 * r
    lo = [max(0, c - R) for c in cell]
    hi = [min(e, c + R + 1) for c, e in zip(cell, ext)]
    sl = tuple(slice(a, b) for a, b in zip(lo, hi))
    sub = u_dev[sl].cpu().numpy()
    loc = np.array([[c - a for c, a in zip(cell, lo)]], dtype=np.int64)
    # a window face that is not a grid face must not be the oracle's ring at distance < R
    return float(oracle.stencil_point(sub, w, r, steps, loc)[0])


@pytest.mark.slow
@pytest.mark.parametrize("ext,shape,r", [((2 ** 31 - 4103,), "star", 1), ((2 ** 31 - 6400,), "star", 1),
                                         ((46341, 46341), "star", 1), ((46400, 46400), "box", 1),
                                         ((1296, 1296, 1296), "star", 1),
                                         ((1291, 1291, 1291), "box", 1)])
def test_beyond_int32_cells_sampled(fs, ext, shape, r):
    """The maximum-size edge case: 1D at the per-axis limit (extents < 2^31; unaligned ->
    cp.async loads, 64-aligned -> TMA), 2D and 3D grids of more than 2^31 cells (every cell
    offset needs 64 bits; odd row pitch -> cp.async, 16-byte pitch -> TMA); automatic T, two or more passes plus a remainder, sampled against the
    oracle on the cells' dependency cones (interior, flat offset 2^31, band, ring)."""
    w = wl.seeded_weights(shape, len(ext), r)
    g = torch.Generator(device="cuda")
    g.manual_seed(2 ** 31 + len(ext))
    u = torch.rand(ext, dtype=torch.float64, device="cuda", generator=g)
    p = fs.Plan(ext, w, r, 0)
    T = p.info()["T"]
    steps = 2 * T + 3 if len(ext) > 1 else T + 5
    out = torch.empty_like(u)
    p.run(u, out, steps)
    torch.cuda.synchronize()
    h = p.info()["halo"]
    total = int(np.prod(ext))
    flat = [f for f in (2 ** 31 - 1, 2 ** 31, 2 ** 31 + 1, total - 1) if f < total]
    cells = []
    for f in flat:   # cells around flat offset 2^31
        c, idx = int(f), []
        for e in reversed(ext):
            idx.append(c % e)
            c //= e
        cells.append(tuple(reversed(idx)))
    rng = np.random.default_rng(7)
    for _ in range(12):
        cells.append(tuple(int(rng.integers(0, e)) for e in ext))
    for d in (0, r - 1, r, h - 1, h, h + 1):
        cells.append(tuple(min(d, e - 1) for e in ext))
        cells.append(tuple(max(0, e - 1 - d) for e in ext))
    scale = float(u.abs().max())
    for cell in cells:
        ref = _window_ref(u, w, r, steps, cell, ext)
        got = float(out[cell].item())
        assert abs(got - ref) <= TOL * scale, (cell, got, ref, p.info())
    del u, out
    p.close()
    torch.cuda.empty_cache()
