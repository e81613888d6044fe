"""CPU tests of the C-ABI library's host side: symbols, plan builder tables, schedule.

No GPU is needed: libfftstencil.so loads without a device and fftstencil_describe /
fftstencil_export_aux run the host plan builder only.  The tables are pinned against
numpy's FFT (an independent route), the oracle's spectrum, and exhaustive coverage
checks; a numpy model of the fused tile algorithm that consumes the exported tables is
compared with the direct-stencil oracle.
"""
import os
import re

import numpy as np
import pytest

import oracle
from oracle import spectrum
from synth import workloads as wl

fs = pytest.importorskip("paper_conf_ppopp_hanlcbzyczcy25_b200")
from paper_conf_ppopp_hanlcbzyczcy25_b200 import _native  # noqa: E402

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_library_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "fftstencil.h")).read()
    declared = set(re.findall(r"\b(fftstencil_[a-z0-9_]+)\s*\(", hdr))
    assert declared == set(_native.EXPORTS)
    lib = _native.lib()
    for name in declared:
        assert hasattr(lib, name), name


def test_describe_rejects_invalid():
    w = wl.seeded_weights("box", 2, 1)
    with pytest.raises(fs.FftStencilError):
        fs.describe((2, 100), w, 1)          # extent <= 2r
    with pytest.raises(fs.FftStencilError):
        fs.describe((100, 100), w, 1, T=-1)
    with pytest.raises(ValueError):
        fs.describe((100, 100), w.reshape(-1)[:5], 1)
    bad = w.copy()
    bad[0] = np.nan
    with pytest.raises(fs.FftStencilError):
        fs.describe((100, 100), bad, 1)


@pytest.fixture
def dense(monkeypatch):
    monkeypatch.setenv("FFTSTENCIL_ALGO", "dense")


@pytest.fixture
def factored(monkeypatch):
    """The factored tile with its DFT-8-GEMM (DMMA) line engine."""
    monkeypatch.setenv("FFTSTENCIL_ALGO", "factored")
    monkeypatch.setenv("FFTSTENCIL_ENGINE", "dmma")


@pytest.fixture
def alu(monkeypatch):
    """The factored tile with its radix butterfly (FP64 ALU) line engine (the default)."""
    monkeypatch.setenv("FFTSTENCIL_ALGO", "factored")
    monkeypatch.setenv("FFTSTENCIL_ENGINE", "alu")


@pytest.mark.parametrize("r,T,L", [(1, 8, 48), (1, 1, 16), (1, 4, 24), (3, 4, 64)])
def test_describe_2d_geometry(dense, r, T, L):
    info = fs.describe((10240, 10240), wl.seeded_weights("box", 2, r), r, T)
    assert info["T"] == T and info["halo"] == r * T
    assert info["tile"] == [L, L] and info["valid"] == [L - 2 * r * T] * 2
    nt = -(-(10240 - 2 * r * T) // (L - 2 * r * T))
    assert info["tiles"] == nt * nt and info["pairs"] == (nt * nt + 1) // 2


def test_describe_auto_T_and_clamping():
    w = wl.seeded_weights("star", 2, 1)
    info = fs.describe((10240, 10240), w, 1, 0)
    assert 1 <= info["T"] <= 16
    small = fs.describe((20, 20), w, 1, 16)    # 2h < 20 forces T <= 9; tile forces S >= 8
    assert 2 * small["halo"] < 20 and small["valid"][0] >= 8
    one = fs.describe((4096,), wl.seeded_weights("star", 1, 1), 1, 8)
    assert one["tile"] == [56] and one["valid"] == [40] and one["pfa"] == [8, 7]


# ---------------------------------------------------------------- P1: DFT matrices
@pytest.mark.parametrize("T", [1, 4, 8, 12, 16])
def test_dft_matrix_vs_numpy(dense, T):
    w = wl.seeded_weights("box", 2, 1)
    info = fs.describe((4000, 4000), w, 1, T)
    L = info["tile"][0]
    v = fs.export_aux((4000, 4000), w, 1, T, which=0, axis=0)
    F = (v[0::2] + 1j * v[1::2]).reshape(L, L)
    np.testing.assert_allclose(F, np.fft.fft(np.eye(L), axis=0), atol=1e-14)


def test_pfa_dft_matrices_vs_numpy():
    w = wl.seeded_weights("star", 1, 1)
    for axis, N in ((0, 8), (1, 7)):
        v = fs.export_aux((4096,), w, 1, 8, which=0, axis=axis)
        F = (v[0::2] + 1j * v[1::2]).reshape(N, N)
        np.testing.assert_allclose(F, np.fft.fft(np.eye(N), axis=0), atol=1e-14)


# ---------------------------------------------------------------- P2: powered spectra
@pytest.mark.parametrize("shape,r,T", [("box", 1, 8), ("star", 3, 4), ("star", 1, 3)])
def test_spectra_2d_vs_oracle_spectrum(dense, shape, r, T):
    w = wl.seeded_weights(shape, 2, r)
    info = fs.describe((5000, 5000), w, r, T)
    L = info["tile"][0]
    for t in range(1, info["T"] + 1):
        v = fs.export_aux((5000, 5000), w, r, T, which=1, t=t)
        got = (v[0::2] + 1j * v[1::2]).reshape(L, L)
        ref = spectrum.powered_spectrum(w, r, (L, L), t)
        np.testing.assert_allclose(got, ref, atol=1e-15)


def test_spectrum_1d_ruritanian_vs_numpy_fft():
    """1D spectrum in Ruritanian order: G[k1][k2] = conj(fft(W_t wrapped))[(8 k2... )]/L."""
    w = wl.seeded_weights("star", 1, 1)
    T = 8
    L, N1, N2 = 56, 8, 7
    for t in (1, 5, 8):
        v = fs.export_aux((4096,), w, 1, T, which=1, t=t)
        G = (v[0::2] + 1j * v[1::2]).reshape(8, 8)
        Wt = np.ones(1)
        for _ in range(t):
            Wt = np.convolve(Wt, w)
        wrap = np.zeros(L)
        for i, val in enumerate(Wt):
            wrap[(i - t) % L] += val
        ref = np.conj(np.fft.fft(wrap)) / L
        for k1 in range(N1):
            for k2 in range(N2):
                assert abs(G[k1, k2] - ref[(k1 * N2 + k2 * N1) % L]) < 1e-15
            assert G[k1, 7] == 0


# ---------------------------------------------------------------- P3: PFA identity
def test_pfa_identity_with_exported_maps():
    """F_N1 . X . F_N2^T with X[l mod 8][l mod 7] = x[l] is fft(x) in Ruritanian order."""
    w = wl.seeded_weights("star", 1, 1)
    crt = fs.export_aux((4096,), w, 1, 8, which=3).astype(int).reshape(8, 7)
    assert sorted(crt.reshape(-1)) == list(range(56))
    for l1 in range(8):
        for l2 in range(7):
            assert crt[l1, l2] % 8 == l1 and crt[l1, l2] % 7 == l2
    v1 = fs.export_aux((4096,), w, 1, 8, which=0, axis=0)
    v2 = fs.export_aux((4096,), w, 1, 8, which=0, axis=1)
    F1 = (v1[0::2] + 1j * v1[1::2]).reshape(8, 8)
    F2 = (v2[0::2] + 1j * v2[1::2]).reshape(7, 7)
    x = np.random.default_rng(3).random(56) + 1j * np.random.default_rng(4).random(56)
    X = x[crt]
    G = F1 @ X @ F2.T
    ref = np.fft.fft(x)
    for k1 in range(8):
        for k2 in range(7):
            assert abs(G[k1, k2] - ref[(k1 * 7 + k2 * 8) % 56]) < 1e-12


# ---------------------------------------------------------------- P4: coverage
def _cover(ext, r, T, shape):
    nd = len(ext)
    w = wl.seeded_weights(shape, nd, r)
    info = fs.describe(ext, w, r, T)
    h = info["halo"]
    count = np.zeros(ext, dtype=np.int32)
    tiles = fs.export_aux(ext, w, r, T, which=2).astype(np.int64).reshape(info["tiles"], nd, 3)
    for t in tiles:
        sl = tuple(slice(t[a, 1], t[a, 1] + t[a, 2]) for a in range(nd))
        count[sl] += 1
    off = 3 - nd
    for kind in (4, 5):
        vals = fs.export_aux(ext, w, r, T, which=kind)
        step = 7 if kind == 4 else 6
        for b in vals.astype(np.int64).reshape(-1, step):
            sl = tuple(slice(b[off + a], b[3 + off + a]) for a in range(nd))
            count[sl] += 1
            for e in range(off):
                assert b[e] == 0 and b[3 + e] == 1
    return count, h


@pytest.mark.parametrize("ext,r,T,shape", [((100, 77), 1, 8, "box"), ((33, 41), 3, 2, "star"),
                                            ((4096,), 1, 8, "star"), ((301,), 2, 5, "star"),
                                            ((30, 29), 1, 1, "box")])
def test_tiles_band_ring_partition_grid_exactly(ext, r, T, shape):
    count, h = _cover(ext, r, T, shape)
    assert count.min() == 1 and count.max() == 1


def test_3d_geometry_partitions_grid():
    count, h = _cover((20, 23, 19), 1, 2, "box")
    assert count.min() == 1 and count.max() == 1


# ---------------------------------------------------------------- P5: tile algorithm model
def _model_2d(u, w, r, T, steps):
    """numpy model of the fused pass as the kernel runs it, fed with the exported tables."""
    ext = u.shape
    info = fs.describe(ext, w, r, T)
    L, S, h, T = info["tile"][0], info["valid"][0], info["halo"], info["T"]
    v = fs.export_aux(ext, w, r, T, which=0, axis=0)
    F = (v[0::2] + 1j * v[1::2]).reshape(L, L)
    tiles = fs.export_aux(ext, w, r, T, which=2).astype(np.int64).reshape(info["tiles"], 2, 3)
    rings = fs.export_aux(ext, w, r, T, which=5).astype(np.int64).reshape(-1, 6)
    bands = fs.export_aux(ext, w, r, T, which=4).astype(np.int64).reshape(-1, 7)
    cur = u.copy()
    done = 0
    while done < steps:
        t = min(T, steps - done)
        sv = fs.export_aux(ext, w, r, T, which=1, t=t)
        St = (sv[0::2] + 1j * sv[1::2]).reshape(L, L)
        nxt = np.full_like(cur, np.nan)
        for b in rings:
            sl = (slice(b[1], b[4]), slice(b[2], b[5]))
            nxt[sl] = cur[sl]
        pad = np.zeros((ext[0] + L, ext[1] + L))
        pad[:ext[0], :ext[1]] = cur
        for i in range(0, len(tiles), 2):
            pair = tiles[i:i + 2]
            xa = pad[pair[0, 0, 0]:pair[0, 0, 0] + L, pair[0, 1, 0]:pair[0, 1, 0] + L]
            xb = pad[pair[1, 0, 0]:pair[1, 0, 0] + L, pair[1, 1, 0]:pair[1, 1, 0] + L] if len(pair) > 1 else 0 * xa
            Z = F @ (xa + 1j * xb) @ F.T                    # Alg. 1 line 1
            Z = Z * St                                      # line 2 (Eq. 10)
            G = np.conj(F)[h:h + S]
            Y = G @ Z @ G.T                                 # lines 3-4, crop-aware
            for k, part in enumerate((Y.real, Y.imag)[:len(pair)]):
                tl = pair[k]
                n0, n1 = tl[0, 2], tl[1, 2]
                nxt[tl[0, 1]:tl[0, 1] + n0, tl[1, 1]:tl[1, 1] + n1] = part[:n0, :n1]
        for b in bands:   # band: t direct steps (model uses the oracle definition)
            lo, hi = b[1:3], b[4:6]
            g = r * t
            rl = np.maximum(lo - g, 0)
            rh = np.minimum(hi + g, ext)
            sub = oracle.stencil_run(cur, w, r, t)[lo[0]:hi[0], lo[1]:hi[1]]
            nxt[lo[0]:hi[0], lo[1]:hi[1]] = sub
            del rl, rh
        assert not np.isnan(nxt).any()
        cur = nxt
        done += t
    return cur


@pytest.mark.parametrize("ext,shape,r,T,steps", [((61, 70), "box", 1, 4, 11), ((58, 47), "star", 3, 2, 5),
                                                   ((40, 40), "box", 1, 8, 8)])
def test_tile_algorithm_model_matches_oracle(dense, ext, shape, r, T, steps):
    w = wl.seeded_weights(shape, 2, r)
    u = wl.grid(ext, 99)
    got = _model_2d(u, w, r, T, steps)
    ref = oracle.stencil_run(u, w, r, steps)
    assert np.abs(got - ref).max() <= 1e-12 * np.abs(ref).max()


# ---------------------------------------------------------------- factored (CT 64 = 8 x 8) tables
def test_factored_is_default_for_2d_and_geometry():
    info = fs.describe((10240, 10240), wl.seeded_weights("star", 2, 1), 1, 0)
    assert info["algo"] == "factored" and info["tile"] == [64, 64]
    assert info["valid"][0] == 64 - 2 * info["halo"]


def test_factored_dft8_and_twiddles_vs_numpy(factored):
    w = wl.seeded_weights("box", 2, 1)
    v = fs.export_aux((1000, 1000), w, 1, 8, which=0, axis=0)
    F8 = (v[0::2] + 1j * v[1::2]).reshape(8, 8)
    np.testing.assert_allclose(F8, np.fft.fft(np.eye(8), axis=0), atol=1e-15)
    v = fs.export_aux((1000, 1000), w, 1, 8, which=0, axis=1)
    tw = (v[0::2] + 1j * v[1::2]).reshape(8, 8)
    ref = np.exp(-2j * np.pi * np.outer(np.arange(8), np.arange(8)) / 64)
    np.testing.assert_allclose(tw, ref, atol=1e-15)


@pytest.mark.parametrize("shape,r,T", [("box", 1, 8), ("star", 3, 4), ("box", 2, 5)])
def test_factored_spectrum_digit_order(factored, shape, r, T):
    """Kernel order [k1][8 g + c] holds k0 = g + 8 c (the CT output digit order)."""
    w = wl.seeded_weights(shape, 2, r)
    info = fs.describe((3000, 3000), w, r, T)
    for t in (1, info["T"]):
        v = fs.export_aux((3000, 3000), w, r, T, which=1, t=t)
        G = (v[0::2] + 1j * v[1::2]).reshape(64, 64)
        ref = spectrum.powered_spectrum(w, r, (64, 64), t)    # [k0][k1]
        m = np.arange(64)
        k0 = (m // 8) + 8 * (m % 8)
        np.testing.assert_allclose(G, ref[k0, :].T, atol=1e-15)


def _ct_axis(x, F8, tw, inverse=False):
    """The kernel's per-axis factorisation, stage by stage (numpy, last axis)."""
    sh = x.shape
    x = x.reshape(-1, 64)
    out = np.empty_like(x)
    Fm, T = (np.conj(F8), np.conj(tw)) if inverse else (F8, tw)
    for n, line in enumerate(x):
        if not inverse:
            B = line.reshape(8, 8)               # [la][lb]
            C = (Fm @ B) * T                     # [ka][lb]
            C = C @ Fm.T                         # [ka][kb]
            out[n] = C.T.reshape(-1)             # k = ka + 8 kb
        else:
            B = line.reshape(8, 8)               # [kb][ka]  (k = ka + 8 kb)
            Z = (Fm @ B) * T.T                   # [lb][ka]
            out[n] = (Fm @ Z.T).reshape(-1)      # [la][lb]: l = 8 la + lb
    return out.reshape(sh)


def test_factored_chain_model_matches_numpy_fft(factored):
    w = wl.seeded_weights("box", 2, 1)
    v = fs.export_aux((1000, 1000), w, 1, 8, which=0, axis=0)
    F8 = (v[0::2] + 1j * v[1::2]).reshape(8, 8)
    v = fs.export_aux((1000, 1000), w, 1, 8, which=0, axis=1)
    tw = (v[0::2] + 1j * v[1::2]).reshape(8, 8)
    rng = np.random.default_rng(5)
    X = rng.random((64, 64)) + 1j * rng.random((64, 64))
    np.testing.assert_allclose(_ct_axis(X, F8, tw), np.fft.fft(X, axis=1), atol=1e-12)
    Y = _ct_axis(np.fft.fft2(X), F8, tw, inverse=True) / 64
    np.testing.assert_allclose(Y, np.fft.ifft(np.fft.fft2(X), axis=1), atol=1e-12)


# ---------------------------------------------------------------- periodic mode (NEXT-2)
@pytest.mark.parametrize("ext,shape,r,T", [((100, 77), "box", 1, 8), ((301,), "star", 2, 5), ((20, 23, 19), "box", 1, 2),
                                           ((64, 64), "star", 3, 4)])
def test_periodic_tiles_cover_grid_exactly_once(ext, shape, r, T):
    nd = len(ext)
    w = wl.seeded_weights(shape, nd, r)
    info = fs.describe(ext, w, r, T, periodic=True)
    assert info["periodic"] and info["band_blocks"] == 0
    count = np.zeros(ext, dtype=np.int32)
    # export_aux describes the fixed-ring plan; rebuild the periodic tile ownership from describe
    S = info["valid"]
    nt = [-(-ext[a] // S[a]) for a in range(nd)]
    assert info["tiles"] == int(np.prod(nt))
    for idx in np.ndindex(*nt):
        sl = tuple(slice(idx[a] * S[a], min(idx[a] * S[a] + S[a], ext[a])) for a in range(nd))
        count[sl] += 1
    assert count.min() == 1 and count.max() == 1


# ---------------------------------------------------------------- factored 1D (4096 = 64 x 64)
def test_factored_1d_is_default_for_long_grids(monkeypatch):
    """The cost model takes the long tile for deep fusion: T = L / (4r) maximises S T
    (DMMA line engine; the ALU engine's choice is pinned by test_alu_1d_default_...)."""
    monkeypatch.setenv("FFTSTENCIL_ENGINE", "dmma")
    for r in (1, 2, 3):
        info = fs.describe((1 << 24,), wl.seeded_weights("star", 1, r), r, 0)
        assert info["algo"] == "factored" and info["tile"] == [4096] and info["pfa"] == [64, 64]
        assert info["T"] == 1024 // r and info["valid"] == [4096 - 2 * r * (1024 // r)]
    # BASELINE configs[0] (4096 cells, T = 8 fixed) keeps the paper's 8 x 7 prime-factor tile
    assert fs.describe((4096,), wl.seeded_weights("star", 1, 1), 1, 8)["algo"] == "pfa"


def _tables_1d(n, w, r, T):
    F8 = fs.export_aux((n,), w, r, T, which=0, axis=0)
    tw = fs.export_aux((n,), w, r, T, which=0, axis=1)
    W = fs.export_aux((n,), w, r, T, which=0, axis=2)
    c = lambda v, s: (v[0::2] + 1j * v[1::2]).reshape(s)   # noqa: E731
    return c(F8, (8, 8)), c(tw, (8, 8)), c(W, (64, 64))


def test_factored_1d_tables_vs_numpy(factored):
    F8, tw, W = _tables_1d(20000, wl.seeded_weights("star", 1, 1), 1, 100)
    np.testing.assert_allclose(F8, np.fft.fft(np.eye(8), axis=0), atol=1e-15)
    np.testing.assert_allclose(tw, np.exp(-2j * np.pi * np.outer(np.arange(8), np.arange(8)) / 64), atol=1e-15)
    np.testing.assert_allclose(W, np.exp(-2j * np.pi * np.outer(np.arange(64), np.arange(64)) / 4096), atol=1e-15)


def _four_step_pass(x, F8, tw, W, G):
    """numpy model of kernel_fft1d_ct.cu on one complex tile: the four-step DFT-4096 as the
    kernel orders it (plane[b][a] = x[a + 64 b]), * S in the kernel's [c][8 g + m] order,
    and the inverse steps backwards."""
    P = x.reshape(64, 64)                                # [b][a]
    Y = _ct_axis(P.T, F8, tw).T * W.T                    # phase 1: over b -> [c][a], * w4096^(a c)
    X = _ct_axis(Y, F8, tw)                              # phase 2: over a -> [c][d]
    m = np.arange(64)
    d_of = (m // 8) + 8 * (m % 8)                        # device column 8 g + m' holds d = g + 8 m'
    Sn = np.empty((64, 64), complex)
    Sn[:, d_of] = G                                      # natural [c][d]
    Z = _ct_axis(X * Sn, F8, tw, inverse=True)           # over d -> [c][a]
    Z = Z * np.conj(W.T)                                 # phase 3: * w4096^(-a c)
    return X, _ct_axis(Z.T, F8, tw, inverse=True).T      # over c -> [b][a]


@pytest.mark.parametrize("r,T", [(1, 1024), (2, 300), (3, 17)])
def test_factored_1d_four_step_model_matches_oracle(factored, r, T):
    """The exported tables, run through the kernel's four-step order, give fft(x) at
    k = c + 64 d, and one fused pass equals T direct steps (the oracle) on [h, 4096 - h)."""
    n = 4096
    w = wl.seeded_weights("star", 1, r)
    info = fs.describe((n,), w, r, T)
    assert info["tile"] == [4096] and info["T"] == T
    h = info["halo"]
    F8, tw, W = _tables_1d(n, w, r, T)
    v = fs.export_aux((n,), w, r, T, which=1, t=T)
    G = (v[0::2] + 1j * v[1::2]).reshape(64, 64)
    u = wl.grid((n,), 7)
    u2 = wl.grid((n,), 8)
    X, y = _four_step_pass(u + 1j * u2, F8, tw, W, G)
    ref = np.fft.fft(u + 1j * u2)
    np.testing.assert_allclose(X, ref.reshape(64, 64).T, atol=1e-10)   # X[c][d] = fft[c + 64 d]
    y = y.reshape(-1)
    for part, src in ((y.real, u), (y.imag, u2)):
        want = oracle.stencil_run(src, w, r, T)
        err = np.abs(part[h:n - h] - want[h:n - h]).max()
        assert err <= 1e-11 * np.abs(want).max(), err


@pytest.mark.parametrize("ext,r,T", [((20000,), 1, 1024), ((9000,), 3, 200), ((5000,), 2, 0)])
def test_factored_1d_tiles_band_ring_partition(factored, ext, r, T):
    count, h = _cover(ext, r, T, "star")
    assert count.min() == 1 and count.max() == 1


# ---------------------------------------------------------------- ALU engine (radix butterflies) tables
def test_alu_engine_is_the_default_for_2d_and_3d():
    for ext, shape, r in (((10240, 10240), "star", 1), ((1024, 1024, 1024), "star", 1)):
        info = fs.describe(ext, wl.seeded_weights(shape, len(ext), r), r, 0)
        assert info["algo"] == "factored" and info["engine"] == "alu", info
        assert info["mma_flops_per_pass"] == 0 and info["alu_ops_per_pass"] > 0


def test_alu_w64_table_vs_numpy(alu):
    w = wl.seeded_weights("box", 2, 1)
    v = fs.export_aux((1000, 1000), w, 1, 8, which=0, axis=0)
    tw = v[0::2] + 1j * v[1::2]
    np.testing.assert_allclose(tw, np.fft.fft(np.eye(64)[1]), atol=1e-15)   # w64^m = exp(-2 pi i m / 64)


def _pos(m):
    """Position of frequency m = k0 + 4 k' on an axis of the 2D ALU engine: p = 16 k0 + k'."""
    return 16 * (m % 4) + m // 4


@pytest.mark.parametrize("shape,r,T", [("box", 1, 8), ("star", 3, 4)])
def test_alu_2d_spectrum_position_order(alu, shape, r, T):
    w = wl.seeded_weights(shape, 2, r)
    info = fs.describe((3000, 3000), w, r, T)
    for t in (1, info["T"]):
        v = fs.export_aux((3000, 3000), w, r, T, which=1, t=t)
        G = (v[0::2] + 1j * v[1::2]).reshape(64, 64)
        ref = spectrum.powered_spectrum(w, r, (64, 64), t)    # [k0][k1], 1/4096 folded in
        m = np.arange(64)
        np.testing.assert_allclose(G[np.ix_(_pos(m), _pos(m))], ref, atol=1e-15)


def test_alu_3d_spectrum_natural_order(alu):
    w = wl.seeded_weights("box", 3, 1)
    v = fs.export_aux((200, 200, 200), w, 1, 2, which=1, t=2)
    G = (v[0::2] + 1j * v[1::2]).reshape(16, 16, 16)
    np.testing.assert_allclose(G, spectrum.powered_spectrum(w, 1, (16, 16, 16), 2), atol=1e-15)


def _dft(x, axis, inverse=False):
    """DFT along `axis` (numpy's definition; conj kernel unnormalised for the inverse)."""
    return np.fft.ifft(x, axis=axis) * x.shape[axis] if inverse else np.fft.fft(x, axis=axis)


def _alu_2d_tile(Z, tw, Sp, h, S):
    """The 2D ALU engine's five passes on one complex 64 x 64 tile, index for index
    (kernel_fft2d_bf.cu): element (16 i + rr, 16 j + cc) of the tile is X[i][rr][j][cc];
    twiddles from the exported w64 table, S_T in its exported position order."""
    W = lambda e: tw[np.mod(e, 64)]
    q = np.arange(4)[:, None, None, None], np.arange(16)[None, :, None, None]
    qc = np.arange(4)[None, None, :, None], np.arange(16)[None, None, None, :]
    X = Z.reshape(4, 16, 4, 16).copy()
    # P1: DFT-4 over i and over j, * w64^(rr k0r) w64^(cc k0c)
    X = _dft(_dft(X, 0), 2) * W(q[1] * q[0]) * W(qc[1] * qc[0])
    # P2: DFT-16 over cc (axis 1); position 16 j + k' holds frequency j + 4 k'
    X = _dft(X, 3)
    # P3: DFT-16 over rr (axis 0), * S_T at the positions, inverse DFT-16
    X = _dft(_dft(X, 1) * Sp.reshape(4, 16, 4, 16), 1, inverse=True)
    # P4: inverse DFT-16 over cc
    X = _dft(X, 3, inverse=True)
    # P5: * conj twiddles, inverse DFT-4 over j and i
    X = X * np.conj(W(q[1] * q[0]) * W(qc[1] * qc[0]))
    X = _dft(_dft(X, 2, inverse=True), 0, inverse=True).reshape(64, 64)
    return X[h:h + S, h:h + S]


@pytest.mark.parametrize("shape,r,T", [("box", 1, 11), ("star", 3, 4), ("box", 2, 5)])
def test_alu_2d_stage_model_vs_overlap_save(alu, shape, r, T):
    """The stage sequence with the exported tables equals the tile's T-step circular
    convolution (ifft2(fft2(x) sigma^T)) on the valid window, for two packed real tiles."""
    w = wl.seeded_weights(shape, 2, r)
    ext = (3000, 3000)
    info = fs.describe(ext, w, r, T)
    h, S, T = info["halo"], info["valid"][0], info["T"]
    v = fs.export_aux(ext, w, r, T, which=0, axis=0)
    tw = v[0::2] + 1j * v[1::2]
    v = fs.export_aux(ext, w, r, T, which=1, t=T)
    Sp = (v[0::2] + 1j * v[1::2]).reshape(64, 64)
    rng = np.random.default_rng(5)
    xa, xb = rng.random((64, 64)), rng.random((64, 64))
    got = _alu_2d_tile(xa + 1j * xb, tw, Sp, h, S)
    sig = spectrum.powered_spectrum(w, r, (64, 64), T) * 4096
    for x, part in ((xa, got.real), (xb, got.imag)):
        ref = np.fft.ifft2(np.fft.fft2(x) * sig).real[h:h + S, h:h + S]
        np.testing.assert_allclose(part, ref, atol=1e-12)
        # and the direct-stencil oracle on the tile (valid window = exact T-step result)
        direct = oracle.stencil_run(np.pad(x, 0), w, r, T, periodic=True)[h:h + S, h:h + S]
        np.testing.assert_allclose(part, direct, atol=1e-11)


# ---------------------------------------------------------------- ALU engine, 1D (4096 = 64 x 64)
def test_alu_1d_default_and_aligned_valid_length():
    """The ALU engine is the 1D default for long grids; its cost model prefers T with S a
    multiple of 64 (tile origins on 64-cell rows: TMA staging) at < 1% loss of S T."""
    for r in (1, 2, 3):
        info = fs.describe((1 << 24,), wl.seeded_weights("star", 1, r), r, 0)
        assert info["algo"] == "factored" and info["engine"] == "alu" and info["tile"] == [4096]
        S, T = info["valid"][0], info["T"]
        assert S % 64 == 0 and S * T >= 0.99 * max((4096 - 2 * r * t) * t for t in range(1, 2048 // r))


def _alu_1d_tables(n, w, r, T):
    c = lambda v: v[0::2] + 1j * v[1::2]   # noqa: E731
    return c(fs.export_aux((n,), w, r, T, which=0, axis=0)), c(fs.export_aux((n,), w, r, T, which=0, axis=2))


def test_alu_1d_tables_vs_numpy(alu):
    w64, w4k = _alu_1d_tables(20000, wl.seeded_weights("star", 1, 1), 1, 100)
    np.testing.assert_allclose(w64, np.exp(-2j * np.pi * np.arange(64) / 64), atol=1e-15)
    np.testing.assert_allclose(w4k, np.exp(-2j * np.pi * np.arange(256) / 4096), atol=1e-15)


def _alu_1d_tile(x, w64, w4k, Sq):
    """The 1D ALU engine's seven passes on one complex 4096-cell tile (kernel_fft1d_bf.cu):
    plane[b][a] = x[a + 64 b] viewed as [i][rr][j][cc] with b = 16 i + rr, a = 16 j + cc;
    S_T in its exported [column position][row position] order."""
    W = lambda e: w64[np.mod(e, 64)]                                     # noqa: E731
    i4, r16 = np.arange(4)[:, None, None, None], np.arange(16)[None, :, None, None]
    j4, c16 = np.arange(4)[None, None, :, None], np.arange(16)[None, None, None, :]
    a = 16 * j4 + c16                                                    # column (cell digit a)
    X = x.reshape(4, 16, 4, 16).copy()
    X = _dft(X, 0) * W(r16 * i4)                                         # P1: column stage 1
    X = _dft(X, 1)                                                       # P2: column stage 2 -> c
    c = i4 + 4 * r16                                                     # row position 16 i + rr <-> c
    tw4096 = w4k[np.mod(a * i4, 4096)] * w4k[np.mod(4 * a, 4096)] ** r16   # base * step^c'
    X = X * tw4096
    X = _dft(X, 2) * W(c16 * j4)                                         # P3: row stage 1
    F = _dft(X, 3)                                                       # P4: row stage 2 -> d
    Sp = Sq.T.reshape(4, 16, 4, 16)                                      # [row pos][column pos]
    X = _dft(F * Sp, 3, inverse=True)
    X = _dft(X * np.conj(W(c16 * j4)), 2, inverse=True)                  # P5
    X = _dft(X * np.conj(tw4096), 1, inverse=True)                       # P6
    X = _dft(X * np.conj(W(r16 * i4)), 0, inverse=True)                  # P7
    return F, X.reshape(-1)


@pytest.mark.parametrize("r,T", [(1, 1024), (2, 512), (3, 352), (3, 17)])
def test_alu_1d_pass_model_matches_fft_and_oracle(alu, r, T):
    """Run through the seven passes, the exported tables give fft(x) at the frequency
    positions (row 16 c0 + c' <-> c = c0 + 4 c', column 16 d0 + d' <-> d = d0 + 4 d',
    k = c + 64 d), and one fused pass equals T direct steps (the oracle) on [h, 4096 - h)."""
    n = 4096
    w = wl.seeded_weights("star", 1, r)
    info = fs.describe((n,), w, r, T)
    assert info["engine"] == "alu" and info["T"] == T
    h = info["halo"]
    w64, w4k = _alu_1d_tables(n, w, r, T)
    v = fs.export_aux((n,), w, r, T, which=1, t=T)
    Sq = (v[0::2] + 1j * v[1::2]).reshape(64, 64)
    u, u2 = wl.grid((n,), 7), wl.grid((n,), 8)
    F, y = _alu_1d_tile(u + 1j * u2, w64, w4k, Sq)
    ref = np.fft.fft(u + 1j * u2)
    pos = lambda f: 16 * (f % 4) + f // 4                                 # noqa: E731
    k = np.arange(n)
    got = F.reshape(64, 64)[pos(k % 64), pos(k // 64)]
    np.testing.assert_allclose(got, ref, atol=1e-10)
    for part, src in ((y.real, u), (y.imag, u2)):
        want = oracle.stencil_run(src, w, r, T)
        err = np.abs(part[h:n - h] - want[h:n - h]).max()
        assert err <= 1e-11 * np.abs(want).max(), err
