"""Pins for the CPU oracle (oracle/): checked against things other than itself.

Each test names what fixes the expected value: a hand-worked example
(tests/golden/*.json), a closed form, a library routine on a special case, or an
invariant of the definition (§2.2, Eq. 2, Fig. 2 left, Eq. 10).
"""
import json
import os

import numpy as np
import pytest
from scipy import signal

import oracle
from oracle import spectrum
from synth import workloads as wl

RNG = np.random.default_rng(7)


def _load(golden_dir, name):
    with open(os.path.join(golden_dir, name)) as f:
        return json.load(f)


# ---------------------------------------------------------------- hand-worked examples
def test_golden_hand_1d(golden_dir):
    g = _load(golden_dir, "hand_1d_n7_w123_2steps.json")
    u0 = np.array(g["u0"], dtype=float)
    w = np.array(g["weights"], dtype=float)
    one = oracle.stencil_run(u0, w, g["radius"], 1)
    assert one.tolist() == g["after_step_1"]
    out = oracle.stencil_run(u0, w, g["radius"], g["steps"])
    assert out.tolist() == g["expected"]


def test_golden_hand_2d(golden_dir):
    g = _load(golden_dir, "hand_2d_4x4_star_1step.json")
    out = oracle.stencil_run(np.array(g["u0"], float), np.array(g["weights"], float), 1, 1)
    assert out.tolist() == g["expected"]


def test_golden_hand_3d(golden_dir):
    g = _load(golden_dir, "hand_3d_3x3x3_box_1step.json")
    u0 = np.arange(27, dtype=float).reshape(3, 3, 3)
    w = np.arange(1, 28, dtype=float)
    out = oracle.stencil_run(u0, w, 1, 1)
    assert out[1, 1, 1] == g["centre_expected"]
    mask = np.ones((3, 3, 3), bool)
    mask[1, 1, 1] = False
    assert np.array_equal(out[mask], u0[mask])  # every other cell is ring


def test_golden_binomial(golden_dir):
    g = _load(golden_dir, "heat1d_binomial.json")
    u0 = np.zeros(g["n"])
    u0[g["impulse_at"]] = 1.0
    out = oracle.stencil_run(u0, g["weights"], 1, g["steps"])
    for o, num in zip(g["offsets"], g["numerators"]):
        assert out[g["impulse_at"] + o] == num / g["denominator"]
    assert np.count_nonzero(out) == len(g["offsets"])


def test_hand_expanded_two_steps_symbolic():
    """u2[3] = a^2 u1 + 2ab u2 + (2ac+b^2) u3 + 2bc u4 + c^2 u5 and the ring-adjacent cell."""
    a, b, c = 0.3, 0.5, 0.2 + 1e-3
    u = RNG.random(7)
    out = oracle.stencil_run(u, [a, b, c], 1, 2)
    exp3 = a * a * u[1] + 2 * a * b * u[2] + (2 * a * c + b * b) * u[3] + 2 * b * c * u[4] + c * c * u[5]
    assert out[3] == pytest.approx(exp3, rel=1e-14)
    exp1 = a * u[0] + b * (a * u[0] + b * u[1] + c * u[2]) + c * (a * u[1] + b * u[2] + c * u[3])
    assert out[1] == pytest.approx(exp1, rel=1e-14)
    exp5 = a * (a * u[3] + b * u[4] + c * u[5]) + b * (a * u[4] + b * u[5] + c * u[6]) + c * u[6]
    assert out[5] == pytest.approx(exp5, rel=1e-14)
    assert out[0] == u[0] and out[6] == u[6]


# ---------------------------------------------------------------- library special cases
@pytest.mark.parametrize("nd,r,steps", [(1, 1, 5), (1, 3, 3), (2, 1, 4), (2, 2, 2), (3, 1, 3)])
def test_impulse_response_is_convolution_power(nd, r, steps):
    """delta deep in the interior -> the steps-fold correlation kernel (scipy.signal.convolve)."""
    w = RNG.uniform(0.1, 1.0, size=(2 * r + 1,) * nd)
    h = r * steps
    n = 2 * h + 2 * r + 5
    u0 = np.zeros((n,) * nd)
    centre = (n // 2,) * nd
    u0[centre] = 1.0
    out = oracle.stencil_run(u0, w, r, steps)
    # correlation u'[c] = sum_o w[o] u[c+o] is convolution with the flipped kernel
    wf = w[(slice(None, None, -1),) * nd]
    k = np.ones((1,) * nd)
    for _ in range(steps):
        k = signal.convolve(k, wf, method="direct")
    blk = tuple(slice(cc - h, cc + h + 1) for cc in centre)
    np.testing.assert_allclose(out[blk], k, rtol=1e-13, atol=1e-16)
    rest = out.copy()
    rest[blk] = 0
    assert not rest.any()


# ---------------------------------------------------------------- closed forms
@pytest.mark.parametrize("nd,shape,r", [(1, "box", 1), (2, "box", 1), (2, "star", 3), (3, "star", 1)])
def test_plane_wave_eigenvalue_periodic(nd, shape, r):
    """u0 = cos(theta.c) on a periodic grid -> Re(sigma(theta)^s e^{i theta.c}), sigma = sum w e^{+i o.theta}."""
    n = {1: 64, 2: 24, 3: 12}[nd]
    w = wl.seeded_weights(shape, nd, r)
    ks = [3, 5, 2][:nd]
    theta = [2 * np.pi * k / n for k in ks]
    c = np.meshgrid(*[np.arange(n)] * nd, indexing="ij")
    phase = sum(theta[a] * c[a] for a in range(nd))
    sig = 0j
    for idx in np.ndindex(*w.shape):
        sig += w[idx] * np.exp(1j * sum((idx[a] - r) * theta[a] for a in range(nd)))
    s = 7
    out = oracle.stencil_run(np.cos(phase), w, r, s, periodic=True)
    np.testing.assert_allclose(out, np.real(sig ** s * np.exp(1j * phase)), atol=1e-13)


def test_toeplitz_sine_modes_fixed_ring_1d():
    """Fixed zero ring: v_j = rho^j sin(pi k j/(n-1)), rho = sqrt(a/c), is an eigenvector with
    eigenvalue b + 2 sqrt(ac) cos(pi k/(n-1))  (tridiagonal Toeplitz closed form)."""
    a, b, c = 0.35, 0.4, 0.25
    n = 33
    j = np.arange(n)
    for k in (1, 4, 9):
        v = (np.sqrt(a / c) ** j) * np.sin(np.pi * k * j / (n - 1))
        v[0] = 0.0
        v[-1] = 0.0
        lam = b + 2 * np.sqrt(a * c) * np.cos(np.pi * k / (n - 1))
        out = oracle.stencil_run(v, [a, b, c], 1, 6)
        np.testing.assert_allclose(out, lam ** 6 * v, atol=1e-13 * np.abs(v).max())


@pytest.mark.parametrize("nd", [2, 3])
def test_sine_modes_fixed_ring_star(nd):
    """Separable star with a fixed zero ring: product of per-axis Toeplitz modes;
    eigenvalue = centre + sum_a 2 sqrt(w_-a w_+a) cos(pi k_a/(n_a-1))."""
    n = [14, 11, 9][:nd]
    w = wl.seeded_weights("star", nd, 1)
    centre = w[(1,) * nd]
    vec = np.ones(n)
    lam = centre
    for a in range(nd):
        lo = [1] * nd
        hi = [1] * nd
        lo[a] = 0
        hi[a] = 2
        wm, wp = w[tuple(lo)], w[tuple(hi)]
        k = a + 2
        j = np.arange(n[a])
        m = (np.sqrt(wm / wp) ** j) * np.sin(np.pi * k * j / (n[a] - 1))
        m[0] = m[-1] = 0.0
        shp = [1] * nd
        shp[a] = n[a]
        vec = vec * m.reshape(shp)
        lam = lam + 2 * np.sqrt(wm * wp) * np.cos(np.pi * k / (n[a] - 1))
    out = oracle.stencil_run(vec, w, 1, 5)
    np.testing.assert_allclose(out, lam ** 5 * vec, atol=1e-13 * np.abs(vec).max())


# ---------------------------------------------------------------- invariants
@pytest.mark.parametrize("periodic", [False, True])
@pytest.mark.parametrize("nd,shape,r", [(1, "star", 2), (2, "box", 1), (2, "star", 3), (3, "box", 1)])
def test_constant_field_preserved(nd, shape, r, periodic):
    w = wl.seeded_weights(shape, nd, r)
    n = {1: 40, 2: 17, 3: 9}[nd]
    u0 = np.full((n,) * nd, 0.7317)
    out = oracle.stencil_run(u0, w, r, 4, periodic=periodic)
    np.testing.assert_allclose(out, u0, rtol=1e-14)


def test_linearity():
    w = wl.seeded_weights("box", 2, 1)
    u, v = RNG.random((20, 23)), RNG.random((20, 23))
    lhs = oracle.stencil_run(2.5 * u - 0.75 * v, w, 1, 5)
    rhs = 2.5 * oracle.stencil_run(u, w, 1, 5) - 0.75 * oracle.stencil_run(v, w, 1, 5)
    np.testing.assert_allclose(lhs, rhs, atol=1e-14)


def test_semigroup_bitwise():
    w = wl.seeded_weights("star", 3, 1)
    u = RNG.random((9, 10, 11))
    a = oracle.stencil_run(oracle.stencil_run(u, w, 1, 3), w, 1, 4)
    b = oracle.stencil_run(u, w, 1, 7)
    assert np.array_equal(a, b)


def test_max_principle():
    w = wl.seeded_weights("box", 2, 3)
    u = RNG.random((30, 31))
    out = oracle.stencil_run(u, w, 3, 6)
    assert out.min() >= u.min() - 1e-15 and out.max() <= u.max() + 1e-15


def test_zero_steps_is_identity():
    u = RNG.random((5, 6))
    assert np.array_equal(oracle.stencil_run(u, wl.seeded_weights("box", 2, 1), 1, 0), u)


def test_fixed_equals_periodic_deep_interior_bitwise():
    """Cells at distance >= r*s from the edge never see the ring or the wrap: identical values."""
    r, s = 2, 3
    w = wl.seeded_weights("box", 2, r)
    u = RNG.random((26, 27))
    f = oracle.stencil_run(u, w, r, s)
    p = oracle.stencil_run(u, w, r, s, periodic=True)
    h = r * s
    assert np.array_equal(f[h:-h, h:-h], p[h:-h, h:-h])
    assert not np.array_equal(f, p)


# ---------------------------------------------------------------- internal consistency
@pytest.mark.parametrize("nd,shape,r,n", [(1, "star", 2, 15), (2, "box", 1, 7), (2, "star", 2, 9), (3, "box", 1, 5)])
def test_c_oracle_matches_python_statement(nd, shape, r, n):
    w = wl.seeded_weights(shape, nd, r)
    u = RNG.random((n,) * nd)
    for periodic in (False, True):
        a = oracle.stencil_run(u, w, r, 3, periodic=periodic)
        b = oracle.stencil_run_py(u, w, r, 3, periodic=periodic)
        np.testing.assert_allclose(a, b, rtol=1e-15, atol=1e-16)


@pytest.mark.parametrize("nd,shape,r,n,s", [(1, "star", 1, 300, 9), (2, "box", 1, 40, 7), (2, "star", 3, 45, 4),
                                            (3, "star", 1, 14, 3)])
def test_point_oracle_bitwise_equals_full(nd, shape, r, n, s):
    w = wl.seeded_weights(shape, nd, r)
    u = RNG.random((n,) * nd)
    full = oracle.stencil_run(u, w, r, s)
    cells = RNG.integers(0, n, size=(60, nd))
    cells[0] = 0
    cells[1] = n - 1
    cells[2] = r
    cells[3] = r * s
    vals = oracle.stencil_point(u, w, r, s, cells)
    assert np.array_equal(vals, full[tuple(cells.T)])


def test_oracle_rejects_bad_arguments():
    with pytest.raises(ValueError):
        oracle.stencil_run(np.zeros(5), [1.0, 2.0], 1, 1)


# ---------------------------------------------------------------- spectrum (plain definition)
@pytest.mark.parametrize("nd,shape,r,t", [(1, "star", 1, 8), (2, "box", 1, 3), (2, "star", 3, 2), (3, "box", 1, 2)])
def test_powered_spectrum_vs_fft_of_wrapped_kernel(nd, shape, r, t):
    """prod(L) * S_t = conj(fftn(W_t wrapped)), W_t the t-fold kernel (numpy FFT, scipy convolve)."""
    w = wl.seeded_weights(shape, nd, r)
    tile = {1: (56,), 2: (24, 16), 3: (8, 8, 8)}[nd]
    Wt = np.ones((1,) * nd)
    for _ in range(t):
        Wt = signal.convolve(Wt, w, method="direct")   # offset -r t .. r t, correlation composition
    h = r * t
    wrap = np.zeros(tile)
    for idx in np.ndindex(*Wt.shape):
        pos = tuple((idx[a] - h) % tile[a] for a in range(nd))
        wrap[pos] += Wt[idx]
    ref = np.conj(np.fft.fftn(wrap)) / np.prod(tile)
    got = spectrum.powered_spectrum(w, r, tile, t)
    np.testing.assert_allclose(got, ref, atol=1e-15)


def test_symbol_of_classic_heat1d():
    """sigma(theta) = 1/2 + 1/2 cos(theta) for (1/4, 1/2, 1/4)."""
    th = np.linspace(0, 2 * np.pi, 17)
    np.testing.assert_allclose(spectrum.symbol([0.25, 0.5, 0.25], 1, [th]), 0.5 + 0.5 * np.cos(th), atol=1e-16)
