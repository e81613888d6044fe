"""Stencil symbol and powered spectrum -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

The FFT path multiplies each tile's spectrum by "k_f * ... * k_f" (T factors),
PAPER.md §4 Eq. 10 L290 and Alg. 1 line 2 L256.  With the forward DFT
X[k] = sum_l x[l] exp(-2 pi i k.l / L) (reading Q7) and the correlation-form
weights of reading Q1 (u'[c] = sum_o w[o] u[c+o]), the spectrum of one step is
the stencil symbol

    sigma(theta) = sum_{o in [-r,r]^d} w[o] * exp(+i o.theta),   theta_a = 2 pi k_a / L_a

and T fused steps multiply by sigma^T (Eq. 10).  The inverse DFT's 1/prod(L) is
folded into the powered spectrum (reading Q6/Q7):  S_t[k] = sigma(theta_k)^t / prod(L).

These are written as the plain definition (a direct sum over offsets, a power by
repeated multiplication); tests/test_oracle.py pins them against numpy's FFT of the
wrapped t-fold kernel, which is an independent route to the same numbers.
"""
from __future__ import annotations

import itertools

import numpy as np


def symbol(weights, radius: int, thetas):
    """sigma(theta) for theta given as a list of per-axis 1-D arrays (outer grid)."""
    nd = len(thetas)
    w = np.asarray(weights, dtype=np.float64).reshape((2 * radius + 1,) * nd)
    grids = np.meshgrid(*[np.asarray(t, dtype=np.float64) for t in thetas], indexing="ij")
    acc = np.zeros(grids[0].shape, dtype=np.complex128)
    for idx in itertools.product(range(2 * radius + 1), repeat=nd):
        o = [i - radius for i in idx]
        phase = sum(o[a] * grids[a] for a in range(nd))
        acc += w[idx] * np.exp(1j * phase)
    return acc


def powered_spectrum(weights, radius: int, tile, t: int):
    """S_t[k] = sigma(2 pi k / L)^t / prod(L) on a tile of shape `tile` (natural k order)."""
    thetas = [2.0 * np.pi * np.arange(L) / L for L in tile]
    s = symbol(weights, radius, thetas)
    p = np.ones_like(s)
    for _ in range(t):
        p = p * s
    return p / float(np.prod(tile))
