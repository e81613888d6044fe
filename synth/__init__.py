"""Seeded synthetic inputs shared by the tests, the bench and the oracle legs.

This package holds NO arithmetic of the method (no DFT, no spectrum, no stencil
step): only the benchmark table, stencil shape masks, the seeded weight recipe and
the seeded grid generator.  Both the CUDA path's tests and the oracle consume it.
"""
from .workloads import (CONFIGS, Workload, classic_weights, gain_weights, grid, mask, seeded_weights,  # noqa: F401
                        signed_grid, signed_weights, stencil_weights)
