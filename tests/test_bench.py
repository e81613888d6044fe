"""Host-side accounting of bench.py (no GPU): the whole-job GStencils/s of a weak-scaled run.

bench.py stacks the N=1 workload's rows N times along axis 0 (the global grid the library
decomposes back into per-rank slabs), so the throughput is global cells x time steps / the
max-over-ranks time -- with no extra factor of the world size (reading Q18).
"""
import bench
from synth import workloads as wl


def test_gstencils_definition():
    # 10240^2 cells x 1000 steps in 100 ms = 1048.576 GStencils/s
    assert abs(bench.gstencils(10240 * 10240, 1000, 100.0) - 1048.576) < 1e-9


def test_weak_scaling_counts_each_slab_once():
    wk = wl.CONFIGS["box2d9p_weak"]
    per_gpu = 1
    for e in wk.extents:
        per_gpu *= e
    one = bench.gstencils(per_gpu, 1000, 50.0)
    for world in (2, 4, 8):
        glob = (wk.extents[0] * world,) + tuple(wk.extents[1:])
        cells = 1
        for e in glob:
            cells *= e
        # perfect weak scaling (same time per rank) reports exactly world x the 1-GPU value
        assert abs(bench.gstencils(cells, 1000, 50.0) / one - world) < 1e-12


def test_smem_wavefront_model():
    # 2D five passes (4 read + write, 1 read) + S_T; 3D cropped inverse passes
    assert bench.smem_wavefronts_per_pair({"ndim": 2}) == 10 * 512
    assert bench.smem_wavefronts_per_pair({"ndim": 3, "valid": [12, 12, 12]}) == 4416
    assert bench.smem_wavefronts_per_pair({"ndim": 3, "valid": [16, 16, 16]}) == 10 * 512
    assert bench.smem_wavefronts_per_pair({"ndim": 1}) == 14 * 512
    assert abs(bench.SMEM_PEAK_TBPS - 37.22496) < 1e-9
