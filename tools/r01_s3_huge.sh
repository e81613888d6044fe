# grids beyond 2^31 cells (1D cp.async + TMA, 2D, 3D) against the oracle on sampled cones
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k int32 2>&1 | tail -15
