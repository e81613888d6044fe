# programmatic dependent launch: full GPU suite with PDL on (default), then device / e2e A/B
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 2400 python -m pytest tests -q -m gpu 2>&1 | tail -3
FFTSTENCIL_PDL=0 timeout 1200 python -m pytest tests -q -m gpu -x tests/test_gpu_parity.py -k "sampled or band" 2>&1 | tail -2
timeout 1500 python tools/env_ab.py heat3d box3d27p heat2d box2d49p -- FFTSTENCIL_PDL=0 FFTSTENCIL_PDL=1   # needs the (reverted) PDL build
