# band cone kernel with 128-thread CTAs (FFTSTENCIL_BAND_NTH=128) vs 256, at several block budgets
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
FFTSTENCIL_BAND_NTH=128 timeout 900 python -m pytest -q -x -m gpu tests/test_gpu_parity.py -k "band or 3d or sampled" 2>&1 | tail -2
timeout 1500 python tools/env_ab.py heat3d box3d27p -- - FFTSTENCIL_BAND_NTH=128 FFTSTENCIL_BAND_NTH=128,FFTSTENCIL_BAND_BUDGET=2304 FFTSTENCIL_BAND_NTH=128,FFTSTENCIL_BAND_BUDGET=3200 FFTSTENCIL_BAND_BUDGET=2304
