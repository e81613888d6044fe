# 3D fused kernel: group 1 starts out of phase with group 0 (BF3_STAGGER = 1 / 2 / 3: after group
# 0's P1 / P2 / P3 of its first pair) vs the default simultaneous start
L=paper_conf_ppopp_hanlcbzyczcy25_b200
FFTSTENCIL_LIB=$L/libfftstencil__DBF3_STAGGER_2.so timeout 900 python -m pytest -q -x -m gpu tests/test_gpu_parity.py tests/test_gpu_steady_state.py -k "3d" 2>&1 | tail -2
for rep in 1 2; do
  for v in "" __DBF3_STAGGER_1 __DBF3_STAGGER_2 __DBF3_STAGGER_3; do
    echo "lib=$v"; ENV_AB_ROUNDS=1 FFTSTENCIL_LIB=$L/libfftstencil$v.so timeout 600 python tools/env_ab.py heat3d 2>&1 | grep device | head -1
  done
done
