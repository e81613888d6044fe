# 3D fused kernel: current pair's geometry read from the issuing thread's shared-memory slot
# (BF3_GEO_SMEM=1, default build) vs recomputed by every thread (libfftstencil__DBF3_GEO_SMEM_0.so)
L=paper_conf_ppopp_hanlcbzyczcy25_b200
timeout 900 python -m pytest -q -x -m gpu tests/test_gpu_parity.py tests/test_gpu_steady_state.py -k "3d" 2>&1 | tail -2
for rep in 1 2 3; do
  for v in __DBF3_GEO_SMEM_0 ""; do
    echo "lib=$v"; ENV_AB_ROUNDS=1 FFTSTENCIL_LIB=$L/libfftstencil$v.so timeout 600 python tools/env_ab.py heat3d box3d27p 2>&1 | grep device
  done
done
