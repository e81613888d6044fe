# 3D geometry staging A/B with the HEAD library as the baseline, SM clocks sampled
L=paper_conf_ppopp_hanlcbzyczcy25_b200
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,clocks_throttle_reasons.active --format=csv
for rep in 1 2 3; do
  for v in _head __DBF3_GEO_SMEM_0 ""; do
    echo "lib=$v"; ENV_AB_ROUNDS=1 FFTSTENCIL_LIB=$L/libfftstencil$v.so timeout 600 python tools/env_ab.py heat3d 2>&1 | grep device
  done
done
nvidia-smi --query-gpu=clocks.sm,clocks_throttle_reasons.active --format=csv
