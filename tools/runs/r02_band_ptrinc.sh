# band kernel: pointer-increment global addressing (BAND_PTRINC=1, default build) vs per-cell
# recomputation (libfftstencil__DBAND_PTRINC_0.so)
L=paper_conf_ppopp_hanlcbzyczcy25_b200
timeout 900 python -m pytest -q -x -m gpu tests/test_gpu_parity.py -k "band or 3d or sampled" 2>&1 | tail -2
for rep in 1 2; do
  for v in __DBAND_PTRINC_0 ""; do
    echo "lib=$v"; ENV_AB_ROUNDS=1 FFTSTENCIL_LIB=$L/libfftstencil$v.so timeout 600 python tools/env_ab.py heat3d box3d27p 2>&1 | grep device
  done
done
timeout 600 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum --clock-control none -k regex:band_cone -s 2 -c 1 --csv python bench.py --workload heat3d --steps 1 --warmup 1 --time-steps 8 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | grep -E "duration|inst_exec" | awk -F'","' '{print "ptrinc=1", $(NF-2), $NF}'
FFTSTENCIL_LIB=$L/libfftstencil__DBAND_PTRINC_0.so timeout 600 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum --clock-control none -k regex:band_cone -s 2 -c 1 --csv python bench.py --workload heat3d --steps 1 --warmup 1 --time-steps 8 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | grep -E "duration|inst_exec" | awk -F'","' '{print "ptrinc=0", $(NF-2), $NF}'
