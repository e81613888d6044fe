# 3M vs 4M complex products (FFTSTENCIL_CMUL3), band stream on/off
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "parity_vs_oracle or factored_1d_parity or periodic_parity" 2>&1 | tail -1
rm -f gpurun_out/r01_run17.jsonl
for lib in "" "paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil__DFFTSTENCIL_CMUL3_0.so"; do
 for bs in 1 0; do
  for w in heat2d heat1d_512m; do
   FFTSTENCIL_LIB=$lib FFTSTENCIL_BAND_STREAM=$bs timeout 300 python bench.py --workload $w --steps 3 --warmup 3 --no-e2e --no-cpu-baseline | tail -1 | sed "s/^{/{\"lib\": \"$(basename "$lib")\", \"bs\": $bs, /" >> gpurun_out/r01_run17.jsonl
  done
 done
done
