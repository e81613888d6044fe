# 3M vs 4M complex products (FFTSTENCIL_CMUL3) at 72 registers
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "parity_vs_oracle or factored_1d_parity or periodic_parity or full_size_3d" 2>&1 | tail -1
rm -f gpurun_out/r01_run18.jsonl
for lib in "" "paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil__DFFTSTENCIL_CMUL3_0.so"; do
  for w in heat2d box2d49p heat3d heat1d_512m; do
   FFTSTENCIL_LIB=$lib timeout 300 python bench.py --workload $w --steps 3 --warmup 3 --no-e2e --no-cpu-baseline | tail -1 | sed "s/^{/{\"lib\": \"$(basename "$lib")\", /" >> gpurun_out/r01_run18.jsonl
  done
done
