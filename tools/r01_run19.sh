timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q -m gpu 2>&1 | tail -1
rm -f gpurun_out/r01_run19.jsonl
for rep in 1 2; do
for lib in "" "paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil__DFFTSTENCIL_CT2D_REGS_80.so"; do
  for w in heat2d box2d49p; do
   FFTSTENCIL_LIB=$lib timeout 300 python bench.py --workload $w --steps 3 --warmup 3 --no-e2e --no-cpu-baseline | tail -1 | sed "s/^{/{\"lib\": \"$(basename "$lib")\", /" >> gpurun_out/r01_run19.jsonl
  done
done
done
for w in heat3d box3d27p heat1d_512m; do timeout 300 python bench.py --workload $w --steps 3 --warmup 3 --no-e2e --no-cpu-baseline | tail -1 | sed "s/^{/{\"lib\": \"\", /" >> gpurun_out/r01_run19.jsonl; done
