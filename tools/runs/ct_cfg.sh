rm -f gpurun_out/ct_cfg.jsonl
for C in 81 82 84 161 162; do
  FFTSTENCIL_CT_CFG=$C python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "parity_vs_oracle" 2>&1 | tail -1 | sed "s/^/cfg $C: /"
  FFTSTENCIL_CT_CFG=$C python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 | sed "s/^{/{\"variant\": $C, /" >> gpurun_out/ct_cfg.jsonl
  FFTSTENCIL_CT_CFG=$C python bench.py --workload box2d49p --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 | sed "s/^{/{\"variant\": $C, /" >> gpurun_out/ct_cfg.jsonl
done
