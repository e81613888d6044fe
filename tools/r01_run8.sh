python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "parity_vs_oracle or periodic_parity or full_size_sampled" 2>&1 | tail -2
FFTSTENCIL_TMA=0 FFTSTENCIL_CT_CFG=81 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "parity_vs_oracle" 2>&1 | tail -1
rm -f gpurun_out/r01_run8.jsonl
for cfg in "1 82" "1 81" "1 84" "0 81"; do set -- $cfg
  FFTSTENCIL_TMA=$1 FFTSTENCIL_CT_CFG=$2 python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 | sed "s/^{/{\"variant\": \"tma$1-$2\", /" >> gpurun_out/r01_run8.jsonl
done
