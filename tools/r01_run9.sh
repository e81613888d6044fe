python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "3d or periodic or parity_vs" 2>&1 | tail -2
FFTSTENCIL_TMA=0 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "parity_vs_oracle or 3d or periodic" 2>&1 | tail -1
rm -f gpurun_out/r01_run9.jsonl
for tmaflag in 1 0; do for w in heat3d box3d27p; do FFTSTENCIL_TMA=$tmaflag python bench.py --workload $w --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 | sed "s/^{/{\"variant\": \"tma$tmaflag\", /" >> gpurun_out/r01_run9.jsonl; done; done
