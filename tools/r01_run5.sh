python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q -m gpu 2>&1 | tail -4
FFTSTENCIL_TMA=0 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "parity_vs_oracle or full_size_sampled" 2>&1 | tail -2
rm -f gpurun_out/r01_run5.jsonl
for tmaflag in 1 0; do for w in heat2d box2d49p; do FFTSTENCIL_TMA=$tmaflag python bench.py --workload $w --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 | sed "s/^{/{\"variant\": \"tma$tmaflag\", /" >> gpurun_out/r01_run5.jsonl; done; done
FFTSTENCIL_CT_CFG=84 python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 | sed "s/^{/{\"variant\": \"tma84\", /" >> gpurun_out/r01_run5.jsonl
