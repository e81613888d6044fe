python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q -m gpu 2>&1 | tail -3
FFTSTENCIL_TMA=0 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "parity_vs_oracle or 3d" 2>&1 | tail -2
rm -f gpurun_out/r01_run6.jsonl
for tmaflag in 1 0; do for w in heat3d box3d27p; do FFTSTENCIL_TMA=$tmaflag python bench.py --workload $w --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 | sed "s/^{/{\"variant\": \"tma$tmaflag\", /" >> gpurun_out/r01_run6.jsonl; done; done
