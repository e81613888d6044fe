python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q -m gpu 2>&1 | tail -1
FFTSTENCIL_TMA=0 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "parity_vs_oracle or periodic" 2>&1 | tail -1
rm -f gpurun_out/r01_run13.jsonl
for w in heat2d heat3d heat1d_512m 1d7p_512m; do python bench.py --workload $w --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/r01_run13.jsonl; done
FFTSTENCIL_ALGO=dense python bench.py --workload heat3d --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/r01_run13.jsonl
