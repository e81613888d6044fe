python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q -m gpu 2>&1 | tail -15
for T in 8 11 12; do python bench.py --T $T --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/ct1.jsonl; done
FFTSTENCIL_CT_WARPS=16 python bench.py --T 12 --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/ct1.jsonl
for w in box2d49p star2d13p; do python bench.py --workload $w --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/ct1.jsonl; done
