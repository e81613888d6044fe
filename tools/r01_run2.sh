python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q -m gpu 2>&1 | tail -5
for w in heat2d box2d9p star2d13p box2d49p heat3d box3d27p; do python bench.py --workload $w --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/r01_run2.jsonl; done
