python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q -m gpu 2>&1 | tail -5
rm -f gpurun_out/r01_run4.jsonl
for w in heat3d box3d27p; do for T in 0 1 3; do python bench.py --workload $w --T $T --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/r01_run4.jsonl; done; done
FFTSTENCIL_ALGO=dense python bench.py --workload heat3d --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/r01_run4.jsonl
