python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q -m gpu 2>&1 | tail -1
rm -f gpurun_out/r01_run15.jsonl
for bs in 1 0; do for w in heat2d box2d49p heat3d; do FFTSTENCIL_BAND_STREAM=$bs python bench.py --workload $w --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/r01_run15.jsonl; done; done
