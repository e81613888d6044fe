python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "band or parity_vs_oracle or full_size" 2>&1 | tail -1
rm -f gpurun_out/r01_run14.jsonl
for w in heat2d box2d49p heat3d box3d27p; do python bench.py --workload $w --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/r01_run14.jsonl; done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01_run14_launches.csv python bench.py --steps 1 --warmup 1 --time-steps 110 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01_run14_launches49.csv python bench.py --workload box2d49p --steps 1 --warmup 1 --time-steps 40 --no-e2e --no-cpu-baseline > /dev/null 2>&1
