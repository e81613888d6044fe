timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "1d or parity_vs_oracle or periodic" 2>&1 | tail -3
rm -f gpurun_out/r01_run16.jsonl
for w in heat1d_512m 1d5p_512m 1d7p_512m; do timeout 300 python bench.py --workload $w --steps 3 --warmup 3 --no-cpu-baseline | tail -1 >> gpurun_out/r01_run16.jsonl; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fft1d_ct -c 1 -o gpurun_out/r01_fft1d_ct python bench.py --workload heat1d_512m --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01_run16_launches.csv python bench.py --workload heat1d_512m --steps 1 --warmup 1 --time-steps 3000 --no-e2e --no-cpu-baseline > /dev/null 2>&1
