rm -f gpurun_out/r01_1d.jsonl
for w in heat1d_512m 1d5p_512m 1d7p_512m; do python bench.py --workload $w --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/r01_1d.jsonl; done
python bench.py --workload heat1d_512m --T 8 --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/r01_1d.jsonl
ncu --set full --clock-control none -k regex:fft1d -s 2 -c 1 -o gpurun_out/r01_fft1d python bench.py --workload heat1d_512m --steps 1 --warmup 1 --time-steps 42 --no-e2e --no-cpu-baseline > /dev/null 2>&1
# dense L48 T8: this box vs the recorded 160.9 (box-to-box check)
FFTSTENCIL_ALGO=dense python bench.py --T 8 --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/r01_1d.jsonl
