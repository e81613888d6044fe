python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "band_kernels_agree or parity_vs_oracle" 2>&1 | tail -3
rm -f gpurun_out/r01_run3.jsonl
for w in heat2d box2d49p heat3d; do python bench.py --workload $w --steps 2 --warmup 1 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/r01_run3.jsonl; done
ncu --metrics gpu__time_duration.sum --clock-control none -c 120 --csv --log-file gpurun_out/r01_ct_launches.csv python bench.py --steps 1 --warmup 1 --time-steps 110 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:fft2d_ct -s 2 -c 1 -o gpurun_out/r01_fft2d_ct python bench.py --steps 1 --warmup 1 --time-steps 33 --no-e2e --no-cpu-baseline > gpurun_out/ncu_ct.log 2>&1
tail -2 gpurun_out/ncu_ct.log
