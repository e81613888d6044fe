rm -f gpurun_out/r01_final.jsonl gpurun_out/r01_configs.jsonl
python bench.py 2>&1 | tail -1 | tee gpurun_out/r01_final.jsonl
for w in heat2d box2d9p star2d13p box2d49p heat3d box3d27p heat1d; do python bench.py --workload $w --steps 3 --warmup 3 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/r01_configs.jsonl; done
for T in 1 2 4 8 12 16; do python bench.py --workload heat2d --T $T --steps 2 --warmup 2 --no-e2e --no-cpu-baseline | tail -1 >> gpurun_out/r01_configs.jsonl; done
ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/r01_final_launches.csv python bench.py --steps 1 --warmup 1 --time-steps 110 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:fft2d_ct -s 2 -c 1 -o gpurun_out/r01_final_ct python bench.py --steps 1 --warmup 1 --time-steps 33 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:fft3d_ct -s 2 -c 1 -o gpurun_out/r01_final_3d python bench.py --workload heat3d --steps 1 --warmup 1 --time-steps 6 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ls gpurun_out/*.ncu-rep
