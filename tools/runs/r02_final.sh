# round-2 final evidence: GPU tests, smoke, default bench line (+ reference arm), ncu captures
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -4 | tee gpurun_out/r02f_smoke.txt
timeout 2700 python -m pytest tests -q -m gpu 2>&1 | tail -4 | tee gpurun_out/r02f_gpu_tests.txt
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv | tee gpurun_out/r02f_smi.txt
( time timeout 900 python bench.py > gpurun_out/r02f_bench.jsonl 2> gpurun_out/r02f_bench.err ) 2>&1 | tail -3
( time timeout 600 python bench.py --impl reference > gpurun_out/r02f_reference.jsonl ) 2>&1 | tail -3
# launch list of the default command's main line (no per_config), device times per launch
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r02f_launches.csv python bench.py --steps 2 --warmup 1 --no-per-config --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo launches rc=$?
# one --set full capture of each top kernel
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fft3d_bf -s 3 -c 1 -o gpurun_out/r02f_fft3d python bench.py --workload heat3d --steps 1 --warmup 1 --time-steps 8 --no-e2e --no-cpu-baseline --no-per-config > /dev/null 2>&1; echo ncu3d rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fft2d_bf -s 3 -c 1 -o gpurun_out/r02f_fft2d python bench.py --workload heat2d --steps 1 --warmup 1 --time-steps 44 --no-e2e --no-cpu-baseline --no-per-config > /dev/null 2>&1; echo ncu2d rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:band_cone -s 3 -c 1 -o gpurun_out/r02f_band3d python bench.py --workload heat3d --steps 1 --warmup 1 --time-steps 8 --no-e2e --no-cpu-baseline --no-per-config > /dev/null 2>&1; echo ncuband rc=$?
