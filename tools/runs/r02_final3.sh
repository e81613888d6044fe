# round-2 closing evidence (session 2, after the fused peer stores): smoke, GPU tests, default bench line + reference arm, launch list, ncu captures, e2e probe
# reference arm, launch list, ncu captures, sanitizers (band kernel changed), e2e probe
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -4 | tee gpurun_out/r02h_smoke.txt
timeout 2400 python -m pytest tests -q -m gpu 2>&1 | tail -4 | tee gpurun_out/r02h_gpu_tests.txt
( time timeout 900 python bench.py > gpurun_out/r02h_bench.jsonl 2> gpurun_out/r02h_bench.err ) 2>&1 | tail -3
( time timeout 600 python bench.py --impl reference > gpurun_out/r02h_reference.jsonl ) 2>&1 | tail -3
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r02h_launches.csv python bench.py --steps 2 --warmup 1 --no-per-config --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo launches rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fft3d_bf -s 3 -c 1 -o gpurun_out/r02h_fft3d python bench.py --workload heat3d --steps 1 --warmup 1 --time-steps 8 --no-e2e --no-cpu-baseline --no-per-config > /dev/null 2>&1; echo ncu3d rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fft2d_bf -s 3 -c 1 -o gpurun_out/r02h_fft2d python bench.py --workload heat2d --steps 1 --warmup 1 --time-steps 44 --no-e2e --no-cpu-baseline --no-per-config > /dev/null 2>&1; echo ncu2d rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:band_cone -s 3 -c 1 -o gpurun_out/r02h_band3d python bench.py --workload heat3d --steps 1 --warmup 1 --time-steps 8 --no-e2e --no-cpu-baseline --no-per-config > /dev/null 2>&1; echo ncuband rc=$?
timeout 600 python tools/e2e_probe.py heat3d heat2d > gpurun_out/r02h_e2e_probe.txt 2>&1
