# default bench line, launch list, traffic of the final 2D/3D/1D ALU kernels
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 600 python bench.py > gpurun_out/bench_default.jsonl 2> gpurun_out/bench_default.err; echo bench $?
cat gpurun_out/bench_default.jsonl
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.jsonl 2> gpurun_out/bench_ref.err; echo ref $?
cat gpurun_out/bench_ref.jsonl
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_final.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/b_ncu.log 2>&1; echo ncu $?
for w in heat2d:11 box2d49p:4 heat3d:2 heat1d_512m:1024; do
  wl=${w%%:*}; ts=${w##*:}
  timeout 600 ncu --clock-control none -k regex:"fft[123]d_bf" -c 1 --csv --page raw --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum python bench.py --workload $wl --steps 1 --warmup 0 --time-steps $ts --no-e2e --no-cpu-baseline > gpurun_out/traffic_$wl.csv 2>&1; echo tr $wl $?
done
