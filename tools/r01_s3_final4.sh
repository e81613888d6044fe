# session 3 final closing run (after the 2D band block budget): smoke, all GPU tests, default bench
# line, reference arm, every workload, launch list, DRAM traffic of the 2D kernel
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/s3x_smoke.log 2>&1; echo smoke $?; tail -3 gpurun_out/s3x_smoke.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/s3x_gpu_tests.log 2>&1; echo tests $?; tail -1 gpurun_out/s3x_gpu_tests.log
timeout 600 python bench.py > gpurun_out/s3x_bench_default.jsonl 2> gpurun_out/s3x_bench_default.err; echo bench $?
cat gpurun_out/s3x_bench_default.jsonl
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/s3x_bench_ref.jsonl 2>&1; echo ref $?
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; m=r.get('smem',{}); print(sys.argv[2], d['config']['workload'], 'T', d['config']['T'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'ms', r['bound'], 'frac', round(r['frac'],3), 'smem', round(m.get('frac',0),3), 'share', round(r['fused_share_of_step'],3))" $1 "$2" 2>&1 | tail -1; }
for w in heat1d heat2d box2d9p star2d13p box2d49p heat3d box3d27p heat1d_512m 1d5p_512m 1d7p_512m box2d9p_weak heat3d_weak; do
  timeout 600 python bench.py --workload $w --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/s3x_sw_$w.jsonl 2>&1
  summ gpurun_out/s3x_sw_$w.jsonl "$w"
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/s3x_launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncu $?
timeout 600 ncu --clock-control none -k regex:"fft2d_bf" -c 1 --csv --page raw --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum python bench.py --workload heat2d --steps 1 --warmup 0 --time-steps 11 --no-e2e --no-cpu-baseline > gpurun_out/s3x_traffic_heat2d.csv 2>&1; echo tr $?
