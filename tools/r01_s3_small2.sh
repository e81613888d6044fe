# configs[0] after sizing the 1D band CTA by its region (64 threads for short bands)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "1d or band or 4096 or configs" 2>&1 | tail -1
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], round(d['value'],3), 'GSt/s ms/step', round(d['ms_per_step'],4), 'fused', round(r['fused_ms_avg'],4), 'band', round(r['band_ms_avg'],4), 'launches', d['gpu_launches'])" $1 "$2" 2>&1 | tail -1; }
for rep in 1 2; do
  for bs in 1 0; do
    FFTSTENCIL_BAND_STREAM=$bs timeout 300 python bench.py --workload heat1d --steps 20 --no-cpu-baseline --no-e2e > gpurun_out/sm2_$bs.jsonl 2>&1
    summ gpurun_out/sm2_$bs.jsonl "band_stream=$bs"
  done
done
timeout 300 python bench.py --workload heat1d_512m --steps 2 --no-cpu-baseline --no-e2e > gpurun_out/sm2_512m.jsonl 2>&1; summ gpurun_out/sm2_512m.jsonl "512m"
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/s3_small2_launches.csv python bench.py --workload heat1d --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncu $?
