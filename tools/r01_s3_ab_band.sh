# A/B: 2D band kernel with a warp per cone row (BAND_ROWS=1, default) vs the flattened cone loop (0)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
FFTSTENCIL_NVCC_DEFS="-DBAND_ROWS=0" python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD0 FAILED
D=$PWD/paper_conf_ppopp_hanlcbzyczcy25_b200
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "band or 2d or vs_oracle or full_size_sampled" 2>&1 | tail -1
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'share', round(r['fused_share_of_step'],3), 'band', round(r['band_ms_avg'],4))" $1 "$2" 2>&1 | tail -1; }
for rep in 1 2; do
  for lib in "" __DBAND_ROWS_0; do
    for w in heat2d box2d49p; do
      FFTSTENCIL_LIB=$D/libfftstencil$lib.so timeout 300 python bench.py --workload $w --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/abb_$w$lib.jsonl 2>&1
      summ gpurun_out/abb_$w$lib.jsonl "${lib:-rows}"
    done
  done
done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/s3_band_launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncu $?
