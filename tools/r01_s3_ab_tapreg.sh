# A/B: band kernel with register-resident taps for 5/7/9-tap stencils (BAND_TAPREG=1) vs shared (0)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
FFTSTENCIL_NVCC_DEFS="-DBAND_TAPREG=0" python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD0 FAILED
D=$PWD/paper_conf_ppopp_hanlcbzyczcy25_b200
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "band or vs_oracle or full_size" 2>&1 | tail -1
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'share', round(r['fused_share_of_step'],3), 'band', round(r['band_ms_avg'],4))" $1 "$2" 2>&1 | tail -1; }
for rep in 1 2; do
  for lib in "" __DBAND_TAPREG_0; do
    for w in heat2d box2d9p heat3d; do
      FFTSTENCIL_LIB=$D/libfftstencil$lib.so timeout 300 python bench.py --workload $w --steps 2 --no-cpu-baseline --no-e2e > gpurun_out/abtr_$w$lib.jsonl 2>&1
      summ gpurun_out/abtr_$w$lib.jsonl "${lib:-tapreg}"
    done
  done
done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/s3_tapreg_launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncu $?
