# A/B: band CTA of ALU plans with up to 128 registers (FFTSTENCIL_BAND_WIDE=1, default) vs 40 (0)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "band or vs_oracle or full_size_sampled or 3d_engines or 2d_engines" 2>&1 | tail -1
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'share', round(r['fused_share_of_step'],3), 'band', round(r['band_ms_avg'],4))" $1 "$2" 2>&1 | tail -1; }
for rep in 1 2; do
  for bw in 1 0; do
    for w in heat2d box2d49p heat3d; do
      FFTSTENCIL_BAND_WIDE=$bw timeout 300 python bench.py --workload $w --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/abw2_$w$bw.jsonl 2>&1
      summ gpurun_out/abw2_$w$bw.jsonl "wide=$bw"
    done
  done
done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/s3_bandw_launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncu $?
