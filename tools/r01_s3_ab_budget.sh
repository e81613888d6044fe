# band block budget sweep for ALU plans (FFTSTENCIL_BAND_BUDGET cells per buffer; 1536 = session 2)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'share', round(r['fused_share_of_step'],3), 'band', round(r['band_ms_avg'],4))" $1 "$2" 2>&1 | tail -1; }
for rep in 1 2; do
  for b in 1536 2240 3072 4608; do
    for w in heat2d box2d9p box2d49p heat3d; do
      FFTSTENCIL_BAND_BUDGET=$b timeout 300 python bench.py --workload $w --steps 2 --no-cpu-baseline --no-e2e > gpurun_out/abbg_$w$b.jsonl 2>&1
      summ gpurun_out/abbg_$w$b.jsonl "budget=$b"
    done
  done
done
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "band or vs_oracle or full_size_sampled" 2>&1 | tail -1
