# whole-run on-chip kernel for small 1D grids: parity (both paths) + configs[0] bench
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "small1d or vs_oracle or aliasing or zero_steps or launch_count" 2>&1 | tail -3
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], round(d['value'],3), 'GSt/s ms/step', round(d['ms_per_step'],4), 'fused', round(r['fused_ms_avg'],4), 'launches', d['gpu_launches'])" $1 "$2" 2>&1 | tail -1; }
for rep in 1 2; do
  for sm in 1 0; do
    FFTSTENCIL_SMALL1D=$sm timeout 300 python bench.py --workload heat1d --steps 20 --no-cpu-baseline --no-e2e > gpurun_out/sm3_$sm.jsonl 2>&1
    summ gpurun_out/sm3_$sm.jsonl "small1d=$sm"
  done
done
timeout 300 python bench.py --workload heat1d > gpurun_out/sm3_full.jsonl 2>&1; tail -c 400 gpurun_out/sm3_full.jsonl
