# T sweep around the cost model's choice, final kernels (Heat-2D, Box-2D49P, Heat-3D)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], 'T', d['config']['T'], 'S', d['config']['valid'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'share', round(r['fused_share_of_step'],3))" $1 "$2" 2>&1 | tail -1; }
for T in 9 10 11 12 13; do
  timeout 300 python bench.py --workload heat2d --T $T --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/ts_h2_$T.jsonl 2>&1; summ gpurun_out/ts_h2_$T.jsonl heat2d
done
for T in 3 4 5; do
  timeout 300 python bench.py --workload box2d49p --T $T --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/ts_b49_$T.jsonl 2>&1; summ gpurun_out/ts_b49_$T.jsonl box2d49p
done
for T in 1 2 3; do
  timeout 300 python bench.py --workload heat3d --T $T --steps 2 --no-cpu-baseline --no-e2e > gpurun_out/ts_h3_$T.jsonl 2>&1; summ gpurun_out/ts_h3_$T.jsonl heat3d
done
