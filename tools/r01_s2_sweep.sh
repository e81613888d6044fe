# all workloads + 2D T sweep (Heat-2D) + 3D dmma/alu A/B; one B200 back to back
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], 'T', d['config']['T'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'ms', r['bound'], 'frac', round(r['frac'],3), 'share', round(r['fused_share_of_step'],3), r['kernel'])" $1 "$2" 2>&1 | tail -1; }
for w in heat1d heat2d box2d9p star2d13p box2d49p heat3d box3d27p heat1d_512m 1d5p_512m 1d7p_512m box2d9p_weak heat3d_weak; do
  timeout 600 python bench.py --workload $w --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/sw_$w.jsonl 2>&1
  summ gpurun_out/sw_$w.jsonl "$w"
done
for T in 1 2 4 8 11 12 16; do
  timeout 600 python bench.py --workload heat2d --T $T --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/sw_heat2d_T$T.jsonl 2>&1
  summ gpurun_out/sw_heat2d_T$T.jsonl "heat2d T=$T"
done
for eng in dmma alu; do
  FFTSTENCIL_ENGINE=$eng timeout 600 python bench.py --workload heat2d --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/sw_eng_$eng.jsonl 2>&1
  summ gpurun_out/sw_eng_$eng.jsonl "engine=$eng"
done
