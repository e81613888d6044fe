# A/B: lean band cone loop (BAND_LEAN=1, default: ring clipped out of the cone, incremental
# index) vs the session-2 loop (0)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
FFTSTENCIL_NVCC_DEFS="-DBAND_LEAN=0" python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD0 FAILED
D=$PWD/paper_conf_ppopp_hanlcbzyczcy25_b200
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -m gpu -x -q 2>&1 | tail -1
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'share', round(r['fused_share_of_step'],3), 'band', round(r['band_ms_avg'],4))" $1 "$2" 2>&1 | tail -1; }
for rep in 1 2; do
  for lib in "" __DBAND_LEAN_0; do
    for w in heat2d box2d49p heat3d box3d27p heat1d_512m; do
      FFTSTENCIL_LIB=$D/libfftstencil$lib.so timeout 300 python bench.py --workload $w --steps 2 --no-cpu-baseline --no-e2e > gpurun_out/abl2_$w$lib.jsonl 2>&1
      summ gpurun_out/abl2_$w$lib.jsonl "${lib:-lean}"
    done
  done
done
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/s3_lean_launches.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncu $?
