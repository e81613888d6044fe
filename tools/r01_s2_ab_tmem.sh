# A/B: S_T in tensor memory (BF_TMEM_S=1) vs shared memory, 2D ALU kernel
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'ms frac', round(r['frac'],3))" $1 "$2" 2>&1 | tail -1; }
for rep in 1 2; do
for lib in "" __DBF_TMEM_S_1; do
  for w in heat2d box2d49p; do
    FFTSTENCIL_LIB=$PWD/paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil$lib.so timeout 300 python bench.py --workload $w --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/abt_$w$lib.jsonl 2>&1
    summ gpurun_out/abt_$w$lib.jsonl "${lib:-smem}"
  done
done
done
FFTSTENCIL_LIB=$PWD/paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil__DBF_TMEM_S_1.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "2d_engines or full_size_sampled or periodic" 2>&1 | tail -2
