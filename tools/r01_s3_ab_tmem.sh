# A/B: 2D ALU kernel, S_T in shared memory (default) vs tensor memory (BF_TMEM_S=1: x8 loads,
# =2: x16 loads)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
FFTSTENCIL_NVCC_DEFS="-DBF_TMEM_S=1" python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD0 FAILED
FFTSTENCIL_NVCC_DEFS="-DBF_TMEM_S=2" python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD1 FAILED
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'ms frac', round(r['frac'],3))" $1 "$2" 2>&1 | tail -1; }
for rep in 1 2; do
for lib in "" __DBF_TMEM_S_1 __DBF_TMEM_S_2; do
  for w in heat2d box2d49p; do
    FFTSTENCIL_LIB=$PWD/paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil$lib.so timeout 300 python bench.py --workload $w --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/abt_$w$lib.jsonl 2>&1
    summ gpurun_out/abt_$w$lib.jsonl "${lib:-smem}"
  done
done
done
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "2d" 2>&1 | tail -2
FFTSTENCIL_LIB=$PWD/paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil__DBF_TMEM_S_2.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "2d" 2>&1 | tail -2
