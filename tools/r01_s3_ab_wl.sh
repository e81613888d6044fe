# A/B: 2D ALU kernel, warp-local P1->P2 / P4->P5 (BF_WARP_LOCAL=1, the default when this ran) vs group barriers (=0),
# and combined twiddles (BF_TW_COMB=1)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
FFTSTENCIL_NVCC_DEFS="-DBF_WARP_LOCAL=0" python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD0 FAILED
FFTSTENCIL_NVCC_DEFS="-DBF_TW_COMB=1" python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD1 FAILED
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'ms frac', round(r['frac'],3))" $1 "$2" 2>&1 | tail -1; }
for rep in 1 2; do
for lib in "" __DBF_WARP_LOCAL_0 __DBF_TW_COMB_1; do
  for w in heat2d box2d49p; do
    FFTSTENCIL_LIB=$PWD/paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil$lib.so timeout 300 python bench.py --workload $w --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/abl_$w$lib.jsonl 2>&1
    summ gpurun_out/abl_$w$lib.jsonl "${lib:-wl}"
  done
done
done
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "2d" 2>&1 | tail -2
FFTSTENCIL_LIB=$PWD/paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil__DBF_TW_COMB_1.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "2d" 2>&1 | tail -2
