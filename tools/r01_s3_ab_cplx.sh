# A/B: 2D ALU kernel, interleaved complex words after P1 (BF_CPLX=1) vs separate Re/Im planes (0)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
FFTSTENCIL_NVCC_DEFS="-DBF_CPLX=1" python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD1 FAILED
D=$PWD/paper_conf_ppopp_hanlcbzyczcy25_b200
FFTSTENCIL_LIB=$D/libfftstencil__DBF_CPLX_1.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "2d" 2>&1 | tail -1
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'ms frac', round(r['frac'],3))" $1 "$2" 2>&1 | tail -1; }
for rep in 1 2; do
  for lib in "" __DBF_CPLX_1; do
    for w in heat2d box2d49p; do
      FFTSTENCIL_LIB=$D/libfftstencil$lib.so timeout 300 python bench.py --workload $w --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/abc_$w$lib.jsonl 2>&1
      summ gpurun_out/abc_$w$lib.jsonl "${lib:-planes}"
    done
  done
done
