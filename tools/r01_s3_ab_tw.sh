# A/B: 2D ALU kernel twiddles from register powers (BF_TW_REG=1, the default when this ran) vs the shared table (=0)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
FFTSTENCIL_NVCC_DEFS="-DBF_TW_REG=0" python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD0 FAILED
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'ms frac', round(r['frac'],3))" $1 "$2" 2>&1 | tail -1; }
for rep in 1 2; do
for lib in "" __DBF_TW_REG_0; do
  for w in heat2d box2d49p; do
    FFTSTENCIL_LIB=$PWD/paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil$lib.so timeout 300 python bench.py --workload $w --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/abw_$w$lib.jsonl 2>&1
    summ gpurun_out/abw_$w$lib.jsonl "${lib:-reg}"
  done
done
done
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "2d" 2>&1 | tail -2
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"fft2d_bf" -c 1 -o gpurun_out/s3_fft2d_bf python bench.py --workload heat2d --steps 1 --warmup 0 --time-steps 11 --no-e2e --no-cpu-baseline > gpurun_out/s3_ncu2d.log 2>&1; echo ncu $?
