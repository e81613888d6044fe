# A/B: 32-bit store predicates in the 2D ALU kernel's P5 (BF_PRED32=1, default) vs int64 (0)
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
FFTSTENCIL_NVCC_DEFS="-DBF_PRED32=0" python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD0 FAILED
D=$PWD/paper_conf_ppopp_hanlcbzyczcy25_b200
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "2d or vs_oracle or full_size_sampled or int32 or periodic" 2>&1 | tail -1
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'share', round(r['fused_share_of_step'],3))" $1 "$2" 2>&1 | tail -1; }
for rep in 1 2; do
  for lib in "" __DBF_PRED32_0; do
    for w in heat2d box2d49p; do
      FFTSTENCIL_LIB=$D/libfftstencil$lib.so timeout 300 python bench.py --workload $w --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/abp2_$w$lib.jsonl 2>&1
      summ gpurun_out/abp2_$w$lib.jsonl "${lib:-pred32}"
    done
  done
done
