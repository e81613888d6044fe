# A/B: ping-pong schedules: 2D BF_PINGPONG=2 (arrive at load issue) and 3D BF3_PINGPONG=1 vs free-running
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
FFTSTENCIL_NVCC_DEFS="-DBF_PINGPONG=2" python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD2 FAILED
FFTSTENCIL_NVCC_DEFS="-DBF3_PINGPONG=1" python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD3 FAILED
D=$PWD/paper_conf_ppopp_hanlcbzyczcy25_b200
FFTSTENCIL_LIB=$D/libfftstencil__DBF3_PINGPONG_1.so timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "3d_engines" 2>&1 | tail -1
FFTSTENCIL_LIB=$D/libfftstencil__DBF_PINGPONG_2.so timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "2d_engines" 2>&1 | tail -1
summ() { python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); r=d['roofline']; print(sys.argv[2], d['config']['workload'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],4), 'ms frac', round(r['frac'],3))" $1 "$2" 2>&1 | tail -1; }
for rep in 1 2; do
  for lib in "" __DBF_PINGPONG_2; do
    FFTSTENCIL_LIB=$D/libfftstencil$lib.so timeout 300 python bench.py --workload heat2d --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/abq_heat2d$lib.jsonl 2>&1
    summ gpurun_out/abq_heat2d$lib.jsonl "${lib:-free}"
  done
  for lib in "" __DBF3_PINGPONG_1; do
    FFTSTENCIL_LIB=$D/libfftstencil$lib.so timeout 300 python bench.py --workload heat3d --steps 2 --no-cpu-baseline --no-e2e > gpurun_out/abq_heat3d$lib.jsonl 2>&1
    summ gpurun_out/abq_heat3d$lib.jsonl "${lib:-free}"
  done
done
