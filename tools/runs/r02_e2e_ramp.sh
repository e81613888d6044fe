python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest tests/test_gpu_e2e_pipe.py tests/test_gpu_parity.py -q -x -m gpu -k "pipe or host" 2>&1 | tail -2
for w in heat2d heat3d box2d49p box2d9p; do
  for rep in 1 2; do
  timeout 300 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print('$w', round(d['value'],1), 'e2e', round(d['e2e']['value'],1), round(d['e2e']['ms_per_step'],2), 'ms', d['e2e']['pipelined'])"
  done
done
