# radix ALU engines (2D + 3D, two 256-thread groups per CTA): parity, benches, ncu
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "engines or periodic or parity_vs_oracle" > gpurun_out/pytest_eng.log 2>&1; echo pytest $?
tail -15 gpurun_out/pytest_eng.log
for w in heat2d heat3d box2d49p; do
  timeout 600 python bench.py --workload $w --no-cpu-baseline --no-e2e > gpurun_out/b_$w.jsonl 2>&1; echo b $w $?
  tail -1 gpurun_out/b_$w.jsonl | cut -c1-300
  tail -1 gpurun_out/b_$w.jsonl | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['roofline'])" 2>&1 | cut -c1-600
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fft2d_bf -c 1 -o gpurun_out/r01_fft2d_bf python bench.py --steps 1 --warmup 0 --time-steps 11 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncu2 $?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fft3d_bf -c 1 -o gpurun_out/r01_fft3d_bf_c python bench.py --workload heat3d --steps 1 --warmup 0 --time-steps 2 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncu3 $?
