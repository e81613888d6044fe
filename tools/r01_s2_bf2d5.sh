# 2D ALU engine, 5-pass 64 = 4 x 16 design: parity, benches, ncu
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "2d_engines or periodic or parity_vs_oracle or full_size_sampled or plane_wave" > gpurun_out/pytest_2d.log 2>&1; echo pytest $?
tail -3 gpurun_out/pytest_2d.log
for w in heat2d box2d49p box2d9p star2d13p; do
  timeout 600 python bench.py --workload $w --no-cpu-baseline --no-e2e > gpurun_out/b_$w.jsonl 2>&1; echo b $w $?
  tail -1 gpurun_out/b_$w.jsonl | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print(d['config']['workload'], round(d['value'],1), 'GSt/s fused', round(r['fused_ms_avg'],3), 'ms frac', round(r['frac'],3))"
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fft2d_bf -c 1 -o gpurun_out/r01_fft2d_bf_5p python bench.py --steps 1 --warmup 0 --time-steps 11 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncu2 $?
