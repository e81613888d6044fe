# after the 2D / 3D ablation cleanup: parity of the ALU kernels, sanitizers, bench; Ozaki microbench
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_steady_state.py -q -x -m gpu 2>&1 | tail -3
timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python tools/sanitize.py > gpurun_out/r02_san_clean_memcheck.log 2>&1; echo "memcheck rc=$?"
for w in heat2d heat3d box2d49p; do
  timeout 300 python bench.py --workload $w --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config > gpurun_out/r02_clean_$w.jsonl 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/r02_clean_$w.jsonl').read().strip().splitlines()[-1]);r=d['roofline'];print('$w', round(d['value'],1), 'GSt/s', 'frac', round(r['frac'],3), 'fused ms', round(r['fused_ms_avg'],3), d['clocks'])" || tail -5 gpurun_out/r02_clean_$w.jsonl
done
bash tools/runs/r02_ozaki.sh
