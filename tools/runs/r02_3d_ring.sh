# 3D line kernel with S_T in TMEM + three-buffer TMA ring: parity, sanitizers, bench, ncu; Ozaki microbench
python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_steady_state.py tests/test_gpu_dist.py tests/test_gpu_e2e_pipe.py -q -x -m gpu -k "3d or 3D or vs_oracle or capped or uncapped or loopback or signed or pipe" 2>&1 | tail -4
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize.py > gpurun_out/r02_san_ring_$tool.log 2>&1; echo "$tool rc=$?"; grep -E "ERROR SUMMARY" gpurun_out/r02_san_ring_$tool.log | tail -2
done
for w in heat3d box3d27p; do
  timeout 300 python bench.py --workload $w --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config > gpurun_out/r02_ring_$w.jsonl 2>&1
  python -c "import json;d=json.loads(open('gpurun_out/r02_ring_$w.jsonl').read().strip().splitlines()[-1]);r=d['roofline'];print('$w', round(d['value'],1), 'GSt/s', 'frac', round(r['frac'],3), 'smem', round(r['smem']['frac'],3), 'fused ms', round(r['fused_ms_avg'],3), d['clocks'])" || tail -5 gpurun_out/r02_ring_$w.jsonl
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fft3d_bf -s 2 -c 1 -o gpurun_out/r02_fft3d_ring python bench.py --workload heat3d --steps 1 --warmup 1 --time-steps 8 --no-e2e --no-cpu-baseline --no-per-config > gpurun_out/r02_ncu3d_ring.log 2>&1; echo ncu rc=$?
bash tools/runs/r02_ozaki.sh
