python -m paper_conf_ppopp_hanlcbzyczcy25_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_e2e_pipe.py tests/test_gpu_steady_state.py tests/test_gpu_dist.py -q -x -m gpu -k "3d or 3D or band or e2e or pipe or capped or uncapped or loopback" 2>&1 | tail -2
for w in heat3d box3d27p heat3d_weak; do
  timeout 300 python bench.py --workload $w --steps 5 --warmup 3 --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('$w', round(d['value'],1), 'e2e', round(d['e2e']['value'],1), 'frac', round(r['frac'],3), 'fused_ms', round(r['fused_ms_avg'],4), 'band_ms', round(r['band_ms_avg'],4), 'share', round(r['fused_share_of_step'],3), d['clocks'])"
done
