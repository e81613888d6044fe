# band cone kernel: cp.async region loads (BAND_CPASYNC=1, default build) vs synchronous loads
# (libfftstencil__DBAND_CPASYNC_0.so); band-only times from the bench's live events
timeout 1500 python -m pytest -q -x -m gpu tests/test_gpu_parity.py tests/test_gpu_steady_state.py tests/test_gpu_e2e_pipe.py 2>&1 | tail -2
run() {  # lib workload
  FFTSTENCIL_LIB=$1 timeout 300 python bench.py --workload $2 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('$1'[-12:], '$2', round(d['value'],1), 'fused_ms', round(r['fused_ms_avg'],4), 'band_ms', round(r.get('band_ms_avg') or 0,4), 'ms/step', round(d['ms_per_step'],2), d['clocks']['sm_mhz'])"
}
A=paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil__DBAND_CPASYNC_0.so
B=paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil.so
for rep in 1 2; do for w in heat3d box3d27p heat2d box2d49p star2d13p; do run $A $w; run $B $w; done; done
run $A heat1d; run $B heat1d
timeout 600 python bench.py --workload heat3d --steps 3 --warmup 3 --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());e=d['e2e'];print('default e2e heat3d', round(d['value'],1), round(e['value'],1), e['overlap'])"
timeout 600 ncu --set full --clock-control none -k regex:band_cone -s 3 -c 1 -o gpurun_out/r02_band_async python bench.py --workload heat3d --steps 1 --warmup 1 --time-steps 8 --no-e2e --no-cpu-baseline --no-per-config > /dev/null 2>&1; echo ncu rc=$?
