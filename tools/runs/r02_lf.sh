# fft16 with scaled (Linzer-Feig) twiddles (FFT16_LF=1, default build) vs the round-2 fft16
# (libfftstencil__DFFT16_LF_0.so, FFTSTENCIL_LIB); parity of the ALU kernels first
timeout 1200 python -m pytest -q -x -m gpu tests/test_gpu_parity.py tests/test_gpu_steady_state.py 2>&1 | tail -2
run() {  # lib workload
  FFTSTENCIL_LIB=$1 timeout 300 python bench.py --workload $2 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('$1 $2', round(d['value'],1), 'fused_ms', round(r['fused_ms_avg'],4), 'ms/step', round(d['ms_per_step'],2), d['clocks']['sm_mhz'])"
}
A=paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil__DFFT16_LF_0.so
B=paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil.so
for rep in 1 2; do for w in heat3d box3d27p heat2d box2d49p; do run $A $w; run $B $w; done; done
run $A heat1d_512m; run $B heat1d_512m
