# e2e schedule: symmetric ramps (FFTSTENCIL_E2E_RAMP=2, default) vs first-in / last-out only (1),
# tail depth sweep; band fdiv A/B at the default band budget
timeout 1200 python -m pytest -q -x -m gpu tests/test_gpu_e2e_pipe.py tests/test_gpu_parity.py -k "e2e or pipe or band" 2>&1 | tail -2
e2e() {  # workload ramp Q Qt
  FFTSTENCIL_E2E_RAMP=$2 FFTSTENCIL_E2E_DEPTH=$3 FFTSTENCIL_E2E_DEPTH_TAIL=$4 timeout 600 python bench.py --workload $1 --steps 3 --warmup 3 --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());e=d['e2e'];print('$1 ramp=$2 Q=$3 Qt=$4 device', round(d['value'],1), 'e2e', round(e['value'],1), 'e2e ms', round(e['ms_per_step'],2), 'dev ms', round(d['ms_per_step'],2))"
}
for rep in 1 2; do
  e2e heat3d 1 20 20; e2e heat3d 2 20 20; e2e heat3d 2 20 24; e2e heat3d 2 20 28; e2e heat3d 2 24 24
  e2e heat2d 1 16 16; e2e heat2d 2 16 16; e2e heat2d 2 16 20; e2e heat2d 2 20 20
done
run() {  # lib workload
  FFTSTENCIL_LIB=$1 timeout 300 python bench.py --workload $2 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('$1'[-12:], '$2', round(d['value'],1), 'fused_ms', round(r['fused_ms_avg'],4), 'band_ms', round(r.get('band_ms_avg') or 0,4), 'ms/step', round(d['ms_per_step'],2), d['clocks']['sm_mhz'])"
}
A=paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil__DBAND_FDIV_0.so
B=paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil.so
for rep in 1 2; do for w in heat3d box3d27p box2d49p; do run $A $w; run $B $w; done; done
