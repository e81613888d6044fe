# band cone kernel: float-reciprocal index divisions (BAND_FDIV=1, default build) vs integer
# divisions (libfftstencil__DBAND_FDIV_0.so), and a sweep of the 3D band block budget
timeout 1500 python -m pytest -q -x -m gpu tests/test_gpu_parity.py tests/test_gpu_steady_state.py tests/test_gpu_e2e_pipe.py -k "band or 3d or e2e or sampled" 2>&1 | tail -2
run() {  # lib workload budget
  FFTSTENCIL_BAND_BUDGET=$3 FFTSTENCIL_LIB=$1 timeout 300 python bench.py --workload $2 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('$1'[-12:], '$2', 'budget=$3', round(d['value'],1), 'fused_ms', round(r['fused_ms_avg'],4), 'band_ms', round(r.get('band_ms_avg') or 0,4), 'ms/step', round(d['ms_per_step'],2), d['clocks']['sm_mhz'])"
}
A=paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil__DBAND_FDIV_0.so
B=paper_conf_ppopp_hanlcbzyczcy25_b200/libfftstencil.so
for rep in 1 2; do for w in heat3d box3d27p; do run $A $w ""; run $B $w ""; done; done
for bud in 3600 6400 9000 12800; do run $B heat3d $bud; done
for bud in 3600 6400 9000; do run $B box3d27p $bud; done
for w in heat2d box2d49p; do run $A $w ""; run $B $w ""; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:band_cone -s 3 -c 1 -o gpurun_out/r02_band_fdiv python bench.py --workload heat3d --steps 1 --warmup 1 --time-steps 8 --no-e2e --no-cpu-baseline --no-per-config > /dev/null 2>&1; echo ncu rc=$?
