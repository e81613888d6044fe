# A/B on one box: 2D fused kernel with the next pair's TMA origins staged in shared memory
# (libfftstencil.so) vs computed at the refill (libfftstencil_ab_old.so, commit bf91377)
D=paper_conf_ppopp_hanlcbzyczcy25_b200
timeout 900 python -m pytest -q -x -m gpu tests/test_gpu_parity.py tests/test_gpu_steady_state.py tests/test_gpu_e2e_pipe.py -k "2d" 2>&1 | tail -2
run() {  # lib workload
  FFTSTENCIL_LIB=$D/$1 timeout 300 python bench.py --workload $2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('$1 $2', round(d['value'],1), 'frac', round(r['frac'],3), 'fused_ms', round(r['fused_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])"
}
for rep in 1 2 3; do
  for lib in libfftstencil_ab_old.so libfftstencil.so; do run $lib heat2d; done
done
for lib in libfftstencil_ab_old.so libfftstencil.so; do run $lib box2d49p; run $lib box2d9p; run $lib heat3d; done
