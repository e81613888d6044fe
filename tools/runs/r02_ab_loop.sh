# A/B on one box: round-1 kernels (old) vs counted-loop cleanup (loop) -- 2D and 3D
D=paper_conf_ppopp_hanlcbzyczcy25_b200
run() {  # lib workload
  FFTSTENCIL_LIB=$D/$1 timeout 300 python bench.py --workload $2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('$1 $2', round(d['value'],1), 'frac', round(r['frac'],3), 'fused_ms', round(r['fused_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])"
}
for rep in 1 2; do
  for lib in libfftstencil_ab_old.so libfftstencil_ab_loop.so; do run $lib heat2d; run $lib heat3d; run $lib box2d49p; done
done
FFTSTENCIL_LIB=$D/libfftstencil_ab_loop.so timeout 300 python bench.py --workload heat3d --steps 3 --warmup 3 --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print('default K heat3d device', round(d['value'],1), 'e2e', round(d['e2e']['value'],1), d['e2e']['ms_per_step'])"
