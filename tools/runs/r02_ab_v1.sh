# A/B on one box: 2D kernel variants (old = round 1, v1 = round 1 + permuted twiddles, loop = round-2 cleanup)
D=paper_conf_ppopp_hanlcbzyczcy25_b200
run() {
  FFTSTENCIL_LIB=$D/$1 timeout 300 python bench.py --workload $2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('$1 $2', round(d['value'],1), 'frac', round(r['frac'],3), 'fused_ms', round(r['fused_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])"
}
for rep in 1 2 3; do
  for lib in libfftstencil_ab_old.so libfftstencil_ab_v1.so libfftstencil_ab_loop.so libfftstencil_ab_clean.so; do run $lib heat2d; done
done
for lib in libfftstencil_ab_old.so libfftstencil_ab_v1.so libfftstencil_ab_loop.so; do run $lib box2d49p; run $lib box2d9p; done
