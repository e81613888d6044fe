# band concurrent (side stream) vs serialised on the run stream (FFTSTENCIL_BAND_STREAM=0), one box
run() {  # stream workload
  FFTSTENCIL_BAND_STREAM=$1 timeout 300 python bench.py --workload $2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('stream=$1 $2', round(d['value'],1), 'frac', round(r['frac'],3), 'fused_ms', round(r['fused_ms_avg'],4), 'share', round(r['fused_share_of_step'],3), 'band_ms', round(r['band_ms_avg'],4), 'ms/step', round(d['ms_per_step'],2))"
}
for rep in 1 2; do for w in heat3d box3d27p heat2d box2d49p heat3d_weak; do run 1 $w; run 0 $w; done; done
