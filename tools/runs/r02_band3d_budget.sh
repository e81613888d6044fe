# 3D band block size (FFTSTENCIL_BAND_BUDGET, cells per buffer): band alone (stream=0) and concurrent
run() {  # budget stream workload
  FFTSTENCIL_BAND_BUDGET=$1 FFTSTENCIL_BAND_STREAM=$2 timeout 300 python bench.py --workload $3 --steps 5 --warmup 2 --no-e2e --no-cpu-baseline --no-per-config 2>/dev/null | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());r=d['roofline'];print('budget=$1 stream=$2 $3', round(d['value'],1), 'fused_ms', round(r['fused_ms_avg'],4), 'band_ms', round(r['band_ms_avg'],4), 'ms/step', round(d['ms_per_step'],2))"
}
for b in 1536 4608 9000 16000 24000; do run $b 0 heat3d; run $b 1 heat3d; done
for b in 1536 9000 16000; do run $b 0 box3d27p; run $b 1 box3d27p; done
